// Graph builder of the C ABI (include/astitch.h) and error plumbing.
// The IR mirrors the paper's op taxonomy (Sec. 2.1): element-wise
// unary/binary ops (broadcast is element-wise-like), row- and
// column-reduce, plus the key-padding LENGTHS mask of BASELINE configs[2].
#include <cmath>
#include <cstdint>
#include <string>

#include "internal.h"

namespace astitch {

static thread_local std::string g_last_error;

void set_error(const std::string& msg) { g_last_error = msg; }

astitch_status fail(astitch_status s, const std::string& msg) {
  g_last_error = msg;
  return s;
}

int dtype_size(astitch_dtype d) {
  switch (d) {
    case ASTITCH_F32: return 4;
    case ASTITCH_BF16: return 2;
    case ASTITCH_F16: return 2;
    case ASTITCH_I32: return 4;
  }
  return 0;
}

const char* dtype_name(astitch_dtype d) {
  switch (d) {
    case ASTITCH_F32: return "f32";
    case ASTITCH_BF16: return "bf16";
    case ASTITCH_F16: return "f16";
    case ASTITCH_I32: return "i32";
  }
  return "?";
}

const char* kind_name(astitch_kind k) {
  switch (k) {
    case ASTITCH_FULL: return "FULL";
    case ASTITCH_ROWVEC: return "ROWVEC";
    case ASTITCH_COLVEC: return "COLVEC";
    case ASTITCH_SCALAR: return "SCALAR";
    case ASTITCH_LENGTHS: return "LENGTHS";
    case ASTITCH_SEGMENTS: return "SEGMENTS";
  }
  return "?";
}

const char* unop_name(int op) {
  static const char* n[] = {"NEG", "ABS", "EXP", "LOG", "TANH", "ERF", "SQRT", "RSQRT", "RCP",
                            "SIGMOID", "GELU_TANH", "GELU_ERF", "GELU_TANH_GRAD"};
  return (op >= 0 && op < ASTITCH_UNOP_COUNT) ? n[op] : "?";
}

const char* binop_name(int op) {
  static const char* n[] = {"ADD", "SUB", "MUL", "DIV", "MAX", "MIN", "POW"};
  return (op >= 0 && op < ASTITCH_BINOP_COUNT) ? n[op] : "?";
}

}  // namespace astitch

using namespace astitch;

namespace {

bool valid_value(const Graph& g, astitch_value_t v) {
  return v >= 0 && v < static_cast<int>(g.nodes.size());
}

astitch_status push(Graph& g, const Node& n, astitch_value_t* out) {
  if (g.nodes.size() >= (1u << 20)) return fail(ASTITCH_ERR_INVALID_GRAPH, "graph too large");
  g.nodes.push_back(n);
  *out = static_cast<astitch_value_t>(g.nodes.size() - 1);
  return ASTITCH_OK;
}

}  // namespace

extern "C" {

const char* astitch_status_str(astitch_status s) {
  switch (s) {
    case ASTITCH_OK: return "ASTITCH_OK";
    case ASTITCH_ERR_INVALID_ARGUMENT: return "ASTITCH_ERR_INVALID_ARGUMENT";
    case ASTITCH_ERR_INVALID_GRAPH: return "ASTITCH_ERR_INVALID_GRAPH";
    case ASTITCH_ERR_UNSUPPORTED: return "ASTITCH_ERR_UNSUPPORTED";
    case ASTITCH_ERR_SHAPE: return "ASTITCH_ERR_SHAPE";
    case ASTITCH_ERR_RESOURCE: return "ASTITCH_ERR_RESOURCE";
    case ASTITCH_ERR_CUDA: return "ASTITCH_ERR_CUDA";
    case ASTITCH_ERR_NCCL: return "ASTITCH_ERR_NCCL";
    case ASTITCH_ERR_INTERNAL: return "ASTITCH_ERR_INTERNAL";
  }
  return "ASTITCH_ERR_UNKNOWN";
}

const char* astitch_last_error(void) { return g_last_error.c_str(); }

int astitch_abi_version(void) { return ASTITCH_ABI_VERSION; }

astitch_status astitch_graph_create(astitch_graph_t* out) {
  if (!out) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "out is NULL");
  try {
    *out = new astitch_graph_s();
  } catch (...) {
    return fail(ASTITCH_ERR_INTERNAL, "allocation failed");
  }
  set_error("");
  return ASTITCH_OK;
}

astitch_status astitch_graph_destroy(astitch_graph_t g) {
  delete g;
  return ASTITCH_OK;
}

astitch_status astitch_graph_input(astitch_graph_t g, astitch_kind kind, astitch_dtype dtype,
                                   astitch_value_t* out) {
  if (!g || !out) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL graph or out");
  if (kind != ASTITCH_FULL && kind != ASTITCH_ROWVEC && kind != ASTITCH_COLVEC && kind != ASTITCH_LENGTHS)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "input kind must be FULL, ROWVEC, COLVEC or LENGTHS");
  if (kind == ASTITCH_LENGTHS ? dtype != ASTITCH_I32
                              : (dtype != ASTITCH_F32 && dtype != ASTITCH_BF16 && dtype != ASTITCH_F16))
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "input dtype must be F32, BF16 or F16 (I32 for LENGTHS)");
  if (g->g.inputs.size() >= static_cast<size_t>(kMaxIO))
    return fail(ASTITCH_ERR_UNSUPPORTED, "too many inputs (max 16)");
  Node n;
  n.type = NodeType::Input;
  n.kind = kind;
  n.dtype = dtype;
  n.input_index = static_cast<int>(g->g.inputs.size());
  astitch_status s = push(g->g, n, out);
  if (s == ASTITCH_OK) g->g.inputs.push_back(*out);
  return s;
}

astitch_status astitch_graph_lengths(astitch_graph_t g, int64_t rows_per_segment,
                                     astitch_value_t* out) {
  if (!g || !out) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL graph or out");
  if (rows_per_segment < 1) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "rows_per_segment < 1");
  if (g->g.lengths_node >= 0 || g->g.segments_node >= 0)
    return fail(ASTITCH_ERR_INVALID_GRAPH, "graph already has a mask or segments");
  if (g->g.inputs.size() >= static_cast<size_t>(kMaxIO))
    return fail(ASTITCH_ERR_UNSUPPORTED, "too many inputs (max 16)");
  Node n;
  n.type = NodeType::Input;
  n.kind = ASTITCH_LENGTHS;
  n.dtype = ASTITCH_I32;
  n.input_index = static_cast<int>(g->g.inputs.size());
  astitch_status s = push(g->g, n, out);
  if (s == ASTITCH_OK) {
    g->g.inputs.push_back(*out);
    g->g.lengths_node = *out;
    g->g.rows_per_segment = rows_per_segment;
  }
  return s;
}

astitch_status astitch_graph_set_mask(astitch_graph_t g, astitch_value_t lengths, int64_t rows_per_segment) {
  if (!g) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL graph");
  if (rows_per_segment < 1) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "rows_per_segment < 1");
  if (lengths < 0 || lengths >= static_cast<astitch_value_t>(g->g.nodes.size()))
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad value");
  const Node& n = g->g.nodes[lengths];
  if (n.type != NodeType::Input || n.kind != ASTITCH_LENGTHS)
    return fail(ASTITCH_ERR_INVALID_GRAPH, "the mask must be a LENGTHS input (astitch_graph_input)");
  if (g->g.lengths_node >= 0 || g->g.segments_node >= 0)
    return fail(ASTITCH_ERR_INVALID_GRAPH, "graph already has a mask or segments");
  g->g.lengths_node = lengths;
  g->g.rows_per_segment = rows_per_segment;
  return ASTITCH_OK;
}

astitch_status astitch_graph_segments(astitch_graph_t g, int32_t nseg, int64_t elems,
                                      astitch_value_t* out) {
  if (!g || !out) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL graph or out");
  if (nseg < 1) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "nseg < 1");
  if (elems < 0) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "elems < 0");
  if (g->g.lengths_node >= 0 || g->g.segments_node >= 0)
    return fail(ASTITCH_ERR_INVALID_GRAPH, "graph already has a mask or segments");
  if (g->g.inputs.size() >= static_cast<size_t>(kMaxIO))
    return fail(ASTITCH_ERR_UNSUPPORTED, "too many inputs (max 16)");
  Node n;
  n.type = NodeType::Input;
  n.kind = ASTITCH_SEGMENTS;
  n.dtype = ASTITCH_I32;
  n.input_index = static_cast<int>(g->g.inputs.size());
  astitch_status s = push(g->g, n, out);
  if (s == ASTITCH_OK) {
    g->g.inputs.push_back(*out);
    g->g.segments_node = *out;
    g->g.nseg = nseg;
    g->g.seg_elems = elems;
  }
  return s;
}

astitch_status astitch_segments_layout(int32_t nseg, const int64_t* seg_rows, const int32_t* seg_cols,
                                       int32_t* table, int64_t* rows, int64_t* elems) {
  if (!seg_rows || !seg_cols || !table || !rows || !elems)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL argument");
  if (nseg < 1) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "nseg < 1");
  int64_t r = 0, off = 0;  // off in elements (always a multiple of 8)
  for (int32_t s = 0; s < nseg; ++s) {
    if (seg_rows[s] < 0 || seg_cols[s] < 1) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "segment rows < 0 or cols < 1");
    const int64_t pitch = (static_cast<int64_t>(seg_cols[s]) + 7) / 8 * 8;
    if (r > INT32_MAX || off / 8 > INT32_MAX) return fail(ASTITCH_ERR_SHAPE, "segment table overflows int32");
    table[4 * s + 0] = static_cast<int32_t>(r);
    table[4 * s + 1] = seg_cols[s];
    table[4 * s + 2] = static_cast<int32_t>(pitch);
    table[4 * s + 3] = static_cast<int32_t>(off / 8);
    r += seg_rows[s];
    off += seg_rows[s] * pitch;
  }
  if (r > INT32_MAX) return fail(ASTITCH_ERR_SHAPE, "segment table overflows int32");
  *rows = r;
  *elems = off;
  return ASTITCH_OK;
}

astitch_status astitch_graph_const(astitch_graph_t g, double v, astitch_value_t* out) {
  if (!g || !out) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL graph or out");
  if (!std::isfinite(v)) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "constant must be finite");
  Node n;
  n.type = NodeType::Const;
  n.kind = ASTITCH_SCALAR;
  n.cval = v;
  return push(g->g, n, out);
}

astitch_status astitch_graph_unary(astitch_graph_t g, astitch_unop op, astitch_value_t a,
                                   astitch_value_t* out) {
  if (!g || !out) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL graph or out");
  if (op < 0 || op >= ASTITCH_UNOP_COUNT) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad unop");
  if (!valid_value(g->g, a)) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad operand");
  astitch_kind k = g->g.nodes[a].kind;
  if (k == ASTITCH_LENGTHS || k == ASTITCH_SEGMENTS)
    return fail(ASTITCH_ERR_INVALID_GRAPH, "LENGTHS / SEGMENTS is not an operand");
  if (k == ASTITCH_SCALAR)
    return fail(ASTITCH_ERR_UNSUPPORTED, "unary op on a SCALAR constant (fold it on the host)");
  Node n;
  n.type = NodeType::Unary;
  n.sub = op;
  n.a = a;
  n.kind = k;
  return push(g->g, n, out);
}

astitch_status astitch_graph_binary(astitch_graph_t g, astitch_binop op, astitch_value_t a,
                                    astitch_value_t b, astitch_value_t* out) {
  if (!g || !out) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL graph or out");
  if (op < 0 || op >= ASTITCH_BINOP_COUNT) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad binop");
  if (!valid_value(g->g, a) || !valid_value(g->g, b))
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad operand");
  astitch_kind ka = g->g.nodes[a].kind, kb = g->g.nodes[b].kind;
  if (ka == ASTITCH_LENGTHS || kb == ASTITCH_LENGTHS || ka == ASTITCH_SEGMENTS || kb == ASTITCH_SEGMENTS)
    return fail(ASTITCH_ERR_INVALID_GRAPH, "LENGTHS / SEGMENTS is not an operand");
  if (ka == ASTITCH_SCALAR && kb == ASTITCH_SCALAR)
    return fail(ASTITCH_ERR_UNSUPPORTED, "binary op on two SCALARs (fold it on the host)");
  if (ka != kb && ka != ASTITCH_SCALAR && kb != ASTITCH_SCALAR)
    return fail(ASTITCH_ERR_INVALID_GRAPH,
                std::string("binary operands must have equal kinds or a SCALAR: ") +
                    kind_name(ka) + " vs " + kind_name(kb) + " (insert a broadcast)");
  Node n;
  n.type = NodeType::Binary;
  n.sub = op;
  n.a = a;
  n.b = b;
  n.kind = (ka == ASTITCH_SCALAR) ? kb : ka;
  return push(g->g, n, out);
}

astitch_status astitch_graph_reduce(astitch_graph_t g, astitch_redop op, astitch_axis axis,
                                    astitch_value_t a, astitch_value_t* out) {
  if (!g || !out) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL graph or out");
  if (op != ASTITCH_SUM && op != ASTITCH_RMAX) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad redop");
  if (axis != ASTITCH_AXIS_ROW && axis != ASTITCH_AXIS_COL)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad axis");
  if (!valid_value(g->g, a)) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad operand");
  astitch_kind k = g->g.nodes[a].kind;
  if (k == ASTITCH_LENGTHS || k == ASTITCH_SEGMENTS)
    return fail(ASTITCH_ERR_INVALID_GRAPH, "LENGTHS / SEGMENTS is not an operand");
  if (k != ASTITCH_FULL)
    return fail(ASTITCH_ERR_UNSUPPORTED,
                std::string("reduce needs a FULL operand, got ") + kind_name(k));
  Node n;
  n.type = NodeType::Reduce;
  n.sub = op;
  n.axis = axis;
  n.a = a;
  n.kind = (axis == ASTITCH_AXIS_ROW) ? ASTITCH_ROWVEC : ASTITCH_COLVEC;
  return push(g->g, n, out);
}

astitch_status astitch_graph_broadcast(astitch_graph_t g, astitch_axis axis, astitch_value_t a,
                                       astitch_value_t* out) {
  if (!g || !out) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL graph or out");
  if (axis != ASTITCH_AXIS_ROW && axis != ASTITCH_AXIS_COL)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad axis");
  if (!valid_value(g->g, a)) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad operand");
  astitch_kind k = g->g.nodes[a].kind;
  astitch_kind want = (axis == ASTITCH_AXIS_ROW) ? ASTITCH_ROWVEC : ASTITCH_COLVEC;
  if (k != want)
    return fail(ASTITCH_ERR_INVALID_GRAPH, std::string("broadcast ") +
                                               (axis == ASTITCH_AXIS_ROW ? "ROW" : "COL") +
                                               " needs a " + kind_name(want) + ", got " +
                                               kind_name(k));
  Node n;
  n.type = NodeType::Bcast;
  n.axis = axis;
  n.a = a;
  n.kind = ASTITCH_FULL;
  return push(g->g, n, out);
}

astitch_status astitch_graph_output(astitch_graph_t g, astitch_value_t v, astitch_dtype dtype,
                                    int32_t* out_index) {
  if (!g || !out_index) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL graph or out_index");
  if (!valid_value(g->g, v)) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad value");
  if (dtype != ASTITCH_F32 && dtype != ASTITCH_BF16 && dtype != ASTITCH_F16)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "output dtype must be F32, BF16 or F16");
  astitch_kind k = g->g.nodes[v].kind;
  if (k != ASTITCH_FULL && k != ASTITCH_ROWVEC && k != ASTITCH_COLVEC)
    return fail(ASTITCH_ERR_INVALID_GRAPH, std::string("cannot output a ") + kind_name(k));
  if (g->g.outputs.size() >= static_cast<size_t>(kMaxIO))
    return fail(ASTITCH_ERR_UNSUPPORTED, "too many outputs (max 16)");
  g->g.outputs.push_back(v);
  g->g.output_dtypes.push_back(dtype);
  *out_index = static_cast<int32_t>(g->g.outputs.size() - 1);
  return ASTITCH_OK;
}

astitch_status astitch_shard_rows(int64_t rows, int32_t world, int32_t rank, int64_t* row_begin,
                                  int64_t* row_count) {
  if (!row_begin || !row_count) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL out");
  if (rows < 0) return fail(ASTITCH_ERR_SHAPE, "rows < 0");
  if (world < 1 || rank < 0 || rank >= world)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad world / rank");
  int64_t base = rows / world, rem = rows % world;
  *row_count = base + (rank < rem ? 1 : 0);
  *row_begin = static_cast<int64_t>(rank) * base + (rank < rem ? rank : rem);
  return ASTITCH_OK;
}

}  // extern "C"
