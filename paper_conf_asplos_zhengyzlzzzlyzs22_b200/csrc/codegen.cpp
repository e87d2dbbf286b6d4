// Code generator: plan -> CUDA C++ source of ONE stitched kernel (per role),
// instantiating the scheme templates of kernels/astitch_device.cuh.
//
// Every live op of the subgraph is emitted once per row (element-level data
// reuse): FULL values live in per-lane fp32 register arrays (local
// scheme), ROWVEC values are team-uniform registers produced by shuffle /
// smem team reductions (regional scheme), COLVEC operands are hoisted per lane,
// column reductions accumulate per-lane partials, combine through HBM and a
// grid barrier (global scheme).  Each input element is loaded once and every
// output element stored once (operator-level reuse).
#include <cmath>
#include <cstdio>
#include <sstream>
#include <string>

#include "internal.h"

namespace astitch {
namespace {

std::string flit(double v) {
  char buf[64];
  float f = static_cast<float>(v);
  if (f == 0.0f) return "0.0f";
  snprintf(buf, sizeof(buf), "%af", static_cast<double>(f));
  return buf;
}

int dt_code(astitch_dtype d) { return d == ASTITCH_F32 ? 0 : (d == ASTITCH_BF16 ? 1 : 2); }

struct Gen {
  const Plan& p;
  const Graph& g;
  const Mapping& m;
  std::ostringstream o;
  int T, V, E, NE, RPB, U;
  long long C;
  bool masked, exact, ragged = false;
  int role;

  Gen(const Plan& pp, int r) : p(pp), g(pp.g), m(pp.map), role(r) {
    T = m.team;
    V = m.chunks_per_lane;
    E = m.vec_elems;
    NE = V * E;
    RPB = m.rows_per_block;
    U = m.row_unroll;
    C = p.desc.cols;
    ragged = g.segments_node >= 0;
    masked = g.lengths_node >= 0 || ragged;  // varlen rows: masks of the row's own length
    slab = m.tmpl == Template::GlobalSweep && m.nslab > 1 && role != ROLE_SHARD_FINAL;
    exact = slab ? (C % (static_cast<long long>(T) * V * E) == 0) : (static_cast<long long>(T) * V * E == C);
    if (slab) tile_off = "SLABOFF";
    split = (m.tmpl == Template::SplitRow) || (m.tmpl == Template::RowStream && m.split > 1);
    compute_precise();
    compute_absorb();
  }
  bool split = false;
  bool slab = false;  // column slabs (wide rows): every column index is offset by the CTA's slab
  // chunk index of chunk j of this lane within its row (slab-relative columns + slab offset)
  std::string chx(const std::string& j) const {
    return slab ? "(" + j + " * T + lane + SLABCH)" : "(" + j + " * T + lane)";
  }
  // chunk-count specialisation of masked rows: inside a `switch` on the
  // row's number of fully valid team chunks KF (a compile-time constant in
  // each case), chunk predicates fold at compile time, chunks past the
  // boundary chunk vanish, and row reductions cover only NEV elements
  bool kf = false;
  std::string full_pred(const std::string& lim) const {
    return kf ? "(j < KF)" : "((j + 1) * T * E <= " + lim + ")";
  }
  std::string live_pred(const std::string& lim) const {
    return kf ? "(j <= KF)" : "(j * T * E < " + lim + ")";
  }
  std::string nev() const { return kf ? "NEV" : "NE"; }
  int rowred_index(int node) const {  // ordinal of a row reduction (cluster slot)
    int k = 0;
    for (int i = 0; i < node; ++i)
      if (I(i).live && I(i).cls == OpClass::ReduceRow) ++k;
    return k;
  }

  const Node& N(int i) const { return g.nodes[i]; }
  const NodeInfo& I(int i) const { return p.info[i]; }

  int nb(astitch_dtype d) const { return E * dtype_size(d); }

  // operand reference for element k (a C expression) in slot suffix sfx
  std::string ref(int i, const std::string& k, const std::string& sfx) const {
    const Node& nd = N(i);
    if (nd.type == NodeType::Const) return "k" + std::to_string(i);
    if (nd.type == NodeType::Bcast) {
      int a = nd.a;
      if (nd.axis == ASTITCH_AXIS_ROW) return "s" + std::to_string(a) + sfx;
      return colref(a, k);
    }
    switch (nd.kind) {
      case ASTITCH_FULL: return "v" + std::to_string(i) + sfx + "[" + k + "]";
      case ASTITCH_ROWVEC: return "s" + std::to_string(i) + sfx;
      case ASTITCH_COLVEC: return colref(i, k);
      default: return "0.f";
    }
  }
  std::string colref(int i, const std::string& k) const {
    if (I(i).post) return "cp" + std::to_string(i) + "[" + k + "]";
    return "c" + std::to_string(i) + "[" + k + "]";
  }
  // scalar reference (ROWVEC / SCALAR context)
  std::string sref(int i, const std::string& sfx) const {
    const Node& nd = N(i);
    if (nd.type == NodeType::Const) return "k" + std::to_string(i);
    return "s" + std::to_string(i) + sfx;
  }

  std::string unop(int op, const std::string& x) const {
    switch (op) {
      case ASTITCH_NEG: return "(-(" + x + "))";
      case ASTITCH_ABS: return "fabsf(" + x + ")";
      case ASTITCH_EXP: return "as::fexp(" + x + ")";
      case ASTITCH_LOG: return "as::flog(" + x + ")";
      case ASTITCH_TANH: return "as::ftanh(" + x + ")";
      case ASTITCH_ERF: return "as::ferf(" + x + ")";
      case ASTITCH_SQRT: return "as::sqrt_(" + x + ")";
      case ASTITCH_RSQRT: return "as::rsq(" + x + ")";
      case ASTITCH_RCP: return "as::rcp(" + x + ")";
      case ASTITCH_SIGMOID: return "as::fsigmoid(" + x + ")";
      case ASTITCH_GELU_TANH: return "as::gelu_tanh(" + x + ")";
      case ASTITCH_GELU_ERF: return "as::gelu_erf(" + x + ")";
      case ASTITCH_GELU_TANH_GRAD: return "as::gelu_tanh_grad(" + x + ")";
    }
    return x;
  }
  std::string binop(int op, int bnode, const std::string& a, const std::string& b) const {
    const Node& bn = N(bnode);
    bool bconst = bn.type == NodeType::Const;
    switch (op) {
      case ASTITCH_ADD: return "(" + a + " + " + b + ")";
      case ASTITCH_SUB: return "(" + a + " - " + b + ")";
      case ASTITCH_MUL: return "(" + a + " * " + b + ")";
      case ASTITCH_DIV:
        if (bconst) return "(" + a + " * " + flit(1.0 / bn.cval) + ")";
        return "as::fdiv(" + a + ", " + b + ")";
      case ASTITCH_MAX: return "as::nmax(" + a + ", " + b + ")";
      case ASTITCH_MIN: return "as::nmin(" + a + ", " + b + ")";
      case ASTITCH_POW:
        if (bconst && bn.cval == std::floor(bn.cval) && bn.cval >= 0 && bn.cval <= 8) {
          int n = static_cast<int>(bn.cval);
          if (n == 0) return "1.0f";
          std::string r = "(" + a;
          for (int t = 1; t < n; ++t) r += " * " + a;
          return r + ")";
        }
        return "as::fpow(" + a + ", " + b + ")";
    }
    return a;
  }

  // ------------------------------------------------------------ prologue
  void header(const std::string& name, bool cooperative_sync) {
    (void)cooperative_sync;
    o << "// generated by astitch codegen: " << template_name(m.tmpl) << " role " << role << "\n";
    if (p.desc.flags & ASTITCH_FLAG_DEBUG_BARRIER) o << "#define AS_BARRIER_TIMEOUT_NS 5000000000ULL\n";
    o << "#include \"astitch_device.cuh\"\n";
    o << "struct Params { const void* in[16]; void* out[16]; void* ws; long long rows; long long row_offset; int flags; void* xbuf; unsigned int gen; };\n";
    o << "extern \"C\" __global__ void __launch_bounds__(" << m.threads << ", " << m.blocks_per_sm << ") ";
    if (split) o << "__cluster_dims__(" << m.split << ", 1, 1) ";
    o << name << "(const Params p) {\n";
    // Programmatic dependent launch: wait for the preceding grid's memory
    // (no-op when launched without the attribute), then let the next stitched
    // kernel in the stream be scheduled while this one runs.
    o << "  asm volatile(\"griddepcontrol.wait;\" ::: \"memory\");\n";
    o << "  asm volatile(\"griddepcontrol.launch_dependents;\");\n";
    o << "  constexpr int T = " << T << ", V = " << V << ", E = " << E << ", NE = " << NE << ", RPB = " << RPB
      << ";\n";
    o << "  constexpr long long C = " << C << "LL;\n";
    o << "  constexpr long long CH = " << (C / E) << "LL;  // chunks per row\n";
    o << "  (void)V; (void)NE; (void)RPB; (void)CH;\n";
    o << "  const " << rowt() << " R = (" << rowt() << ")p.rows;\n";
    if (split) {
      // task splitting: the row's team is the whole cluster (K CTAs)
      o << "  const int lane = (int)as::cluster_rank() * (int)blockDim.x + (int)threadIdx.x;\n";
      o << "  const int team = 0;\n";
      o << "  const long long UNIT = as::cluster_idx(), NUNITS = as::cluster_count();\n";
      int nred = 0;
      for (size_t i = 0; i < g.nodes.size(); ++i)
        if (I(i).live && I(i).cls == OpClass::ReduceRow) ++nred;
      o << "  __shared__ float cl_slot[" << std::max(1, nred) << "];\n";
      o << "  __shared__ double cl_slot_d[" << std::max(1, nred) << "];\n";
    } else if (slab) {
      o << "  const int lane = threadIdx.x % T;\n";
      o << "  const int team = threadIdx.x / T;\n";
      o << "  constexpr int NSLAB = " << m.nslab << ";\n  constexpr long long SLABW = (long long)T * V * E;\n";
      o << "  const int SLAB = (int)(blockIdx.x % NSLAB);  // column slab of this CTA\n";
      o << "  const long long SLABOFF = (long long)SLAB * SLABW, SLABCH = (long long)SLAB * T * V;\n";
      o << "  (void)SLABOFF; (void)SLABCH;\n";
      o << "  const long long UNIT = blockIdx.x / NSLAB, NUNITS = gridDim.x / NSLAB;\n";
    } else {
      o << "  const int lane = threadIdx.x % T;\n";
      o << "  const int team = threadIdx.x / T;\n";
      o << "  const long long UNIT = blockIdx.x, NUNITS = gridDim.x;\n";
    }
    o << "  (void)lane; (void)team; (void)UNIT; (void)NUNITS;\n";
    if (T > 32) o << "  __shared__ float red_scratch[32];\n  __shared__ double red_scratch_d[32];\n";
    // constants
    for (size_t i = 0; i < g.nodes.size(); ++i)
      if (N(i).type == NodeType::Const && I(i).live)
        o << "  const float k" << i << " = " << flit(N(i).cval) << ";\n";
    if (g.lengths_node >= 0) {
      o << "  const int* __restrict__ Lp = (const int*)p.in[" << N(g.lengths_node).input_index << "];\n";
      o << "  constexpr long long RPS = " << g.rows_per_segment << "LL;\n";
    }
    if (ragged) {
      o << "  const int4* __restrict__ SG = (const int4*)p.in[" << N(g.segments_node).input_index << "];\n";
      o << "  constexpr int NSEG = " << g.nseg << ";\n";
    }
  }

  std::string col_expr(const std::string& j, const std::string& e) const {
    if (!tile_off.empty()) return "((" + j + " * T + lane) * E + " + e + " + " + tile_off + ")";
    return "((" + j + " * T + lane) * E + " + e + ")";
  }
  std::string tile_off;  // row_stream: column offset of the current tile ("" otherwise)

  // hoisted COLVEC values (pre-barrier): inputs and EW on them
  // in_loop: called inside the row loop (COLVEC operands re-read through L1
  // every row) vs. once per thread (hoisted in registers); the plan's
  // hoist_colvec decides which call site emits (a6 register budget).
  void emit_colvecs(bool in_loop) {
    if (in_loop == m.hoist_colvec) return;
    for (size_t i = 0; i < g.nodes.size(); ++i) {
      const Node& nd = N(i);
      if (!I(i).live || nd.kind != ASTITCH_COLVEC || I(i).post) continue;
      if (nd.type == NodeType::Reduce) continue;
      o << "  float c" << i << "[NE];\n";
      if (nd.type == NodeType::Input) {
        // chunk loads through L1 (the vector is re-read by every row team)
        std::string rt = "as::Raw<" + std::to_string(nb(nd.dtype)) + ">";
        o << "#pragma unroll\n  for (int j = 0; j < V; ++j) {\n";
        o << "    const long long ch = (long long)j * T + lane" << (tile_off.empty() ? "" : " + " + tile_off + " / E") << ";\n";
        o << "    const " << rt << " rc_ = (ch < CH) ? as::ldg_l1((const " << rt << "*)p.in[" << nd.input_index
          << "] + ch) : " << rt << "{};\n";
        o << "    as::Conv<" << dt_code(nd.dtype) << ", E>::unpack(rc_, c" << i << " + j * E);\n  }\n";
        continue;
      }
      o << "#pragma unroll\n  for (int j = 0; j < V; ++j)\n#pragma unroll\n  for (int e = 0; e < E; ++e) {\n";
      o << "    const int k = j * E + e; const long long col = " << col_expr("j", "e") << "; (void)col;\n";
      if (nd.type == NodeType::Unary) {
        o << "    c" << i << "[k] = " << unop(nd.sub, ref(nd.a, "k", "")) << ";\n";
      } else if (nd.type == NodeType::Binary) {
        o << "    c" << i << "[k] = " << binop(nd.sub, nd.b, ref(nd.a, "k", ""), ref(nd.b, "k", "")) << ";\n";
      }
      o << "  }\n";
    }
  }

  // ---- barrier levels ----------------------------------------------------
  // Sweep `cur_level` computes every FULL/ROWVEC op whose level equals it; a
  // column reduction accumulates in the sweep of its operand's level.
  int cur_level = 0;
  int phase_of(int u) const {
    if (I(u).cls == OpClass::ReduceCol) return I(N(u).a).level;
    return I(u).level;
  }
  // is node u evaluated in the current sweep?  Its own level's, plus the
  // later sweeps that recompute it instead of reading an HBM buffer (R22)
  bool runs_here(int u) const { return phase_of(u) == cur_level || ((I(u).remat_mask >> cur_level) & 1u); }
  int last_run(int u) const {
    int l = phase_of(u);
    for (int b = l + 1; b < 32; ++b)
      if ((I(u).remat_mask >> b) & 1u) l = b;
    return l;
  }

  // byte offset of the lo parts of post-barrier COLVEC values (R7c)
  long long colvals_lo() const {
    return static_cast<long long>(p.ws.colvals + (p.post_colvecs.size() + p.colreds.size()) * C * 4);
  }
  // COLVEC values finalised after earlier barriers (loaded from ws)
  void emit_post_colvec_loads() {
    for (size_t q = 0; q < p.post_colvecs.size(); ++q) {
      int i = p.post_colvecs[q];
      if (I(i).level > cur_level) continue;  // not computed yet
      o << "  float cp" << i << "[NE];\n";
      o << "  { const float* cv = (const float*)((char*)p.ws + " << p.ws.colvals << "LL) + " << q << "LL * C;\n";
      o << "#pragma unroll\n  for (int j = 0; j < V; ++j)\n#pragma unroll\n  for (int e = 0; e < E; ++e) {\n";
      o << "    const long long col = " << col_expr("j", "e") << ";\n";
      o << "    cp" << i << "[j * E + e] = (col < C) ? as::ld_cg(cv + col) : 0.f;\n  }}\n";
      if (pc(i)) {  // lo part (R7c)
        o << "  float cp" << i << "lo[NE];\n";
        o << "  { const float* cv = (const float*)((char*)p.ws + " << colvals_lo() << "LL) + " << q << "LL * C;\n";
        o << "#pragma unroll\n  for (int j = 0; j < V; ++j)\n#pragma unroll\n  for (int e = 0; e < E; ++e) {\n";
        o << "    const long long col = " << col_expr("j", "e") << ";\n";
        o << "    cp" << i << "lo[j * E + e] = (col < C) ? as::ld_cg(cv + col) : 0.f;\n  }}\n";
      }
    }
  }

  // ------------------------------------------------------------ loads
  // FULL inputs read in this phase (pre: live inputs; post: global FULL
  // buffers + FULL inputs consumed after the barrier)
  struct Stream {
    int node;         // node id
    bool ws_buf;      // read from the workspace global buffer (fp32)
    astitch_dtype dt;
    long long ws_off;
  };
  std::vector<Stream> streams;

  // does any consumer of node i run in the current sweep?
  bool node_used_in_phase(int i, bool post = false) const {
    for (int u : I(i).consumers) {
      if (!I(u).live) continue;
      // broadcasts are folded into their consumers: look through them
      if (N(u).type == NodeType::Bcast) {
        if (node_used_in_phase(u, post)) return true;
        continue;
      }
      if (runs_here(u)) return true;
    }
    return false;
  }

  // FULL bf16 / f16 input streams whose raw 32-bit words (two elements) are
  // kept next to their fp32 unpack: an ADD of such an element and an fp32
  // value is ONE sm_100a mixed-precision add (add.rn.f32.bf16 -> FHADD.BF16,
  // exact widening + one fp32 rounding: bitwise the same as unpack + FADD)
  // and the unpack of that element disappears when nothing else reads it.
  // Unmasked rows only (an absorbed mask rewrites invalid elements).
  std::vector<bool> rawok;
  void collect_streams(bool /*post*/) {
    streams.clear();
    rawok.assign(g.nodes.size(), false);
    for (int id : g.inputs) {
      const Node& nd = N(id);
      if (nd.kind == ASTITCH_FULL && I(id).live && node_used_in_phase(id, false)) {
        streams.push_back({id, false, nd.dtype, 0});  // re-read from HBM in later sweeps
        rawok[id] = !masked && (E % 2) == 0 && (nd.dtype == ASTITCH_BF16 || nd.dtype == ASTITCH_F16) &&
                    m.tmpl != Template::RowStream;
      }
    }
    for (size_t q = 0; q < p.global_fulls.size(); ++q) {
      int id = p.global_fulls[q];
      if (N(id).kind == ASTITCH_FULL && I(id).level < cur_level && node_used_in_phase(id, false))
        streams.push_back({id, true, ASTITCH_F32, static_cast<long long>(p.ws.globals + gbuf_offset(q))});
    }
  }
  size_t gbuf_offset(size_t q) const { return p.gbuf_off[q]; }

  std::string raw_t(const Stream& s) const { return "as::Raw<" + std::to_string(nb(s.dt)) + ">"; }

  void emit_stream_ptrs() {
    for (size_t s = 0; s < streams.size(); ++s) {
      const Stream& st = streams[s];
      if (st.ws_buf)
        o << "  const " << raw_t(st) << "* __restrict__ gs" << s << " = (const " << raw_t(st)
          << "*)((const char*)p.ws + " << st.ws_off << "LL);\n";
      else
        o << "  const " << raw_t(st) << "* __restrict__ gs" << s << " = (const " << raw_t(st) << "*)p.in["
          << N(st.node).input_index << "];\n";
    }
  }

  // emit: raw loads of all streams for row `row` into arrays r{s}{sfx}[V]
  void emit_loads(const std::string& row, const std::string& act, const std::string& lim,
                  const std::string& sfx, bool declare) {
    for (size_t s = 0; s < streams.size(); ++s) {
      const Stream& st = streams[s];
      if (declare) o << "    " << raw_t(st) << " r" << s << sfx << "[V];\n";
      o << "#pragma unroll\n    for (int j = 0; j < V; ++j) {\n";
      o << "      const long long c0 = " << chx("j") << " * E;\n";
      std::string cond = act;
      if (!exact || masked) cond += " && c0 < " + lim;
      o << "      if (" << cond << ") r" << s << sfx << "[j] = "
        << (st.ws_buf ? "as::ldg_cg(" : "as::ldg(") << "gs" << s << " + " << rowbase(row, lim)
        << " + " << chx("j") << ");\n";
      // chunks that are not loaded need no defined bits when the mask is
      // absorbed: the unpack step overwrites every invalid element with S
      if (!(absorb && !st.ws_buf)) o << "      else r" << s << sfx << "[j] = " << raw_t(st) << "{};\n";
      o << "    }\n";
    }
  }

  // unpack = convert (raw vectors -> fp32 registers) + mask (absorbed
  // substitute for invalid elements).  The early-unpack row loop emits the
  // convert step before the next row's prefetch is issued (the raw registers
  // die there, so the prefetch reuses them: no register copies) and the
  // mask step later, inside the (possibly KF-specialised) row block.
  bool early_unpack = false;   // convert already emitted for the current row
  void emit_unpack(const std::string& sfx, const std::string& lim = "") {
    if (!early_unpack) emit_unpack_convert(sfx, sfx);
    emit_unpack_mask(sfx, lim);
  }
  void emit_unpack_convert(const std::string& sfx, const std::string& src) {
    for (size_t s = 0; s < streams.size(); ++s) {
      const Stream& st = streams[s];
      int id = st.node;
      std::string dst = "v" + std::to_string(id) + sfx;
      int dt = st.ws_buf ? 0 : dt_code(st.dt);
      o << "    float " << dst << "[NE];\n";
      o << "#pragma unroll\n    for (int j = 0; j < V; ++j) as::Conv<" << dt << ", E>::unpack(r" << s << src
        << "[j], " << dst << " + j * E);\n";
      if (rawok.size() > static_cast<size_t>(id) && rawok[id]) {
        o << "    unsigned int w" << id << sfx << "[NE / 2];\n";
        o << "#pragma unroll\n    for (int j = 0; j < V; ++j)\n#pragma unroll\n    for (int q = 0; q < E / 2; ++q) w" << id << sfx
          << "[j * (E / 2) + q] = as::word(r" << s << src << "[j], q);\n";
      }
    }
  }
  void emit_unpack_mask(const std::string& sfx, const std::string& lim) {
    for (size_t s = 0; s < streams.size(); ++s) {
      const Stream& st = streams[s];
      int id = st.node;
      std::string dst = "v" + std::to_string(id) + sfx;
      if (absorb && masked && !st.ws_buf && !lim.empty()) {
        // mask absorption: invalid elements take the substitute value
        // d_ = elements of this lane's chunk that are valid (may be <= 0)
        o << "#pragma unroll\n    for (int j = 0; j < V; ++j) {\n      if (!" << full_pred(lim)
          << ") {\n        const int d_ = " << lim << " - (j * T + lane) * E;\n#pragma unroll\n"
          << "        for (int e = 0; e < E; ++e) if (e >= d_) " << dst << "[j * E + e] = " << fconst(absorb_sub)
          << ";\n      }\n    }\n";
      }
    }
  }

  // ---- mask absorption (reading R18) -------------------------------------
  // With a key-padding mask, choose a substitute S for the invalid input
  // elements such that, evaluating the subgraph on S, every row reduction
  // receives its identity (0 for SUM, -inf for RMAX).  Then reductions need no
  // per-element selects at all; only stores zero the invalid tail.  The
  // abstract value of each FULL node is found by evaluating the ops on S with
  // three sets of representative finite values for the per-row / per-column
  // scalars; a value is "known" when all three agree.  Softmax: S = -inf gives
  // max(-inf)=identity and exp(-inf - m) = 0 = identity of the sum.
  bool absorb = false;
  double absorb_sub = 0.0;
  std::vector<double> inval;      // known invalid-element value per node (NaN = unknown)
  std::vector<bool> inval_known;

  static std::string fconst(double v) {
    if (std::isinf(v)) return v > 0 ? "AS_INF" : "(-AS_INF)";
    return flit(v);
  }

  static double ap_un(int op, double x) {
    switch (op) {
      case ASTITCH_NEG: return -x;
      case ASTITCH_ABS: return std::fabs(x);
      case ASTITCH_EXP: return std::exp(x);
      case ASTITCH_LOG: return std::log(x);
      case ASTITCH_TANH: return std::tanh(x);
      case ASTITCH_ERF: return std::erf(x);
      case ASTITCH_SQRT: return std::sqrt(x);
      case ASTITCH_RSQRT: return 1.0 / std::sqrt(x);
      case ASTITCH_RCP: return 1.0 / x;
      case ASTITCH_SIGMOID: return 1.0 / (1.0 + std::exp(-x));
      case ASTITCH_GELU_TANH:
        return 0.5 * x * (1.0 + std::tanh(0.7978845608028654 * (x + 0.044715 * x * x * x)));
      case ASTITCH_GELU_ERF: return 0.5 * x * (1.0 + std::erf(x / std::sqrt(2.0)));
      default: return std::nan("");
    }
  }
  static double ap_bin(int op, double a, double b) {
    switch (op) {
      case ASTITCH_ADD: return a + b;
      case ASTITCH_SUB: return a - b;
      case ASTITCH_MUL: return a * b;
      case ASTITCH_DIV: return a / b;
      case ASTITCH_MAX: return (std::isnan(a) || std::isnan(b)) ? a + b : std::fmax(a, b);
      case ASTITCH_MIN: return (std::isnan(a) || std::isnan(b)) ? a + b : std::fmin(a, b);
      case ASTITCH_POW: return std::pow(a, b);
      default: return std::nan("");
    }
  }

  // shifted fp32 form of a precise row sum: rows wholly inside one warp (or
  // one thread), every column valid up to C (no masks: an invalid element
  // would have to be excluded from both the terms and the count)
  bool shifted_sum_ok() const {
    return !masked && !split && T <= 32 && (m.tmpl == Template::RowTeam || m.tmpl == Template::PackedTile);
  }
  // a FULL value whose (transitive) consumers include a reduction
  bool feeds_reduction(int i) const {
    for (int u : I(i).consumers) {
      if (!I(u).live) continue;
      const Node& un = N(u);
      if (un.type == NodeType::Reduce) return true;
      if (un.kind == ASTITCH_FULL && feeds_reduction(u)) return true;
    }
    return false;
  }
  // FULL light op computed over every chunk of an absorbed-mask row (no
  // live-chunk branch): its invalid elements take the known value inval[i]
  // whenever the row's scalars are finite, i.e. whenever the row has a valid
  // prefix; no reduction reads it (so fully-masked rows cannot leak a NaN into
  // a row scalar) and it is not buffered across a barrier
  bool light_unguarded(int i) const {
    if (!absorb || kf || !inval_known[i]) return false;
    const Node& nd = N(i);
    bool light = false;
    if (nd.type == NodeType::Binary)
      light = nd.sub == ASTITCH_ADD || nd.sub == ASTITCH_SUB || nd.sub == ASTITCH_MUL || nd.sub == ASTITCH_MAX ||
              nd.sub == ASTITCH_MIN || row_div(i) || (nd.sub == ASTITCH_DIV && N(nd.b).type == NodeType::Const);
    else if (nd.type == NodeType::Unary)
      light = nd.sub == ASTITCH_NEG || nd.sub == ASTITCH_ABS;
    return light && !feeds_reduction(i) && !I(i).global_full;
  }
  // FULL output whose invalid elements are known to be exactly 0 under the
  // absorbed mask: stored without per-element selects
  bool store_absorbed(int id) const {
    return absorb && masked && inval_known[id] && inval[id] == 0.0;
  }

  // abstract evaluation for substitute S; returns true if every row (and
  // column) reduction fed by FULL data receives its identity
  bool try_absorb(double S, std::vector<double> (&vals)[3]) {
    const int n = static_cast<int>(g.nodes.size());
    static const double reps[3][2] = {{1.75, -0.625}, {-2.375, 3.5}, {0.8125, 7.25}};
    for (int r = 0; r < 3; ++r) {
      vals[r].assign(n, std::nan(""));
      for (int i = 0; i < n; ++i) {
        const Node& nd = N(i);
        if (!I(i).live) continue;
        double v = std::nan("");
        if (nd.type == NodeType::Const) v = nd.cval;
        else if (nd.kind == ASTITCH_ROWVEC || nd.kind == ASTITCH_COLVEC) v = reps[r][(nd.kind == ASTITCH_COLVEC) ? 1 : 0] + 0.03125 * (i % 7);
        else if (nd.type == NodeType::Input && nd.kind == ASTITCH_FULL) v = S;
        else if (nd.type == NodeType::Bcast) v = vals[r][nd.a];
        else if (nd.type == NodeType::Unary) v = ap_un(nd.sub, vals[r][nd.a]);
        else if (nd.type == NodeType::Binary) v = ap_bin(nd.sub, vals[r][nd.a], vals[r][nd.b]);
        vals[r][i] = v;
      }
    }
    for (int i = 0; i < n; ++i) {
      const Node& nd = N(i);
      if (!I(i).live || nd.type != NodeType::Reduce) continue;
      double ident = nd.sub == ASTITCH_SUM ? 0.0 : -INFINITY;
      for (int r = 0; r < 3; ++r)
        if (!(vals[r][nd.a] == ident)) return false;
    }
    return true;
  }

  void compute_absorb() {
    absorb = false;
    if (!masked) return;
    for (size_t k = 0; k < g.outputs.size(); ++k)
      if (N(g.outputs[k]).kind != ASTITCH_FULL) return;  // fully-masked rows would expose S
    bool any_reduce = false;
    for (size_t i = 0; i < g.nodes.size(); ++i)
      if (I(i).live && N(i).type == NodeType::Reduce) any_reduce = true;
    if (!any_reduce) return;
    // values buffered in HBM across a barrier are re-read for the valid
    // prefix only (chunks past it load as 0), which is not S: keep selects
    if (!p.global_fulls.empty()) return;
    const double cands[3] = {-HUGE_VAL, 0.0, HUGE_VAL};
    for (double S : cands) {
      std::vector<double> vals[3];
      if (!try_absorb(S, vals)) continue;
      absorb = true;
      absorb_sub = S;
      const int n = static_cast<int>(g.nodes.size());
      inval.assign(n, std::nan(""));
      inval_known.assign(n, false);
      for (int i = 0; i < n; ++i) {
        if (vals[0][i] == vals[1][i] && vals[1][i] == vals[2][i]) {
          inval[i] = vals[0][i];
          inval_known[i] = true;
        }
      }
      return;
    }
  }

  // ------------------------------------------------------------ per-row body
  // Emits the ops of one phase for one row slot.  lim = valid column bound.
  void emit_body(bool post, const std::string& sfx, const std::string& row, const std::string& act,
                 const std::string& lim) {
    const bool check = masked || !exact;
    for (size_t ii = 0; ii < g.nodes.size(); ++ii) {
      int i = static_cast<int>(ii);
      const Node& nd = N(i);
      const NodeInfo& in = I(i);
      if (!in.live || nd.type == NodeType::Input || nd.type == NodeType::Const) continue;
      if (nd.type == NodeType::Bcast) continue;  // folded into operand references
      (void)post;
      // only the ops of this sweep's level; a column reduction accumulates in
      // the sweep of its operand (earlier levels come from HBM buffers)
      if (!runs_here(i)) continue;
      // COLVEC values: level 0 hoisted per lane, later ones finalised per column
      if (nd.kind == ASTITCH_COLVEC && !(nd.type == NodeType::Reduce && nd.axis == ASTITCH_AXIS_COL)) continue;
      std::string id = std::to_string(i);
      if (nd.type == NodeType::Reduce && nd.axis == ASTITCH_AXIS_COL) {
        bool mx = nd.sub == ASTITCH_RMAX;
        if (pc(i)) {  // fp64 accumulation of a cancellation-prone column sum (R7c)
          std::string okc = act;
          if (check && !absorb) okc += " && " + col_expr("(k / E)", "(k % E)") + " < " + lim;
          o << "#pragma unroll\n    for (int k = 0; k < NE; ++k) acc" << id << "[k] += (" << okc << ") ? (double)"
            << ref(nd.a, "k", sfx) << " : 0.0;\n";
          continue;
        }
        if (!mx && (E % 2) == 0 && !(check && !absorb)) {
          // paired accumulation (FADD2); inactive rows contribute zeros
          o << "#pragma unroll\n    for (int k = 0; k < NE; k += 2) {\n";
          o << "      const as::f2 a_ = as::add2(as::f2{acc" << id << "[k], acc" << id << "[k + 1]}, " << act << " ? "
            << ref2(nd.a, sfx) << " : as::bc2(0.f));\n";
          o << "      acc" << id << "[k] = a_.x; acc" << id << "[k + 1] = a_.y;\n    }\n";
          continue;
        }
        o << "#pragma unroll\n    for (int k = 0; k < NE; ++k) {\n";
        std::string val = ref(nd.a, "k", sfx);
        std::string okc = act;
        if (check && !absorb) okc += " && " + col_expr("(k / E)", "(k % E)") + " < " + lim;
        if (mx) o << "      if (" << okc << ") acc" << id << "[k] = as::nmax(acc" << id << "[k], " << val << ");\n";
        else o << "      if (" << okc << ") acc" << id << "[k] += " << val << ";\n";
        o << "    }\n";
        continue;
      }
      if (nd.type == NodeType::Reduce && precise[i] && shifted_sum_ok()) {
        // cancellation-prone row sum, shifted form: sum the row's values
        // minus its first value x0 (team-uniform) in fp32, then
        // d = C*x0 + sum(v - x0) in fp64 once per row.  The fp32 terms are of
        // the size of the row's spread, not of its mean, so the mean is
        // accurate to ~log2(C) ulps of the spread (as the fp64 tree, reading
        // R7b) without an F2F + DADD per element.
        const std::string v0 = ref(nd.a, "0", sfx);
        o << "    double d" << id << sfx << ";\n    {\n";
        o << "      const float x0_ = " << (T == 1 ? v0 : "__shfl_sync(0xffffffffu, " + v0 + ", 0, T)") << ";\n";
        o << "      float t_[NE];\n";
        if (check) {
          o << "#pragma unroll\n      for (int k = 0; k < NE; ++k) t_[k] = (" << col_expr("(k / E)", "(k % E)") << " < " << lim
            << ") ? " << ref(nd.a, "k", sfx) << " - x0_ : 0.f;\n";
        } else if ((NE % 2) == 0) {
          o << "#pragma unroll\n      for (int k = 0; k < NE; k += 2) { const as::f2 r_ = as::sub2(" << ref2(nd.a, sfx)
            << ", as::bc2(x0_)); t_[k] = r_.x; t_[k + 1] = r_.y; }\n";
        } else {
          o << "#pragma unroll\n      for (int k = 0; k < NE; ++k) t_[k] = " << ref(nd.a, "k", sfx) << " - x0_;\n";
        }
        o << "      float r_ = as::TreeSum<NE>::reduce(t_);\n";
        if (T > 1) o << "      r_ = as::team_sum<T>(r_);\n";
        o << "      d" << id << sfx << " = fma((double)x0_, (double)C, (double)r_);\n    }\n";
        emit_split(id, sfx);
        continue;
      }
      if (nd.type == NodeType::Reduce && precise[i]) {  // cancellation-prone row sum: fp64
        o << "    double d" << id << sfx << ";\n    {\n      float t_[NE];\n";
        o << "#pragma unroll\n      for (int k = 0; k < NE; ++k) t_[k] = ";
        if (check && !absorb) o << "(" << col_expr("(k / E)", "(k % E)") << " < " << lim << ") ? " << ref(nd.a, "k", sfx)
                     << " : 0.f;\n";
        else o << ref(nd.a, "k", sfx) << ";\n";
        o << "      double r_ = as::TreeD<" << nev() << ">::reduce(t_);\n";
        if (T <= 32) o << "      r_ = as::team_sum_d<T>(r_);\n";
        else if (split)
          o << "      r_ = as::cluster_team_sum_d<" << m.threads << ", " << m.split << ">(r_, red_scratch_d, &cl_slot_d["
            << rowred_index(i) << "]);\n";
        else o << "      r_ = as::block_team_sum_d<T>(r_, red_scratch_d);\n";
        o << "      d" << id << sfx << " = r_;\n    }\n";
        emit_split(id, sfx);
        continue;
      }
      if (nd.type == NodeType::Reduce) {  // row reduce: regional (team)
        bool mx = nd.sub == ASTITCH_RMAX;
        std::string ident = mx ? "-AS_INF" : "0.f";
        // max(c * x) == c * max(x) exactly for c > 0 (rounding is monotonic):
        // reduce the unscaled operand and scale the row scalar once
        int src = nd.a;
        std::string post_scale;
        {
          const Node& sn = N(src);
          if (mx && sn.type == NodeType::Binary && sn.sub == ASTITCH_MUL && sn.kind == ASTITCH_FULL &&
              runs_here(src)) {
            if (N(sn.b).type == NodeType::Const && N(sn.b).cval > 0) { post_scale = flit(N(sn.b).cval); src = sn.a; }
            else if (N(sn.a).type == NodeType::Const && N(sn.a).cval > 0) { post_scale = flit(N(sn.a).cval); src = sn.b; }
          }
        }
        o << "    float s" << id << sfx << ";\n    {\n      float t_[NE];\n";
        if (absorb) {
          // mask absorbed: invalid elements already hold the identity
          o << "#pragma unroll\n      for (int k = 0; k < NE; ++k) t_[k] = " << ref(src, "k", sfx) << ";\n";
        } else if (masked) {
          // chunk-uniform mask handling: a chunk index j covers columns
          // [j*T*E, (j+1)*T*E) across the team, so "fully valid" is uniform
          // over the team and only the boundary chunk pays per-element selects
          o << "#pragma unroll\n      for (int j = 0; j < V; ++j) {\n";
          o << "        if (" << full_pred(lim) << ") {\n#pragma unroll\n          for (int e = 0; e < E; ++e) { const int k = j * E + e; t_[k] = " << ref(src, "k", sfx) << "; }\n";
          o << "        } else {\n#pragma unroll\n          for (int e = 0; e < E; ++e) { const int k = j * E + e; t_[k] = ("
            << col_expr("j", "e") << " < " << lim << ") ? " << ref(src, "k", sfx) << " : " << ident << "; }\n        }\n      }\n";
        } else {
          o << "#pragma unroll\n      for (int k = 0; k < NE; ++k) t_[k] = ";
          if (check) o << "(" << col_expr("(k / E)", "(k % E)") << " < " << lim << ") ? " << ref(src, "k", sfx)
                       << " : " << ident << ";\n";
          else o << ref(src, "k", sfx) << ";\n";
        }
        if (mx) o << "      float r_ = as::Tree<" << nev() << ", true>::reduce(t_);\n";
        else o << "      float r_ = as::TreeSum<" << nev() << ">::reduce(t_);\n";
        if (T <= 32) o << "      r_ = as::team_" << (mx ? "max" : "sum") << "<T>(r_);\n";
        else if (split)
          o << "      r_ = as::cluster_team_reduce<" << m.threads << ", " << m.split << ", " << (mx ? "true" : "false")
            << ">(r_, red_scratch, &cl_slot[" << rowred_index(i) << "]);\n";
        else o << "      r_ = as::block_team_reduce<T, " << (mx ? "true" : "false") << ">(r_, red_scratch);\n";
        if (!post_scale.empty()) o << "      r_ = r_ * " << post_scale << ";\n";
        o << "      s" << id << sfx << " = r_;\n    }\n";
        continue;
      }
      if (nd.kind == ASTITCH_ROWVEC && precise[i]) {
        o << "    const double d" << id << sfx << " = ";
        if (nd.type == NodeType::Unary) o << (nd.sub == ASTITCH_NEG ? "-" : "fabs") << "(" << dref(nd.a, sfx) << ");\n";
        else o << dbinop(nd.sub, nd.a, nd.b, sfx) << ";\n";
        emit_split(id, sfx);
        continue;
      }
      if (nd.kind == ASTITCH_ROWVEC) {
        if (nd.type == NodeType::Unary)
          o << "    const float s" << id << sfx << " = " << unop(nd.sub, sref(nd.a, sfx)) << ";\n";
        else
          o << "    const float s" << id << sfx << " = "
            << binop(nd.sub, nd.b, sref(nd.a, sfx), sref(nd.b, sfx)) << ";\n";
        continue;
      }
      if (nd.kind == ASTITCH_FULL) {
        const bool paired = (E % 2) == 0;
        std::string expr = full_expr(i, sfx);
        std::string body;  // statement computing element(s) at index k
        if (paired) {
          body = "{ const as::f2 r_ = " + full_expr2(i, sfx) + "; v" + id + sfx + "[k] = r_.x; v" + id + sfx +
                 "[k + 1] = r_.y; }";
        } else {
          body = "v" + id + sfx + "[k] = " + expr + ";";
        }
        const std::string estep = paired ? "e += 2" : "++e";
        if (row_div(i)) o << "    " << row_div_decl(i, sfx) << "\n";
        o << "    float v" << id << sfx << "[NE];\n";
        if (masked && light_unguarded(i)) {
          // absorbed mask, light op that no reduction reads: past the valid
          // length it computes its known invalid value anyway, cheaper than a
          // branch per chunk plus a zero fill
          o << "#pragma unroll\n    for (int k = 0; k < NE; k += " << (paired ? 2 : 1) << ") " << body << "\n";
        } else if (masked) {
          // chunks wholly past the valid length are not computed (team-uniform branch)
          o << "#pragma unroll\n    for (int j = 0; j < V; ++j) {\n      if (" << live_pred(lim) << ") {\n";
          o << "#pragma unroll\n        for (int e = 0; e < E; " << estep << ") { const int k = j * E + e; " << body
            << " }\n";
          std::string skip = (absorb && inval_known[i]) ? fconst(inval[i]) : "0.f";
          o << "      } else {\n#pragma unroll\n        for (int e = 0; e < E; ++e) v" << id << sfx
            << "[j * E + e] = " << skip << ";\n      }\n    }\n";
        } else {
          o << "#pragma unroll\n    for (int k = 0; k < NE; k += " << (paired ? 2 : 1) << ") " << body << "\n";
        }
        continue;
      }
    }
  }

  // ---- double-float handling of cancellation-prone row scalars (reading R7b)
  // A row sum whose value (through light per-row ops) is broadcast into a FULL
  // add/sub (a mean that is subtracted) is reduced in fp64 and applied as an
  // fp32 hi + lo pair, so x - mean is accurate to fp32 even when the row's
  // spread is small relative to its mean.
  std::vector<bool> precise;

  void compute_precise() {
    const int n = static_cast<int>(g.nodes.size());
    precise.assign(n, false);
    std::vector<bool> need(n, false);
    for (int b = 0; b < n; ++b) {
      const Node& bn = N(b);
      if (!I(b).live || bn.type != NodeType::Bcast || bn.axis != ASTITCH_AXIS_ROW) continue;
      for (int u : I(b).consumers) {
        const Node& un = N(u);
        if (I(u).live && un.type == NodeType::Binary && un.kind == ASTITCH_FULL &&
            (un.sub == ASTITCH_ADD || un.sub == ASTITCH_SUB))
          need[bn.a] = true;
      }
    }
    for (int i = n - 1; i >= 0; --i) {  // backward closure through light per-row ops
      if (!need[i]) continue;
      const Node& nd = N(i);
      bool light = (nd.type == NodeType::Binary && nd.sub != ASTITCH_POW) ||
                   (nd.type == NodeType::Unary && (nd.sub == ASTITCH_NEG || nd.sub == ASTITCH_ABS));
      if (nd.kind != ASTITCH_ROWVEC) continue;
      if (nd.type == NodeType::Reduce && nd.sub == ASTITCH_SUM && nd.axis == ASTITCH_AXIS_ROW) precise[i] = true;
      if (light) {
        precise[i] = true;
        if (nd.a >= 0 && N(nd.a).kind == ASTITCH_ROWVEC) need[nd.a] = true;
        if (nd.b >= 0 && N(nd.b).kind == ASTITCH_ROWVEC) need[nd.b] = true;
      }
    }
    // row values read after a grid barrier (FORCE_GLOBAL) stay precise: the
    // ROWVEC buffer carries the lo part next to the value (R floats later)
    for (int i = 0; i < n; ++i)
      if ((I(i).post || I(i).global_full) && N(i).kind != ASTITCH_ROWVEC) precise[i] = false;
  }
  void emit_split(const std::string& id, const std::string& sfx) {
    o << "    const float s" << id << sfx << " = (float)d" << id << sfx << ";\n";
    o << "    const float s" << id << sfx << "lo = (float)(d" << id << sfx << " - (double)s" << id << sfx << ");\n";
  }
  std::string dref(int i, const std::string& sfx) const {
    const Node& nd = N(i);
    if (nd.type == NodeType::Const) {
      char buf[64];
      snprintf(buf, sizeof(buf), "%a", nd.cval);
      return std::string("(") + buf + ")";
    }
    if (precise[i]) return "d" + std::to_string(i) + sfx;
    return "(double)s" + std::to_string(i) + sfx;
  }
  std::string dbinop(int op, int a, int b, const std::string& sfx) const {
    std::string x = dref(a, sfx), y = dref(b, sfx);
    switch (op) {
      case ASTITCH_ADD: return "(" + x + " + " + y + ")";
      case ASTITCH_SUB: return "(" + x + " - " + y + ")";
      case ASTITCH_MUL: return "(" + x + " * " + y + ")";
      case ASTITCH_DIV:
        if (N(b).type == NodeType::Const) {  // fp64 reciprocal: error ~1e-16, no DDIV
          char buf[64];
          snprintf(buf, sizeof(buf), "%a", 1.0 / N(b).cval);
          return "(" + x + " * " + buf + ")";
        }
        return "(" + x + " / " + y + ")";
      case ASTITCH_MAX: return "as::dmaxn(" + x + ", " + y + ")";
      case ASTITCH_MIN: return "as::dminn(" + x + ", " + y + ")";
    }
    return x;
  }
  // ---- paired (f32x2) emission: FADD2 / FMUL2 / FFMA2 on element pairs ----
  std::string ref2(int i, const std::string& sfx) const {
    const Node& nd = N(i);
    if (nd.type == NodeType::Const) return "as::bc2(k" + std::to_string(i) + ")";
    if (nd.type == NodeType::Bcast && nd.axis == ASTITCH_AXIS_ROW) return "as::bc2(s" + std::to_string(nd.a) + sfx + ")";
    if (nd.kind == ASTITCH_ROWVEC) return "as::bc2(s" + std::to_string(i) + sfx + ")";
    return "as::f2{" + ref(i, "k", sfx) + ", " + ref(i, "k + 1", sfx) + "}";
  }
  std::string unop2(int op, const std::string& x) const {
    switch (op) {
      case ASTITCH_NEG: return "as::neg2(" + x + ")";
      case ASTITCH_ABS: return "as::abs2(" + x + ")";
      case ASTITCH_EXP: return "as::fexp2(" + x + ")";
      case ASTITCH_LOG: return "as::flog2_(" + x + ")";
      case ASTITCH_TANH: return "as::ftanh2(" + x + ")";
      case ASTITCH_ERF: return "as::ferf2(" + x + ")";
      case ASTITCH_SQRT: return "as::sqrt2_(" + x + ")";
      case ASTITCH_RSQRT: return "as::rsq2(" + x + ")";
      case ASTITCH_RCP: return "as::rcp_2(" + x + ")";
      case ASTITCH_SIGMOID: return "as::fsigmoid2(" + x + ")";
      case ASTITCH_GELU_TANH: return "as::gelu_tanh2(" + x + ")";
      case ASTITCH_GELU_ERF: return "as::gelu_erf2(" + x + ")";
      case ASTITCH_GELU_TANH_GRAD: return "as::gelu_tanh_grad2(" + x + ")";
    }
    return x;
  }
  std::string binop2(int op, int bnode, const std::string& a, const std::string& b) const {
    const Node& bn = N(bnode);
    bool bconst = bn.type == NodeType::Const;
    switch (op) {
      case ASTITCH_ADD: return "as::add2(" + a + ", " + b + ")";
      case ASTITCH_SUB: return "as::sub2(" + a + ", " + b + ")";
      case ASTITCH_MUL: return "as::mul2(" + a + ", " + b + ")";
      case ASTITCH_DIV:
        if (bconst) return "as::mul2(" + a + ", as::bc2(" + flit(1.0 / bn.cval) + "))";
        return "as::fdiv2(" + a + ", " + b + ")";
      case ASTITCH_MAX: return "as::max2(" + a + ", " + b + ")";
      case ASTITCH_MIN: return "as::min2(" + a + ", " + b + ")";
      case ASTITCH_POW:
        if (bconst && bn.cval == std::floor(bn.cval) && bn.cval >= 0 && bn.cval <= 8) {
          int n = static_cast<int>(bn.cval);
          if (n == 0) return "as::bc2(1.0f)";
          std::string r = a;
          for (int t = 1; t < n; ++t) r = "as::mul2(" + r + ", " + a + ")";
          return r;
        }
        return "as::fpow2(" + a + ", " + b + ")";
    }
    return a;
  }
  std::string full_expr2(int i, const std::string& sfx) const {
    const Node& nd = N(i);
    if (nd.type == NodeType::Unary && nd.sub == ASTITCH_EXP) {
      const Node& a = N(nd.a);
      if (a.type == NodeType::Binary && a.sub == ASTITCH_SUB && a.kind == ASTITCH_FULL) {
        const Node& b = N(a.b);
        bool b_row = b.type == NodeType::Bcast && b.axis == ASTITCH_AXIS_ROW && !precise[b.a];
        bool b_const = b.type == NodeType::Const;
        if (b_row || b_const) {
          std::string bs = b_row ? ("s" + std::to_string(b.a) + sfx) : ("k" + std::to_string(a.b));
          std::string nbs = "as::bc2(-(" + bs + ") * 1.4426950408889634f)";
          const Node& x = N(a.a);
          if (x.type == NodeType::Binary && x.sub == ASTITCH_MUL && x.kind == ASTITCH_FULL &&
              runs_here(a.a)) {
            if (N(x.b).type == NodeType::Const)
              return "as::ex2_2(as::fma2(" + ref2(x.a, sfx) + ", as::bc2(" +
                     flit(N(x.b).cval * 1.4426950408889634) + "), " + nbs + "))";
            if (N(x.a).type == NodeType::Const)
              return "as::ex2_2(as::fma2(" + ref2(x.b, sfx) + ", as::bc2(" +
                     flit(N(x.a).cval * 1.4426950408889634) + "), " + nbs + "))";
          }
          return "as::ex2_2(as::fma2(" + ref2(a.a, sfx) + ", as::bc2(1.4426950408889634f), " + nbs + "))";
        }
      }
    }
    if (nd.type == NodeType::Unary) return unop2(nd.sub, ref2(nd.a, sfx));
    if (row_div(i)) return "as::mul2(" + ref2(nd.a, sfx) + ", as::bc2(rq" + std::to_string(i) + sfx + "))";
    if (nd.type == NodeType::Binary && nd.sub == ASTITCH_ADD && !precise_bcast(nd.a) && !precise_bcast(nd.b) &&
        !precise_bcast_col(nd.a) && !precise_bcast_col(nd.b)) {
      const std::string hf = N(nd.a).dtype == ASTITCH_F16 ? "f16" : "bf16";
      if (raw_operand(nd.a))
        return "as::hadd2_" + hf + "(w" + std::to_string(nd.a) + sfx + "[k / 2], " + ref2(nd.b, sfx) + ")";
      if (raw_operand(nd.b))
        return "as::hadd2_" + std::string(N(nd.b).dtype == ASTITCH_F16 ? "f16" : "bf16") + "(w" + std::to_string(nd.b) +
               sfx + "[k / 2], " + ref2(nd.a, sfx) + ")";
    }
    std::string a = ref2(nd.a, sfx), b = ref2(nd.b, sfx);
    // hi + lo operands (R7b row means, R7c column means): (a_hi ± b_hi) + (a_lo ± b_lo),
    // every lo part that exists (both operands may carry one, e.g. m - m)
    if (nd.type == NodeType::Binary && (nd.sub == ASTITCH_ADD || nd.sub == ASTITCH_SUB)) {
      auto lo2 = [&](int v) -> std::string {
        if (precise_bcast_col(v)) return "as::f2{" + col_lo(v, "k") + ", " + col_lo(v, "k + 1") + "}";
        if (precise_bcast(v)) return "as::bc2(s" + std::to_string(N(v).a) + sfx + "lo)";
        return "";
      };
      const std::string la = lo2(nd.a), lb = lo2(nd.b);
      if (!la.empty() || !lb.empty()) {
        const bool sub = nd.sub == ASTITCH_SUB;
        std::string hi = std::string(sub ? "as::sub2(" : "as::add2(") + a + ", " + b + ")";
        std::string lo;
        if (!la.empty() && !lb.empty()) lo = std::string(sub ? "as::sub2(" : "as::add2(") + la + ", " + lb + ")";
        else if (!la.empty()) lo = la;
        else return std::string(sub ? "as::sub2(" : "as::add2(") + hi + ", " + lb + ")";
        return "as::add2(" + hi + ", " + lo + ")";
      }
    }
    return binop2(nd.sub, nd.b, a, b);
  }

  bool raw_operand(int v) const {
    return v >= 0 && static_cast<size_t>(v) < rawok.size() && rawok[v] && N(v).type == NodeType::Input &&
           N(v).kind == ASTITCH_FULL;
  }
  // Per-element expression of a FULL op.  Peephole (local stitching lets the
  // whole chain sit in registers, so it can be re-associated once):
  //   exp((k*x) - s)  ->  ex2(fma(x, k*log2e, -s*log2e))   (s: row scalar / const)
  // which is one FFMA + one MUFU.EX2 per element; -s*log2e is row-uniform.
  std::string full_expr(int i, const std::string& sfx) const {
    const Node& nd = N(i);
    if (nd.type == NodeType::Unary && nd.sub == ASTITCH_EXP) {
      const Node& a = N(nd.a);
      if (a.type == NodeType::Binary && a.sub == ASTITCH_SUB && a.kind == ASTITCH_FULL) {
        const Node& b = N(a.b);
        bool b_row = b.type == NodeType::Bcast && b.axis == ASTITCH_AXIS_ROW && !precise[b.a];
        bool b_const = b.type == NodeType::Const;
        if (b_row || b_const) {
          std::string bs = b_row ? ("s" + std::to_string(b.a) + sfx) : ("k" + std::to_string(a.b));
          std::string nbs = "(-(" + bs + ") * 1.4426950408889634f)";
          const Node& x = N(a.a);
          if (x.type == NodeType::Binary && x.sub == ASTITCH_MUL && x.kind == ASTITCH_FULL &&
              runs_here(a.a)) {
            if (N(x.b).type == NodeType::Const)
              return "as::ex2(fmaf(" + ref(x.a, "k", sfx) + ", " + flit(N(x.b).cval * 1.4426950408889634) + ", " +
                     nbs + "))";
            if (N(x.a).type == NodeType::Const)
              return "as::ex2(fmaf(" + ref(x.b, "k", sfx) + ", " + flit(N(x.a).cval * 1.4426950408889634) + ", " +
                     nbs + "))";
          }
          return "as::ex2(fmaf(" + ref(a.a, "k", sfx) + ", 1.4426950408889634f, " + nbs + "))";
        }
      }
    }
    if (nd.type == NodeType::Unary) return unop(nd.sub, ref(nd.a, "k", sfx));
    if (row_div(i)) return "(" + ref(nd.a, "k", sfx) + " * rq" + std::to_string(i) + sfx + ")";
    return full_binop(nd, sfx);
  }

  // x / bcast_row(s): multiply by the row's reciprocal, computed once per
  // row (rq<i>) instead of a MUFU.RCP per element (same arithmetic as fdiv)
  bool row_div(int i) const {
    const Node& nd = N(i);
    if (nd.type != NodeType::Binary || nd.sub != ASTITCH_DIV || nd.kind != ASTITCH_FULL) return false;
    const Node& b = N(nd.b);
    return b.type == NodeType::Bcast && b.axis == ASTITCH_AXIS_ROW && !precise[b.a];
  }
  std::string row_div_decl(int i, const std::string& sfx) const {
    return "const float rq" + std::to_string(i) + sfx + " = as::rcp(s" + std::to_string(N(N(i).b).a) + sfx + ");";
  }
  bool precise_bcast(int v) const {
    const Node& nd = N(v);
    return nd.type == NodeType::Bcast && nd.axis == ASTITCH_AXIS_ROW && precise[nd.a];
  }
  // ---- cancellation-prone column values (reading R7c): fp64 column sums,
  // fp64 per-column chain, applied to FULL add/sub as an fp32 hi + lo pair.
  // Unsharded stitched kernel only (the sharded / chunked roles combine fp32
  // totals across launches and keep the plain fp32 path).
  bool pc(int i) const { return role == ROLE_MAIN && I(i).precise_col; }
  int nslots() const { return static_cast<int>(p.colreds.size()) + p.n_precise_colreds; }
  int lo_slot(int q) const {  // partial slot of the lo part of precise column sum q
    int k = static_cast<int>(p.colreds.size());
    for (int j = 0; j < q; ++j)
      if (I(p.colreds[j]).precise_col) ++k;
    return k;
  }
  bool any_pc() const {
    for (int id : p.colreds)
      if (pc(id)) return true;
    return false;
  }
  // FULL operand v = bcast_col(c) of a precise post-barrier column value
  bool precise_bcast_col(int v) const {
    const Node& nd = N(v);
    return nd.type == NodeType::Bcast && nd.axis == ASTITCH_AXIS_COL && pc(nd.a) && I(nd.a).post;
  }
  std::string col_lo(int v, const std::string& k) const { return "cp" + std::to_string(N(v).a) + "lo[" + k + "]"; }
  std::string full_binop(const Node& nd, const std::string& sfx) const {
    std::string a = ref(nd.a, "k", sfx), b = ref(nd.b, "k", sfx);
    if (nd.sub == ASTITCH_ADD || nd.sub == ASTITCH_SUB) {  // hi + lo operands (R7b / R7c)
      auto lo1 = [&](int v, const std::string& r) -> std::string {
        if (precise_bcast_col(v)) return col_lo(v, "k");
        if (precise_bcast(v)) return r + "lo";
        return "";
      };
      const std::string la = lo1(nd.a, a), lb = lo1(nd.b, b);
      if (!la.empty() || !lb.empty()) {
        const std::string op = nd.sub == ASTITCH_SUB ? " - " : " + ";
        std::string lo;
        if (!la.empty() && !lb.empty()) lo = "(" + la + op + lb + ")";
        else if (!la.empty()) lo = la;
        else return "((" + a + op + b + ")" + op + lb + ")";
        return "((" + a + op + b + ") + " + lo + ")";
      }
    }
    return binop(nd.sub, nd.b, a, b);
  }

  void emit_rowvec_inputs(bool post, const std::string& sfx, const std::string& row, const std::string& act) {
    for (int id : g.inputs) {
      const Node& nd = N(id);
      if (nd.kind != ASTITCH_ROWVEC || !I(id).live || !node_used_in_phase(id, post)) continue;
      o << "    const float s" << id << sfx << " = (" << act << ") ? as::ld_scalar<" << dt_code(nd.dtype)
        << ">(p.in[" << nd.input_index << "], " << row << ") : 0.f;\n";
    }
    if (cur_level > 0) {  // earlier-level ROWVEC values: global row buffers
      for (size_t q = 0; q < p.global_fulls.size(); ++q) {
        int id = p.global_fulls[q];
        if (N(id).kind != ASTITCH_ROWVEC || I(id).level >= cur_level || !node_used_in_phase(id, true)) continue;
        o << "    const float s" << id << sfx << " = (" << act << ") ? as::ld_cg((const float*)((const char*)p.ws + "
          << (p.ws.globals + gbuf_offset(q)) << "LL) + " << row << ") : 0.f;\n";
        if (precise[id]) {  // R7b across the barrier: hi + lo
          o << "    const float s" << id << sfx << "lo = (" << act << ") ? as::ld_cg((const float*)((const char*)p.ws + "
            << (p.ws.globals + gbuf_offset(q)) << "LL) + " << p.desc.rows << "LL + " << row << ") : 0.f;\n";
          o << "    const double d" << id << sfx << " = (double)s" << id << sfx << " + (double)s" << id << sfx << "lo;\n";
        }
      }
    }
  }

  // stores of one phase's outputs (+ global buffers written in sweep 1)
  void emit_stores(bool post, const std::string& sfx, const std::string& row, const std::string& act,
                   const std::string& lim) {
    const bool check = masked || !exact;
    for (size_t k = 0; k < g.outputs.size(); ++k) {
      int id = g.outputs[k];
      const Node& nd = N(id);
      if (I(id).level != cur_level) continue;
      astitch_dtype dt = g.output_dtypes[k];
      if (nd.kind == ASTITCH_FULL) {
        std::string rt = "as::Raw<" + std::to_string(nb(dt)) + ">";
        o << "    if (" << act << ") {\n      " << rt << "* __restrict__ op_ = (" << rt << "*)p.out[" << k
          << "] + " << rowbase(row, lim) << ";\n";
        std::string val = ref(id, "(j * E + e)", sfx);
        const std::string cguard = exact ? "" : "        if ((long long)" + chx("j") + " < CH)\n";
        if (store_absorbed(id) && !ragged) {
          // every invalid element already holds 0 (absorbed mask): no
          // per-element selects; fully-masked rows (the only ones whose row
          // scalars may be non-finite) store zeros on a team-uniform branch
          o << "      if (" << lim << " > 0) {\n#pragma unroll\n      for (int j = 0; j < V; ++j) {\n        float t_[E];\n"
            << "#pragma unroll\n        for (int e = 0; e < E; ++e) t_[e] = " << val << ";\n"
            << cguard << "        as::stg(op_ + " << chx("j") << ", as::Conv<" << dt_code(dt) << ", E>::pack(t_));\n"
            << "      }\n      } else {\n#pragma unroll\n      for (int j = 0; j < V; ++j) {\n"
            << cguard << "        as::stg(op_ + " << chx("j") << ", " << rt << "{});\n      }\n      }\n    }\n";
          continue;
        }
        o << "#pragma unroll\n      for (int j = 0; j < V; ++j) {\n";
        o << "        float t_[E];\n";
        if (store_absorbed(id)) {
          // packed varlen rows: only the row's own chunks are stored, and
          // its invalid tail elements already hold 0
          o << "#pragma unroll\n        for (int e = 0; e < E; ++e) t_[e] = " << val << ";\n";
        } else if (masked) {
          o << "        if (" << full_pred(lim) << ") {\n#pragma unroll\n          for (int e = 0; e < E; ++e) t_[e] = "
            << val << ";\n        } else {\n#pragma unroll\n          for (int e = 0; e < E; ++e) t_[e] = ("
            << col_expr("j", "e") << " < " << lim << ") ? " << val << " : 0.f;\n        }\n";
        } else {
          o << "#pragma unroll\n        for (int e = 0; e < E; ++e) t_[e] = " << val << ";\n";
        }
        if (ragged) o << "        if (" << live_pred(lim) << " && (j * T + lane) * E < " << lim << ")  // chunks of the row only (packed)\n";
        else if (!exact) o << "        if ((long long)" << chx("j") << " < CH)\n";
        o << "        as::stg(op_ + " << chx("j") << ", as::Conv<" << dt_code(dt) << ", E>::pack(t_));\n";
        o << "      }\n    }\n";
      } else if (nd.kind == ASTITCH_ROWVEC) {
        o << "    if ((" << act << ") && lane == 0) as::st_scalar<" << dt_code(dt) << ">(p.out[" << k << "], " << row
          << ", " << sref(id, sfx) << ");\n";
      }
    }
    (void)check;
    (void)post;
    {  // values of this level read by later sweeps: buffered in HBM (global scheme)
      for (size_t q = 0; q < p.global_fulls.size(); ++q) {
        int id = p.global_fulls[q];
        if (I(id).level != cur_level) continue;
        long long off = static_cast<long long>(p.ws.globals + gbuf_offset(q));
        if (N(id).kind == ASTITCH_FULL) {
          std::string rt = "as::Raw<" + std::to_string(E * 4) + ">";
          o << "    if (" << act << ") {\n      " << rt << "* gb_ = (" << rt << "*)((char*)p.ws + " << off
            << "LL) + (" << row << ") * CH;\n";
          o << "#pragma unroll\n      for (int j = 0; j < V; ++j) {\n";
          if (!exact) o << "        if ((long long)" << chx("j") << " < CH)\n";
          o << "        as::stg(gb_ + " << chx("j") << ", as::Conv<0, E>::pack(v" << id << sfx << " + j * E));\n";
          o << "      }\n    }\n";
        } else if (N(id).kind == ASTITCH_ROWVEC) {
          o << "    if ((" << act << ") && lane == 0) ((float*)((char*)p.ws + " << off << "LL))[" << row << "] = s"
            << id << sfx << ";\n";
          if (precise[id])
            o << "    if ((" << act << ") && lane == 0) ((float*)((char*)p.ws + " << off << "LL))[" << p.desc.rows << "LL + "
              << row << "] = s" << id << sfx << "lo;\n";
        }
      }
    }
    (void)lim;
  }

  // declaration of the valid bound `lim` of row `row` (active flag `act`); for
  // packed varlen rows also `lim`_b = the row's first chunk in every FULL tensor
  // seg: (ragged) an int4 expression holding the row's table entry already
  // looked up (the prefetch of the previous iteration), else "" = look it up
  std::string limdecl(const std::string& lim, const std::string& act, const std::string& row,
                      const std::string& seg = "") const {
    if (!ragged) {
      if (!masked) return "const int " + lim + " = (int)C;";
      return "const int " + lim + " = " + act + " ? " + lim_expr(row) + " : 0;";
    }
    std::string find = seg.empty() ? act + " ? as::seg_find<NSEG>(SG, (int)(" + row + ")) : make_int4(0, 0, 0, 0)" : seg;
    return "const int4 " + lim + "_s = " + find + ";\n    const int " + lim + " = min(" + lim +
           "_s.y, (int)C);\n    const long long " + lim + "_b = ((long long)" + lim + "_s.w * 8 + (long long)((" + row +
           ") - " + lim + "_s.x) * " + lim + "_s.z) / E; (void)" + lim + "_b;";
  }
  // first chunk of row `row` in a FULL tensor (row-major [R, C] or packed varlen)
  std::string rowbase(const std::string& row, const std::string& lim) const {
    if (ragged) return lim + "_b";
    return "(" + row + ") * CH";
  }

  std::string lim_expr(const std::string& row) const {
    if (!masked) return "C";
    // 32-bit valid bound; the segment index is an unsigned division by the
    // compile-time rows-per-segment (a shift when it is a power of two)
    // p.row_offset: global row of local row 0 (chunked host pipelines)
    return "min(max(__ldg(Lp + (unsigned long long)((" + row + ") + p.row_offset) / (unsigned long long)RPS), 0), (int)C)";
  }

  // ------------------------------------------------------------ row sweep
  // Block-uniform loop over row groups; each team owns rows base + team.
  // Row indices fit 32 bits for every plan below 2^30 rows (cheaper compares
  // and increments than 64-bit); addresses are still formed in 64 bits.
  std::string rowt() const { return p.desc.rows < (1LL << 30) ? "int" : "long long"; }

  // one ping-pong half of the software-pipelined row loop: loads of the rows
  // one stride ahead go to buffer `nx` while the rows of `base` are computed
  // from buffer `cu` (no register copies between the halves)
  void emit_pingpong_half(bool post, const std::string& cu, const std::string& nx) {
    const std::string su = "_u";
    const std::string rt = rowt();
    for (int u = 0; u < U; ++u) {
      const std::string us = std::to_string(u);
      o << "    const " << rt << " row" << u << " = base + " << u << " * RPB + team;\n";
      o << "    const bool act" << u << " = row" << u << " < R;\n";
      o << "    const int lim" << u << " = "
        << (masked ? "act" + us + " ? " + lim_expr("row" + us) + " : 0" : "(int)C") << ";\n";
      o << "    (void)lim" << u << ";\n";
    }
    for (int u = 0; u < U; ++u) {
      const std::string us = std::to_string(u);
      o << "    {\n      const " << rt << " nrow = base + rstride + " << u
        << " * RPB + team;\n";
      o << "      const bool pact = nrow < R;\n";
      o << "      const int plim = " << (masked ? "pact ? " + lim_expr("nrow") + " : 0" : "(int)C") << ";\n";
      o << "      (void)plim;\n";
      emit_loads("nrow", "pact", "plim", su + us + nx, false);
      o << "    }\n";
    }
    for (int u = 0; u < U; ++u) {
      std::string s = su + std::to_string(u) + cu;
      std::string row = "row" + std::to_string(u), act = "act" + std::to_string(u), lim = "lim" + std::to_string(u);
      o << "    {\n";
      emit_unpack(s, lim);
      emit_colvecs(true);
      emit_rowvec_inputs(post, s, row, act);
      emit_body(post, s, row, act, lim);
      emit_stores(post, s, row, act, lim);
      o << "    }\n";
    }
  }


  void emit_sweep(bool post) {
    collect_streams(post);
    emit_stream_ptrs();
    // prefetching the next row only pays when a team sweeps more than one row
    const bool pf = m.prefetch && m.vertical_trips > 1;
    const std::string su = "_u";
    const std::string rt = rowt();
    o << "  const " << rt << " rstride = (" << rt << ")(NUNITS * RPB * " << U << ");\n";
    o << "  " << rt << " base = (" << rt << ")(UNIT * RPB * " << U << ");\n";
    // Ping-pong buffers (the loop body emitted twice, rows alternating between
    // two raw register sets: no copies, and each prefetch has a whole row step
    // to land) are the default for padded rows.  Measured on B200 against the
    // early-unpack copy form: C3 143.8 vs 146.1 us (80 vs 72 registers), C2 at
    // 32768 rows 29.1 vs 29.9 us, C5 and fig6a equal.  Packed varlen rows keep
    // the copy form (their KF-specialised body would be emitted 2 x (V+1)
    // times).
    if (pf && !ragged) {
      // ping-pong buffers a / b
      for (int u = 0; u < U; ++u)
        for (const char* bf : {"a", "b"})
          for (size_t q = 0; q < streams.size(); ++q)
            o << "  " << raw_t(streams[q]) << " r" << q << su << u << bf << "[V];\n";
      for (int u = 0; u < U; ++u) {
        const std::string us = std::to_string(u);
        o << "  {\n    const " << rt << " nrow = base + " << u << " * RPB + team;\n";
        o << "    const bool pact = nrow < R;\n";
        o << "    const int plim = " << (masked ? "pact ? " + lim_expr("nrow") + " : 0" : "(int)C") << ";\n";
        o << "    (void)plim;\n";
        emit_loads("nrow", "pact", "plim", su + std::to_string(u) + "a", false);
        o << "  }\n";
      }
      // (sync_steps) a block barrier per row step keeps the CTA's warps on
      // the same rows: drifting warps widen the window of concurrently
      // accessed addresses (measured on B200, 2R:1W stream: 6.41 -> 6.73 TB/s)
      const std::string sync = m.sync_steps ? "    __syncthreads();\n" : "";
      o << "  while (base < R) {\n";
      o << "   {\n" << sync;
      emit_pingpong_half(post, "a", "b");
      o << "   }\n    base += rstride;\n    if (base >= R) break;\n";
      o << "   {\n" << sync;
      emit_pingpong_half(post, "b", "a");
      o << "   }\n    base += rstride;\n  }\n";
      return;
    }
    if (pf) {
      for (int u = 0; u < U; ++u) {
        std::string row = "(base + " + std::to_string(u) + " * RPB + team)";
        o << "  const " << rt << " prow" << u << " = " << row << ";\n";
      }
      for (int u = 0; u < U; ++u) {
        std::string s = su + std::to_string(u) + "n";
        for (size_t q = 0; q < streams.size(); ++q) o << "  " << raw_t(streams[q]) << " r" << q << s << "[V];\n";
        // (ragged) the segment entry of the prefetched row, reused by the compute step
        if (ragged) {
          o << "  int4 nsg" << u << " = (prow" << u << " < R) ? as::seg_find<NSEG>(SG, (int)prow" << u
            << ") : make_int4(0, 0, 0, 0);\n";
          // two-deep segment lookahead: the entry of the row after the
          // prefetched one is searched an iteration early, so the prefetch's
          // load addresses never wait on a binary search
          o << "  int nnsg" << u << " = (prow" << u << " + rstride < R) ? as::seg_find_idx<NSEG>(SG, (int)(prow" << u
              << " + rstride)) : -1;\n";
        }
        o << "  {\n    const bool pact = prow" << u << " < R;\n";
        o << "    " << limdecl("plim", "pact", "prow" + std::to_string(u), ragged ? "nsg" + std::to_string(u) : "")
          << "\n";
        o << "    (void)plim;\n";
        emit_loads("prow" + std::to_string(u), "pact", "plim", s, false);
        o << "  }\n";
      }
    }
    o << "  for (; base < R; base += rstride) {\n";
    if (m.sync_steps) o << "    __syncthreads();  // keep the CTA's warps on the same rows\n";
    for (int u = 0; u < U; ++u) {
      std::string s = su + std::to_string(u);
      o << "    const " << rt << " row" << u << " = base + " << u << " * RPB + team;\n";
      o << "    const bool act" << u << " = row" << u << " < R;\n";
      o << "    " << limdecl("lim" + std::to_string(u), "act" + std::to_string(u), "row" + std::to_string(u),
                           (ragged && pf) ? "nsg" + std::to_string(u) : "") << "\n";
      o << "    (void)lim" << u << ";\n";
    }
    // early unpack: convert the prefetched raw vectors to fp32 before the
    // next prefetch is issued into the same registers (a raw copy kept live
    // across the prefetch stalled on the next row's loads: long scoreboard at
    // the loop back-edge, C3 ncu source view, round 1)
    if (pf) {
      for (int u = 0; u < U; ++u) {
        std::string s = su + std::to_string(u);
        emit_unpack_convert(s, s + "n");
      }
    }
    if (pf) {
      for (int u = 0; u < U; ++u) {
        std::string s = su + std::to_string(u) + "n";
        o << "    {\n";
        o << "      const " << rt << " nrow = base + rstride + " << u << " * RPB + team;\n";
        o << "      const bool pact = nrow < R;\n";
        const bool la = ragged;
        if (la) o << "      nsg" << u << " = (nnsg" << u << " >= 0) ? __ldg(SG + nnsg" << u << ") : make_int4(0, 0, 0, 0);\n";
        else if (ragged) o << "      nsg" << u << " = pact ? as::seg_find<NSEG>(SG, (int)nrow) : make_int4(0, 0, 0, 0);\n";
        o << "      " << limdecl("plim", "pact", "nrow", ragged ? "nsg" + std::to_string(u) : "") << "\n";
        o << "      (void)plim;\n";
        emit_loads("nrow", "pact", "plim", s, false);
        if (la)
          o << "      nnsg" << u << " = (nrow + rstride < R) ? as::seg_find_idx<NSEG>(SG, (int)(nrow + rstride)) : -1;\n";
        o << "    }\n";
      }
    } else {
      for (int u = 0; u < U; ++u) {
        std::string s = su + std::to_string(u);
        emit_loads("row" + std::to_string(u), "act" + std::to_string(u), "lim" + std::to_string(u), s, true);
      }
    }
    early_unpack = pf;
    for (int u = 0; u < U; ++u) {
      std::string s = su + std::to_string(u);
      std::string row = "row" + std::to_string(u), act = "act" + std::to_string(u), lim = "lim" + std::to_string(u);
      emit_row_block(post, s, row, act, lim);
    }
    early_unpack = false;
    o << "  }\n";
  }

  // one row's compute (unpack, ops, stores).  Packed varlen row teams
  // specialise it on KF = the number of fully valid team chunks (0..V), a
  // warp-uniform switch for rows of one segment: per-chunk mask tests fold at
  // compile time and chunks past the valid prefix cost nothing (measured on
  // B200: C3v 81 vs 95 us; the padded C3 rows gain nothing: stores of the
  // whole padded row dominate, and the 5x code loses 1-4%).
  void emit_row_block(bool post, const std::string& s, const std::string& row, const std::string& act,
                      const std::string& lim) {
    const bool spec = ragged && m.tmpl == Template::RowTeam && V >= 2 && !split;
    if (!spec) {
      o << "    {\n";
      emit_unpack(s, lim);
      emit_colvecs(true);
      emit_rowvec_inputs(post, s, row, act);
      emit_body(post, s, row, act, lim);
      emit_stores(post, s, row, act, lim);
      o << "    }\n";
      return;
    }
    o << "    switch (min(" << lim << " / (T * E), V)) {\n";
    kf = true;
    for (int k = 0; k <= V; ++k) {
      o << (k == V ? "    default" : "    case " + std::to_string(k)) << ": {\n";
      o << "    constexpr int KF = " << k << ", NEV = " << std::min(k + 1, V) << " * E; (void)KF; (void)NEV;\n";
      emit_unpack(s, lim);
      emit_colvecs(true);
      emit_rowvec_inputs(post, s, row, act);
      emit_body(post, s, row, act, lim);
      emit_stores(post, s, row, act, lim);
      o << "    } break;\n";
    }
    kf = false;
    o << "    }\n";
  }

  // ------------------------------------------------------------ global pieces
  void emit_colred_acc_decl() {
    for (int id : p.colreds) {
      if (phase_of(id) != cur_level) continue;
      bool mx = N(id).sub == ASTITCH_RMAX;
      if (pc(id)) {  // fp64 per-lane column sums (R7c)
        o << "  double acc" << id << "[NE];\n#pragma unroll\n  for (int k = 0; k < NE; ++k) acc" << id << "[k] = 0.0;\n";
        continue;
      }
      o << "  float acc" << id << "[NE];\n#pragma unroll\n  for (int k = 0; k < NE; ++k) acc" << id
        << "[k] = " << (mx ? "-AS_INF" : "0.f") << ";\n";
    }
  }

  // partial row written by this block
  const std::string part_idx = "blockIdx.x";
  // block partial of every column reduction -> ws partial row blockIdx.x
  // (precise sums, R7c: the block's fp64 sum stored as fp32 hi in slot q and
  // lo in slot lo_slot(q); hi + lo keeps ~48 bits)
  void emit_block_partials() {
    const int ncr = static_cast<int>(p.colreds.size());
    const int NS = nslots();
    o << "  {\n    float* part = (float*)((char*)p.ws + " << p.ws.partials << "LL);\n";
    if (RPB == 1) {
      for (int q = 0; q < ncr; ++q) {
        int id = p.colreds[q];
        if (phase_of(id) != cur_level) continue;
        o << "#pragma unroll\n    for (int k = 0; k < NE; ++k) {\n      const long long col = "
          << col_expr("(k / E)", "(k % E)") << ";\n";
        if (pc(id)) {
          o << "      const float h_ = (float)acc" << id << "[k];\n";
          o << "      if (col < C) { part[((long long)" << part_idx << " * " << NS << " + " << q << ") * C + col] = h_;\n";
          o << "        part[((long long)" << part_idx << " * " << NS << " + " << lo_slot(q) << ") * C + col] = (float)(acc"
            << id << "[k] - (double)h_); }\n    }\n";
          continue;
        }
        o << "      if (col < C) part[((long long)" << part_idx << " * " << NS << " + " << q << ") * C + col] = acc" << id
          << "[k];\n    }\n";
      }
    } else {
      o << "    extern __shared__ __align__(16) float cp_smem[];\n";
      o << "    const long long CC = (long long)T * V * E;\n";
      for (int q = 0; q < ncr; ++q) {
        int id = p.colreds[q];
        if (phase_of(id) != cur_level) continue;
        bool mx = N(id).sub == ASTITCH_RMAX;
        o << "    __syncthreads();\n";
        if (pc(id)) {
          o << "#pragma unroll\n    for (int k = 0; k < NE; ++k) {\n      const long long c_ = " << col_expr("(k / E)", "(k % E)")
            << ";\n      const float h_ = (float)acc" << id << "[k];\n      cp_smem[team * CC + c_] = h_;\n"
            << "      cp_smem[(RPB + team) * CC + c_] = (float)(acc" << id << "[k] - (double)h_);\n    }\n";
          o << "    __syncthreads();\n";
          o << "    for (long long col = threadIdx.x; col < C; col += blockDim.x) {\n";
          o << "      double a_ = 0.0;\n";
          o << "      for (int t = 0; t < RPB; ++t) a_ += (double)cp_smem[t * CC + col] + (double)cp_smem[(RPB + t) * CC + col];\n";
          o << "      const float h_ = (float)a_;\n";
          o << "      part[((long long)" << part_idx << " * " << NS << " + " << q << ") * C + col] = h_;\n";
          o << "      part[((long long)" << part_idx << " * " << NS << " + " << lo_slot(q) << ") * C + col] = (float)(a_ - (double)h_);\n    }\n";
          continue;
        }
        o << "#pragma unroll\n    for (int k = 0; k < NE; ++k) cp_smem[team * CC + " << col_expr("(k / E)", "(k % E)")
          << "] = acc" << id << "[k];\n";
        o << "    __syncthreads();\n";
        o << "    for (long long col = threadIdx.x; col < C; col += blockDim.x) {\n";
        o << "      float a_ = cp_smem[col];\n";
        o << "      for (int t = 1; t < RPB; ++t) a_ = " << (mx ? "as::nmax(a_, cp_smem[t * CC + col])" : "a_ + cp_smem[t * CC + col]") << ";\n";
        o << "      part[((long long)" << part_idx << " * " << NS << " + " << q << ") * C + col] = a_;\n    }\n";
      }
    }
    o << "  }\n";
  }

  // ------------------------------------------------------------ tma_sweep
  // Global sweep with address-ordered dynamic row tiles (reading R23): a
  // producer warp takes tile indices from a workspace counter and stages the
  // tile's rows of every FULL input in a ring of shared-memory stages with
  // bulk copies (cp.async.bulk, mbarrier complete_tx); the compute teams read
  // their rows from shared memory, store FULL outputs from registers, sum
  // each column over their rows of the tile in fp32 (fixed order) and
  // deposit that tile partial into an exact binned accumulator (as::bins_add),
  // so the column totals do not depend on which CTA took which tile.
  // Column MAX is order-independent as it is (nmax).
  bool binned(int id) const { return m.tma_sweep && N(id).sub != ASTITCH_RMAX; }
  // byte address of (CTA g, partial slot q, column col) in the tma_sweep
  // partial region (48-byte slots: as::BinSlot / as::BinSlotP / an fp32 max)
  // (32-byte slots unless a precise sum needs as::BinSlotP's 48)
  std::string slot_at(const std::string& base, const std::string& gi, int q, const std::string& col) const {
    return "((const char*)(" + base + ") + (((long long)(" + gi + ") * " + std::to_string(nslots()) + " + " +
           std::to_string(q) + ") * C + (" + col + ")) * " + (p.n_precise_colreds > 0 ? "48LL)" : "32LL)");
  }
  // prologue (once per kernel): ring, mbarriers, the running stage counters
  // of the producer (kt_p) and of the consumers (kt_c), which continue across
  // barrier levels so the mbarrier phases stay in step
  void emit_tma_prologue() {
    const int TR = m.tma_rows, S = m.tma_stages;
    const int CT = RPB * T;  // compute threads (the producer warp follows)
    o << "  constexpr int TR = " << TR << ", NSTG = " << S << ", CT = " << CT << ";\n";
    o << "  extern __shared__ __align__(128) unsigned char tma_smem[];\n";
    o << "  __shared__ __align__(8) unsigned long long tma_full[NSTG], tma_empty[NSTG];\n";
    o << "  __shared__ int tma_tile[NSTG];\n";
    o << "  const int NTILES = (int)((R + TR - 1) / TR);\n";
    o << "  const unsigned sbase_ = as::smem_addr(tma_smem);\n";
    o << "  int kt_p = 0, kt_c = 0;\n  (void)kt_p; (void)kt_c;\n";
    o << "  if (threadIdx.x == 0) {\n    for (int s = 0; s < NSTG; ++s) { as::mbar_init(as::smem_addr(&tma_full[s]), 1u); "
         "as::mbar_init(as::smem_addr(&tma_empty[s]), (unsigned)(CT / 32)); }\n    as::fence_mbar_init();\n  }\n";
    o << "  __syncthreads();\n";
  }
  // does a later barrier level sweep the rows again (FULL values or column
  // reductions of a later level, recomputed values)?
  bool sweep_after(int lv) const {
    for (size_t i = 0; i < g.nodes.size(); ++i) {
      if (!I(i).live) continue;
      if (N(i).kind == ASTITCH_FULL && (I(i).level > lv || (I(i).remat_mask >> (lv + 1)) != 0u)) return true;
      if (I(i).cls == OpClass::ReduceCol && phase_of(static_cast<int>(i)) > lv) return true;
    }
    return false;
  }
  // the tile counter of barrier level lv; [60]: CTAs done (the last resets them)
  long long tctr_off(int lv) const { return static_cast<long long>(p.ws.barrier + 64 + 4 * lv); }
  void emit_tma_epilogue() {
    o << "  __syncthreads();\n";
    o << "  if (threadIdx.x == 0) {\n    __threadfence();\n";
    o << "    const unsigned d_ = atomicAdd((unsigned*)((char*)p.ws + " << (p.ws.barrier + 60) << "LL), 1u);\n";
    o << "    if (d_ == gridDim.x - 1) {\n";
    for (int lv = 0; lv <= p.max_level; ++lv)
      o << "      *(volatile unsigned*)((char*)p.ws + " << tctr_off(lv) << "LL) = 0u;\n";
    o << "      *(volatile unsigned*)((char*)p.ws + " << (p.ws.barrier + 60) << "LL) = 0u;\n      __threadfence();\n    }\n  }\n";
  }

  // one sweep (barrier level cur_level) of the tma_sweep: the producer warp
  // stages this level's row streams (FULL inputs re-read, HBM buffers of
  // earlier levels), the consumers compute this level's ops, deposit the tile
  // partials of this level's column reductions, then the CTA combine writes
  // this CTA's partial slots
  void emit_tma_level() {
    const int lv = cur_level;
    collect_streams(lv > 0);
    const int TR = m.tma_rows, S = m.tma_stages;
    std::vector<long long> soff(streams.size()), rb(streams.size());
    long long stage_bytes = 0;
    for (size_t s = 0; s < streams.size(); ++s) {
      rb[s] = C * dtype_size(streams[s].dt);
      // ring layout: stream s occupies S x TR rows starting at S * TR * (sum of earlier row bytes)
      soff[s] = static_cast<long long>(S) * TR * stage_bytes;
      stage_bytes += rb[s];
    }
    std::vector<int> crs;
    for (int id : p.colreds)
      if (phase_of(id) == lv) crs.push_back(id);
    // accumulators that live across tiles
    for (int id : crs) {
      if (binned(id) && pc(id)) {  // precise (R7c): fp64 tile partials, 4 x 16-bit bins
        o << "  int bJ" << id << "[NE];\n  long long bq" << id << "[NE * 4];\n  float bs" << id
          << "[NE];\n#pragma unroll\n  for (int k = 0; k < NE; ++k) { bJ" << id << "[k] = AS_BIN_EMPTY; bs" << id
          << "[k] = 0.f; bq" << id << "[4 * k] = bq" << id << "[4 * k + 1] = bq" << id << "[4 * k + 2] = bq" << id << "[4 * k + 3] = 0; }\n";
      } else if (binned(id)) {
        o << "  int bJ" << id << "[NE];\n  long long bh" << id << "[NE], bl" << id << "[NE];\n  float bs" << id
          << "[NE];\n#pragma unroll\n  for (int k = 0; k < NE; ++k) { bJ" << id << "[k] = AS_BIN_EMPTY; bh" << id << "[k] = 0; bl" << id
          << "[k] = 0; bs" << id << "[k] = 0.f; }\n";
      } else {
        o << "  float acc" << id << "[NE];\n#pragma unroll\n  for (int k = 0; k < NE; ++k) acc" << id << "[k] = -AS_INF;\n";
      }
    }
    o << "  unsigned int* tctr = (unsigned int*)((char*)p.ws + " << tctr_off(lv) << "LL);\n";
    // producer: one elected thread of the extra warp (after a level's
    // barriers: the ring held generic-proxy scratch, order it before the
    // bulk copies' async-proxy writes)
    o << "  if (threadIdx.x >= CT) {\n    if (threadIdx.x == CT) {\n";
    if (lv > 0) o << "      as::fence_proxy_async_smem();\n";
    o << "      for (;; ++kt_p) {\n";
    o << "        const int st = kt_p % NSTG;\n";
    o << "        if (kt_p >= NSTG) as::mbar_wait(as::smem_addr(&tma_empty[st]), (unsigned)((kt_p / NSTG - 1) & 1));\n";
    o << "        const int tile = (int)atomicAdd(tctr, 1u);\n";
    o << "        tma_tile[st] = tile;\n";
    o << "        const unsigned fb = as::smem_addr(&tma_full[st]);\n";
    o << "        if (tile >= NTILES) { asm volatile(\"mbarrier.arrive.shared::cta.b64 _, [%0];\" ::\"r\"(fb) : \"memory\"); ++kt_p; break; }\n";
    o << "        const int trows = min(TR, R - tile * TR);\n";
    o << "        as::mbar_expect_tx(fb, (unsigned)(trows * " << stage_bytes << "LL));\n";
    for (size_t s = 0; s < streams.size(); ++s) {
      std::string src = streams[s].ws_buf ? "(const char*)p.ws + " + std::to_string(streams[s].ws_off) + "LL"
                                          : "(const char*)p.in[" + std::to_string(N(streams[s].node).input_index) + "]";
      o << "        as::bulk_g2s(as::smem_addr(tma_smem + " << soff[s] << "LL + (long long)st * TR * " << rb[s]
        << "LL), " << src << " + (long long)tile * TR * " << rb[s] << "LL, (unsigned)(trows * " << rb[s] << "LL), fb);\n";
    }
    o << "      }\n    }\n  } else {\n";
    // consumers
    o << "  for (;; ++kt_c) {\n";
    o << "    const int st = kt_c % NSTG;\n";
    o << "    as::mbar_wait(as::smem_addr(&tma_full[st]), (unsigned)((kt_c / NSTG) & 1));\n";
    o << "    const int tile = tma_tile[st];\n";
    // the sentinel's stage is released too when a later level's producer reuses it
    if (sweep_after(lv))
      o << "    if (tile >= NTILES) {\n      __syncwarp();\n      if ((threadIdx.x & 31) == 0) asm volatile(\"mbarrier.arrive.shared::cta.b64 _, [%0];\" ::\"r\"(as::smem_addr(&tma_empty[st])) : \"memory\");\n      ++kt_c;\n      break;\n    }\n";
    else
      o << "    if (tile >= NTILES) break;\n";
    o << "    const int trows = min(TR, R - tile * TR);\n";
    for (int id : crs)
      if (binned(id))
        o << "    " << (pc(id) ? "double" : "float") << " acc" << id << "[NE];\n#pragma unroll\n    for (int k = 0; k < NE; ++k) acc" << id
          << "[k] = 0;\n";
    o << "#pragma unroll\n    for (int rr_ = 0; rr_ < TR / RPB; ++rr_) {\n";
    o << "    const int rl_ = team + RPB * rr_;\n";
    o << "    const int row0 = tile * TR + rl_;\n";
    o << "    const bool act0 = rl_ < trows;\n";
    o << "    const int lim0 = (int)C;\n    (void)lim0;\n";
    for (size_t s = 0; s < streams.size(); ++s) {
      o << "    " << raw_t(streams[s]) << " r" << s << "_u0[V];\n";
      o << "    r" << s << "_u0[0] = act0 ? as::lds_chunk<" << nb(streams[s].dt) << ">(sbase_ + (unsigned)(" << soff[s]
        << "LL + ((long long)st * TR + rl_) * " << rb[s] << "LL + (long long)lane * " << nb(streams[s].dt) << ")) : "
        << raw_t(streams[s]) << "{};\n";
    }
    emit_row_block(lv > 0, "_u0", "row0", "act0", "lim0");
    o << "    }\n";
    // release the stage, then deposit the tile partials
    o << "    __syncwarp();\n    if ((threadIdx.x & 31) == 0) asm volatile(\"mbarrier.arrive.shared::cta.b64 _, [%0];\" ::\"r\"(as::smem_addr(&tma_empty[st])) : \"memory\");\n";
    for (int id : crs) {
      if (binned(id) && pc(id))
        o << "    as::bins_add_p<NE>(bJ" << id << ", bq" << id << ", bs" << id << ", acc" << id << ");\n";
      else if (binned(id))
        o << "    as::bins_add<NE>(bJ" << id << ", bh" << id << ", bl" << id << ", bs" << id << ", acc" << id << ");\n";
    }
    o << "  }\n  }\n";
    if (crs.empty()) return;
    // CTA combine (teams in order) -> partial slot of this CTA; the ring is free now
    o << "  {\n    char* part = (char*)p.ws + " << p.ws.partials << "LL;\n";
    for (size_t q = 0; q < p.colreds.size(); ++q) {
      int id = p.colreds[q];
      if (phase_of(id) != lv) continue;
      o << "    __syncthreads();\n";
      if (binned(id) && pc(id)) {
        o << "    {\n      as::BinSlotP* sc_ = (as::BinSlotP*)tma_smem;  // [team][lane][k]\n";
        o << "      if (threadIdx.x < CT) {\n#pragma unroll\n        for (int k = 0; k < NE; ++k) { as::BinSlotP b_; b_.J = bJ" << id
          << "[k]; b_.sp = bs" << id << "[k]; b_.pad = 0;\n#pragma unroll\n          for (int q_ = 0; q_ < 4; ++q_) b_.b[q_] = bq" << id
          << "[4 * k + q_];\n          sc_[(team * T + lane) * NE + k] = b_; }\n      }\n";
        o << "      __syncthreads();\n";
        o << "      for (int c_ = threadIdx.x; c_ < (int)C; c_ += blockDim.x) {\n";
        o << "        const int l_ = c_ / E, k_ = c_ % E;\n";
        o << "        as::BinSlotP a_ = sc_[l_ * NE + k_];\n";
        o << "        for (int t_ = 1; t_ < RPB; ++t_) { const as::BinSlotP b_ = sc_[(t_ * T + l_) * NE + k_]; "
             "as::bins_merge_p(a_.J, a_.b, a_.sp, b_.J, b_.b, b_.sp); }\n";
        o << "        *(as::BinSlotP*)" << slot_at("part", "blockIdx.x", static_cast<int>(q), "c_") << " = a_;\n";
        o << "      }\n    }\n";
      } else if (binned(id)) {
        o << "    {\n      as::BinSlot* sc_ = (as::BinSlot*)tma_smem;  // [team][lane][k]\n";
        o << "      if (threadIdx.x < CT) {\n#pragma unroll\n        for (int k = 0; k < NE; ++k) { as::BinSlot b_; b_.J = bJ" << id
          << "[k]; b_.sp = bs" << id << "[k]; b_.hi = bh" << id << "[k]; b_.lo = bl" << id << "[k]; b_.pad = 0; sc_[(team * T + lane) * NE + k] = b_; }\n      }\n";
        o << "      __syncthreads();\n";
        o << "      for (int c_ = threadIdx.x; c_ < (int)C; c_ += blockDim.x) {\n";
        o << "        const int l_ = c_ / E, k_ = c_ % E;\n";
        o << "        as::BinSlot a_ = sc_[l_ * NE + k_];\n";
        o << "        for (int t_ = 1; t_ < RPB; ++t_) { const as::BinSlot b_ = sc_[(t_ * T + l_) * NE + k_]; "
             "as::bins_merge(a_.J, a_.hi, a_.lo, a_.sp, b_.J, b_.hi, b_.lo, b_.sp); }\n";
        o << "        *(as::BinSlot*)" << slot_at("part", "blockIdx.x", static_cast<int>(q), "c_") << " = a_;\n";
        o << "      }\n    }\n";
      } else {
        o << "    {\n      float* sc_ = (float*)tma_smem;\n";
        o << "      if (threadIdx.x < CT) {\n#pragma unroll\n        for (int k = 0; k < NE; ++k) sc_[(team * T + lane) * NE + k] = acc" << id
          << "[k];\n      }\n      __syncthreads();\n";
        o << "      for (int c_ = threadIdx.x; c_ < (int)C; c_ += blockDim.x) {\n";
        o << "        const int l_ = c_ / E, k_ = c_ % E;\n        float a_ = sc_[l_ * NE + k_];\n";
        o << "        for (int t_ = 1; t_ < RPB; ++t_) a_ = as::nmax(a_, sc_[(t_ * T + l_) * NE + k_]);\n";
        o << "        ((as::BinSlot*)" << slot_at("part", "blockIdx.x", static_cast<int>(q), "c_") << ")->sp = a_;\n";
        o << "      }\n    }\n";
      }
    }
    o << "  }\n";
  }

  // ------------------------------------------------------------ tma_team
  // Row teams fed by a producer warp: tiles of TR rows are taken from a
  // workspace counter (address order); lane r of the producer warp copies
  // row r's valid prefix of every FULL input (rounded up to 16 bytes) into
  // its slot of the stage with one bulk copy; the teams read their rows'
  // chunks from shared memory and run the usual row body (masks, KF
  // specialisation, stores).  The last CTA to finish resets the counters.
  void emit_tma_team(const std::string& name) {
    header(name, false);
    collect_streams(false);
    const int TR = m.tma_rows, S = m.tma_stages;
    const int CT = RPB * T;
    std::vector<long long> soff(streams.size()), slot(streams.size());
    long long acc = 0;
    for (size_t s = 0; s < streams.size(); ++s) {
      slot[s] = (C * dtype_size(streams[s].dt) + 15) / 16 * 16;
      soff[s] = static_cast<long long>(S) * TR * acc;
      acc += slot[s];
    }
    emit_colvecs(false);
    emit_pre_colvec_outputs();  // COLVEC outputs of the row plan (block 0; fuzz seeds 4039 / 4161)
    o << "  constexpr int TR = " << TR << ", NSTG = " << S << ", CT = " << CT << ";\n";
    o << "  extern __shared__ __align__(128) unsigned char tma_smem[];\n";
    o << "  __shared__ __align__(8) unsigned long long tma_full[NSTG], tma_empty[NSTG];\n";
    o << "  __shared__ int tma_tile[NSTG];\n";
    o << "  unsigned int* tctr = (unsigned int*)((char*)p.ws + " << (p.ws.barrier + 64) << "LL);\n";
    o << "  unsigned int* tdone = (unsigned int*)((char*)p.ws + " << (p.ws.barrier + 68) << "LL);\n";
    // (ragged) per stage: the segment pitch (elements) when the tile's rows
    // were copied with ONE bulk copy (all in one segment: contiguous), else 0
    if (ragged) o << "  __shared__ int tma_pk[NSTG];\n";
    o << "  const int NTILES = (int)((R + TR - 1) / TR);\n";
    o << "  const unsigned sbase_ = as::smem_addr(tma_smem);\n";
    o << "  if (threadIdx.x == 0) {\n    for (int s = 0; s < NSTG; ++s) { as::mbar_init(as::smem_addr(&tma_full[s]), 1u); "
         "as::mbar_init(as::smem_addr(&tma_empty[s]), (unsigned)(CT / 32)); }\n    as::fence_mbar_init();\n  }\n";
    o << "  __syncthreads();\n";
    // producer warp: lane r copies row r of the tile
    o << "  if (threadIdx.x >= CT) {\n    const int pl = threadIdx.x - CT;\n";
    o << "    for (int kt = 0;; ++kt) {\n";
    o << "      const int st = kt % NSTG;\n";
    o << "      if (kt >= NSTG) as::mbar_wait(as::smem_addr(&tma_empty[st]), (unsigned)((kt / NSTG - 1) & 1));\n";
    o << "      int tile = 0;\n      if (pl == 0) tile = (int)atomicAdd(tctr, 1u);\n";
    o << "      tile = __shfl_sync(0xffffffffu, tile, 0);\n";
    o << "      const unsigned fb = as::smem_addr(&tma_full[st]);\n";
    o << "      if (tile >= NTILES) {\n        if (pl == 0) { tma_tile[st] = tile; asm volatile(\"mbarrier.arrive.shared::cta.b64 _, [%0];\" ::\"r\"(fb) : \"memory\"); }\n        break;\n      }\n";
    o << "      const int prow = tile * TR + pl;\n";
    o << "      const bool pact = pl < TR && prow < R;\n";
    o << "      " << limdecl("plim", "pact", "prow") << "\n      (void)plim;\n";
    if (ragged) {
      // rows of one segment are contiguous at the segment's pitch (a multiple
      // of 8 elements): the whole tile in one bulk copy per stream
      o << "      const int fx_ = __shfl_sync(0xffffffffu, plim_s.x, 0);\n";
      o << "      if (__all_sync(0xffffffffu, !pact || plim_s.x == fx_)) {\n";
      o << "        const int nact_ = __popc(__ballot_sync(0xffffffffu, pact));\n";
      o << "        if (pl == 0) {\n          tma_tile[st] = tile; tma_pk[st] = plim_s.z;\n";
      long long tot = 0;
      for (size_t s = 0; s < streams.size(); ++s) tot += dtype_size(streams[s].dt);
      o << "          as::mbar_expect_tx(fb, (unsigned)(nact_ * plim_s.z * " << tot << "));\n";
      for (size_t s = 0; s < streams.size(); ++s)
        o << "          as::bulk_g2s(sbase_ + (unsigned)(" << soff[s] << "LL + (long long)st * TR * " << slot[s]
          << "LL), (const char*)p.in[" << N(streams[s].node).input_index << "] + (long long)plim_b * " << nb(streams[s].dt)
          << "LL, (unsigned)(nact_ * plim_s.z * " << dtype_size(streams[s].dt) << "), fb);\n";
      o << "        }\n        continue;\n      }\n";
      o << "      if (pl == 0) tma_pk[st] = 0;\n";
    }
    o << "      unsigned nbytes_ = 0;\n";
    for (size_t s = 0; s < streams.size(); ++s) {
      const int es = dtype_size(streams[s].dt);
      o << "      const unsigned nb" << s << " = pact ? (unsigned)((min(plim, (int)C) * " << es << " + 15) & ~15) : 0u;\n";
      o << "      nbytes_ += nb" << s << ";\n";
    }
    o << "#pragma unroll\n      for (int o_ = 16; o_ > 0; o_ /= 2) nbytes_ += __shfl_xor_sync(0xffffffffu, nbytes_, o_);\n";
    o << "      if (pl == 0) { tma_tile[st] = tile; as::mbar_expect_tx(fb, nbytes_); }\n";
    o << "      __syncwarp();\n";
    for (size_t s = 0; s < streams.size(); ++s) {
      o << "      if (nb" << s << ") as::bulk_g2s(sbase_ + (unsigned)(" << soff[s] << "LL + ((long long)st * TR + pl) * " << slot[s]
        << "LL), (const char*)p.in[" << N(streams[s].node).input_index << "] + (long long)" << rowbase("prow", "plim")
        << " * " << nb(streams[s].dt) << "LL, nb" << s << ", fb);\n";
    }
    o << "    }\n  } else {\n";
    // consumers
    o << "  for (int kt = 0;; ++kt) {\n";
    o << "    const int st = kt % NSTG;\n";
    o << "    as::mbar_wait(as::smem_addr(&tma_full[st]), (unsigned)((kt / NSTG) & 1));\n";
    o << "    const int tile = tma_tile[st];\n";
    o << "    if (tile >= NTILES) break;\n";
    o << "#pragma unroll 1\n    for (int rr_ = 0; rr_ < TR / RPB; ++rr_) {\n";
    o << "    const int rl_ = team + RPB * rr_;\n";
    o << "    const int row0 = tile * TR + rl_;\n";
    o << "    const bool act0 = row0 < R;\n";
    // (a per-stage table of the lengths the producer lanes looked up measured
    // slower on B200, C3 137.8 vs 136.1 us: one more register, a 4-byte spill)
    o << "    " << limdecl("lim0", "act0", "row0") << "\n    (void)lim0;\n";
    for (size_t s = 0; s < streams.size(); ++s) {
      const Stream& stv = streams[s];
      o << "    " << raw_t(stv) << " r" << s << "_u0[V];\n";
      o << "#pragma unroll\n    for (int j = 0; j < V; ++j) {\n";
      o << "      const long long c0 = " << chx("j") << " * E;\n";
      std::string cond = "act0";
      if (!exact || masked) cond += " && c0 < lim0";
      if (ragged)  // the row's offset: segment pitch when the tile came in one copy, else its slot
        o << "      if (" << cond << ") r" << s << "_u0[j] = as::lds_chunk<" << nb(stv.dt) << ">(sbase_ + (unsigned)(" << soff[s]
          << "LL + (long long)st * TR * " << slot[s] << "LL + (tma_pk[st] ? (long long)rl_ * tma_pk[st] * " << dtype_size(stv.dt)
          << "LL : (long long)rl_ * " << slot[s] << "LL) + " << chx("j") << " * " << nb(stv.dt) << "LL));\n";
      else
        o << "      if (" << cond << ") r" << s << "_u0[j] = as::lds_chunk<" << nb(stv.dt) << ">(sbase_ + (unsigned)(" << soff[s]
          << "LL + ((long long)st * TR + rl_) * " << slot[s] << "LL + " << chx("j") << " * " << nb(stv.dt) << "LL));\n";
      if (!absorb) o << "      else r" << s << "_u0[j] = " << raw_t(stv) << "{};\n";
      o << "    }\n";
    }
    emit_row_block(false, "_u0", "row0", "act0", "lim0");
    o << "    }\n";
    o << "    __syncwarp();\n    if ((threadIdx.x & 31) == 0) asm volatile(\"mbarrier.arrive.shared::cta.b64 _, [%0];\" ::\"r\"(as::smem_addr(&tma_empty[st])) : \"memory\");\n";
    o << "  }\n  }\n";
    // the last CTA to finish resets the counters for the next run
    o << "  __syncthreads();\n";
    o << "  if (threadIdx.x == 0) {\n    __threadfence();\n    const unsigned d_ = atomicAdd(tdone, 1u);\n";
    o << "    if (d_ == gridDim.x - 1) { *(volatile unsigned*)tctr = 0u; *(volatile unsigned*)tdone = 0u; __threadfence(); }\n  }\n";
    o << "}\n";
  }

  // partial rows of column `col` combined by the finalise: every CTA's, or
  // (column slabs) the CTAs of col's slab, r = slab + k * NSLAB, in k order
  std::string fin_r0() const { return slab ? "(int)(col / SLABW) + pi * NSLAB" : "pi"; }
  std::string fin_rs() const { return slab ? "P * NSLAB" : "P"; }
  // after the barrier: fixed-order combine of the grid partials per column
  // (deterministic), then the COLVEC consumers (global stage) for that column.
  // final == false (sharded): write the rank-local totals to ws colpart only.
  void emit_column_finalize(bool final_chain) {
    const int ncr = static_cast<int>(p.colreds.size());
    o << "  {\n    const float* part = (const float*)((const char*)p.ws + " << p.ws.partials << "LL);\n";
    o << "    float* colpart = (float*)((char*)p.ws + " << (p.ws.colvals + p.post_colvecs.size() * C * 4) << "LL);\n";
    o << "    const int G = gridDim.x;\n";
    o << "    const long long W = (C + G - 1) / G;\n";
    o << "    const long long c0 = (long long)blockIdx.x * W;\n";
    o << "    const long long c1 = min(C, c0 + W);\n";
    o << "    __shared__ float fin_smem[" << m.threads << "];\n";
    if (any_pc()) o << "    __shared__ double fin_smem_d[" << m.threads << "];\n";
    o << "    int P = 1; while (P * 2 * W <= blockDim.x && P * 2 <= 256) P *= 2;\n";
    o << "    for (long long cb = c0; cb < c1; cb += blockDim.x / P) {\n";
    o << "      const int wi = threadIdx.x / P, pi = threadIdx.x % P;\n";
    o << "      const long long col = cb + wi;\n";
    o << "      const bool own = (wi < (int)(blockDim.x / P)) && col < c1;\n";
    const int NS = nslots();
    for (int q = 0; q < ncr; ++q) {
      int id = p.colreds[q];
      if (phase_of(id) != cur_level) continue;
      bool mx = N(id).sub == ASTITCH_RMAX;
      std::string ident = mx ? "-AS_INF" : "0.f";
      if (binned(id) && pc(id)) {  // tma_sweep, precise (R7c): merge the CTAs' fp64 bins, value in fp64
        o << "      float t" << id << ";\n      double t" << id << "d;\n      {\n";
        o << "        as::BinSlotP a_; a_.J = AS_BIN_EMPTY; a_.sp = 0.f; a_.b[0] = a_.b[1] = a_.b[2] = a_.b[3] = 0; a_.pad = 0;\n";
        o << "        if (own) for (int r = pi; r < G; r += P) { const as::BinSlotP b_ = as::ld_cg_binsp((const as::BinSlotP*)"
          << slot_at("part", "r", q, "col") << "); as::bins_merge_p(a_.J, a_.b, a_.sp, b_.J, b_.b, b_.sp); }\n";
        o << "        as::BinSlotP* fs_ = (as::BinSlotP*)tma_smem;\n        fs_[threadIdx.x] = a_;\n        __syncthreads();\n";
        o << "        for (int s = P / 2; s > 0; s /= 2) {\n          if (pi < s) { as::BinSlotP c_ = fs_[threadIdx.x]; const as::BinSlotP d_ = fs_[threadIdx.x + s]; "
             "as::bins_merge_p(c_.J, c_.b, c_.sp, d_.J, d_.b, d_.sp); fs_[threadIdx.x] = c_; }\n          __syncthreads();\n        }\n";
        o << "        const as::BinSlotP r_ = fs_[threadIdx.x - pi];\n        __syncthreads();\n";
        o << "        t" << id << "d = as::bins_value_p(r_.J, r_.b, r_.sp);\n        t" << id << " = (float)t" << id << "d;\n      }\n";
        continue;
      }
      if (binned(id)) {  // tma_sweep: merge the CTAs' binned accumulators (exact, any order: R23)
        o << "      float t" << id << ";\n      {\n";
        o << "        as::BinSlot a_; a_.J = AS_BIN_EMPTY; a_.sp = 0.f; a_.hi = 0; a_.lo = 0; a_.pad = 0;\n";
        o << "        if (own) for (int r = pi; r < G; r += P) { const as::BinSlot b_ = as::ld_cg_bins((const as::BinSlot*)"
          << slot_at("part", "r", q, "col") << "); as::bins_merge(a_.J, a_.hi, a_.lo, a_.sp, b_.J, b_.hi, b_.lo, b_.sp); }\n";
        o << "        as::BinSlot* fs_ = (as::BinSlot*)tma_smem;\n        fs_[threadIdx.x] = a_;\n        __syncthreads();\n";
        o << "        for (int s = P / 2; s > 0; s /= 2) {\n          if (pi < s) { as::BinSlot c_ = fs_[threadIdx.x]; const as::BinSlot d_ = fs_[threadIdx.x + s]; "
             "as::bins_merge(c_.J, c_.hi, c_.lo, c_.sp, d_.J, d_.hi, d_.lo, d_.sp); fs_[threadIdx.x] = c_; }\n          __syncthreads();\n        }\n";
        o << "        const as::BinSlot r_ = fs_[threadIdx.x - pi];\n        __syncthreads();\n";
        o << "        t" << id << " = (float)as::bins_value_d(r_.J, r_.hi, r_.lo, r_.sp);\n      }\n";
        continue;
      }
      if (m.tma_sweep) {  // tma_sweep column MAX: the CTA maxima sit in the slots' sp words
        o << "      float t" << id << " = -AS_INF;\n";
        o << "      if (own) for (int r = pi; r < G; r += P) t" << id << " = as::nmax(t" << id
          << ", as::ld_cg(&((const as::BinSlot*)" << slot_at("part", "r", q, "col") << ")->sp));\n";
        o << "      fin_smem[threadIdx.x] = t" << id << ";\n      __syncthreads();\n";
        o << "      for (int s = P / 2; s > 0; s /= 2) { if (pi < s) fin_smem[threadIdx.x] = as::nmax(fin_smem[threadIdx.x], fin_smem[threadIdx.x + s]); __syncthreads(); }\n";
        o << "      t" << id << " = fin_smem[threadIdx.x - pi];\n      __syncthreads();\n";
        continue;
      }
      if (pc(id)) {  // fp64 combine of the hi + lo partials (R7c)
        o << "      double t" << id << "d = 0.0;\n";
        o << "      if (own) for (int r = " << fin_r0() << "; r < G; r += " << fin_rs() << ") t" << id
          << "d += (double)as::ld_cg(part + ((long long)r * " << NS << " + " << q << ") * C + col) + (double)as::ld_cg(part + ((long long)r * "
          << NS << " + " << lo_slot(q) << ") * C + col);\n";
        o << "      fin_smem_d[threadIdx.x] = t" << id << "d;\n      __syncthreads();\n";
        o << "      for (int s = P / 2; s > 0; s /= 2) { if (pi < s) fin_smem_d[threadIdx.x] += fin_smem_d[threadIdx.x + s]; __syncthreads(); }\n";
        o << "      t" << id << "d = fin_smem_d[threadIdx.x - pi];\n      __syncthreads();\n";
        o << "      const float t" << id << " = (float)t" << id << "d; (void)t" << id << ";\n";
        continue;
      }
      o << "      float t" << id << " = " << ident << ";\n";
      o << "      if (own) for (int r = " << fin_r0() << "; r < G; r += " << fin_rs() << ") { const float x_ = as::ld_cg(part + ((long long)r * " << NS
        << " + " << q << ") * C + col); t" << id << " = " << (mx ? "as::nmax(t" + std::to_string(id) + ", x_)" : "t" + std::to_string(id) + " + x_") << "; }\n";
      o << "      fin_smem[threadIdx.x] = t" << id << ";\n      __syncthreads();\n";
      o << "      for (int s = P / 2; s > 0; s /= 2) { if (pi < s) fin_smem[threadIdx.x] = "
        << (mx ? "as::nmax(fin_smem[threadIdx.x], fin_smem[threadIdx.x + s])" : "fin_smem[threadIdx.x] + fin_smem[threadIdx.x + s]")
        << "; __syncthreads(); }\n";
      o << "      t" << id << " = fin_smem[threadIdx.x - pi];\n      __syncthreads();\n";
    }
    o << "      if (own && pi == 0) {\n";
    if (!final_chain) {
      // p.flags & 1: accumulate onto the totals of earlier row chunks
      for (int q = 0; q < ncr; ++q) {
        bool mx = N(p.colreds[q]).sub == ASTITCH_RMAX;
        std::string slot = "colpart[" + std::to_string(q) + "LL * C + col]";
        std::string t = "t" + std::to_string(p.colreds[q]);
        if (mx && role == ROLE_SHARD_MAIN) {
          // sharded stage 0: a MAX slot holds int32 order keys (as::okey) so
          // the cross-rank combine is an integer max that keeps NaN (R12)
          std::string islot = "((int*)colpart)[" + std::to_string(q) + "LL * C + col]";
          o << "        " << islot << " = as::okey((p.flags & 1) ? as::nmax(as::okey_dec(" << islot << "), " << t
            << ") : " << t << ");\n";
          continue;
        }
        o << "        " << slot << " = (p.flags & 1) ? "
          << (mx ? "as::nmax(" + slot + ", " + t + ")" : "(" + slot + " + " + t + ")") << " : " << t << ";\n";
      }
    } else {
      emit_colvec_chain("t");
    }
    o << "      }\n    }\n  }\n";
  }

  // Fused sharded stage (astitch_run_fused, NEXT f1): the rank-local column
  // totals of this block's columns (ws colpart) are pushed with plain stores
  // into slot [gen parity][this rank] of EVERY rank's exchange buffer (peer
  // memory over NVLink), published by a system fence + grid barrier + one
  // release flag per rank; each block then waits for all ranks' flags (bounded)
  // and combines the world slots in rank order 0..world-1 (identical on every
  // rank: deterministic) before the column consumers.  One kernel, no NCCL.
  void emit_fused_exchange() {
    const int ncr = static_cast<int>(p.colreds.size());
    const int XW = p.desc.shard_world, XR = p.desc.shard_rank;
    const long long colpart = static_cast<long long>(p.ws.colvals + p.post_colvecs.size() * C * 4);
    o << "  __syncthreads();\n";
    o << "  {  // ---- fused exchange of the column totals over peer memory\n";
    o << "    constexpr int XW = " << XW << ", XR = " << XR << ", NCR = " << ncr << ";\n";
    o << "    unsigned char* X = (unsigned char*)p.xbuf;\n";
    o << "    const float* colpart = (const float*)((const char*)p.ws + " << colpart << "LL);\n";
    o << "    const int G = gridDim.x;\n    const long long W = (C + G - 1) / G;\n";
    o << "    const long long c0 = (long long)blockIdx.x * W, c1 = min(C, c0 + W);\n";
    // every block read xgen before the grid barrier above: publish it
    o << "    if (blockIdx.x == 0 && threadIdx.x == 0) *(volatile unsigned int*)(X + " << kXGen << ") = xgen;\n";
    o << "    const int par = (int)(xgen & 1u);\n";
    o << "    for (int q = 0; q < XW; ++q) {\n";
    o << "      float* dst = (float*)(__ldcg((const unsigned long long*)X + q) + " << kXSlots
      << "ULL) + ((long long)(par * XW + XR) * NCR) * C;\n";
    o << "      for (long long col = c0 + threadIdx.x; col < c1; col += blockDim.x)\n";
    o << "#pragma unroll\n        for (int r = 0; r < NCR; ++r) dst[r * C + col] = colpart[r * C + col];\n";
    o << "    }\n";
    o << "    __threadfence_system();\n";
    o << "    as::grid_barrier(bar);\n";
    o << "    if (blockIdx.x == 0 && threadIdx.x < XW)\n";
    o << "      as::st_release_sys((unsigned int*)(__ldcg((const unsigned long long*)X + threadIdx.x) + " << kXFlags
      << "ULL) + XR, xgen);\n";
    o << "    if (threadIdx.x == 0) as::wait_flags((const unsigned int*)(X + " << kXFlags << "), XW, xgen, (unsigned int*)(X + "
      << kXErr << "));\n";
    o << "    __syncthreads();\n";
    o << "    const float* slots = (const float*)(X + " << kXSlots << ") + (long long)par * XW * NCR * C;\n";
    o << "    for (long long col = c0 + threadIdx.x; col < c1; col += blockDim.x) {\n";
    for (int q = 0; q < ncr; ++q) {
      int id = p.colreds[q];
      bool mx = N(id).sub == ASTITCH_RMAX;
      o << "      float t" << id << " = " << (mx ? "-AS_INF" : "0.f") << ";\n";
      o << "      for (int q = 0; q < XW; ++q) { const float x_ = as::ld_cg(slots + ((long long)q * NCR + " << q
        << ") * C + col); t" << id << " = " << (mx ? "as::nmax(t" + std::to_string(id) + ", x_)" : "t" + std::to_string(id) + " + x_")
        << "; }\n";
    }
    emit_colvec_chain("t");
    o << "    }\n  }\n";
  }

  // COLVEC chain for one column `col` given totals t<id> of the column
  // reductions finalised at this barrier (level cur_level + 1); values of
  // earlier barriers are read back from the workspace, level-0 ones recomputed
  int post_index(int id) const {
    for (size_t q = 0; q < p.post_colvecs.size(); ++q)
      if (p.post_colvecs[q] == id) return static_cast<int>(q);
    return -1;
  }
  void emit_colvec_chain(const std::string& tpref) {
    const int lv = cur_level + 1;
    for (size_t ii = 0; ii < g.nodes.size(); ++ii) {
      int i = static_cast<int>(ii);
      const Node& nd = N(i);
      if (!I(i).live || nd.kind != ASTITCH_COLVEC) continue;
      if (I(i).level > lv) continue;
      std::string id = std::to_string(i);
      if (I(i).level >= 1 && I(i).level < lv) {
        o << "        const float x" << id << " = as::ld_cg((const float*)((const char*)p.ws + " << p.ws.colvals
          << "LL) + " << post_index(i) << "LL * C + col);\n";
        if (pc(i))  // R7c: the fp64 value = hi + lo
          o << "        const double x" << id << "d = (double)x" << id << " + (double)as::ld_cg((const float*)((const char*)p.ws + "
            << colvals_lo() << "LL) + " << post_index(i) << "LL * C + col);\n";
      } else if (pc(i)) {  // R7c: the per-column chain of a precise value in fp64
        if (nd.type == NodeType::Reduce)
          o << "        const double x" << id << "d = " << tpref << id << "d;\n";
        else if (nd.type == NodeType::Unary)
          o << "        const double x" << id << "d = " << (nd.sub == ASTITCH_NEG ? "-" : "fabs") << "(" << xdref(nd.a) << ");\n";
        else
          o << "        const double x" << id << "d = " << xdbinop(nd.sub, nd.a, nd.b) << ";\n";
        o << "        const float x" << id << " = (float)x" << id << "d;\n";
      } else if (nd.type == NodeType::Reduce) {
        o << "        const float x" << id << " = " << tpref << id << ";\n";
      } else if (nd.type == NodeType::Input) {
        o << "        const float x" << id << " = as::ld_scalar<" << dt_code(nd.dtype) << ">(p.in[" << nd.input_index
          << "], col);\n";
      } else if (nd.type == NodeType::Unary) {
        o << "        const float x" << id << " = " << unop(nd.sub, xref(nd.a)) << ";\n";
      } else if (nd.type == NodeType::Binary) {
        o << "        const float x" << id << " = " << binop(nd.sub, nd.b, xref(nd.a), xref(nd.b)) << ";\n";
      }
    }
    for (size_t k = 0; k < g.outputs.size(); ++k) {
      int id = g.outputs[k];
      if (N(id).kind != ASTITCH_COLVEC || I(id).level != lv) continue;
      o << "        as::st_scalar<" << dt_code(g.output_dtypes[k]) << ">(p.out[" << k << "], col, x" << id << ");\n";
    }
    for (size_t q = 0; q < p.post_colvecs.size(); ++q) {
      int id = p.post_colvecs[q];
      if (I(id).level != lv || !read_later(id)) continue;
      o << "        ((float*)((char*)p.ws + " << p.ws.colvals << "LL))[" << q << "LL * C + col] = x" << id << ";\n";
      if (pc(id))
        o << "        ((float*)((char*)p.ws + " << colvals_lo() << "LL))[" << q << "LL * C + col] = (float)(x" << id
          << "d - (double)x" << id << ");\n";
    }
  }
  // is post-barrier COLVEC value id read by a later sweep or a later level's
  // column chain?  (only then is it published to the workspace)
  bool read_later(int id) const {
    const int lv = I(id).level;
    for (int u : I(id).consumers) {
      if (!I(u).live) continue;
      const Node& un = N(u);
      if (un.type == NodeType::Bcast) {
        for (int w : I(u).consumers)
          if (I(w).live && last_run(w) >= lv) return true;
        continue;
      }
      if (un.kind == ASTITCH_COLVEC) {
        if (I(u).level > lv) return true;       // a later level's column chain reads it back
        if (read_later(u)) return true;         // same level: computed from it, recursively
        continue;
      }
      if (last_run(u) >= lv) return true;       // FULL / ROWVEC consumer in a later sweep
    }
    return false;
  }
  std::string xdref(int i) const {
    if (N(i).type == NodeType::Const) {
      char buf[64];
      snprintf(buf, sizeof(buf), "%a", N(i).cval);
      return std::string("(") + buf + ")";
    }
    if (pc(i)) return "x" + std::to_string(i) + "d";
    return "(double)x" + std::to_string(i);
  }
  std::string xdbinop(int op, int a, int b) const {
    std::string x = xdref(a), y = xdref(b);
    switch (op) {
      case ASTITCH_ADD: return "(" + x + " + " + y + ")";
      case ASTITCH_SUB: return "(" + x + " - " + y + ")";
      case ASTITCH_MUL: return "(" + x + " * " + y + ")";
      case ASTITCH_DIV: return "(" + x + " / " + y + ")";
      case ASTITCH_MAX: return "as::dmaxn(" + x + ", " + y + ")";
      case ASTITCH_MIN: return "as::dminn(" + x + ", " + y + ")";
    }
    return x;
  }
  std::string xref(int i) const {
    if (N(i).type == NodeType::Const) return "k" + std::to_string(i);
    return "x" + std::to_string(i);
  }

  // pre-barrier COLVEC outputs (not from a column reduction): block 0 writes them
  void emit_pre_colvec_outputs() {
    bool any = false;
    for (size_t k = 0; k < g.outputs.size(); ++k)
      if (N(g.outputs[k]).kind == ASTITCH_COLVEC && !I(g.outputs[k]).post) any = true;
    if (!any) return;
    o << "  if (blockIdx.x == 0) {\n    for (long long col = threadIdx.x; col < C; col += blockDim.x) {\n";
    for (size_t ii = 0; ii < g.nodes.size(); ++ii) {
      int i = static_cast<int>(ii);
      const Node& nd = N(i);
      if (!I(i).live || nd.kind != ASTITCH_COLVEC || I(i).post) continue;
      std::string id = std::to_string(i);
      if (nd.type == NodeType::Input)
        o << "      const float x" << id << " = as::ld_scalar<" << dt_code(nd.dtype) << ">(p.in[" << nd.input_index
          << "], col);\n";
      else if (nd.type == NodeType::Unary)
        o << "      const float x" << id << " = " << unop(nd.sub, xref(nd.a)) << ";\n";
      else if (nd.type == NodeType::Binary)
        o << "      const float x" << id << " = " << binop(nd.sub, nd.b, xref(nd.a), xref(nd.b)) << ";\n";
    }
    for (size_t k = 0; k < g.outputs.size(); ++k) {
      int id = g.outputs[k];
      if (N(id).kind != ASTITCH_COLVEC || I(id).post) continue;
      o << "      as::st_scalar<" << dt_code(g.output_dtypes[k]) << ">(p.out[" << k << "], col, x" << id << ");\n";
    }
    o << "    }\n  }\n";
  }

  // ------------------------------------------------------------ packed tile
  void emit_packed(const std::string& name) {
    header(name, false);
    collect_streams(false);
    const int S = m.stages, TR = m.tile_rows;
    // stage layout: input tiles, then output tiles (outputs written in place
    // over an input tile of the same element size when possible)
    std::vector<long long> in_off(streams.size()), in_bytes(streams.size());
    long long off = 0;
    for (size_t s = 0; s < streams.size(); ++s) {
      in_bytes[s] = static_cast<long long>(C) * dtype_size(streams[s].dt);
      in_off[s] = off;
      off += ((TR * in_bytes[s] + 127) / 128) * 128;
    }
    std::vector<long long> out_off(g.outputs.size(), -1), out_bytes(g.outputs.size(), 0);
    std::vector<bool> in_used(streams.size(), false);
    for (size_t k = 0; k < g.outputs.size(); ++k) {
      if (N(g.outputs[k]).kind != ASTITCH_FULL) continue;
      out_bytes[k] = static_cast<long long>(C) * dtype_size(g.output_dtypes[k]);
      for (size_t s = 0; s < streams.size(); ++s)
        if (!in_used[s] && in_bytes[s] == out_bytes[k]) {
          in_used[s] = true;
          out_off[k] = in_off[s];
          break;
        }
      if (out_off[k] < 0) {
        out_off[k] = off;
        off += ((TR * out_bytes[k] + 127) / 128) * 128;
      }
    }
    const long long stage_bytes = off;
    o << "  extern __shared__ __align__(128) unsigned char smem[];\n";
    o << "  constexpr int S = " << S << ", TR = " << TR << ";\n";
    o << "  constexpr long long STAGE = " << stage_bytes << "LL;\n";
    o << "  const u32 sbase = as::smem_addr(smem);\n";
    o << "  const u32 bars = sbase + (u32)(S * STAGE);\n";
    o << "  const long long ntiles = (R + TR - 1) / TR;\n";
    o << "  if (threadIdx.x == 0) { for (int s = 0; s < S; ++s) as::mbar_init(bars + 8 * s, 1); as::fence_mbar_init(); }\n";
    o << "  __syncthreads();\n";
    o << "  const int warp = threadIdx.x >> 5, wl = threadIdx.x & 31; (void)wl;\n";
    emit_colvecs(false);
    // producer: warp 0 issues the TMA bulk copies of one tile into stage s.
    // Unmasked: one contiguous copy per input.  Masked (key padding): one copy
    // per row of only its valid prefix (rounded up to whole 16-byte chunks), so
    // the padded tail is never read from HBM.
    o << "  auto issue = [&](long long t, int s) {\n";
    o << "    const long long r0 = t * TR; const long long nr = min((long long)TR, R - r0);\n";
    long long per_row = 0;
    for (size_t s = 0; s < streams.size(); ++s) per_row += in_bytes[s];
    if (!masked) {
      o << "    if (wl == 0) {\n";
      o << "      as::mbar_expect_tx(bars + 8 * s, (u32)(nr * " << per_row << "LL));\n";
      for (size_t s = 0; s < streams.size(); ++s)
        o << "      as::bulk_g2s(sbase + (u32)(s * STAGE + " << in_off[s] << "LL), (const char*)p.in["
          << N(streams[s].node).input_index << "] + r0 * " << in_bytes[s] << "LL, (u32)(nr * " << in_bytes[s]
          << "LL), bars + 8 * s);\n";
      o << "    }\n";
    } else {
      o << "    u32 tot = 0;\n";
      o << "    for (int q = wl; q < TR; q += 32) {\n";
      o << "      if (q < nr) {\n        const long long Lr = " << lim_expr("(r0 + q)") << ";\n";
      o << "        const long long nch = (Lr + E - 1) / E;\n";
      for (size_t s = 0; s < streams.size(); ++s) {
        int es = dtype_size(streams[s].dt);
        o << "        tot += (u32)min((long long)" << in_bytes[s] << ", ((nch * E * " << es << " + 15) / 16) * 16);\n";
      }
      o << "      }\n    }\n";
      o << "    tot = __reduce_add_sync(0xffffffffu, tot);\n";
      o << "    if (wl == 0) as::mbar_expect_tx(bars + 8 * s, tot);\n";
      o << "    __syncwarp();\n";
      o << "    for (int q = wl; q < nr; q += 32) {\n";
      o << "      const long long Lr = " << lim_expr("(r0 + q)") << ";\n";
      o << "      const long long nch = (Lr + E - 1) / E;\n";
      for (size_t s = 0; s < streams.size(); ++s) {
        int es = dtype_size(streams[s].dt);
        o << "      { const u32 nbq = (u32)min((long long)" << in_bytes[s] << ", ((nch * E * " << es
          << " + 15) / 16) * 16);\n";
        o << "        if (nbq) as::bulk_g2s(sbase + (u32)(s * STAGE + " << in_off[s] << "LL + q * " << in_bytes[s]
          << "LL), (const char*)p.in[" << N(streams[s].node).input_index << "] + (r0 + q) * " << in_bytes[s]
          << "LL, nbq, bars + 8 * s); }\n";
      }
      o << "    }\n";
    }
    o << "  };\n";
    o << "  const int DIST = S - 2;\n";
    o << "  if (warp == 0) for (int k = 0; k < DIST; ++k) { long long t = blockIdx.x + (long long)k * gridDim.x; if (t < ntiles) issue(t, k); }\n";
    o << "  int k = 0;\n";
    o << "  for (long long t = blockIdx.x; t < ntiles; t += gridDim.x, ++k) {\n";
    o << "    const int st = k % S; const u32 ph = (u32)((k / S) & 1);\n";
    o << "    if (warp == 0) {\n      if (wl == 0) as::bulk_wait_read<1>();\n      __syncwarp();\n";
    o << "      const long long tn = t + (long long)DIST * gridDim.x;\n";
    o << "      if (tn < ntiles) issue(tn, (k + DIST) % S);\n    }\n";
    o << "    as::mbar_wait(bars + 8 * st, ph);\n";
    o << "    const long long r0 = t * TR; const long long nr = min((long long)TR, R - r0);\n";
    // consumers: a team of T lanes per row; rows of the tile strided by the
    // number of teams (TR is a multiple of it, so the loop is warp-uniform)
    o << "    for (int rr = team; rr < TR; rr += RPB) {\n";
    o << "      const bool act_u0 = rr < nr; const long long row_u0 = r0 + rr; (void)row_u0;\n";
    o << "      const int lim_u0 = " << (masked ? "act_u0 ? " + lim_expr("row_u0") + " : 0" : "(int)C")
      << "; (void)lim_u0;\n";
    // loads from smem (chunks of the valid prefix only when masked)
    for (size_t s = 0; s < streams.size(); ++s) {
      int nbs = nb(streams[s].dt);
      std::string cond = "act_u0";
      if (masked || !exact) cond += " && (j * T + lane) * E < lim_u0";
      o << "      as::Raw<" << nbs << "> r" << s << "_u0[V];\n";
      o << "#pragma unroll\n      for (int j = 0; j < V; ++j) r" << s << "_u0[j] = (" << cond << ") ? as::lds_chunk<"
        << nbs << ">(sbase + (u32)(st * STAGE + " << in_off[s] << "LL + rr * " << in_bytes[s]
        << "LL + (j * T + lane) * " << nbs << ")) : as::Raw<" << nbs << ">{};\n";
    }
    o << "      {\n";
    emit_unpack("_u0", "lim_u0");
    emit_colvecs(true);
    emit_rowvec_inputs(false, "_u0", "row_u0", "act_u0");
    emit_body(false, "_u0", "row_u0", "act_u0", "lim_u0");
    // FULL outputs to smem; ROWVEC outputs direct
    for (size_t k = 0; k < g.outputs.size(); ++k) {
      int id = g.outputs[k];
      astitch_dtype dt = g.output_dtypes[k];
      if (N(id).kind == ASTITCH_FULL) {
        int nbo = nb(dt);
        o << "      if (act_u0) {\n#pragma unroll\n        for (int j = 0; j < V; ++j) {\n";
        std::string val = ref(id, "(j * E + e)", "_u0");
        o << "          float t_[E];\n";
        if (masked) {
          o << "          if ((j + 1) * T * E <= lim_u0) {\n#pragma unroll\n            for (int e = 0; e < E; ++e) t_[e] = "
            << val << ";\n          } else {\n#pragma unroll\n            for (int e = 0; e < E; ++e) t_[e] = ("
            << col_expr("j", "e") << " < lim_u0) ? " << val << " : 0.f;\n          }\n";
        } else {
          o << "#pragma unroll\n          for (int e = 0; e < E; ++e) t_[e] = " << val << ";\n";
        }
        if (!exact) o << "          if ((long long)(j * T + lane) < CH)\n";
        o << "          as::sts_chunk<" << nbo << ">(sbase + (u32)(st * STAGE + " << out_off[k] << "LL + rr * "
          << out_bytes[k] << "LL + (j * T + lane) * " << nbo << "), as::Conv<" << dt_code(dt) << ", E>::pack(t_));\n";
        o << "        }\n      }\n";
      } else if (N(id).kind == ASTITCH_ROWVEC) {
        o << "      if (act_u0 && lane == 0) as::st_scalar<" << dt_code(dt) << ">(p.out[" << k << "], row_u0, s" << id
          << "_u0);\n";
      }
    }
    o << "      }\n    }\n";
    o << "    as::fence_proxy_async_smem();\n    __syncthreads();\n";
    o << "    if (threadIdx.x == 0) {\n";
    for (size_t k = 0; k < g.outputs.size(); ++k) {
      if (N(g.outputs[k]).kind != ASTITCH_FULL) continue;
      o << "      as::bulk_s2g((char*)p.out[" << k << "] + r0 * " << out_bytes[k] << "LL, sbase + (u32)(st * STAGE + "
        << out_off[k] << "LL), (u32)(nr * " << out_bytes[k] << "LL));\n";
    }
    o << "      as::bulk_commit();\n    }\n  }\n";
    o << "  if (threadIdx.x == 0) as::bulk_wait_all();\n";
    o << "}\n";
  }

  // ------------------------------------------------------------ row stream
  // Rows longer than the team's registers (planner: RowStream).  A team (a
  // block, or a cluster when rows are few) owns a row and walks it in column
  // tiles of T lanes x V chunks.  Row-local levels: rl(v) = number of row
  // reductions on v's dependency path.  Pass p re-reads the tile's inputs,
  // recomputes the FULL values of levels <= p, accumulates the row reductions
  // of level p (per-lane fp32 / fp64 accumulators in tile order, then one
  // team reduction) and stores the FULL outputs of level p; the row scalars
  // of level p+1 are then computed in registers.  Deterministic (fixed tile
  // order and trees).
  std::vector<int> rl;
  void compute_row_levels() {
    const int n = static_cast<int>(g.nodes.size());
    rl.assign(n, 0);
    for (int i = 0; i < n; ++i) {
      const Node& nd = N(i);
      int lv = 0;
      for (int a : {nd.a, nd.b}) {
        if (a < 0) continue;
        lv = std::max(lv, rl[a] + (I(a).cls == OpClass::ReduceRow ? 1 : 0));
      }
      rl[i] = lv;
    }
  }
  // values pass `pass` of a streamed row needs: its reductions' operands and
  // its FULL outputs, closed backwards over FULL values; COLVEC operands in *cv
  std::vector<bool> stream_need(int pass, int n, std::vector<bool>* cv = nullptr) const {
    std::vector<bool> need(n, false), need_cv(n, false);
    for (int i = 0; i < n; ++i)
      if (I(i).live && I(i).cls == OpClass::ReduceRow && rl[i] == pass) need[N(i).a] = true;
    for (size_t k = 0; k < g.outputs.size(); ++k)
      if (N(g.outputs[k]).kind == ASTITCH_FULL && rl[g.outputs[k]] == pass) need[g.outputs[k]] = true;
    for (int i = n - 1; i >= 0; --i) {
      if (!need[i]) continue;
      const Node& nd = N(i);
      if (nd.type == NodeType::Bcast) {
        if (nd.axis == ASTITCH_AXIS_COL) need_cv[nd.a] = true;
        continue;
      }
      for (int a : {nd.a, nd.b}) {
        if (a < 0) continue;
        if (N(a).kind == ASTITCH_FULL) need[a] = true;
        else if (N(a).kind == ASTITCH_COLVEC) need_cv[a] = true;
      }
    }
    for (int i = n - 1; i >= 0; --i)  // COLVEC closure
      if (need_cv[i])
        for (int a : {N(i).a, N(i).b})
          if (a >= 0 && N(a).kind == ASTITCH_COLVEC) need_cv[a] = true;
    if (cv) *cv = need_cv;
    return need;
  }

  // ROWVEC value i (not an input) computed from row scalars
  void emit_stream_rowvec(int i) {
    const Node& nd = N(i);
    std::string id = std::to_string(i);
    if (precise[i]) {
      o << "    const double d" << id << " = ";
      if (nd.type == NodeType::Unary) o << (nd.sub == ASTITCH_NEG ? "-" : "fabs") << "(" << dref(nd.a, "") << ");\n";
      else o << dbinop(nd.sub, nd.a, nd.b, "") << ";\n";
      emit_split(id, "");
      return;
    }
    if (nd.type == NodeType::Unary) o << "    const float s" << id << " = " << unop(nd.sub, sref(nd.a, "")) << ";\n";
    else o << "    const float s" << id << " = " << binop(nd.sub, nd.b, sref(nd.a, ""), sref(nd.b, "")) << ";\n";
  }
  void emit_stream_rowvec_output(int i) {
    for (size_t k = 0; k < g.outputs.size(); ++k)
      if (g.outputs[k] == i)
        o << "    if (lane == 0) as::st_scalar<" << dt_code(g.output_dtypes[k]) << ">(p.out[" << k << "], row, s"
          << i << ");\n";
  }
  void emit_stream(const std::string& name) {
    header(name, false);
    compute_row_levels();
    const int n = static_cast<int>(g.nodes.size());
    int P = 1;
    for (int i = 0; i < n; ++i)
      if (I(i).live && N(i).kind == ASTITCH_FULL && N(i).type != NodeType::Bcast) P = std::max(P, rl[i] + 1);
    std::vector<int> fin;  // live FULL inputs
    for (int id : g.inputs)
      if (N(id).kind == ASTITCH_FULL && I(id).live) fin.push_back(id);
    for (size_t s = 0; s < fin.size(); ++s) {
      std::string rt = "as::Raw<" + std::to_string(nb(N(fin[s]).dtype)) + ">";
      o << "  const " << rt << "* __restrict__ gs" << s << " = (const " << rt << "*)p.in[" << N(fin[s]).input_index
        << "];\n";
    }
    emit_pre_colvec_outputs();
    // (staged rows) first pass that reads each FULL input: it loads from HBM
    // and keeps the lane's raw chunks in smem for the later passes
    std::vector<int> first_pass(n, -1);
    std::vector<long long> soff(fin.size(), 0);
    if (m.stage_row) {
      o << "  extern __shared__ __align__(16) unsigned char smem[];\n";
      o << "  const u32 sbase = as::smem_addr(smem);\n";
    }
    o << "  constexpr long long TCH = (long long)T * V;            // chunks per tile\n";
    o << "  constexpr long long NT = (CH + TCH - 1) / TCH;          // tiles per row\n";
    if (m.stage_row) {
      const long long tch = static_cast<long long>(m.team) * V;
      const long long nt = (C / E + tch - 1) / tch;
      long long off = 0;
      for (size_t s = 0; s < fin.size(); ++s) {
        soff[s] = off;
        off += nt * V * m.threads * nb(N(fin[s]).dtype);
      }
      for (int pass = 0; pass < P; ++pass) {
        std::vector<bool> need = stream_need(pass, n);
        for (size_t s = 0; s < fin.size(); ++s)
          if (need[fin[s]] && first_pass[fin[s]] < 0) first_pass[fin[s]] = pass;
      }
    }
    o << "  for (long long row = UNIT; row < (long long)R; row += NUNITS) {\n";
    // ROWVEC inputs and level-0 row scalars
    for (int id : g.inputs)
      if (N(id).kind == ASTITCH_ROWVEC && I(id).live)
        o << "    const float s" << id << " = as::ld_scalar<" << dt_code(N(id).dtype) << ">(p.in[" << N(id).input_index
          << "], row);\n";
    for (int i = 0; i < n; ++i)
      if (I(i).live && N(i).kind == ASTITCH_ROWVEC && rl[i] == 0 && N(i).type != NodeType::Input &&
          N(i).type != NodeType::Reduce)
        emit_stream_rowvec(i);
    for (int i = 0; i < n; ++i)
      if (I(i).live && N(i).kind == ASTITCH_ROWVEC && rl[i] == 0 && N(i).type != NodeType::Reduce)
        emit_stream_rowvec_output(i);
    for (int pass = 0; pass < P; ++pass) {
      // what this pass needs: its reductions' operands and its FULL outputs,
      // closed backwards over FULL values (row / column scalars are at hand)
      std::vector<bool> need_cv;
      std::vector<bool> need = stream_need(pass, n, &need_cv);
      std::vector<int> reds;
      for (int i = 0; i < n; ++i)
        if (I(i).live && I(i).cls == OpClass::ReduceRow && rl[i] == pass) reds.push_back(i);
      std::vector<int> fouts;
      for (size_t k = 0; k < g.outputs.size(); ++k) {
        int id = g.outputs[k];
        if (N(id).kind == ASTITCH_FULL && rl[id] == pass) fouts.push_back(static_cast<int>(k));
      }
      o << "    // ---- pass " << pass << ": " << reds.size() << " row reduction(s), " << fouts.size()
        << " FULL output(s)\n";
      for (int r : reds) {
        if (precise[r]) o << "    double ad" << r << " = 0.0;\n";
        else o << "    float a" << r << " = " << (N(r).sub == ASTITCH_RMAX ? "-AS_INF" : "0.f") << ";\n";
      }
      o << "    for (long long t = 0; t < NT; ++t) {\n";
      o << "      const long long TOFF = t * TCH * E;  // first column of the tile\n";
      tile_off = "TOFF";
      for (size_t s = 0; s < fin.size(); ++s) {
        int id = fin[s];
        if (!need[id]) continue;
        std::string rt = "as::Raw<" + std::to_string(nb(N(id).dtype)) + ">";
        o << "      " << rt << " r" << s << "[V];\n";
        o << "#pragma unroll\n      for (int j = 0; j < V; ++j) {\n";
        o << "        const long long ch = t * TCH + j * T + lane;\n";
        if (m.stage_row) {
          const int nbs = nb(N(id).dtype);
          o << "        const u32 sa = sbase + (u32)(" << soff[s] << "LL + ((t * V + j) * (long long)blockDim.x + threadIdx.x) * "
            << nbs << ");\n";
          if (first_pass[id] == pass) {
            o << "        r" << s << "[j] = (ch < CH) ? as::ldg(gs" << s << " + row * CH + ch) : " << rt << "{};\n";
            o << "        if (ch < CH) as::sts_chunk<" << nbs << ">(sa, r" << s << "[j]);  // stage for later passes\n";
          } else {
            o << "        r" << s << "[j] = (ch < CH) ? as::lds_chunk<" << nbs << ">(sa) : " << rt << "{};\n";
          }
        } else {
          o << "        r" << s << "[j] = (ch < CH) ? as::ldg(gs" << s << " + row * CH + ch) : " << rt << "{};\n";
        }
        o << "      }\n";
        o << "      float v" << id << "[NE];\n";
        o << "#pragma unroll\n      for (int j = 0; j < V; ++j) as::Conv<" << dt_code(N(id).dtype) << ", E>::unpack(r" << s
          << "[j], v" << id << " + j * E);\n";
      }
      // COLVEC operands of the tile (inputs through L1, EW on them)
      for (int i = 0; i < n; ++i) {
        if (!need_cv[i] || !I(i).live) continue;
        const Node& nd = N(i);
        o << "      float c" << i << "[NE];\n";
        if (nd.type == NodeType::Input) {
          std::string rt = "as::Raw<" + std::to_string(nb(nd.dtype)) + ">";
          o << "#pragma unroll\n      for (int j = 0; j < V; ++j) {\n";
          o << "        const long long ch = t * TCH + j * T + lane;\n";
          o << "        const " << rt << " rc_ = (ch < CH) ? as::ldg_l1((const " << rt << "*)p.in[" << nd.input_index
            << "] + ch) : " << rt << "{};\n";
          o << "        as::Conv<" << dt_code(nd.dtype) << ", E>::unpack(rc_, c" << i << " + j * E);\n      }\n";
        } else {
          o << "#pragma unroll\n      for (int k = 0; k < NE; ++k) c" << i << "[k] = ";
          if (nd.type == NodeType::Unary) o << unop(nd.sub, ref(nd.a, "k", "")) << ";\n";
          else o << binop(nd.sub, nd.b, ref(nd.a, "k", ""), ref(nd.b, "k", "")) << ";\n";
        }
      }
      // FULL values of levels <= pass (recomputed)
      for (int i = 0; i < n; ++i) {
        const Node& nd = N(i);
        if (!need[i] || !I(i).live || nd.kind != ASTITCH_FULL || nd.type == NodeType::Input ||
            nd.type == NodeType::Bcast)
          continue;
        if (row_div(i)) o << "      " << row_div_decl(i, "") << "\n";
        o << "      float v" << i << "[NE];\n";
        o << "#pragma unroll\n      for (int k = 0; k < NE; ++k) v" << i << "[k] = " << full_expr(i, "") << ";\n";
      }
      // row reductions of this level: per-lane accumulation in tile order
      const bool tail = (C % (static_cast<long long>(m.team) * V * E)) != 0;
      for (int r : reds) {
        bool mx = N(r).sub == ASTITCH_RMAX;
        std::string ident = mx ? "-AS_INF" : "0.f";
        o << "      {\n        float t_[NE];\n#pragma unroll\n        for (int k = 0; k < NE; ++k) t_[k] = ";
        if (tail) o << "(" << col_expr("(k / E)", "(k % E)") << " < C) ? " << ref(N(r).a, "k", "") << " : " << ident << ";\n";
        else o << ref(N(r).a, "k", "") << ";\n";
        if (precise[r]) o << "        ad" << r << " += as::TreeD<NE>::reduce(t_);\n";
        else if (mx) o << "        a" << r << " = as::nmax(a" << r << ", as::Tree<NE, true>::reduce(t_));\n";
        else o << "        a" << r << " += as::TreeSum<NE>::reduce(t_);\n";
        o << "      }\n";
      }
      // FULL outputs of this level
      for (int k : fouts) {
        int id = g.outputs[k];
        astitch_dtype dt = g.output_dtypes[k];
        std::string rt = "as::Raw<" + std::to_string(nb(dt)) + ">";
        o << "#pragma unroll\n      for (int j = 0; j < V; ++j) {\n";
        o << "        const long long ch = t * TCH + j * T + lane;\n";
        o << "        float t_[E];\n#pragma unroll\n        for (int e = 0; e < E; ++e) t_[e] = " << ref(id, "(j * E + e)", "")
          << ";\n";
        o << "        if (ch < CH) as::stg((" << rt << "*)p.out[" << k << "] + row * CH + ch, as::Conv<" << dt_code(dt)
          << ", E>::pack(t_));\n      }\n";
      }
      tile_off.clear();
      o << "    }\n";
      // team reductions -> row scalars of level pass+1
      for (int r : reds) {
        bool mx = N(r).sub == ASTITCH_RMAX;
        std::string id = std::to_string(r);
        if (precise[r]) {
          o << "    double d" << id << ";\n    {\n      double r_ = ad" << id << ";\n";
          if (split)
            o << "      r_ = as::cluster_team_sum_d<" << m.threads << ", " << m.split << ">(r_, red_scratch_d, &cl_slot_d["
              << rowred_index(r) << "]);\n";
          else o << "      r_ = as::block_team_sum_d<T>(r_, red_scratch_d);\n";
          o << "      d" << id << " = r_;\n    }\n";
          emit_split(id, "");
        } else {
          o << "    float s" << id << ";\n    {\n      float r_ = a" << id << ";\n";
          if (split)
            o << "      r_ = as::cluster_team_reduce<" << m.threads << ", " << m.split << ", " << (mx ? "true" : "false")
              << ">(r_, red_scratch, &cl_slot[" << rowred_index(r) << "]);\n";
          else o << "      r_ = as::block_team_reduce<T, " << (mx ? "true" : "false") << ">(r_, red_scratch);\n";
          o << "      s" << id << " = r_;\n    }\n";
        }
        emit_stream_rowvec_output(r);
      }
      for (int i = 0; i < n; ++i)
        if (I(i).live && N(i).kind == ASTITCH_ROWVEC && rl[i] == pass + 1 && N(i).type != NodeType::Reduce &&
            N(i).type != NodeType::Input) {
          emit_stream_rowvec(i);
          emit_stream_rowvec_output(i);
        }
    }
    o << "  }\n}\n";
  }

  // ------------------------------------------------------------ roles
  std::string run(const std::string& name) {
    if (m.tmpl == Template::RowTeam && m.tma_team) {
      emit_tma_team(name);
      return o.str();
    }
    if (m.tmpl == Template::PackedTile) {
      emit_packed(name);
      return o.str();
    }
    if (m.tmpl == Template::RowStream) {
      emit_stream(name);
      return o.str();
    }
    if (role == ROLE_SHARD_FINAL) {
      // small epilogue: one thread per column, consumers of the all-reduced
      // column totals (sharded global stage)
      o << "#include \"astitch_device.cuh\"\n";
      o << "struct Params { const void* in[16]; void* out[16]; void* ws; long long rows; long long row_offset; int flags; void* xbuf; unsigned int gen; };\n";
      o << "extern \"C\" __global__ void __launch_bounds__(256) " << name << "(const Params p) {\n";
      o << "  constexpr long long C = " << C << "LL;\n";
      for (size_t i = 0; i < g.nodes.size(); ++i)
        if (N(i).type == NodeType::Const && I(i).live)
          o << "  const float k" << i << " = " << flit(N(i).cval) << ";\n";
      o << "  const float* colpart = (const float*)((const char*)p.ws + "
        << (p.ws.colvals + p.post_colvecs.size() * C * 4) << "LL);\n";
      o << "  for (long long col = blockIdx.x * 256LL + threadIdx.x; col < C; col += gridDim.x * 256LL) {\n";
      for (size_t q = 0; q < p.colreds.size(); ++q) {
        if (N(p.colreds[q]).sub == ASTITCH_RMAX)  // int32 order keys (stage 0)
          o << "    const float t" << p.colreds[q] << " = as::okey_dec(((const int*)colpart)[" << q << "LL * C + col]);\n";
        else
          o << "    const float t" << p.colreds[q] << " = colpart[" << q << "LL * C + col];\n";
      }
      emit_colvec_chain("t");
      o << "  }\n}\n";
      return o.str();
    }
    header(name, m.tmpl == Template::GlobalSweep);
    if (m.tmpl == Template::GlobalSweep) {
      o << "  unsigned int* bar = (unsigned int*)((char*)p.ws + " << p.ws.barrier << "LL);\n  (void)bar;\n";
    }
    if (role == ROLE_FUSED) {
      // this run's generation: read by every block BEFORE the first grid
      // barrier, bumped in the buffer by block 0 after it (emit_fused_exchange),
      // so eager runs and CUDA-graph replays alike get a fresh generation; and
      // this run's wait status (set only after the grid barriers below)
      o << "  const unsigned int xgen = *(volatile unsigned int*)((unsigned char*)p.xbuf + " << kXGen << ") + 1u;\n";
      o << "  if (blockIdx.x == 0 && threadIdx.x == 0) *(volatile unsigned int*)((unsigned char*)p.xbuf + " << kXErr
        << ") = 0u;\n";
    }
    if (m.tma_sweep && role != ROLE_SHARD_SWEEP2) {
      // tma_sweep: per barrier level, a bulk-copy sweep -> CTA partials ->
      // grid barrier -> finalise (+ fused exchange) [-> grid barrier when a
      // later level reads what it published]
      emit_colvecs(false);
      emit_pre_colvec_outputs();
      emit_tma_prologue();
      const int D = p.max_level;
      auto colred_at = [&](int lv) {
        for (int id : p.colreds)
          if (phase_of(id) == lv) return true;
        return false;
      };
      auto sweep_at = [&](int lv) {
        if (lv == 0) return true;
        for (size_t i = 0; i < g.nodes.size(); ++i)
          if (I(i).live && I(i).level == lv && N(i).kind == ASTITCH_FULL) return true;
        for (size_t i = 0; i < g.nodes.size(); ++i)
          if (I(i).live && N(i).kind == ASTITCH_FULL && ((I(i).remat_mask >> lv) & 1u)) return true;
        return false;
      };
      auto later_work = [&](int lv) {
        for (int l = lv + 1; l <= D; ++l)
          if (sweep_at(l) || colred_at(l)) return true;
        return false;
      };
      for (int lv = 0; lv <= D; ++lv) {
        cur_level = lv;
        const bool colred_here = colred_at(lv), sweep_here = sweep_at(lv);
        if (!sweep_here && !colred_here) continue;
        o << "  {  // ---- level " << lv << "\n";
        if (lv > 0) emit_post_colvec_loads();
        emit_tma_level();
        if (colred_here) {
          o << "  as::grid_barrier(bar);\n";
          if (role == ROLE_SHARD_MAIN) {
            emit_column_finalize(false);
          } else if (role == ROLE_FUSED) {
            emit_column_finalize(false);
            emit_fused_exchange();
            if (later_work(lv)) o << "  as::grid_barrier(bar);\n";
          } else {
            emit_column_finalize(true);
            if (later_work(lv)) o << "  as::grid_barrier(bar);\n";
          }
        } else if (later_work(lv)) {
          o << "  as::grid_barrier(bar);\n";
        }
        o << "  }\n";
        if (role == ROLE_SHARD_MAIN) break;
      }
      emit_tma_epilogue();
      o << "}\n";
      return o.str();
    }
    if (role == ROLE_SHARD_SWEEP2) {  // sharded plans have one barrier level
      cur_level = 1;
      emit_colvecs(false);
      emit_post_colvec_loads();
      emit_sweep(true);
      o << "}\n";
      return o.str();
    }
    emit_colvecs(false);
    emit_pre_colvec_outputs();
    if (m.tmpl != Template::GlobalSweep) {
      cur_level = 0;
      emit_sweep(false);
      o << "}\n";
      return o.str();
    }
    // global stitching: sweep level 0 -> [partials -> barrier -> finalise
    // level 1 -> barrier -> sweep level 1 -> ...]: one grid barrier pair per
    // level of dependent column reductions
    const int D = p.max_level;
    auto colred_at = [&](int lv) {
      for (int id : p.colreds)
        if (phase_of(id) == lv) return true;
      return false;
    };
    auto sweep_at = [&](int lv) {
      if (lv == 0) return true;
      for (size_t i = 0; i < g.nodes.size(); ++i)
        if (I(i).live && I(i).level == lv && (N(i).kind == ASTITCH_FULL || N(i).kind == ASTITCH_ROWVEC)) return true;
      return false;
    };
    // a grid barrier after a level's column finalise only when a later level
    // reads what it published (a last level ends the kernel with no barrier)
    auto later_work = [&](int lv) {
      for (int l = lv + 1; l <= D; ++l)
        if (sweep_at(l) || colred_at(l)) return true;
      return false;
    };
    for (int lv = 0; lv <= D; ++lv) {
      cur_level = lv;
      const bool colred_here = colred_at(lv), sweep_here = sweep_at(lv);
      if (!sweep_here && !colred_here) continue;
      o << "  {  // ---- level " << lv << "\n";
      if (lv > 0) emit_post_colvec_loads();
      if (colred_here) emit_colred_acc_decl();
      emit_sweep(lv > 0);
      if (colred_here) {
        emit_block_partials();
        o << "  as::grid_barrier(bar);\n";
        if (role == ROLE_SHARD_MAIN) {
          emit_column_finalize(false);
        } else if (role == ROLE_FUSED) {
          emit_column_finalize(false);
          emit_fused_exchange();
          if (later_work(lv)) o << "  as::grid_barrier(bar);\n";
        } else {
          emit_column_finalize(true);
          if (later_work(lv)) o << "  as::grid_barrier(bar);\n";
        }
      } else if (later_work(lv)) {
        // FORCE_GLOBAL: row-reduction results of this level are in HBM
        o << "  as::grid_barrier(bar);\n";
      }
      o << "  }\n";
      if (role == ROLE_SHARD_MAIN) break;
    }
    o << "}\n";
    return o.str();
  }
};

}  // namespace

std::string generate_kernel(const Plan& p, int role, const std::string& name) {
  Gen gen(p, role);
  return gen.run(name);
}

}  // namespace astitch
