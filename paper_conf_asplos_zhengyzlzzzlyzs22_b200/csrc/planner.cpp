// Planner: the paper's Sec. 4 pipeline, re-derived for B200.
//
//   a1  classify ops (light / heavy EW, broadcast, row / column reduce)
//   a2  dominant candidates -> dominant merging -> op groups
//   a3  adaptive thread mapping (packing / splitting)
//   a4  schedule propagation (every op inherits its group's mapping)
//   a5  scheme finalisation (passive / proactive block locality)
//   a6  memory plan (smem per block, HBM workspace)
//   a7  launch configuration (assume-relax-apply register bound)
//
// Constants that the paper gives for V100 (1024-element split threshold,
// 1024-thread blocks, 160 blocks per wave) are recomputed from B200 limits
// (reading R15).
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <numeric>
#include <sstream>

#include "internal.h"

namespace astitch {

const char* opclass_name(OpClass c) {
  switch (c) {
    case OpClass::Input: return "input";
    case OpClass::Const: return "const";
    case OpClass::LightEW: return "light_ew";
    case OpClass::HeavyEW: return "heavy_ew";
    case OpClass::BcastRow: return "broadcast_row";
    case OpClass::BcastCol: return "broadcast_col";
    case OpClass::ReduceRow: return "reduce_row";
    case OpClass::ReduceCol: return "reduce_col";
  }
  return "?";
}

const char* scheme_name(Scheme s) {
  switch (s) {
    case Scheme::Independent: return "independent";
    case Scheme::Local: return "local";
    case Scheme::Regional: return "regional";
    case Scheme::Global: return "global";
  }
  return "?";
}

const char* template_name(Template t) {
  switch (t) {
    case Template::RowTeam: return "row_team";
    case Template::PackedTile: return "packed_tile";
    case Template::GlobalSweep: return "global_sweep";
    case Template::SplitRow: return "split_row";
    case Template::RowStream: return "row_stream";
  }
  return "?";
}

namespace {

// Heavy element-wise ops ("tanh, power, and log"; we add the other
// transcendental / division ops that cost a MUFU or a multi-instruction sequence).
bool is_heavy_unop(int op) {
  switch (op) {
    case ASTITCH_NEG:
    case ASTITCH_ABS: return false;
    default: return true;
  }
}
// Division is light: in Fig. 7(a)/9 divide.1 is not a dominant candidate while
// power.1 is, so only POW counts as a heavy binary op.
bool is_heavy_binop(int op) { return op == ASTITCH_POW; }

struct DSU {
  std::vector<int> p;
  explicit DSU(int n) : p(n) { std::iota(p.begin(), p.end(), 0); }
  int find(int x) { return p[x] == x ? x : p[x] = find(p[x]); }
  void unite(int a, int b) { p[find(a)] = find(b); }
};

}  // namespace

// ------------------------------------------------------------------------ a1/a2/a5
void analyse(Plan& p) {
  const Graph& g = p.g;
  const int n = static_cast<int>(g.nodes.size());
  p.info.assign(n, NodeInfo());
  auto& info = p.info;

  // consumers
  for (int i = 0; i < n; ++i) {
    const Node& nd = g.nodes[i];
    if (nd.a >= 0) info[nd.a].consumers.push_back(i);
    if (nd.b >= 0 && nd.b != nd.a) info[nd.b].consumers.push_back(i);
  }
  // liveness: reverse reachability from outputs
  std::function<void(int)> mark = [&](int i) {
    if (info[i].live) return;
    info[i].live = true;
    if (g.nodes[i].a >= 0) mark(g.nodes[i].a);
    if (g.nodes[i].b >= 0) mark(g.nodes[i].b);
  };
  for (int o : g.outputs) mark(o);
  if (g.lengths_node >= 0) info[g.lengths_node].live = true;
  if (g.segments_node >= 0) info[g.segments_node].live = true;

  // a1: classification
  for (int i = 0; i < n; ++i) {
    const Node& nd = g.nodes[i];
    OpClass c = OpClass::Input;
    switch (nd.type) {
      case NodeType::Input: c = OpClass::Input; break;
      case NodeType::Const: c = OpClass::Const; break;
      case NodeType::Unary: c = is_heavy_unop(nd.sub) ? OpClass::HeavyEW : OpClass::LightEW; break;
      case NodeType::Binary: c = is_heavy_binop(nd.sub) ? OpClass::HeavyEW : OpClass::LightEW; break;
      case NodeType::Reduce:
        c = nd.axis == ASTITCH_AXIS_ROW ? OpClass::ReduceRow : OpClass::ReduceCol;
        break;
      case NodeType::Bcast:
        c = nd.axis == ASTITCH_AXIS_ROW ? OpClass::BcastRow : OpClass::BcastCol;
        break;
    }
    info[i].cls = c;
  }

  // Barrier levels: a value's level is the number of column reductions on
  // its dependency path (each needs a grid barrier before it is usable);
  // values downstream of a column reduction run after the grid barrier.
  // A column reduction accumulates during the sweep of its operand's level.
  // FORCE_GLOBAL ablation (the paper's regional -> global demotion, P:L288;
  // Table 4 mirror): a row reduction's result is stored to HBM and its
  // consumers read it back after a grid barrier, so every consumer of a row
  // reduction sits one barrier level above it (FULL operands are re-read from
  // HBM or buffered there, like the values of a column-reduction level).
  const bool force_global = (p.desc.flags & ASTITCH_FLAG_FORCE_GLOBAL) != 0;
  p.colreds.clear();
  p.max_level = 0;
  auto operand_level = [&](int a) {
    if (a < 0) return 0;
    return info[a].level + ((force_global && info[a].cls == OpClass::ReduceRow) ? 1 : 0);
  };
  for (int i = 0; i < n; ++i) {
    const Node& nd = g.nodes[i];
    if (!info[i].live) continue;
    int lv = std::max(operand_level(nd.a), operand_level(nd.b));
    if (info[i].cls == OpClass::ReduceCol) {
      lv += 1;
      p.colreds.push_back(i);
    }
    info[i].level = lv;
    info[i].post = lv > 0;
    p.max_level = std::max(p.max_level, lv);
  }
  if (g.segments_node >= 0 && (!p.colreds.empty() || force_global || p.desc.shard_world > 1))
    throw Error{ASTITCH_ERR_UNSUPPORTED,
                "packed varlen segments support row-wise subgraphs only (no column reduction, "
                "FORCE_GLOBAL or sharding)"};
  if (p.max_level > 4)
    throw Error{ASTITCH_ERR_UNSUPPORTED, "more than 4 dependent column reductions (grid barriers)"};

  // Recomputation instead of an HBM buffer (reading R22).  A FULL element-wise
  // value read in a later barrier level (BatchNorm's centred x, Fig. 7(a)'s
  // power.1) is, in the paper's global scheme, written to HBM by its own
  // sweep and read back by the later one: 4 + 4 B per element in fp32.  When
  // the FULL inputs its element-wise cone starts from cost fewer bytes per
  // element than that, the later sweep re-reads those inputs and recomputes
  // the cone instead (row scalars and column values it needs are tiny
  // buffers).  Same ops in the same order as the buffered value (up to the
  // compiler's FMA contraction).  Off under FORCE_GLOBAL (the ablation
  // measures buffering) and with remat=0.
  auto phase = [&](int u) { return info[u].cls == OpClass::ReduceCol ? info[g.nodes[u].a].level : info[u].level; };
  if (p.max_level > 0 && !force_global && p.tune.remat != 0) {
    auto ew_full = [&](int v) {
      const Node& nd = g.nodes[v];
      return v >= 0 && info[v].live && nd.kind == ASTITCH_FULL &&
             (nd.type == NodeType::Unary || nd.type == NodeType::Binary);
    };
    for (int v = n - 1; v >= 0; --v) {
      if (!ew_full(v)) continue;
      unsigned later = 0;
      for (int u : info[v].consumers)
        if (info[u].live && g.nodes[u].type != NodeType::Bcast && info[u].cls != OpClass::ReduceCol &&
            phase(u) > info[v].level)
          later |= 1u << phase(u);
      later |= info[v].remat_mask;  // levels where a recomputed consumer needs it
      if (!later) continue;
      // the element-wise cone of v and the FULL inputs it starts from
      std::vector<int> cone, stack = {v};
      std::vector<bool> seen(n, false);
      std::vector<int> leaves;
      bool ok = true;
      while (!stack.empty() && ok) {
        int w = stack.back();
        stack.pop_back();
        if (w < 0 || seen[w]) continue;
        seen[w] = true;
        const Node& wn = g.nodes[w];
        if (ew_full(w)) {
          cone.push_back(w);
          stack.push_back(wn.a);
          stack.push_back(wn.b);
        } else if (wn.type == NodeType::Input && wn.kind == ASTITCH_FULL) {
          leaves.push_back(w);
        } else if (wn.kind == ASTITCH_FULL && wn.type != NodeType::Bcast) {
          ok = false;  // (not reached: FULL values are inputs, broadcasts or element-wise)
        }
      }
      if (!ok || cone.size() > 32) continue;
      int bytes = 0;
      for (int x : leaves) bytes += dtype_size(g.nodes[x].dtype);
      if (bytes >= 8) continue;  // the fp32 buffer's write + read is no more
      for (int w : cone) info[w].remat_mask |= later;
    }
  }

  // a2 step 1: dominant candidates = reduces, heavy EW followed by a broadcast,
  // and the outputs of the stitch op.
  std::vector<bool> is_output(n, false);
  for (int o : g.outputs) is_output[o] = true;
  for (int i = 0; i < n; ++i) {
    if (!info[i].live) continue;
    OpClass c = info[i].cls;
    bool cand = (c == OpClass::ReduceRow || c == OpClass::ReduceCol || is_output[i]);
    if (c == OpClass::HeavyEW) {
      for (int u : info[i].consumers)
        if (info[u].live && (info[u].cls == OpClass::BcastRow || info[u].cls == OpClass::BcastCol))
          cand = true;
    }
    // Reading R17: a value read after the grid barrier (by anything but the
    // column reduce that accumulates it) has a one-to-many dependency across
    // groups too, so it is a candidate (power.1 of Fig. 7(a)).
    if (c != OpClass::Input && c != OpClass::Const &&
        (g.nodes[i].kind == ASTITCH_FULL || g.nodes[i].kind == ASTITCH_ROWVEC)) {
      for (int u : info[i].consumers)
        if (info[u].live && info[u].level > info[i].level && info[u].cls != OpClass::ReduceCol) cand = true;
    }
    info[i].candidate = cand;
  }

  // a2 step 2: dominant merging / grouping.  Ops connected through local-only
  // paths share one schedule.  Two kinds of edges are cut: the
  // edge into a column reduction (its one-to-many dependency spans all rows,
  // so its consumers need the grid barrier) and any edge crossing that barrier.
  DSU dsu(n);
  for (int i = 0; i < n; ++i) {
    if (!info[i].live || info[i].cls == OpClass::Const) continue;
    const Node& nd = g.nodes[i];
    for (int src : {nd.a, nd.b}) {
      if (src < 0 || info[src].cls == OpClass::Const) continue;
      if (info[i].cls == OpClass::ReduceCol) continue;
      if (info[src].level < info[i].level) continue;
      dsu.unite(src, i);
    }
  }
  std::vector<int> gid(n, -1);
  p.groups.clear();
  for (int i = 0; i < n; ++i) {
    if (!info[i].live || info[i].cls == OpClass::Const || info[i].cls == OpClass::Input) continue;
    int r = dsu.find(i);
    if (gid[r] < 0) {
      gid[r] = static_cast<int>(p.groups.size());
      p.groups.emplace_back();
    }
    info[i].group = gid[r];
    p.groups[gid[r]].push_back(i);
  }
  for (int i = 0; i < n; ++i)
    if (info[i].live && info[i].cls == OpClass::Input && gid[dsu.find(i)] >= 0)
      info[i].group = gid[dsu.find(i)];

  // final dominant per group: prefer a reduction, column reduce first
  // (it fixes the whole sweep's mapping), then the first row reduce, then a
  // heavy-EW candidate, then an output.  Other candidates are sub-dominants.
  for (auto& grp : p.groups) {
    int best = -1, best_rank = 99;
    for (int i : grp) {
      if (!info[i].candidate) continue;
      int rank = 9;
      if (info[i].cls == OpClass::ReduceCol) rank = 0;
      else if (info[i].cls == OpClass::ReduceRow) rank = 1;
      else if (info[i].cls == OpClass::HeavyEW) rank = 2;
      else rank = 3;
      if (rank < best_rank) { best_rank = rank; best = i; }
    }
    for (int i : grp) {
      if (!info[i].candidate) continue;
      if (i == best) info[i].dominant = true;
      else info[i].sub_dominant = true;
    }
  }

  // a5: scheme finalisation.  Passive block-locality check for reduce-
  // dominated groups: a row reduce is produced and consumed by the same row
  // team inside one block (or one cluster when split) -> regional.  A column
  // reduce's consumers need every row -> global.  FULL values that cross the
  // barrier are buffered in HBM -> global.  EW-only groups adapt their mapping
  // to the producer's (proactive adaptation) and stay local.
  p.global_fulls.clear();
  p.post_colvecs.clear();
  p.needs_sweep2 = false;
  for (int i = 0; i < n; ++i) {
    if (!info[i].live) continue;
    Scheme s = Scheme::Local;
    OpClass c = info[i].cls;
    if (c == OpClass::ReduceRow) s = force_global ? Scheme::Global : Scheme::Regional;
    else if (c == OpClass::ReduceCol) s = Scheme::Global;
    else if (c == OpClass::HeavyEW && info[i].candidate && !is_output[i])
      s = (g.nodes[i].kind == ASTITCH_ROWVEC || g.nodes[i].kind == ASTITCH_COLVEC)
              ? Scheme::Regional : Scheme::Local;
    // a pre-barrier FULL / ROWVEC value read after the barrier (by anything
    // but the column reduction that accumulates it before the barrier)
    // (broadcasts are folded into their consumers: look through them)
    // (a column reduction accumulates in the sweep of its operand's level:
    // it reads v after the barrier iff that operand sits above v's level,
    // e.g. the broadcast of a row reduction demoted by FORCE_GLOBAL)
    // (a consumer also runs in the sweeps that recompute it, R22; a level
    // where the value itself is recomputed needs no buffer)
    std::function<bool(int, int, unsigned)> later_use = [&](int v, int lvl, unsigned own) {
      for (int u : info[v].consumers) {
        if (!info[u].live) continue;
        if (g.nodes[u].type == NodeType::Bcast) {
          if (later_use(u, lvl, own)) return true;
        } else if (info[u].cls == OpClass::ReduceCol) {
          if (info[g.nodes[u].a].level > lvl) return true;
        } else {
          const unsigned runs = (1u << info[u].level) | info[u].remat_mask;
          if ((runs & ~own) >> (lvl + 1)) return true;
        }
      }
      return false;
    };
    auto used_after_barrier = [&](int v) { return later_use(v, info[v].level, info[v].remat_mask); };
    if (c != OpClass::Const && c != OpClass::Input && g.nodes[i].type != NodeType::Bcast &&
        (g.nodes[i].kind == ASTITCH_FULL || g.nodes[i].kind == ASTITCH_ROWVEC) && used_after_barrier(i)) {
      s = Scheme::Global;
      info[i].global_full = true;
    }
    // crosses the barrier by recomputation from the HBM inputs (R22): still
    // the global scheme of the paper, without the buffer
    if (info[i].remat_mask >> (info[i].level + 1) && info[i].candidate) s = Scheme::Global;
    if (c == OpClass::Input && g.nodes[i].kind == ASTITCH_FULL && used_after_barrier(i))
      info[i].global_full = true;  // re-read from HBM after the barrier
    bool has_live_consumer = false;
    for (int u : info[i].consumers) has_live_consumer |= info[u].live;
    if (is_output[i] && !has_live_consumer && s == Scheme::Local) s = Scheme::Independent;
    info[i].scheme = s;
    if (info[i].global_full && c != OpClass::Input) p.global_fulls.push_back(i);
    if (info[i].post && g.nodes[i].kind == ASTITCH_COLVEC) p.post_colvecs.push_back(i);
    if (info[i].post && (g.nodes[i].kind == ASTITCH_FULL || g.nodes[i].kind == ASTITCH_ROWVEC))
      p.needs_sweep2 = true;
  }

  // Reading R7c (the column analogue of R7b): a column SUM whose value, through
  // light per-column ops, is broadcast into a FULL add / sub (a column mean
  // that is subtracted: BatchNorm) must keep the column's spread.  It is
  // accumulated in fp64 (per lane, per block, per column), its per-column
  // chain is evaluated in fp64, and the value is applied as an fp32 hi + lo pair.
  std::vector<bool> need(n, false);
  for (int b = 0; b < n; ++b) {
    const Node& bn = g.nodes[b];
    if (!info[b].live || bn.type != NodeType::Bcast || bn.axis != ASTITCH_AXIS_COL) continue;
    for (int u : info[b].consumers) {
      const Node& un = g.nodes[u];
      if (info[u].live && un.type == NodeType::Binary && un.kind == ASTITCH_FULL &&
          (un.sub == ASTITCH_ADD || un.sub == ASTITCH_SUB))
        need[bn.a] = true;
    }
  }
  p.n_precise_colreds = 0;
  for (int i = n - 1; i >= 0; --i) {
    if (!need[i] || !info[i].post) continue;
    const Node& nd = g.nodes[i];
    if (nd.kind != ASTITCH_COLVEC) continue;
    if (nd.type == NodeType::Reduce && nd.sub == ASTITCH_SUM && nd.axis == ASTITCH_AXIS_COL) {
      info[i].precise_col = true;
      continue;
    }
    const bool light = (nd.type == NodeType::Binary && nd.sub != ASTITCH_POW) ||
                       (nd.type == NodeType::Unary && (nd.sub == ASTITCH_NEG || nd.sub == ASTITCH_ABS));
    if (!light) continue;
    info[i].precise_col = true;
    for (int a : {nd.a, nd.b})
      if (a >= 0 && g.nodes[a].kind == ASTITCH_COLVEC && info[a].post) need[a] = true;
  }
  // keep only chains that start at a precise column SUM (a MIN / MAX of an
  // RMAX, for example, has no cancellation-prone sum behind it)
  for (int i = 0; i < n; ++i) {
    if (!info[i].precise_col || g.nodes[i].type == NodeType::Reduce) continue;
    bool from_sum = false;
    for (int a : {g.nodes[i].a, g.nodes[i].b})
      if (a >= 0 && info[a].precise_col) from_sum = true;
    info[i].precise_col = from_sum;
  }
  for (int id : p.colreds)
    if (info[id].precise_col) ++p.n_precise_colreds;
}

// ------------------------------------------------------------------------ a3/a4/a6/a7
namespace {

int pow2_floor(int x) {
  int r = 1;
  while (r * 2 <= x) r *= 2;
  return r;
}

// Shared-memory bank-conflict degree of a quarter-warp reading 16-byte chunks
// at a byte stride `stride` (thread-per-row staging, LDS.128).
int lds128_conflict_ways(int stride) {
  // LDS.128 serves 8 lanes per wavefront; lanes collide when their 16-byte
  // bank groups (addr / 16 mod 8) coincide.
  int cnt[8] = {0};
  for (int l = 0; l < 8; ++l) cnt[((l * stride) / 16) % 8]++;
  return *std::max_element(cnt, cnt + 8);
}

}  // namespace

void select_mapping(Plan& p) {
  const Graph& g = p.g;
  Mapping m;
  p.demotions.clear();
  const int64_t R = p.desc.rows, C = p.desc.cols;
  const int sms = p.sm_count;
  std::ostringstream why;

  // element sizes over FULL tensors (inputs and outputs)
  int es_min = 16, es_max = 1;
  bool any_full = false;
  for (int id : g.inputs) {
    const Node& nd = g.nodes[id];
    if (nd.kind == ASTITCH_FULL && p.info[id].live) {
      es_min = std::min(es_min, dtype_size(nd.dtype));
      es_max = std::max(es_max, dtype_size(nd.dtype));
      any_full = true;
    }
  }
  for (size_t k = 0; k < g.outputs.size(); ++k) {
    if (g.nodes[g.outputs[k]].kind == ASTITCH_FULL) {
      es_min = std::min(es_min, dtype_size(g.output_dtypes[k]));
      es_max = std::max(es_max, dtype_size(g.output_dtypes[k]));
      any_full = true;
    }
  }
  if (!p.global_fulls.empty()) es_max = 4, es_min = std::min(es_min, 4);
  if (!any_full) es_min = es_max = 4;

  // E: the widest power-of-two vector (<= 16 bytes of the narrowest tensor)
  // that divides C, so every chunk is aligned and never straddles a row.
  const Tuning& tu = p.tune;
  int vec_bytes = tu.vec_bytes == 32 ? 32 : 16;  // 128-bit vectors (tuning vec_bytes=32: 256-bit)
  int E = std::max(1, vec_bytes / es_min);
  while (E > 1 && (C % E) != 0) E /= 2;
  m.vec_elems = E;
  m.chunks = static_cast<int>((C + E - 1) / E);
  const int chunks = m.chunks;
  // packed varlen rows behave like masked rows of the maximum length
  const bool ragged = g.segments_node >= 0;
  const bool has_mask = g.lengths_node >= 0 || ragged;
  const bool has_colred = !p.colreds.empty();
  const int row_bytes_max = static_cast<int>(std::min<int64_t>(C * es_max, 1 << 30));

  // number of live FULL inputs (memory streams per row)
  int nfull_in = 0;
  for (int id : g.inputs)
    if (g.nodes[id].kind == ASTITCH_FULL && p.info[id].live) ++nfull_in;
  nfull_in = std::max(nfull_in, 1);

  // Team choice: lanes T (power of two) x chunks per lane V, T*V >= chunks.
  // Score: lane utilisation first, then per-lane elements near the target
  // (enough bytes in flight, few registers), then fewer lanes (cheaper team
  // reduction).  Depends on C and dtypes only, never on R, so a row's
  // reduction tree is identical for every shard (reading R13).
  auto choose_team = [&](int max_team, int target_ne, int max_ne) {
    int bestT = 1, bestV = chunks;
    double best_score = -1e30;
    for (int T = 1; T <= max_team; T *= 2) {
      int V = (chunks + T - 1) / T;
      int ne = V * E;
      if (ne > max_ne && T < max_team) continue;
      double util = static_cast<double>(chunks) / (T * V);
      double score = util * 100.0 - std::fabs(std::log2(static_cast<double>(ne) / target_ne)) * 4.0 -
                     (T > 32 ? 6.0 : 0.0) - (T < 4 ? 3.0 : 0.0);
      if (score > best_score) { best_score = score; bestT = T; bestV = V; }
    }
    m.team = bestT;
    m.chunks_per_lane = bestV;
    m.lane_util = static_cast<double>(chunks) / (bestT * bestV);
  };

  bool no_pack = (p.desc.flags & ASTITCH_FLAG_NO_PACK) != 0;
  bool no_split = (p.desc.flags & ASTITCH_FLAG_NO_SPLIT) != 0;
  bool no_tma = (p.desc.flags & ASTITCH_FLAG_NO_TMA) != 0;
  m.prefetch = (p.desc.flags & ASTITCH_FLAG_NO_PREFETCH) == 0;

  // Blocks-per-wave reference for the paper's shape rule: the number
  // of 1024-thread-equivalent blocks the chip runs at once = 2 per SM.
  const int64_t blocks_per_wave_1024 = 2LL * sms;
  // Cluster size for few long rows: the largest power of two K <= 8 with
  // R * K <= SMs, i.e. every row's cluster resident in ONE wave of the
  // 512-thread CTAs these templates use (one per SM at their register
  // counts).  Measured on B200, <64, 300000> fp32 row sum: K = 8 (18
  // clusters, 4 row trips) 29.1 us; one CTA per row, streamed, 20.8 us.
  int k_wave = 1;
  while (k_wave < 8 && R * (k_wave * 2) <= sms) k_wave *= 2;
  // rows <= 9: non-portable clusters of 16 (validated at load time against
  // cuOccupancyMaxActiveClusters, else back to 8)
  if (k_wave == 8 && R * 16 <= sms && !p.portable_clusters && !tu.portable_clusters)
    k_wave = 16;

  if (has_colred || p.max_level > 0) {
    // ---------------------------------------------------------- global sweep
    // Column reductions (K3) need all rows: a one-wave persistent grid sweeps
    // the rows (vertical packing), each lane keeps fp32 column
    // partials in registers, blocks combine in smem, then the grid barrier
    // and a deterministic fixed-order final combine.
    m.tmpl = Template::GlobalSweep;
    choose_team(1024, 8, 16);
    if (no_pack && m.team < 32) { m.team = 32; m.chunks_per_lane = (chunks + 31) / 32; }
    bool has_rowred = false, has_rowvec = false;
    for (size_t i = 0; i < g.nodes.size(); ++i) {
      if (p.info[i].live && p.info[i].cls == OpClass::ReduceRow) has_rowred = true;
      if (p.info[i].live && g.nodes[i].kind == ASTITCH_ROWVEC) has_rowvec = true;
    }
    // Wide rows (a vocabulary-sized bias gradient, P:L103-L109 K3): a team
    // keeps its row's columns in registers, so past ~16 values per lane it
    // would spill.  Column slabs instead: the columns are cut into slabs of
    // T x V x E (V*E ~ 8 values per lane) and CTA b sweeps slab b % nslab over
    // its row group (b / nslab); each CTA's column partials cover its slab
    // only, and the finalise sums the row groups of each column's slab in
    // order (deterministic).  Element-wise + column-reduction graphs only (a
    // row reduction needs the whole row in one team).
    m.nslab = 1;
    if (m.chunks_per_lane * E > 16 && !has_rowred && !has_rowvec && !has_mask && !ragged &&
        (p.desc.flags & ASTITCH_FLAG_FORCE_GLOBAL) == 0) {
      const int T = 512;
      const int64_t wave = 2LL * sms;                      // 2 x 512-thread CTAs per SM
      int V = std::max(1, 8 / E);
      int64_t ns = (chunks + static_cast<int64_t>(T) * V - 1) / (static_cast<int64_t>(T) * V);
      while (ns > wave / 4 && V * E < 32) {               // keep >= 4 row groups per slab
        V *= 2;
        ns = (chunks + static_cast<int64_t>(T) * V - 1) / (static_cast<int64_t>(T) * V);
      }
      if (ns <= wave / 4) {
        m.team = T;
        m.chunks_per_lane = V;
        m.nslab = static_cast<int>(ns);
        m.lane_util = static_cast<double>(chunks) / (static_cast<double>(ns) * T * V);
        why << "wide rows: " << ns << " column slabs of " << (T * V * E) << " columns (team " << T << " x " << V
            << " chunks), CTA b -> slab b % " << ns << "; ";
      }
    }
    // a multi-warp team reduces through block-wide smem: one team per block.
    // Long sweeps (>= 32 row steps per CTA: bandwidth-bound): one 1024-thread
    // CTA per SM, no software prefetch, a block barrier per row step
    // (sync_steps, retune_grid): the SM's warps sweep the same rows in lock
    // step.  Measured on B200 (C5): 981 us vs 1012 us for the round-1 mapping
    // (512 threads, register ping-pong prefetch).  Short sweeps (latency-
    // bound: BatchNorm 25088 x 128 fp32, 32 vs 48 us) keep 512 threads with
    // prefetch and no per-step barrier.  (scripts/sweeps/r02_*.txt)
    const int ne0 = m.chunks_per_lane * E;
    const int u0 = std::max(1, std::min(4, 64 / std::max(1, ne0 * nfull_in)));
    const int64_t steps_1024 = R / std::max<int64_t>(1, static_cast<int64_t>(sms) * std::max(1, 1024 / m.team) * u0);
    const bool long_sweep = steps_1024 >= 32;
    m.threads = (m.team > 32 && has_rowred) ? m.team : std::max(long_sweep ? 1024 : 512, m.team);
    if (tu.threads >= m.team && tu.threads <= 1024 && tu.threads % m.team == 0) m.threads = tu.threads;
    if (m.nslab > 1) m.threads = m.team;  // one 512-lane team per CTA (2 CTAs per SM)
    if (long_sweep) m.prefetch = false;
    if (tu.prefetch >= 0) m.prefetch = tu.prefetch == 1 && (p.desc.flags & ASTITCH_FLAG_NO_PREFETCH) == 0;
    m.rows_per_block = m.threads / m.team;
    int ne = m.chunks_per_lane * E;
    // rows per team per iteration: ~64 input elements in flight per lane
    // (measured on B200 for C5: U=4 reaches 98% of the copy roofline, U=2 94%)
    m.row_unroll = std::max(1, std::min(4, 64 / std::max(1, ne * nfull_in)));
    if (m.nslab > 1) m.row_unroll = std::min(m.row_unroll, 2);  // 2 x 512-thread CTAs per SM at <= 64 registers
    if (tu.unroll >= 1 && tu.unroll <= 8) m.row_unroll = tu.unroll;
    // a6: block-level combine of the teams' column partials in smem
    // (rows_per_block teams x the team's columns, fp32; hi + lo for precise
    // sums).  Over the budget: fewer teams per block (demotion), down to one
    // team per block, whose partials go straight to the workspace (no smem).
    if (m.rows_per_block > 1 && has_colred) {
      auto cbytes = [&]() {
        int64_t cb = static_cast<int64_t>(m.rows_per_block) * m.team * m.chunks_per_lane * E * 4;
        return p.n_precise_colreds > 0 ? 2 * cb : cb;  // hi and lo parts of fp64 column partials (R7c)
      };
      const int64_t budget = std::min<int64_t>(96 * 1024, p.smem_optin - 16 * 1024);
      const int rpb0 = m.rows_per_block;
      while (m.rows_per_block > 1 && (m.rows_per_block / 2) * m.team >= 32 && cbytes() > budget) {
        m.rows_per_block /= 2;
        m.threads = m.rows_per_block * m.team;
      }
      if (m.rows_per_block != rpb0)
        p.demotions.push_back("global sweep block combine: " + std::to_string(rpb0) + " -> " +
                              std::to_string(m.rows_per_block) + " teams per block (smem)");
      if (m.rows_per_block > 1) m.smem_bytes = static_cast<int>(cbytes());
    }
    why << (has_colred ? "column reduce -> global sweep (vertical packing, grid barrier); "
                       : "FORCE_GLOBAL: row reductions demoted to global (HBM + grid barrier); ");
    // tma_sweep (reading R23): element-wise + column-reduction graphs with one
    // barrier level.  Row tiles are staged in shared memory by bulk copies
    // (UBLKCP) that one producer warp issues for tiles taken from a counter in
    // address order; the teams compute from shared memory.  Measured on B200
    // (scripts/micro/tma_stream.cu, c5_dyn.cu): address-ordered tiles move
    // C5's 2R:1W mix at 7.0 TB/s where any static ownership of rows (register
    // or bulk-copy loads alike) stays at 6.5-6.6.  Dynamic ownership makes
    // per-CTA fp32 column partials scheduling-dependent, so column sums go
    // to exact binned accumulators (bins_add): the totals stay bitwise
    // deterministic (R13).  Each lane owns E = 4 columns (8 B bf16 / 16 B
    // fp32 chunks; E = 8 past 2048 columns), teams of T = C / E lanes share
    // the tile's rows (TR / teams rows per lane per tile, one deposit each).
    {
      // barrier levels (dependent column reductions, values read after a
      // barrier) are swept one after the other by the same ring; sharded
      // plans keep one sweep per kernel (their level-1 sweep is a separate
      // role); precise column sums (R7c) deposit fp64 tile partials into
      // 4 x 16-bit bins (>= 48 bits, as::bins_add_p)
      bool one_sweep = true;
      for (size_t i = 0; i < g.nodes.size(); ++i) {
        if (!p.info[i].live) continue;
        if (g.nodes[i].kind == ASTITCH_FULL && p.info[i].level > 0) one_sweep = false;
        if (p.info[i].cls == OpClass::ReduceCol && p.info[g.nodes[i].a].level > 0) one_sweep = false;
      }
      const bool levels_ok = one_sweep || p.desc.shard_world <= 1;
      bool ok = tu.tma != 0 && !no_tma && has_colred && levels_ok && !has_rowred && !has_rowvec &&
                !has_mask && !ragged && m.nslab == 1 &&
                R < (1LL << 30) && (p.desc.flags & ASTITCH_FLAG_FORCE_GLOBAL) == 0 && es_max <= 4;
      int64_t rowbytes = 0;
      for (int id : g.inputs) {
        const Node& nd = g.nodes[id];
        if (nd.kind != ASTITCH_FULL || !p.info[id].live) continue;
        if ((C * dtype_size(nd.dtype)) % 16) ok = false;  // bulk copies: 16-byte rows
        rowbytes += C * dtype_size(nd.dtype);
      }
      // fp32 HBM buffers of values read by later levels (upper bound of any level's streams)
      rowbytes += static_cast<int64_t>(p.global_fulls.size()) * C * 4;
      const int Et = C / 4 > 512 ? 8 : 4;
      ok = ok && rowbytes > 0 && C % Et == 0 && (C / Et) % 32 == 0 && C / Et <= 512;
      if (ok) {
        const int T = static_cast<int>(C / Et);
        // teams: >= 8 compute warps; beyond that, fewer teams = more rows per
        // lane per tile = fewer binned deposits per element (measured on B200,
        // C5: 1 team of 8 warps 914 us, 2 teams 929 us, 3 teams 1011 us)
        const int TM = (tu.tma_teams >= 1 && tu.tma_teams * T <= 1024) ? tu.tma_teams : std::max(1, 256 / T);
        const int S = (tu.tma_stages >= 2 && tu.tma_stages <= 8) ? tu.tma_stages : 3;
        const int64_t budget = p.smem_optin - 8 * 1024;  // static smem: barriers, finalise scratch
        // power-of-two tiles (C5: 16 rows 914 us, 18 rows 918 us)
        int64_t TR = pow2_floor(static_cast<int>(std::min<int64_t>(64, budget / (S * rowbytes))));
        if (tu.tma_rows > 0) TR = tu.tma_rows;
        TR -= TR % TM;
        const int64_t ring = S * TR * rowbytes;
        // the CTA combine of the teams' accumulators (one as::BinSlot /
        // as::BinSlotP, <= 48 bytes, per lane column) and the finalise
        // scratch reuse the ring
        const int64_t comb = std::max<int64_t>(static_cast<int64_t>(TM) * T * Et * 48, (TM * T + 32) * 48);
        // long sweeps only (>= 16 tiles per CTA): a short sweep is latency-
        // bound and pays the ring's fill and the producer hop (measured on
        // B200, BatchNorm fp32 [25088, 128]: 35.3 us vs 30.4 us static;
        // [1M, 1024]: 2.54 ms vs 2.77 ms); tuning tma=1 forces it
        const int64_t trips = ((R + TR - 1) / std::max<int64_t>(TR, 1) + sms - 1) / sms;
        if (TR >= std::max(4, TM) && ring <= budget && ring >= comb && (trips >= 16 || tu.tma == 1)) {
          m.tma_sweep = true;
          m.vec_elems = E = Et;
          m.chunks = static_cast<int>(C / Et);
          m.team = T;
          m.chunks_per_lane = 1;
          m.lane_util = 1.0;
          m.rows_per_block = TM;
          m.threads = TM * T + 32;  // + one producer warp
          m.row_unroll = 1;
          m.prefetch = false;
          m.hoist_colvec = true;
          m.tma_rows = static_cast<int>(TR);
          m.tma_stages = S;
          m.smem_bytes = static_cast<int>(ring);
          m.blocks_per_sm = 1;
          why << "tma_sweep: " << TR << "-row tiles x " << S << " stages (" << ring << " B smem), " << TM
              << " teams x " << T << " lanes x " << Et << " columns, producer warp, address-ordered tiles, exact "
              << "binned column sums (R23); ";
        }
      }
    }
  } else {
    // ---------------------------------------------------------- row-wise
    // Masked rows: a chunk index spans T*E columns across the team, and the
    // chunk-uniform mask branches skip whole chunks past the valid length, so
    // a finer chunk (smaller team, more chunks per lane) wastes less work on
    // padding; it also puts several rows of one segment (same length) in a warp.
    // Packed varlen rows (measured on B200, C3v): T=8 x 8 chunks of 8 bf16 +
    // the KF chunk-count specialisation (codegen) 81 us vs 95 us at T=16;
    // padded masked rows (C3) are store-bound and keep T=16 without it.
    choose_team(1024, ragged ? 64 : (has_mask ? 32 : 16), ragged ? 64 : 32);
    if (const int t = tu.team; t >= 1 && t <= 1024 && ((t & (t - 1)) == 0 || t % 32 == 0)) {
      m.team = t;
      m.chunks_per_lane = (chunks + t - 1) / t;
      m.lane_util = static_cast<double>(chunks) / (t * m.chunks_per_lane);
    }
    if (no_pack && m.team < 32 && chunks >= 1) {
      // ablation: XLA-style one row per warp (no horizontal packing)
      m.team = 32;
      m.chunks_per_lane = (chunks + 31) / 32;
      m.lane_util = static_cast<double>(chunks) / (32 * m.chunks_per_lane);
    }
    bool row16 = true;  // every FULL row is a multiple of 16 bytes
    for (int id : g.inputs)
      if (g.nodes[id].kind == ASTITCH_FULL && (C * dtype_size(g.nodes[id].dtype)) % 16) row16 = false;
    for (size_t k = 0; k < g.outputs.size(); ++k)
      if (g.nodes[g.outputs[k]].kind == ASTITCH_FULL && (C * dtype_size(g.output_dtypes[k])) % 16)
        row16 = false;
    bool has_colvec_in = false;
    for (int id : g.inputs)
      if (g.nodes[id].kind == ASTITCH_COLVEC && p.info[id].live) has_colvec_in = true;
    // Horizontal packing of many tiny rows: when a row is too
    // short for a power-of-two team to tile it (e.g. 9 x 16-byte chunks),
    // stage row tiles in smem with TMA bulk copies and give each thread a row.
    bool tile_common = !no_tma && row16 && p.global_fulls.empty() && R >= 4096;
    bool packed_ok = tile_common && !no_pack && !has_mask && !has_colvec_in && row_bytes_max <= 512 &&
                     m.lane_util < 0.95 && chunks <= 32;
    // (Round 1 measured TMA-staged tiles with a power-of-two TEAM per row
    // against register row teams on B200: C2 8.7 vs 8.0 us, C3 3.8 vs 4.6 TB/s;
    // the register row team wins whenever a team tiles the row, so only the
    // T=1 packed tiles -- rows no team can tile, C4 -- use the TMA template.)
    // Task splitting (rule P:L270): rows < blocks-per-wave and row > 1024.
    // B200 threshold (reading R15): measured on <64,30000> fp32 (120 KB rows)
    // one block per row is still faster (4.2 vs 4.7 us, latency-bound), on
    // <64,300000> (1.2 MB rows) a cluster of 8 is 5x faster; split from 256 KB.
    const bool force_split = (p.desc.flags & ASTITCH_FLAG_FORCE_SPLIT) != 0;
    bool split_rule = !no_split && !ragged && R < blocks_per_wave_1024 && C > 1024 &&
                      (force_split || C * es_max >= 256 * 1024);
    // packed-tile stage bytes per row: input tiles + output tiles that cannot
    // be written in place over an input tile of the same element size
    // (mirrors codegen)
    int64_t pk_in_bytes = 0, pk_out_bytes = 0;
    {
      int64_t& in_bytes = pk_in_bytes;
      int64_t& out_bytes = pk_out_bytes;
      std::vector<int> in_sizes;
      for (int id : g.inputs)
        if (g.nodes[id].kind == ASTITCH_FULL && p.info[id].live) {
          in_bytes += C * dtype_size(g.nodes[id].dtype);
          in_sizes.push_back(dtype_size(g.nodes[id].dtype));
        }
      for (size_t k = 0; k < g.outputs.size(); ++k)
        if (g.nodes[g.outputs[k]].kind == ASTITCH_FULL) {
          int es = dtype_size(g.output_dtypes[k]);
          auto it = std::find(in_sizes.begin(), in_sizes.end(), es);
          if (it != in_sizes.end()) in_sizes.erase(it);
          else out_bytes += C * es;
        }
    }
    // a6 shared-memory plan with demotion ("demote ... one by one
    // until the memory usage is under the limit"): the staged tile ring of
    // S stages x TR rows must fit HALF the SM's shared memory (>= 2 blocks per
    // SM, so the producer warp of one block overlaps the other's compute).
    // Demote in order of cost: 3 stages (prefetch distance 1), 64-row tiles;
    // if it still does not fit, the staged tile is abandoned for a register
    // row team (no smem staging at all) -- one warp of 32-row tiles per SM
    // would starve HBM.
    int pk_stages = 4, pk_threads = 128;  // prefetch distance 2 tiles + 2 tiles draining (bulk stores)
    if (tu.tile_stages >= 2 && tu.tile_stages <= 8) pk_stages = tu.tile_stages;
    if (tu.tile_threads >= 32 && tu.tile_threads <= 1024 && tu.tile_threads % 32 == 0) pk_threads = tu.tile_threads;
    int pk_rows = (tu.tile_rows >= 1 && tu.tile_rows % pk_threads == 0) ? tu.tile_rows : pk_threads;
    const int64_t smem_budget = std::min<int64_t>(100 * 1024, p.smem_optin / 2 - 4096);
    auto pk_smem = [&]() {
      return static_cast<int64_t>(pk_stages) * pk_rows * (pk_in_bytes + pk_out_bytes) + 64 * pk_stages;
    };
    if (packed_ok) {
      while (pk_smem() > smem_budget) {
        if (pk_stages > 3) --pk_stages;
        else if (pk_threads > 64) { pk_threads /= 2; pk_rows = pk_threads; }
        else break;
      }
      if (pk_smem() > smem_budget) {
        packed_ok = false;
        p.demotions.push_back("packed_tile needs " + std::to_string(pk_smem()) + " B of smem at " +
                              std::to_string(pk_stages) + " stages x " + std::to_string(pk_rows) + " rows > " +
                              std::to_string(smem_budget) + " -> row team (no staging)");
      } else if (pk_stages != 4 || pk_threads != 128) {
        p.demotions.push_back("packed_tile smem: " + std::to_string(pk_stages) + " stages x " + std::to_string(pk_rows) +
                              " rows (" + std::to_string(pk_smem()) + " B <= " + std::to_string(smem_budget) + ")");
      }
    }
    if (packed_ok) {
      m.tmpl = Template::PackedTile;
      m.team = 1;
      m.chunks_per_lane = chunks;
      m.lane_util = 1.0;
      m.threads = pk_threads;
      m.tile_rows = pk_rows;
      m.stages = pk_stages;
      m.rows_per_block = m.threads / m.team;
      m.smem_bytes = static_cast<int>(pk_smem());
      m.grid_waves = tu.waves > 0 ? tu.waves : 0;
      m.bank_conflict_ways = lds128_conflict_ways(static_cast<int>(C) * es_min);
      why << "row of " << chunks << " x " << (E * es_min)
          << "B chunks does not tile a power-of-two team -> TMA-staged packed tiles, thread per row; ";
    } else if (split_rule && p.global_fulls.empty()) {
      // Task splitting: each row is split over a thread-block cluster
      // of K CTAs (K ~ blocks-per-wave / rows, power of two, <= 8 portable);
      // block partials combine through DSMEM in a fixed order.
      m.tmpl = Template::SplitRow;
      m.split = std::max(2, k_wave);
      m.threads = 512;
      if (const int kk = tu.split; kk >= 1 && kk <= 16 && (kk & (kk - 1)) == 0) m.split = kk;
      if (const int t = tu.split_threads; t >= 32 && t <= 1024 && t % 32 == 0) m.threads = t;
      m.team = m.split * m.threads;
      m.chunks_per_lane = std::max(1, (chunks + m.team - 1) / m.team);
      m.lane_util = static_cast<double>(chunks) / (static_cast<double>(m.team) * m.chunks_per_lane);
      m.rows_per_block = 1;
      m.row_unroll = 1;
      why << "paper split rule holds (rows " << R << " < per-wave " << blocks_per_wave_1024 << " and row " << C
          << " > 1024): each row split over a cluster of " << m.split << " CTAs x " << m.threads
          << " threads, partials combined through DSMEM; ";
    } else {
      m.tmpl = Template::RowTeam;
      // a multi-warp team reduces through block-wide smem: one team per block
      m.threads = m.team > 32 ? m.team : 256;
      if (const int t = tu.threads; t >= m.team && t <= 1024 && t % m.team == 0 && t % 32 == 0) m.threads = t;
      // One wave of teams for every row: when the rows need at most 28 warps
      // per SM (>= 72 registers per thread), give each row its own team in a
      // single wave of 4-warp blocks, sized to exactly the warps needed (no
      // vertical trips, so no prefetch pipeline; the finest block granularity
      // wastes the fewest warps).  Measured on B200 (C2, 4096 rows of 768
      // bf16): 128 x 7 blocks/SM, one row per warp, 6.79 us vs 7.10 us for
      // 256-thread blocks at 2 blocks/SM sweeping two rows per warp.
      m.single_wave_bps = 0;
      if (m.team <= 32 && tu.threads == 0) {
        const int64_t teams_per_warp = 32 / m.team;
        const int64_t warps = (R + teams_per_warp - 1) / teams_per_warp;
        const int64_t warps_per_sm = (warps + sms - 1) / std::max(1, sms);
        if (warps_per_sm > 8 && warps_per_sm <= 28) {
          m.threads = 128;
          m.single_wave_bps = static_cast<int>((warps_per_sm + 3) / 4);
        }
      }
      m.rows_per_block = m.threads / m.team;
      m.row_unroll = (tu.unroll >= 1 && tu.unroll <= 8) ? tu.unroll : 1;
      // Light rows (<= 16 values per lane over all input streams, no mask):
      // a non-persistent grid, one row group per CTA, so the hardware block
      // scheduler streams the CTAs through the rows in address order and the
      // low register count keeps many warps per SM.  Measured on B200
      // (scripts/sweeps/r02_readmostly.txt): row sums [4M, 32] fp32 87.6 ->
      // 75.1 us, [1M, 256] 153 -> 144 us; softmax fp32 [1M, 128] 184 -> 157 us.
      // Heavier rows keep the persistent prefetching sweep (LayerNorm+GELU
      // [65536, 768] 52.9 vs 54.7 us, masked softmax C3 145 vs 165 us).
      m.nonpersistent = !has_mask && !ragged && m.single_wave_bps == 0 &&
                        nfull_in * m.chunks_per_lane * E <= 16;
      if (tu.persistent >= 0) m.nonpersistent = tu.persistent == 0;
      m.grid_waves = tu.waves > 0 ? tu.waves : 0;
      why << (m.single_wave_bps ? "one wave of teams (one row per team); " : "") << "row team of " << m.team << " lanes x " << m.chunks_per_lane << " chunks ("
          << m.rows_per_block << " rows / block, packing), regional via shuffles" << (m.team > 32 ? "+smem" : "")
          << "; ";
    }
    // Rows longer than the team's registers (more than kStreamNE fp32 values
    // per lane even with the largest team / cluster): stream the row in
    // column tiles, one pass over the row per level of dependent row
    // reductions (FULL values of lower levels are recomputed from the
    // re-read inputs, L2-resident for a row in flight), the regional values
    // (row scalars) stay in registers.  The paper's answer to a regional
    // buffer over the on-chip limit is demotion to global; a
    // per-row re-read keeps it in one pass of the grid with no barrier.
    constexpr int kStreamNE = 128;
    const bool stream_ok = !has_mask && p.global_fulls.empty() && tu.stream != 0 &&
                           (m.tmpl == Template::RowTeam || m.tmpl == Template::SplitRow);
    const bool force_stream = tu.stream == 1;
    if (stream_ok && (m.chunks_per_lane * E > kStreamNE || force_stream || p.stream_fallback)) {
      m.tmpl = Template::RowStream;
      m.threads = 512;
      m.split = 1;
      if (!no_split && R < blocks_per_wave_1024) {
        m.split = k_wave;
      }
      m.chunks_per_lane = std::max(1, 32 / E);  // V: 32 values per lane per tile
      // Regional stitching proper: when the row's inputs fit the
      // shared memory of a cluster (<= 160 KB per CTA, <= 8 CTAs), the first
      // pass that reads an input stages the lane's raw chunks in its CTA's
      // smem and the later passes re-read them from there (each lane reads
      // back only its own chunks: no barrier); else the passes re-read L2/HBM.
      int in_row_bytes = 0;
      for (int id : g.inputs)
        if (g.nodes[id].kind == ASTITCH_FULL && p.info[id].live)
          in_row_bytes += static_cast<int>(std::min<int64_t>(C * dtype_size(g.nodes[id].dtype), 1 << 30));
      // Measured on B200 (LM-head softmax 4096 x 128256 bf16: 741 us staged vs
      // 660 us re-reading L2; fp32 4096 x 100000: 1896 vs 1049 us): staging
      // costs occupancy (one 512-thread CTA per SM) that the L2-resident
      // re-reads do not, so it is opt-in (tuning stage=1) until the staged
      // pass pipelines its loads.
      const bool no_stage = tu.stage != 1;
      m.stage_row = false;
      m.smem_bytes = 0;
      int stage_budget = 72 * 1024;  // per CTA: keeps 3 CTAs of 512 threads per SM
      if (tu.stage_kb > 0) stage_budget = std::max(8, tu.stage_kb) * 1024;
      if (!no_stage && in_row_bytes > 0) {
        int k = m.split;
        while (k < 8 && (in_row_bytes + k - 1) / k > stage_budget) k *= 2;
        if ((in_row_bytes + k - 1) / k <= stage_budget && !(no_split && k > 1)) {
          m.split = k;
          m.stage_row = true;
          const int64_t tch = static_cast<int64_t>(k) * m.threads * m.chunks_per_lane;
          const int64_t nt = (m.chunks + tch - 1) / tch;
          int64_t sm = 0;
          for (int id : g.inputs)
            if (g.nodes[id].kind == ASTITCH_FULL && p.info[id].live)
              sm += nt * m.chunks_per_lane * m.threads * E * dtype_size(g.nodes[id].dtype);
          m.smem_bytes = static_cast<int>(sm);
        }
      }
      m.team = m.split * m.threads;
      m.lane_util = 1.0;
      m.rows_per_block = 1;
      m.row_unroll = 1;
      m.prefetch = false;
      why << "row of " << C << " exceeds the team's registers -> streamed in tiles of " << m.team << " lanes x "
          << m.chunks_per_lane << " chunks" << (m.split > 1 ? " over a cluster of " + std::to_string(m.split) + " CTAs" : "")
          << ", one pass per row-reduction level" << (m.stage_row ? ", inputs staged in shared memory" : "") << "; ";
    }
  }

  // colvec operands: hoist in registers when the footprint is small (a6)
  {
    int ncv = 0;
    for (int i = 0; i < static_cast<int>(g.nodes.size()); ++i)
      if (p.info[i].live && !p.info[i].post && g.nodes[i].kind == ASTITCH_COLVEC) ++ncv;
    m.hoist_colvec = (ncv * m.chunks_per_lane * E) <= 48;
    if (tu.hoist >= 0) m.hoist_colvec = tu.hoist == 1;
  }

  // a7: assume-relax-apply.  Assume the 32-register bound (full occupancy),
  // compute blocks per SM from threads and smem, relax the register cap to the
  // largest value that keeps those blocks resident; the caller
  // recompiles with a lower target if ptxas reports spills.
  // Register row teams that write whole rows: cap the resident warps at those
  // needed for ~48 KB of row stores per SM per row step; more concurrent
  // row-write streams only add DRAM page contention (measured on B200: C3
  // masked softmax, 2 KB of stores per warp step: 24 warps/SM 146 us, 32
  // warps 153.5 us, 16 warps 163 us).  Read-mostly rows (a row sum, fig6a:
  // 64 B of stores per warp step) keep the full occupancy.
  // tma_team: row teams fed by the tma_sweep machinery -- a producer warp
  // takes TR-row tiles from a counter in address order and bulk-copies each
  // row's valid prefix (lane r of the warp: row r of the tile) into a ring of
  // shared-memory stages; the teams compute from shared memory.  Rows must
  // start 16-byte aligned in every FULL input.  Default for key-padding
  // masked rows of >= 512 bytes (measured on B200, C3: 16-row tiles x 4
  // stages, 3 CTAs/SM, 135.8 us vs 140.4 us for the oversubscribed register
  // row teams; 1 CTA/SM with 128 KB rings 193 us); opt-in (tuning
  // tma_team=1) elsewhere: packed varlen rows (C3v: 80.9 us with 16-lane
  // teams and one bulk copy per single-segment tile vs 78.9 us register
  // rows), unmasked rows are not better served than by register rows.
  const bool tma_team_default = has_mask && !ragged && C * es_min >= 512;
  if (m.tmpl == Template::RowTeam && (tu.tma_team == 1 || (tu.tma_team != 0 && tma_team_default)) && !no_tma &&
      R < (1LL << 30) && es_max <= 4) {
    bool ok = true;
    int64_t pitch = 0;  // smem bytes of one row slot, all FULL inputs
    for (int id : g.inputs) {
      const Node& nd = g.nodes[id];
      if (nd.kind != ASTITCH_FULL || !p.info[id].live) continue;
      const int64_t rb = C * dtype_size(nd.dtype);
      if (!ragged && rb % 16) ok = false;
      pitch += (rb + 15) / 16 * 16;
    }
    const int S = (tu.tma_stages >= 2 && tu.tma_stages <= 8) ? tu.tma_stages : 4;
    const int teams = (tu.tma_teams >= 1 && tu.tma_teams * m.team <= 1024) ? tu.tma_teams : m.rows_per_block;
    // 16-row tiles, at least one row per team (<= 32: one producer lane per row)
    const int TRq = tu.tma_rows > 0 ? tu.tma_rows : std::max(16, teams);
    const int64_t ring = static_cast<int64_t>(S) * TRq * pitch;
    // whole compute warps (the producer warp follows them)
    if (ok && pitch > 0 && TRq <= 32 && TRq % teams == 0 && (teams * m.team) % 32 == 0 &&
        ring <= p.smem_optin - 8 * 1024) {
      m.tma_team = true;
      m.tma_rows = TRq;
      m.tma_stages = S;
      m.rows_per_block = teams;
      m.threads = teams * m.team + 32;
      m.row_unroll = 1;
      m.prefetch = false;
      m.nonpersistent = false;
      m.single_wave_bps = 0;
      m.grid_waves = 0;
      m.smem_bytes = static_cast<int>(ring);
      why << "tma_team: " << TRq << "-row tiles x " << S << " stages (" << ring << " B), " << teams << " teams, "
          << "producer warp (one bulk copy per row), address-ordered tiles; ";
    }
  }
  int max_threads_sm = 2048;
  if (m.tmpl == Template::RowTeam && !m.tma_team) {
    if (m.single_wave_bps > 0) {
      max_threads_sm = m.single_wave_bps * m.threads;
    } else {
      int64_t out_row_bytes = 0;
      for (size_t k = 0; k < g.outputs.size(); ++k)
        if (g.nodes[g.outputs[k]].kind == ASTITCH_FULL)
          out_row_bytes += std::min<int64_t>(C * dtype_size(g.output_dtypes[k]), 1 << 30);
      const double bytes_per_warp = std::max<double>(1.0, static_cast<double>(out_row_bytes) * m.row_unroll * 32.0 / m.team);
      const int cap_warps = static_cast<int>(std::min(64.0, std::max(4.0, std::ceil(48.0 * 1024 / bytes_per_warp))));
      const int wpb = std::max(1, m.threads / 32);
      max_threads_sm = std::min(2048, ((cap_warps + wpb - 1) / wpb) * m.threads);
    }
  }
  int by_threads = std::max(1, max_threads_sm / m.threads);
  int by_smem = m.smem_bytes > 0 ? (228 * 1024) / (m.smem_bytes + 1024) : 32;
  m.blocks_per_sm = std::max(1, std::min({32, by_threads, by_smem}));
  if (tu.bps >= 1 && tu.bps <= 32) m.blocks_per_sm = tu.bps;
  m.reg_cap = std::min(255, (65536 / (m.blocks_per_sm * m.threads)) & ~7);

  m.reason = why.str();
  p.map = m;
  retune_grid(p);
}

// grid: one wave (persistent, vertical packing); never more blocks
// than there is work.  Recomputed whenever blocks_per_sm is relaxed.
void retune_grid(Plan& p) {
  Mapping& m = p.map;
  const int64_t R = p.desc.rows;
  int64_t work_units = 0;
  if (m.tmpl == Template::PackedTile) work_units = (R + m.tile_rows - 1) / m.tile_rows;
  else work_units = (R + (int64_t)m.rows_per_block * m.row_unroll - 1) / ((int64_t)m.rows_per_block * m.row_unroll);
  int64_t wave = static_cast<int64_t>(m.blocks_per_sm) * p.sm_count;
  if (m.tmpl == Template::SplitRow || (m.tmpl == Template::RowStream && m.split > 1)) {
    // clusters of `split` CTAs, one row per cluster per iteration
    int64_t clusters = std::max<int64_t>(1, std::min(work_units, wave / m.split));
    m.grid = clusters * m.split;
    m.vertical_trips = (work_units + clusters - 1) / clusters;
  } else if (m.tmpl == Template::RowTeam && m.tma_team) {
    const int64_t tiles = (R + m.tma_rows - 1) / m.tma_rows;
    m.grid = std::max<int64_t>(1, std::min<int64_t>(tiles, wave));
    m.vertical_trips = (tiles + m.grid - 1) / m.grid;
  } else if (m.tmpl == Template::GlobalSweep && m.tma_sweep) {
    // one CTA per SM (the ring fills its shared memory); tiles are taken
    // from the counter, so the grid never needs more CTAs than tiles
    const int64_t tiles = (R + m.tma_rows - 1) / m.tma_rows;
    m.grid = std::max<int64_t>(1, std::min<int64_t>(tiles, wave));
    m.vertical_trips = (tiles + m.grid - 1) / m.grid;
  } else if (m.tmpl == Template::GlobalSweep && m.nslab > 1) {
    // column slabs: nslab CTAs per row group, grid a multiple of nslab
    const int64_t groups = std::max<int64_t>(1, std::min(work_units, wave / m.nslab));
    m.grid = groups * m.nslab;
    m.vertical_trips = (work_units + groups - 1) / groups;
  } else if (m.tmpl == Template::RowTeam && m.nonpersistent && work_units < (1LL << 31)) {
    // one row group per CTA: the hardware block scheduler streams the CTAs
    // through the rows in address order (no software prefetch needed)
    m.grid = std::max<int64_t>(1, work_units);
    m.vertical_trips = 1;
  } else {
    // Oversubscribed grids (non-cooperative templates): CTAs beyond the
    // resident ones start as earlier CTAs finish, which balances the tail.
    // Measured on B200 (scripts/sweeps/r02_waves*.txt): TMA packed tiles
    // best at ~2.5 tiles per CTA (C4: 95.1 -> 86.1 us; 1 tile per CTA loses
    // the TMA pipeline: 95.2 us); masked register row teams best at ~8 row
    // steps per CTA (C3: 143.5 -> 140.4 us).  Packed varlen rows and
    // unmasked heavy rows measured slower oversubscribed (C3v 78.5 vs 84+ us;
    // LayerNorm+GELU [65536, 768] 52.2 vs 53.7 us): one wave.
    int64_t target = wave;
    if (m.tmpl == Template::PackedTile) target = std::max<int64_t>(wave, (work_units * 2 + 4) / 5);
    else if (m.tmpl == Template::RowTeam && p.g.lengths_node >= 0 && p.g.segments_node < 0 && m.single_wave_bps == 0)
      target = std::max<int64_t>(wave, std::min<int64_t>(wave * 16, work_units / 8));
    if (m.grid_waves > 1 && (m.tmpl == Template::PackedTile || m.tmpl == Template::RowTeam)) target = wave * m.grid_waves;
    m.grid = std::max<int64_t>(1, std::min({work_units, target, static_cast<int64_t>(INT32_MAX)}));
    m.vertical_trips = (work_units + m.grid - 1) / m.grid;
  }
  // block barrier per row step of a persistent multi-trip sweep (the CTA's
  // warps stay on the same rows): default for the global sweep (measured on
  // B200); tuning sync=0/1 overrides
  m.sync_steps = (m.tmpl == Template::GlobalSweep) && m.vertical_trips >= 32 && !m.prefetch && !m.tma_sweep;
  if (p.tune.sync >= 0)
    m.sync_steps = p.tune.sync == 1 && m.vertical_trips > 1 &&
                   (m.tmpl == Template::GlobalSweep || m.tmpl == Template::RowTeam) && !m.tma_sweep;
  plan_workspace(p);
}

// ------------------------------------------------------------------------ a6 workspace
void plan_workspace(Plan& p) {
  WsLayout w;
  size_t off = 0;
  auto align = [](size_t x) { return (x + 255) & ~static_cast<size_t>(255); };
  const int64_t C = p.desc.cols, R = p.desc.rows;
  if (p.map.tmpl == Template::GlobalSweep) {
    w.barrier = off;
    off = align(off + 256);
    w.partials = off;
    const int64_t nparts = p.map.grid;
    // partial slots: one per column reduction + a lo slot per precise sum (R7c)
    const size_t nslots = p.colreds.size() + static_cast<size_t>(p.n_precise_colreds);
    // (tma_sweep: a binned accumulator per slot and column, as::BinSlot 32 B,
    // as::BinSlotP 48 B when a precise sum needs it)
    const size_t slot_bytes = !p.map.tma_sweep ? 4 : (p.n_precise_colreds > 0 ? 48 : 32);
    off = align(off + static_cast<size_t>(nparts) * nslots * C * slot_bytes);
    w.colvals = off;
    // [post COLVEC hi][rank-local column totals][post COLVEC lo (R7c)]
    bool any_precise_post = false;
    for (int id : p.post_colvecs) any_precise_post |= p.info[id].precise_col;
    off = align(off + std::max<size_t>(p.post_colvecs.size(), 1) * C * 4 + C * 4 * p.colreds.size() +
                (any_precise_post ? p.post_colvecs.size() * C * 4 : 0));
    w.globals = off;
    // a6 memory reuse: a global buffer is live from the sweep that
    // writes it to the last sweep that reads it; a later value of the same
    // kind whose writing sweep starts after that (a grid barrier in between)
    // takes over the buffer (interval colouring in definition order, the
    // role of the paper's dominance-tree data-flow analysis).  ROWVEC values
    // need R floats, FULL values R x C floats.
    const int n = static_cast<int>(p.g.nodes.size());
    std::function<int(int)> last_read = [&](int v) {
      int last = -1;
      for (int u : p.info[v].consumers) {
        if (!p.info[u].live) continue;
        if (p.g.nodes[u].type == NodeType::Bcast) { last = std::max(last, last_read(u)); continue; }
        int ph = p.info[u].cls == OpClass::ReduceCol ? p.info[p.g.nodes[u].a].level : p.info[u].level;
        last = std::max(last, ph);
      }
      return last;
    };
    struct Slot { astitch_kind kind; int free_after; size_t off; };
    std::vector<Slot> slots;
    size_t goff = 0;
    p.gbuf_off.assign(p.global_fulls.size(), 0);
    std::vector<size_t> order(p.global_fulls.size());
    std::iota(order.begin(), order.end(), 0);
    std::stable_sort(order.begin(), order.end(), [&](size_t a, size_t b) {
      return p.info[p.global_fulls[a]].level < p.info[p.global_fulls[b]].level;
    });
    for (size_t q : order) {
      const int id = p.global_fulls[q];
      const astitch_kind k = p.g.nodes[id].kind;
      const int def = p.info[id].level;
      int chosen = -1;
      for (size_t s = 0; s < slots.size(); ++s)
        if (slots[s].kind == k && slots[s].free_after < def) { chosen = static_cast<int>(s); break; }
      if (chosen < 0) {
        slots.push_back({k, -1, goff});
        // ROWVEC buffers hold 2 R floats: the value and, for a cancellation-
        // prone row sum demoted to global (FORCE_GLOBAL), its lo part (R7b)
        goff = align(goff + static_cast<size_t>(R) * (k == ASTITCH_FULL ? C : 2) * 4);
        chosen = static_cast<int>(slots.size()) - 1;
      }
      slots[chosen].free_after = last_read(id);
      p.gbuf_off[q] = slots[chosen].off;
    }
    (void)n;
    p.gbuf_slots = static_cast<int>(slots.size());
    off = align(off + goff);
  }
  if (p.map.tmpl == Template::RowTeam && p.map.tma_team) {
    w.barrier = off;  // [64]: tile counter, [68]: CTAs done (the last one resets both)
    off = align(off + 256);
  }
  w.total = off;
  p.ws = w;
}

uint64_t compulsory_bytes(const Plan& p) {
  const Graph& g = p.g;
  const uint64_t R = p.desc.rows, C = p.desc.cols;
  uint64_t b = 0;
  for (int id : g.inputs) {
    const Node& nd = g.nodes[id];
    if (!p.info[id].live) continue;
    uint64_t es = dtype_size(nd.dtype);
    // packed varlen: the whole packed buffer (incl. pitch padding: an upper bound)
    if (nd.kind == ASTITCH_FULL && g.segments_node >= 0) b += static_cast<uint64_t>(g.seg_elems) * es;
    else if (nd.kind == ASTITCH_SEGMENTS) b += 16ULL * g.nseg;
    else if (nd.kind == ASTITCH_FULL) b += R * C * es;
    else if (nd.kind == ASTITCH_ROWVEC) b += R * es;
    else if (nd.kind == ASTITCH_COLVEC) b += C * es;
    else if (nd.kind == ASTITCH_LENGTHS)
      b += 4 * ((R + g.rows_per_segment - 1) / std::max<int64_t>(g.rows_per_segment, 1));
  }
  for (size_t k = 0; k < g.outputs.size(); ++k) {
    uint64_t es = dtype_size(g.output_dtypes[k]);
    astitch_kind kd = g.nodes[g.outputs[k]].kind;
    if (kd == ASTITCH_FULL && g.segments_node >= 0) b += static_cast<uint64_t>(g.seg_elems) * es;
    else if (kd == ASTITCH_FULL) b += R * C * es;
    else if (kd == ASTITCH_ROWVEC) b += R * es;
    else b += C * es;
  }
  return b;
}

// ------------------------------------------------------------------------ describe
std::string describe_json(const Plan& p) {
  std::ostringstream o;
  const Graph& g = p.g;
  const Mapping& m = p.map;
  auto esc = [](const std::string& s) {
    std::string r;
    for (char c : s) {
      if (c == '"' || c == '\\') r += '\\';
      if (c == '\n') { r += "\\n"; continue; }
      r += c;
    }
    return r;
  };
  o << "{\"rows\":" << p.desc.rows << ",\"cols\":" << p.desc.cols << ",\"device\":" << p.desc.device
    << ",\"shard_rank\":" << p.desc.shard_rank << ",\"shard_world\":" << p.desc.shard_world
    << ",\"sm_count\":" << p.sm_count << ",\"flags\":" << p.desc.flags << ",\"tuning\":\"" << esc(p.tune.text) << "\"";
  o << ",\"ops\":[";
  for (size_t i = 0; i < g.nodes.size(); ++i) {
    const Node& nd = g.nodes[i];
    const NodeInfo& in = p.info[i];
    if (i) o << ",";
    o << "{\"id\":" << i << ",\"class\":\"" << opclass_name(in.cls) << "\",\"kind\":\""
      << kind_name(nd.kind) << "\"";
    if (nd.type == NodeType::Unary) o << ",\"op\":\"" << unop_name(nd.sub) << "\"";
    if (nd.type == NodeType::Binary) o << ",\"op\":\"" << binop_name(nd.sub) << "\"";
    if (nd.type == NodeType::Reduce) o << ",\"op\":\"" << (nd.sub == ASTITCH_SUM ? "SUM" : "RMAX") << "\"";
    if (nd.a >= 0) o << ",\"a\":" << nd.a;
    if (nd.b >= 0) o << ",\"b\":" << nd.b;
    o << ",\"live\":" << (in.live ? "true" : "false") << ",\"post_barrier\":" << (in.post ? "true" : "false")
      << ",\"candidate\":" << (in.candidate ? "true" : "false")
      << ",\"dominant\":" << (in.dominant ? "true" : "false")
      << ",\"sub_dominant\":" << (in.sub_dominant ? "true" : "false") << ",\"group\":" << in.group
      << ",\"scheme\":\"" << scheme_name(in.scheme) << "\"";
    if (in.remat_mask) {  // levels whose sweeps recompute this value (R22)
      o << ",\"recomputed_at\":[";
      bool first = true;
      for (int b = 0; b < 32; ++b)
        if ((in.remat_mask >> b) & 1u) { o << (first ? "" : ",") << b; first = false; }
      o << "]";
    }
    o << "}";
  }
  o << "],\"groups\":[";
  for (size_t k = 0; k < p.groups.size(); ++k) {
    if (k) o << ",";
    o << "[";
    for (size_t j = 0; j < p.groups[k].size(); ++j) o << (j ? "," : "") << p.groups[k][j];
    o << "]";
  }
  // Step 2: each group's schedule = its dominant's.  Every group of
  // one stitched kernel shares the block and the lane -> (row, columns)
  // assignment of the template (the team shape is a function of C and the
  // dtypes only); groups differ in the index space their dominant iterates:
  o << "],\"group_mappings\":[";
  for (size_t k = 0; k < p.groups.size(); ++k) {
    int dom = -1;
    bool any_full = false, any_row = false, any_col = false;
    for (int i : p.groups[k]) {
      if (p.info[i].dominant) dom = i;
      any_full |= g.nodes[i].kind == ASTITCH_FULL;
      any_row |= g.nodes[i].kind == ASTITCH_ROWVEC;
      any_col |= g.nodes[i].kind == ASTITCH_COLVEC;
    }
    std::string how;
    const OpClass dc = dom >= 0 ? p.info[dom].cls : OpClass::LightEW;
    if (dc == OpClass::ReduceCol)
      how = "column reduce: each lane accumulates its columns over its rows (vertical packing), block + grid "
            "partials, then one thread per column after the grid barrier";
    else if (dc == OpClass::ReduceRow)
      how = "row reduce: a team of T lanes per row (elements (j*T+lane)*E..), shuffle / smem / DSMEM tree, "
            "row scalar team-uniform";
    else if (!any_full && any_col)
      how = "column values: one thread per column (finalise after the barrier) or per lane chunk (hoisted)";
    else if (!any_full && any_row)
      how = "row values: team-uniform scalars";
    else
      how = "element-wise only: adopts its producer group's mapping (proactive block locality, P:L282)";
    o << (k ? "," : "") << "{\"group\":" << k << ",\"dominant\":" << dom << ",\"level\":"
      << (dom >= 0 ? p.info[dom].level : 0) << ",\"schedule\":\"" << how << "\"}";
  }
  o << "],\"mapping\":{\"template\":\"" << template_name(m.tmpl) << "\",\"vec_elems\":" << m.vec_elems
    << ",\"chunks\":" << m.chunks << ",\"team\":" << m.team << ",\"chunks_per_lane\":" << m.chunks_per_lane
    << ",\"lane_util\":" << m.lane_util << ",\"threads\":" << m.threads
    << ",\"rows_per_block\":" << m.rows_per_block << ",\"row_unroll\":" << m.row_unroll
    << ",\"prefetch\":" << (m.prefetch ? "true" : "false") << ",\"single_wave_bps\":" << m.single_wave_bps << ",\"sync_steps\":" << (m.sync_steps ? "true" : "false") << ",\"nslab\":" << m.nslab << ",\"nonpersistent\":" << (m.nonpersistent ? "true" : "false")
    << ",\"hoist_colvec\":" << (m.hoist_colvec ? "true" : "false") << ",\"tile_rows\":" << m.tile_rows
    << ",\"stages\":" << m.stages << ",\"split\":" << m.split << ",\"stage_row\":" << (m.stage_row ? "true" : "false")
    << ",\"tma_sweep\":" << (m.tma_sweep ? "true" : "false") << ",\"tma_team\":" << (m.tma_team ? "true" : "false")
    << ",\"tma_rows\":" << m.tma_rows
    << ",\"tma_stages\":" << m.tma_stages << ",\"grid\":" << m.grid
    << ",\"blocks_per_sm\":" << m.blocks_per_sm << ",\"reg_cap\":" << m.reg_cap
    << ",\"vertical_trips\":" << m.vertical_trips << ",\"smem_bytes\":" << m.smem_bytes
    << ",\"lds128_conflict_ways\":" << m.bank_conflict_ways << ",\"reason\":\"" << esc(m.reason)
    << "\"}";
  o << ",\"workspace\":{\"total\":" << p.ws.total << ",\"barrier\":" << p.ws.barrier
    << ",\"partials\":" << p.ws.partials << ",\"colvals\":" << p.ws.colvals << ",\"globals\":" << p.ws.globals
    << "}";
  o << ",\"global_fulls\":[";
  for (size_t k = 0; k < p.global_fulls.size(); ++k) o << (k ? "," : "") << p.global_fulls[k];
  o << "],\"global_buffers\":" << p.gbuf_slots;
  o << ",\"demotions\":[";
  for (size_t k = 0; k < p.demotions.size(); ++k) o << (k ? "," : "") << "\"" << esc(p.demotions[k]) << "\"";
  o << "]";
  o << ",\"needs_sweep2\":" << (p.needs_sweep2 ? "true" : "false");
  if (g.segments_node >= 0)
    o << ",\"ragged\":{\"nseg\":" << g.nseg << ",\"elems\":" << g.seg_elems << "}";
  o << ",\"kernel_count\":" << p.kernels.size() << ",\"memsets_per_run\":0";
  o << ",\"kernels\":[";
  for (size_t k = 0; k < p.kernels.size(); ++k) {
    const Kernel& kk = p.kernels[k];
    if (k) o << ",";
    o << "{\"name\":\"" << kk.name << "\",\"threads\":" << kk.threads << ",\"grid\":" << kk.grid
      << ",\"smem\":" << kk.smem << ",\"cooperative\":" << (kk.cooperative ? "true" : "false")
      << ",\"regs\":" << kk.regs << ",\"spill_bytes\":" << kk.spill_bytes
      << ",\"occupancy_blocks_per_sm\":" << kk.occupancy << ",\"cubin_bytes\":" << kk.cubin.size() << "}";
  }
  o << "],\"shard_kernels\":" << p.shard_kernels.size();
  o << ",\"plan_time_ms\":{\"analyse_map\":" << p.ms_analyse << ",\"codegen\":" << p.ms_codegen
    << ",\"nvrtc\":" << p.ms_nvrtc << ",\"load\":" << p.ms_load << ",\"total\":" << p.ms_total
    << ",\"nvrtc_compiles\":" << p.n_compiles << ",\"cache_hits_memory\":" << p.n_mem_hits
    << ",\"cache_hits_disk\":" << p.n_disk_hits << "}";
  o << ",\"compulsory_bytes\":" << p.compulsory_bytes << "}";
  return o.str();
}

}  // namespace astitch
