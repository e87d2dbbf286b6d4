// Plan construction (JIT) and execution entry points of the C ABI.
#include <chrono>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <regex>
#include <string>

#include "internal.h"

// NVTX ranges (header-only nvtx3: a no-op unless a profiler injects its
// library) around planning and every run, so nsys / ncu timelines show the
// plan (JIT) phases and which plan launched which kernel
#include <nvtx3/nvToolsExt.h>

using namespace astitch;

namespace {
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};
}  // namespace

namespace {

double ms_since(std::chrono::steady_clock::time_point t0) {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}

uint64_t fnv1a(const std::string& s) {
  uint64_t h = 1469598103934665603ULL;
  for (unsigned char c : s) {
    h ^= c;
    h *= 1099511628211ULL;
  }
  return h;
}

void parse_ptxas(Kernel& k) {
  std::smatch mt;
  std::regex rr("Used ([0-9]+) registers");
  if (std::regex_search(k.log, mt, rr)) k.regs = std::stoi(mt[1]);
  std::regex rs("([0-9]+) bytes spill stores");
  if (std::regex_search(k.log, mt, rs)) k.spill_bytes = std::stoi(mt[1]);
}

size_t io_bytes(const Plan& p, int node, astitch_dtype dt) {
  const Node& nd = p.g.nodes[node];
  const size_t R = static_cast<size_t>(p.desc.rows), C = static_cast<size_t>(p.desc.cols);
  const size_t es = dtype_size(dt);
  switch (nd.kind) {
    case ASTITCH_FULL:
      if (p.g.segments_node >= 0) return static_cast<size_t>(p.g.seg_elems) * es;
      return R * C * es;
    case ASTITCH_SEGMENTS: return 16 * static_cast<size_t>(p.g.nseg);
    case ASTITCH_ROWVEC: return R * es;
    case ASTITCH_COLVEC: return C * es;
    case ASTITCH_LENGTHS: {
      size_t rps = static_cast<size_t>(p.g.rows_per_segment);
      return 4 * ((R + rps - 1) / rps);
    }
    default: return 0;
  }
}

const char* role_suffix(int role) {
  switch (role) {
    case ROLE_MAIN: return "";
    case ROLE_SHARD_MAIN: return "_shard";
    case ROLE_SHARD_FINAL: return "_shard_final";
    case ROLE_SHARD_SWEEP2: return "_shard_sweep2";
    case ROLE_FUSED: return "_fused";
  }
  return "";
}

// Build (generate + compile + load) one kernel of the plan.  Applies the
// assume-relax-apply loop: if ptxas spills under the assumed
// register bound, relax the target blocks per SM and recompile.
// Register use and spills come from the loaded function's attributes when a
// device is present (authoritative), else from the ptxas -v log.
static astitch_status compile_and_inspect(Plan& p, Kernel& k, bool load) {
  std::string err;
  if (k.module) drv_unload(k);
  k.regs = -1;
  k.spill_bytes = -1;
  auto t0 = std::chrono::steady_clock::now();
  int cs = 0;
  if (!nvrtc_compile(k.source, k.name, k.cubin, k.log, err, &cs)) return fail(ASTITCH_ERR_CUDA, err);
  p.ms_nvrtc += ms_since(t0);
  if (cs == 0) ++p.n_compiles;
  else if (cs == 1) ++p.n_mem_hits;
  else ++p.n_disk_hits;
  parse_ptxas(k);
  if (load) {
    int log_spill = k.spill_bytes;
    k.spill_bytes = -1;
    auto t1 = std::chrono::steady_clock::now();
    if (!drv_load(p, k, err)) return fail(ASTITCH_ERR_CUDA, err);
    p.ms_load += ms_since(t1);
    k.spill_bytes = std::max(log_spill, k.spill_bytes);
  }
  return ASTITCH_OK;
}

astitch_status build_kernel(Plan& p, int role, Kernel& k) {
  const bool compile = (p.desc.flags & ASTITCH_FLAG_NO_COMPILE) == 0;
  const bool load = compile && p.device >= 0;
  const bool may_relax = (role == ROLE_MAIN);  // later kernels share the main kernel's layout
  // assume-relax-apply as a bisection on blocks per SM: the largest occupancy
  // whose register bound (65536 / (bps * threads)) compiles without spills
  int good = 0, bad = 0;  // best spill-free / smallest spilling bps seen
  // generate + compile for the current p.map (called again after the loop if
  // its attempts run out, so the kernel always matches the final mapping and
  // workspace layout)
  auto gen_compile = [&]() -> astitch_status {
    std::string base = std::string("astitch_") + template_name(p.map.tmpl) + role_suffix(role);
    k.name = base;
    auto tg = std::chrono::steady_clock::now();
    k.source = generate_kernel(p, role, base);
    p.ms_codegen += ms_since(tg);
    char hb[32];
    snprintf(hb, sizeof(hb), "_%012llx", static_cast<unsigned long long>(fnv1a(k.source) & 0xffffffffffffULL));
    // give each specialisation a unique, recognisable symbol
    std::string uniq = base + hb;
    size_t pos = k.source.find(" " + base + "(");
    if (pos != std::string::npos) k.source.replace(pos + 1, base.size(), uniq);
    k.name = uniq;
    k.threads = (role == ROLE_SHARD_FINAL) ? 256 : p.map.threads;
    k.grid = (role == ROLE_SHARD_FINAL) ? std::max<int64_t>(1, (p.desc.cols + 255) / 256) : p.map.grid;
    k.smem = (role == ROLE_SHARD_FINAL) ? 0 : p.map.smem_bytes;
    k.cooperative = (p.map.tmpl == Template::GlobalSweep) &&
                    (role == ROLE_MAIN || role == ROLE_SHARD_MAIN || role == ROLE_FUSED);
    k.pdl = !k.cooperative && role != ROLE_SHARD_FINAL && (p.desc.flags & ASTITCH_FLAG_NO_PDL) == 0;
    const bool clustered = role != ROLE_SHARD_FINAL &&
                           (p.map.tmpl == Template::SplitRow || p.map.tmpl == Template::RowStream) && p.map.split > 1;
    k.cluster = clustered ? p.map.split : 1;
    if (!compile) return ASTITCH_OK;
    return compile_and_inspect(p, k, load);
  };
  for (int attempt = 0; attempt < 10; ++attempt) {
    astitch_status st = gen_compile();
    if (st != ASTITCH_OK || !compile) return st;
    // non-portable clusters (9-16 CTAs): keep them only if every row's
    // cluster is co-resident in one wave; else fall back to portable 8
    if (k.cluster > 8 && load && k.max_clusters >= 0 && k.max_clusters * k.cluster < k.grid && !p.portable_clusters) {
      p.portable_clusters = true;
      select_mapping(p);  // re-plan the row's lanes / chunks for clusters of <= 8
      good = bad = 0;
      continue;
    }
    if (!may_relax || p.tune.bps > 0) return ASTITCH_OK;
    const int cur = p.map.blocks_per_sm;
    // (measured on B200, fp32 softmax rows of 4096 x C: a 116-byte spill
    // (C=30000) costs less than streaming, 448+ bytes (C >= 60000) more)
    if (k.spill_bytes >= 256 && cur == 1 && !p.stream_fallback && p.tune.stream != 0 &&
        (p.map.tmpl == Template::RowTeam || p.map.tmpl == Template::SplitRow) && p.g.lengths_node < 0 &&
        p.g.segments_node < 0 && p.global_fulls.empty()) {
      // the row does not fit the team's registers even at one block per SM:
      // re-plan it as a streamed row (column tiles, one pass per level)
      p.stream_fallback = true;
      select_mapping(p);
      good = bad = 0;
      continue;
    }
    if (k.spill_bytes > 0 && cur == 1 && p.map.row_unroll > 1) {
      // even one block per SM spills: fewer rows in flight per team
      p.map.row_unroll /= 2;
      good = bad = 0;
      retune_grid(p);
      continue;
    }
    // a one-wave row team (every row its own team) tolerates a small spill
    // at its target occupancy: measured on B200 (C2), 40 spilled bytes at
    // 7 blocks/SM 6.8 us vs 7.1 us spill-free at 4 blocks/SM (two row trips)
    // A register row team tolerates a spill of a few registers (<= 32 bytes,
    // L1-resident local memory) rather than halving its occupancy (C3v: 8
    // bytes at 2 blocks/SM 79 us; 1 block/SM spill-free 100 us).
    const bool tolerable = p.map.tmpl == Template::RowTeam &&
                           (k.spill_bytes <= 32 || (p.map.single_wave_bps == cur && k.spill_bytes <= 64));
    if (k.spill_bytes > 0 && cur > 1 && !tolerable) bad = cur;
    else good = cur;
    if (good == cur && (bad == 0 || bad - good <= 1)) return ASTITCH_OK;  // best found
    int next = good > 0 ? (good + bad) / 2 : std::max(1, bad / 2);
    if (next == cur || next < 1) return ASTITCH_OK;
    if (good > 0 && next <= good) next = good;  // re-emit the best spill-free version
    p.map.blocks_per_sm = next;
    p.map.reg_cap = std::min(255, (65536 / (p.map.blocks_per_sm * p.map.threads)) & ~7);
    retune_grid(p);
  }
  // attempts exhausted after a retune: the last compiled kernel may not match
  // p.map / p.ws any more -- compile the final mapping once more
  return gen_compile();
}

}  // namespace

namespace astitch {
// "key=value,key=value" -> Tuning (integers only; unknown keys are errors)
bool parse_tuning(const char* s, Tuning& t, std::string& err) {
  t = Tuning();
  if (!s) return true;
  t.text = s;
  std::string str(s);
  size_t pos = 0;
  while (pos < str.size()) {
    size_t end = str.find(',', pos);
    if (end == std::string::npos) end = str.size();
    std::string item = str.substr(pos, end - pos);
    pos = end + 1;
    if (item.empty()) continue;
    size_t eq = item.find('=');
    if (eq == std::string::npos) { err = "tuning item without '=': " + item; return false; }
    std::string key = item.substr(0, eq), val = item.substr(eq + 1);
    char* ep = nullptr;
    long v = strtol(val.c_str(), &ep, 10);
    if (val.empty() || *ep != '\0') { err = "tuning value is not an integer: " + item; return false; }
    const int iv = static_cast<int>(v);
    struct { const char* k; int* f; } keys[] = {
        {"threads", &t.threads}, {"unroll", &t.unroll}, {"team", &t.team}, {"bps", &t.bps},
        {"vec_bytes", &t.vec_bytes}, {"hoist", &t.hoist}, {"tile_stages", &t.tile_stages},
        {"tile_rows", &t.tile_rows}, {"tile_threads", &t.tile_threads}, {"split", &t.split},
        {"split_threads", &t.split_threads}, {"stream", &t.stream}, {"stage", &t.stage},
        {"stage_kb", &t.stage_kb}, {"portable_clusters", &t.portable_clusters},
        {"sync", &t.sync}, {"prefetch", &t.prefetch}, {"persistent", &t.persistent}, {"waves", &t.waves},
        {"remat", &t.remat}, {"tma", &t.tma}, {"tma_rows", &t.tma_rows}, {"tma_stages", &t.tma_stages}, {"tma_teams", &t.tma_teams}, {"tma_team", &t.tma_team}};
    bool found = false;
    for (auto& kv : keys)
      if (key == kv.k) { *kv.f = iv; found = true; }
    if (!found) { err = "unknown tuning key: " + key; return false; }
  }
  return true;
}
}  // namespace astitch

namespace astitch {
// (comm.cpp) build one more kernel of a plan, e.g. the fused sharded role
astitch_status build_plan_kernel(Plan& p, int role, Kernel& k) { return build_kernel(p, role, k); }
}  // namespace astitch

extern "C" {

astitch_status astitch_plan(astitch_graph_t gr, const astitch_plan_desc* desc, astitch_plan_t* out) {
  return astitch_plan_ex(gr, desc, nullptr, out);
}

astitch_status astitch_plan_ex(astitch_graph_t gr, const astitch_plan_desc* desc, const char* tuning,
                               astitch_plan_t* out) {
  if (!gr || !desc || !out) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL graph, desc or out");
  NvtxRange nvtx("astitch_plan");
  *out = nullptr;
  if (desc->rows < 0) return fail(ASTITCH_ERR_SHAPE, "rows < 0");
  if (desc->cols < 1) return fail(ASTITCH_ERR_SHAPE, "cols < 1");
  if (desc->cols > (1LL << 31) || desc->rows > (1LL << 40) ||
      static_cast<double>(desc->rows) * static_cast<double>(desc->cols) > 4.0e12)
    return fail(ASTITCH_ERR_SHAPE, "shape too large");
  if (desc->shard_world < 0 || (desc->shard_world > 0 && (desc->shard_rank < 0 || desc->shard_rank >= desc->shard_world)))
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad shard_rank / shard_world");
  if (gr->g.outputs.empty()) return fail(ASTITCH_ERR_INVALID_GRAPH, "graph has no outputs");
  for (int id : gr->g.inputs)
    if (gr->g.nodes[id].kind == ASTITCH_LENGTHS && id != gr->g.lengths_node)
      return fail(ASTITCH_ERR_INVALID_GRAPH, "LENGTHS input not bound by astitch_graph_set_mask");
  try {
    const auto t_start = std::chrono::steady_clock::now();
    auto plan = std::make_unique<Plan>();
    Plan& p = *plan;
    p.g = gr->g;
    p.desc = *desc;
    {
      std::string terr;
      if (!parse_tuning(tuning, p.tune, terr)) return fail(ASTITCH_ERR_INVALID_ARGUMENT, terr);
    }
    if (p.desc.shard_world == 0) p.desc.shard_world = 1;
    p.device = desc->device;
    p.sm_count = desc->sm_count > 0 ? desc->sm_count : 148;
    if (p.device >= 0) {
      std::string err;
      int sms = 0, smem_optin = 0;
      if (!drv_device_info(p.device, sms, smem_optin, err)) return fail(ASTITCH_ERR_CUDA, err);
      if (desc->sm_count <= 0) p.sm_count = sms;
      if (smem_optin > 0) p.smem_optin = smem_optin;
    }
    analyse(p);
    if (p.desc.shard_world > 1 && (p.desc.flags & ASTITCH_FLAG_FORCE_GLOBAL))
      return fail(ASTITCH_ERR_UNSUPPORTED, "FORCE_GLOBAL ablation runs unsharded only");
    if (p.desc.shard_world > 1 && p.max_level > 1)
      return fail(ASTITCH_ERR_UNSUPPORTED,
                  "row-sharded plans support one level of column reductions (one allreduce)");
    select_mapping(p);
    plan_workspace(p);
    p.compulsory_bytes = compulsory_bytes(p);
    p.ms_analyse = ms_since(t_start);

    std::vector<int> roles = {ROLE_MAIN};
    p.kernels.resize(1);
    astitch_status s = build_kernel(p, ROLE_MAIN, p.kernels[0]);
    if (s != ASTITCH_OK) return s;
    if (p.map.tmpl == Template::GlobalSweep && p.desc.shard_world > 1) {
      std::vector<int> sr = {ROLE_SHARD_MAIN, ROLE_SHARD_FINAL};
      if (p.needs_sweep2) sr.push_back(ROLE_SHARD_SWEEP2);
      p.shard_kernels.resize(sr.size());
      for (size_t i = 0; i < sr.size(); ++i) {
        s = build_kernel(p, sr[i], p.shard_kernels[i]);
        if (s != ASTITCH_OK) return s;
      }
    }
    // workspace offsets are baked into the sources: keep the layout computed
    // for the planned (maximum) grid; the launch grid may only shrink.
    if (p.device >= 0 && (p.desc.flags & ASTITCH_FLAG_NO_COMPILE) == 0) {
      auto load = [&](Kernel& k) -> astitch_status {
        std::string err;
        if (!k.module && !drv_load(p, k, err)) return fail(ASTITCH_ERR_CUDA, err);
        if (k.cooperative) {
          int64_t max_grid = static_cast<int64_t>(k.occupancy) * p.sm_count;
          if (max_grid < 1)
            return fail(ASTITCH_ERR_RESOURCE, "kernel " + k.name + " cannot be resident (occupancy 0)");
          if (p.map.nslab > 1) max_grid = (max_grid / p.map.nslab) * p.map.nslab;  // whole row groups
          if (max_grid < 1)
            return fail(ASTITCH_ERR_RESOURCE, "kernel " + k.name + ": fewer resident CTAs than column slabs");
          if (k.grid > max_grid) {
            // the planned one-wave grid is not co-resident (the register /
            // smem estimate was optimistic): STRICT refuses, otherwise the
            // persistent grid shrinks to what is resident (still one kernel)
            if (p.desc.flags & ASTITCH_FLAG_STRICT_SINGLE_KERNEL)
              return fail(ASTITCH_ERR_RESOURCE, "kernel " + k.name + ": planned grid " + std::to_string(k.grid) +
                                                    " > resident " + std::to_string(max_grid) + " (STRICT_SINGLE_KERNEL)");
            p.demotions.push_back("grid " + std::to_string(k.grid) + " -> " + std::to_string(max_grid) + " (residency)");
            k.grid = max_grid;
          }
        }
        return ASTITCH_OK;
      };
      for (auto& k : p.kernels)
        if ((s = load(k)) != ASTITCH_OK) return s;
      for (auto& k : p.shard_kernels)
        if ((s = load(k)) != ASTITCH_OK) return s;
    }
    p.ms_total = ms_since(t_start);
    p.describe = describe_json(p);
    if (log_enabled())
      fprintf(stderr, "[astitch] plan %lldx%lld: %s, kernel %s grid %lld x %d threads, %d regs, %d B smem, "
              "%zu demotion(s), %.1f ms (nvrtc %.1f ms, %d compiled, %d cached)\n",
              static_cast<long long>(p.desc.rows), static_cast<long long>(p.desc.cols), template_name(p.map.tmpl),
              p.kernels.empty() ? "-" : p.kernels[0].name.c_str(),
              static_cast<long long>(p.kernels.empty() ? 0 : p.kernels[0].grid), p.map.threads,
              p.kernels.empty() ? -1 : p.kernels[0].regs, p.map.smem_bytes, p.demotions.size(), p.ms_total,
              p.ms_nvrtc, p.n_compiles, p.n_mem_hits + p.n_disk_hits);
    auto* h = new astitch_plan_s();
    h->p = std::move(plan);
    *out = h;
    set_error("");
    return ASTITCH_OK;
  } catch (const Error& e) {
    return fail(e.status, e.msg);
  } catch (const std::exception& e) {
    return fail(ASTITCH_ERR_INTERNAL, e.what());
  }
}

astitch_status astitch_set_cache_dir(const char* dir) {
  set_cache_dir(dir);
  return ASTITCH_OK;
}

astitch_status astitch_plan_destroy(astitch_plan_t h) {
  if (!h) return ASTITCH_OK;
  for (auto& k : h->p->kernels) drv_unload(k);
  for (auto& k : h->p->shard_kernels) drv_unload(k);
  for (auto& k : h->p->chunk_kernels) drv_unload(k);
  for (auto& k : h->p->fused_kernels) drv_unload(k);
  for (void* s : h->p->pipe_streams) drv_stream_destroy(s);
  for (void* e : h->p->pipe_events) drv_event_destroy(e);
  delete h;
  return ASTITCH_OK;
}

astitch_status astitch_plan_workspace_bytes(astitch_plan_t h, size_t* bytes) {
  if (!h || !bytes) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL plan or bytes");
  *bytes = h->p->ws.total;
  return ASTITCH_OK;
}

static astitch_status copy_out(const std::string& s, char* buf, size_t cap, size_t* len) {
  if (len) *len = s.size();
  if (buf && cap > 0) {
    size_t n = std::min(cap - 1, s.size());
    memcpy(buf, s.data(), n);
    buf[n] = '\0';
  }
  return ASTITCH_OK;
}

astitch_status astitch_plan_describe(astitch_plan_t h, char* json, size_t cap, size_t* len) {
  if (!h) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL plan");
  return copy_out(h->p->describe, json, cap, len);
}

static const Kernel* kernel_at(const Plan& p, int32_t k) {
  if (k < 0) return nullptr;
  if (k < static_cast<int32_t>(p.kernels.size())) return &p.kernels[k];
  k -= static_cast<int32_t>(p.kernels.size());
  if (k < static_cast<int32_t>(p.shard_kernels.size())) return &p.shard_kernels[k];
  return nullptr;
}

astitch_status astitch_plan_source(astitch_plan_t h, int32_t k, char* buf, size_t cap, size_t* len) {
  if (!h) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL plan");
  const Kernel* kk = kernel_at(*h->p, k);
  if (!kk) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "kernel index out of range");
  return copy_out(kk->source, buf, cap, len);
}

astitch_status astitch_plan_cubin(astitch_plan_t h, int32_t k, void* buf, size_t cap, size_t* len) {
  if (!h) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL plan");
  const Kernel* kk = kernel_at(*h->p, k);
  if (!kk) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "kernel index out of range");
  if (len) *len = kk->cubin.size();
  if (buf && cap >= kk->cubin.size()) memcpy(buf, kk->cubin.data(), kk->cubin.size());
  return ASTITCH_OK;
}

astitch_status astitch_plan_kernel_count(astitch_plan_t h, int32_t* n) {
  if (!h || !n) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL plan or n");
  *n = static_cast<int32_t>(h->p->kernels.size());
  return ASTITCH_OK;
}

astitch_status astitch_plan_io_count(astitch_plan_t h, int32_t* ni, int32_t* no) {
  if (!h || !ni || !no) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL argument");
  *ni = static_cast<int32_t>(h->p->g.inputs.size());
  *no = static_cast<int32_t>(h->p->g.outputs.size());
  return ASTITCH_OK;
}

astitch_status astitch_plan_io(astitch_plan_t h, int32_t is_output, int32_t index, astitch_kind* kind,
                               astitch_dtype* dtype) {
  if (!h || !kind || !dtype) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL argument");
  const Graph& g = h->p->g;
  if (is_output) {
    if (index < 0 || index >= static_cast<int32_t>(g.outputs.size()))
      return fail(ASTITCH_ERR_INVALID_ARGUMENT, "output index out of range");
    *kind = g.nodes[g.outputs[index]].kind;
    *dtype = g.output_dtypes[index];
  } else {
    if (index < 0 || index >= static_cast<int32_t>(g.inputs.size()))
      return fail(ASTITCH_ERR_INVALID_ARGUMENT, "input index out of range");
    *kind = g.nodes[g.inputs[index]].kind;
    *dtype = g.nodes[g.inputs[index]].dtype;
  }
  return ASTITCH_OK;
}

astitch_status astitch_workspace_init(astitch_plan_t h, void* ws, void* stream) {
  if (!h) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL plan");
  const Plan& p = *h->p;
  if (p.ws.total == 0) return ASTITCH_OK;
  if (!ws) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "plan needs a workspace");
  std::string err;
  if (!drv_memset_async(static_cast<char*>(ws) + p.ws.barrier, 256, stream, err))
    return fail(ASTITCH_ERR_CUDA, err);
  return ASTITCH_OK;
}

}  // extern "C"

namespace astitch {

astitch_status check_io(const Plan& p, const void* const* inputs, void* const* outputs, void* ws) {
  const Graph& g = p.g;
  if (!inputs && !g.inputs.empty()) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "inputs is NULL");
  if (!outputs) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "outputs is NULL");
  for (size_t i = 0; i < g.inputs.size(); ++i) {
    if (!inputs[i]) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "input " + std::to_string(i) + " is NULL");
    if (reinterpret_cast<uintptr_t>(inputs[i]) % 16)
      return fail(ASTITCH_ERR_INVALID_ARGUMENT, "input " + std::to_string(i) + " is not 16-byte aligned");
  }
  for (size_t i = 0; i < g.outputs.size(); ++i) {
    if (!outputs[i]) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "output " + std::to_string(i) + " is NULL");
    if (reinterpret_cast<uintptr_t>(outputs[i]) % 16)
      return fail(ASTITCH_ERR_INVALID_ARGUMENT, "output " + std::to_string(i) + " is not 16-byte aligned");
  }
  if (p.ws.total > 0 && !ws) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "plan needs a workspace");
  if (ws && reinterpret_cast<uintptr_t>(ws) % 256) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "workspace not 256-byte aligned");
  if (p.kernels.empty() || !p.kernels[0].function)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "plan was built without a device (device = -1 or NO_COMPILE)");
  return ASTITCH_OK;
}

KernelParams make_params(const Plan& p, const void* const* inputs, void* const* outputs, void* ws) {
  KernelParams kp;
  memset(&kp, 0, sizeof(kp));
  for (size_t i = 0; i < p.g.inputs.size(); ++i) kp.in[i] = inputs[i];
  for (size_t i = 0; i < p.g.outputs.size(); ++i) kp.out[i] = outputs[i];
  kp.ws = ws;
  kp.rows = p.desc.rows;
  kp.row_offset = 0;
  return kp;
}

astitch_status launch(const Plan& p, const Kernel& k, KernelParams& kp, void* stream) {
  std::string err;
  if (!drv_launch(k, &kp, sizeof(kp), stream, err)) return fail(ASTITCH_ERR_CUDA, err);
  if (p.desc.flags & ASTITCH_FLAG_LAUNCH_CHECK) {
    if (!drv_sync(stream, err)) return fail(ASTITCH_ERR_CUDA, err);
  }
  return ASTITCH_OK;
}

}  // namespace astitch

extern "C" {

astitch_status astitch_run(astitch_plan_t h, const void* const* inputs, void* const* outputs, void* ws,
                           void* stream) {
  if (!h) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL plan");
  const Plan& p = *h->p;
  if (p.desc.rows == 0) return ASTITCH_OK;
  NvtxRange nvtx("astitch_run");
  astitch_status s = check_io(p, inputs, outputs, ws);
  if (s != ASTITCH_OK) return s;
  KernelParams kp = make_params(p, inputs, outputs, ws);
  for (const Kernel& k : p.kernels)
    if ((s = launch(p, k, kp, stream)) != ASTITCH_OK) return s;
  return ASTITCH_OK;
}

}  // extern "C"

namespace astitch {
// H2D of every input, `run` (the stitched kernel(s) on the device buffers),
// D2H of every output, all asynchronous on `stream`
template <typename F>
astitch_status run_with_host_copies(astitch_plan_t h, const void* const* host_inputs, void* const* host_outputs,
                                    const void* const* dev_inputs, void* const* dev_outputs, void* stream, F run) {
  if (!h || !host_inputs || !host_outputs || !dev_inputs || !dev_outputs)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL argument");
  const Plan& p = *h->p;
  if (p.desc.rows == 0) return ASTITCH_OK;
  std::string err;
  for (size_t i = 0; i < p.g.inputs.size(); ++i) {
    int node = p.g.inputs[i];
    size_t nbytes = io_bytes(p, node, p.g.nodes[node].dtype);
    if (!host_inputs[i]) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "host input NULL");
    if (!drv_memcpy_async(const_cast<void*>(dev_inputs[i]), host_inputs[i], nbytes, 1, stream, err))
      return fail(ASTITCH_ERR_CUDA, err);
  }
  astitch_status s = run();
  if (s != ASTITCH_OK) return s;
  for (size_t i = 0; i < p.g.outputs.size(); ++i) {
    size_t nbytes = io_bytes(p, p.g.outputs[i], p.g.output_dtypes[i]);
    if (!host_outputs[i]) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "host output NULL");
    if (!drv_memcpy_async(host_outputs[i], dev_outputs[i], nbytes, 2, stream, err))
      return fail(ASTITCH_ERR_CUDA, err);
  }
  return ASTITCH_OK;
}
}  // namespace astitch

extern "C" {

astitch_status astitch_run_sharded_host(astitch_plan_t h, astitch_comm_t c, astitch_peer_t x,
                                        const void* const* host_inputs, void* const* host_outputs,
                                        const void* const* dev_inputs, void* const* dev_outputs, void* ws,
                                        void* stream) {
  return run_with_host_copies(h, host_inputs, host_outputs, dev_inputs, dev_outputs, stream, [&]() {
    return x ? astitch_run_fused(h, x, dev_inputs, dev_outputs, ws, stream)
             : astitch_run_sharded(h, c, dev_inputs, dev_outputs, ws, stream);
  });
}

astitch_status astitch_run_host(astitch_plan_t h, const void* const* host_inputs, void* const* host_outputs,
                                const void* const* dev_inputs, void* const* dev_outputs, void* ws, void* stream) {
  return run_with_host_copies(h, host_inputs, host_outputs, dev_inputs, dev_outputs, stream,
                              [&]() { return astitch_run(h, dev_inputs, dev_outputs, ws, stream); });
}

astitch_status astitch_run_host_pipelined(astitch_plan_t h, const void* const* host_inputs,
                                          void* const* host_outputs, const void* const* dev_inputs,
                                          void* const* dev_outputs, void* ws, void* stream, int32_t chunks) {
  if (!h || !host_inputs || !host_outputs || !dev_inputs || !dev_outputs)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL argument");
  Plan& p = *h->p;
  const int64_t R = p.desc.rows;
  const bool global = p.map.tmpl == Template::GlobalSweep;
  // rows are the independent units: chunk them; a column reduction accumulates
  // its totals across chunks and its consumers run once at the end
  if (chunks <= 1 || R < static_cast<int64_t>(chunks) * 64 || (global && p.needs_sweep2) ||
      p.desc.shard_world > 1 || p.map.tmpl == Template::SplitRow || p.map.tmpl == Template::RowStream || p.device < 0 || p.g.segments_node >= 0)
    return astitch_run_host(h, host_inputs, host_outputs, dev_inputs, dev_outputs, ws, stream);
  if (chunks > 64) chunks = 64;
  astitch_status s = check_io(p, dev_inputs, dev_outputs, ws);
  if (s != ASTITCH_OK) return s;
  std::string err;
  if (global && p.chunk_kernels.empty()) {
    p.chunk_kernels.resize(2);
    if ((s = build_kernel(p, ROLE_SHARD_MAIN, p.chunk_kernels[0])) != ASTITCH_OK) return s;
    if ((s = build_kernel(p, ROLE_SHARD_FINAL, p.chunk_kernels[1])) != ASTITCH_OK) return s;
    for (Kernel& k : p.chunk_kernels) {
      if (!k.module && !drv_load(p, k, err)) return fail(ASTITCH_ERR_CUDA, err);
      if (k.cooperative) {
        k.grid = resident_grid(p, k);
        if (k.grid < 1) return fail(ASTITCH_ERR_RESOURCE, "chunk kernel cannot be resident");
      }
    }
  }
  for (int i = 0; i < 3; ++i)
    if (!p.pipe_streams[i] && !drv_stream_create(&p.pipe_streams[i], err)) return fail(ASTITCH_ERR_CUDA, err);
  while (p.pipe_events.size() < static_cast<size_t>(2 * chunks + 3)) {
    void* e = nullptr;
    if (!drv_event_create(&e, err)) return fail(ASTITCH_ERR_CUDA, err);
    p.pipe_events.push_back(e);
  }
  void* s_in = p.pipe_streams[0];
  void* s_comp = p.pipe_streams[1];
  void* s_out = p.pipe_streams[2];
  auto& ev = p.pipe_events;
  auto ck = [&](bool ok) { return ok ? ASTITCH_OK : fail(ASTITCH_ERR_CUDA, err); };
  // fork from the caller's stream
  if ((s = ck(drv_event_record(ev[0], stream, err))) != ASTITCH_OK) return s;
  for (void* st : {s_in, s_comp, s_out})
    if ((s = ck(drv_stream_wait(st, ev[0], err))) != ASTITCH_OK) return s;
  const size_t C = static_cast<size_t>(p.desc.cols);
  auto row_scaled = [&](astitch_kind k, int64_t rows, astitch_dtype dt) -> size_t {
    if (k == ASTITCH_FULL) return static_cast<size_t>(rows) * C * dtype_size(dt);
    if (k == ASTITCH_ROWVEC) return static_cast<size_t>(rows) * dtype_size(dt);
    return 0;
  };
  for (int c = 0; c < chunks; ++c) {
    const int64_t b = (R * c) / chunks, n = (R * (c + 1)) / chunks - b;
    // copy-in of the chunk's rows (vectors and lengths once, with chunk 0)
    for (size_t i = 0; i < p.g.inputs.size(); ++i) {
      const Node& nd = p.g.nodes[p.g.inputs[i]];
      size_t off = row_scaled(nd.kind, b, nd.dtype), nb = row_scaled(nd.kind, n, nd.dtype);
      if (nd.kind != ASTITCH_FULL && nd.kind != ASTITCH_ROWVEC) {
        if (c != 0) continue;
        off = 0;
        nb = io_bytes(p, p.g.inputs[i], nd.dtype);
      }
      if (!host_inputs[i]) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "host input NULL");
      if (!drv_memcpy_async(static_cast<char*>(const_cast<void*>(dev_inputs[i])) + off,
                            static_cast<const char*>(host_inputs[i]) + off, nb, 1, s_in, err))
        return fail(ASTITCH_ERR_CUDA, err);
    }
    if ((s = ck(drv_event_record(ev[1 + 2 * c], s_in, err))) != ASTITCH_OK) return s;
    if ((s = ck(drv_stream_wait(s_comp, ev[1 + 2 * c], err))) != ASTITCH_OK) return s;
    // the stitched kernel on the chunk's rows
    KernelParams kp = make_params(p, dev_inputs, dev_outputs, ws);
    for (size_t i = 0; i < p.g.inputs.size(); ++i) {
      const Node& nd = p.g.nodes[p.g.inputs[i]];
      kp.in[i] = static_cast<const char*>(dev_inputs[i]) + row_scaled(nd.kind, b, nd.dtype);
    }
    for (size_t i = 0; i < p.g.outputs.size(); ++i)
      kp.out[i] = static_cast<char*>(dev_outputs[i]) +
                  row_scaled(p.g.nodes[p.g.outputs[i]].kind, b, p.g.output_dtypes[i]);
    kp.rows = n;
    kp.row_offset = b;
    kp.flags = (global && c > 0) ? 1 : 0;
    if ((s = launch(p, global ? p.chunk_kernels[0] : p.kernels[0], kp, s_comp)) != ASTITCH_OK) return s;
    if ((s = ck(drv_event_record(ev[2 + 2 * c], s_comp, err))) != ASTITCH_OK) return s;
    if ((s = ck(drv_stream_wait(s_out, ev[2 + 2 * c], err))) != ASTITCH_OK) return s;
    // copy-out of the chunk's row outputs
    for (size_t i = 0; i < p.g.outputs.size(); ++i) {
      const astitch_kind k = p.g.nodes[p.g.outputs[i]].kind;
      if (k != ASTITCH_FULL && k != ASTITCH_ROWVEC) continue;
      size_t off = row_scaled(k, b, p.g.output_dtypes[i]), nb = row_scaled(k, n, p.g.output_dtypes[i]);
      if (!host_outputs[i]) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "host output NULL");
      if (!drv_memcpy_async(static_cast<char*>(host_outputs[i]) + off, static_cast<char*>(dev_outputs[i]) + off, nb,
                            2, s_out, err))
        return fail(ASTITCH_ERR_CUDA, err);
    }
  }
  if (global) {  // column consumers once every chunk has accumulated
    KernelParams kp = make_params(p, dev_inputs, dev_outputs, ws);
    if ((s = launch(p, p.chunk_kernels[1], kp, s_comp)) != ASTITCH_OK) return s;
    if ((s = ck(drv_event_record(ev[2 * chunks + 1], s_comp, err))) != ASTITCH_OK) return s;
    if ((s = ck(drv_stream_wait(s_out, ev[2 * chunks + 1], err))) != ASTITCH_OK) return s;
    for (size_t i = 0; i < p.g.outputs.size(); ++i) {
      if (p.g.nodes[p.g.outputs[i]].kind != ASTITCH_COLVEC) continue;
      if (!drv_memcpy_async(host_outputs[i], dev_outputs[i], io_bytes(p, p.g.outputs[i], p.g.output_dtypes[i]), 2,
                            s_out, err))
        return fail(ASTITCH_ERR_CUDA, err);
    }
  }
  // join back into the caller's stream
  if ((s = ck(drv_event_record(ev[2 * chunks + 2], s_out, err))) != ASTITCH_OK) return s;
  return ck(drv_stream_wait(stream, ev[2 * chunks + 2], err));
}

}  // extern "C"

// ------------------------------------------------------------------ measurement aids
namespace {
struct BenchModule {
  Kernel barrier, copy;
  bool ok = false;
};
std::mutex g_bench_mu;
BenchModule g_bench[64];

astitch_status bench_module(int device, BenchModule*& out) {
  if (device < 0 || device >= 64) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad device");
  std::lock_guard<std::mutex> lk(g_bench_mu);
  BenchModule& b = g_bench[device];
  if (!b.ok) {
    std::string err, log;
    std::vector<char> cubin;
    std::string src = "#define ASTITCH_BENCH_KERNELS 1\n#include \"astitch_device.cuh\"\n";
    if (!nvrtc_compile(src, "astitch_bench", cubin, log, err)) return fail(ASTITCH_ERR_CUDA, err);
    Plan tmp;
    tmp.device = device;
    b.barrier.cubin = cubin;
    b.barrier.name = "astitch_barrier_bench";
    b.barrier.threads = 1024;
    b.copy.cubin = cubin;
    b.copy.name = "astitch_copy_bench";
    b.copy.threads = 256;
    if (!drv_load(tmp, b.barrier, err)) return fail(ASTITCH_ERR_CUDA, err);
    if (!drv_load(tmp, b.copy, err)) return fail(ASTITCH_ERR_CUDA, err);
    b.ok = true;
  }
  out = &b;
  return ASTITCH_OK;
}
}  // namespace

extern "C" {

astitch_status astitch_bench_barrier(int32_t device, int32_t blocks, int32_t threads, int32_t iters, void* ws,
                                     void* stream) {
  if (blocks < 1 || threads < 32 || threads > 1024 || iters < 0 || !ws)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad barrier bench arguments");
  BenchModule* b = nullptr;
  astitch_status s = bench_module(device, b);
  if (s != ASTITCH_OK) return s;
  Kernel k = b->barrier;
  k.grid = blocks;
  k.threads = threads;
  k.cooperative = true;
  void* bar = ws;
  int it = iters;
  void* argv[] = {&bar, &it};
  std::string err;
  if (!drv_launch_args(k, argv, stream, err)) return fail(ASTITCH_ERR_CUDA, err);
  return ASTITCH_OK;
}

astitch_status astitch_bench_copy(int32_t device, const void* src, void* dst, size_t bytes, void* stream) {
  if (!src || !dst || bytes % 16) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad copy arguments");
  BenchModule* b = nullptr;
  astitch_status s = bench_module(device, b);
  if (s != ASTITCH_OK) return s;
  Kernel k = b->copy;
  k.threads = 256;
  int sms = 148, smem = 0;
  std::string err;
  drv_device_info(device, sms, smem, err);
  k.grid = static_cast<int64_t>(sms) * 8;
  long long n16 = static_cast<long long>(bytes / 16);
  const void* s_ = src;
  void* d_ = dst;
  void* argv[] = {&s_, &d_, &n16};
  if (!drv_launch_args(k, argv, stream, err)) return fail(ASTITCH_ERR_CUDA, err);
  return ASTITCH_OK;
}

}  // extern "C"
