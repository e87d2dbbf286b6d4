// Row-sharded multi-GPU execution (BASELINE north_star (4); not in the paper,
// which is single-GPU).  Rows are independent units: a row-only
// subgraph runs unchanged on each rank's row slice.  A column reduction over
// the sharded row dimension is completed with ONE ncclAllReduce of the
// per-rank fp32 partials on the caller's stream (over NVLink / NVSwitch),
// followed by a small epilogue kernel for the column consumers.
//
// libnccl is dlopen'ed (PyTorch's copy is already loaded in-process).
#include <dlfcn.h>

#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "internal.h"
#include "nccl.h"

using namespace astitch;

namespace {

struct Nccl {
  void* h = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*);
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int);
  ncclResult_t (*CommDestroy)(ncclComm_t);
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t);
  const char* (*GetErrorString)(ncclResult_t);
};

Nccl* nccl(std::string& err) {
  static Nccl n;
  static bool tried = false;
  static std::string load_err;
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  if (tried) {
    if (!n.h) err = load_err;
    return n.h ? &n : nullptr;
  }
  tried = true;
  const char* cands[] = {getenv("ASTITCH_NCCL"), "libnccl.so.2", "libnccl.so"};
  for (const char* c : cands) {
    if (!c) continue;
    n.h = dlopen(c, RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
    if (!n.h) n.h = dlopen(c, RTLD_NOW | RTLD_GLOBAL);
    if (n.h) break;
  }
  if (!n.h) {
    load_err = "cannot dlopen libnccl.so.2 (import torch first or set ASTITCH_NCCL)";
    err = load_err;
    return nullptr;
  }
#define SYM(field, name)                                   \
  *reinterpret_cast<void**>(&n.field) = dlsym(n.h, name);  \
  if (!n.field) {                                          \
    load_err = std::string("libnccl lacks ") + name;       \
    err = load_err;                                        \
    n.h = nullptr;                                         \
    return nullptr;                                        \
  }
  SYM(GetUniqueId, "ncclGetUniqueId");
  SYM(CommInitRank, "ncclCommInitRank");
  SYM(CommDestroy, "ncclCommDestroy");
  SYM(AllReduce, "ncclAllReduce");
  SYM(GetErrorString, "ncclGetErrorString");
#undef SYM
  return &n;
}

}  // namespace

struct astitch_comm_s {
  ncclComm_t comm = nullptr;
  int world = 1, rank = 0, device = 0;
};

struct astitch_peer_s {
  int world = 1, rank = 0, device = 0;
  size_t bytes = 0;
  void* local = nullptr;                  // this rank's exchange buffer (cuMemAlloc)
  std::vector<void*> ptrs;                // every rank's buffer as addressed from this process
  std::vector<bool> opened;               // ptrs[q] came from cuIpcOpenMemHandle (close on destroy)
  bool table_dirty = true;
};

namespace astitch {
astitch_status build_plan_kernel(Plan& p, int role, Kernel& k);
astitch_status check_io(const Plan& p, const void* const* inputs, void* const* outputs, void* ws);
KernelParams make_params(const Plan& p, const void* const* inputs, void* const* outputs, void* ws);
astitch_status launch(const Plan& p, const Kernel& k, KernelParams& kp, void* stream);
}  // namespace astitch

extern "C" {

astitch_status astitch_comm_unique_id(uint8_t id[128]) {
  if (!id) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL id");
  std::string err;
  Nccl* n = nccl(err);
  if (!n) return fail(ASTITCH_ERR_NCCL, err);
  ncclUniqueId u;
  ncclResult_t r = n->GetUniqueId(&u);
  if (r != ncclSuccess) return fail(ASTITCH_ERR_NCCL, n->GetErrorString(r));
  static_assert(sizeof(u) == 128, "ncclUniqueId size");
  memcpy(id, &u, 128);
  return ASTITCH_OK;
}

astitch_status astitch_comm_create(int32_t world, int32_t rank, const uint8_t id[128], int32_t device,
                                   astitch_comm_t* out) {
  if (!id || !out || world < 1 || rank < 0 || rank >= world || device < 0)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "bad comm arguments");
  std::string err;
  Nccl* n = nccl(err);
  if (!n) return fail(ASTITCH_ERR_NCCL, err);
  int sms = 0, smem = 0;
  if (!drv_device_info(device, sms, smem, err)) return fail(ASTITCH_ERR_CUDA, err);
  ncclUniqueId u;
  memcpy(&u, id, 128);
  auto* c = new astitch_comm_s();
  ncclResult_t r = n->CommInitRank(&c->comm, world, u, rank);
  if (r != ncclSuccess) {
    delete c;
    return fail(ASTITCH_ERR_NCCL, std::string("ncclCommInitRank: ") + n->GetErrorString(r));
  }
  c->world = world;
  c->rank = rank;
  c->device = device;
  *out = c;
  return ASTITCH_OK;
}

astitch_status astitch_comm_destroy(astitch_comm_t c) {
  if (!c) return ASTITCH_OK;
  std::string err;
  Nccl* n = nccl(err);
  if (n && c->comm) n->CommDestroy(c->comm);
  delete c;
  return ASTITCH_OK;
}

astitch_status astitch_run_sharded(astitch_plan_t h, astitch_comm_t c, const void* const* inputs,
                                   void* const* outputs, void* ws, void* stream) {
  if (!h) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL plan");
  const Plan& p = *h->p;
  // row-local subgraphs: no communication at all
  if (p.colreds.empty() || p.desc.shard_world <= 1) return astitch_run(h, inputs, outputs, ws, stream);
  if (!c) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "column reduction over shards needs a comm");
  if (c->world != p.desc.shard_world || c->rank != p.desc.shard_rank)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "comm world/rank do not match the plan's shard");
  if (p.shard_kernels.empty() || !p.shard_kernels[0].function)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "plan has no loaded sharded kernels");
  astitch_status s = ASTITCH_OK;
  // empty shard: contribute identity partials (the main kernel still runs its
  // combine with zero rows, writing 0 / -inf partials)
  s = check_io(p, inputs, outputs, ws);
  if (s != ASTITCH_OK) return s;
  KernelParams kp = make_params(p, inputs, outputs, ws);
  if ((s = launch(p, p.shard_kernels[0], kp, stream)) != ASTITCH_OK) return s;
  std::string err;
  Nccl* n = nccl(err);
  if (!n) return fail(ASTITCH_ERR_NCCL, err);
  const size_t C = static_cast<size_t>(p.desc.cols);
  char* colpart = static_cast<char*>(ws) + p.ws.colvals + p.post_colvecs.size() * C * 4;
  for (size_t q = 0; q < p.colreds.size(); ++q) {
    // MAX slots hold int32 order keys (codegen: as::okey): an integer max
    // keeps NaN, which ncclMax on fp32 would drop (reading R12)
    const bool mx = p.g.nodes[p.colreds[q]].sub == ASTITCH_RMAX;
    float* buf = reinterpret_cast<float*>(colpart) + q * C;
    ncclResult_t r = n->AllReduce(buf, buf, C, mx ? ncclInt32 : ncclFloat32, mx ? ncclMax : ncclSum, c->comm,
                                  static_cast<cudaStream_t>(stream));
    if (r != ncclSuccess) return fail(ASTITCH_ERR_NCCL, std::string("ncclAllReduce: ") + n->GetErrorString(r));
  }
  for (size_t i = 1; i < p.shard_kernels.size(); ++i)
    if ((s = launch(p, p.shard_kernels[i], kp, stream)) != ASTITCH_OK) return s;
  return ASTITCH_OK;
}

// ---------------------------------------------------------------- fused sharded run (NEXT f1)
astitch_status astitch_peer_create(astitch_plan_t h, astitch_peer_t* out, uint8_t ipc_handle[64]) {
  if (!h || !out) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL plan or out");
  *out = nullptr;
  const Plan& p = *h->p;
  if (p.device < 0) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "host-only plan");
  if (p.desc.shard_world > 64) return fail(ASTITCH_ERR_UNSUPPORTED, "fused exchange supports up to 64 ranks");
  // compile + load the fused kernel now: ranks must not JIT at different
  // times inside the first exchange (a late peer looks like a missing one)
  Plan& pm = *h->p;
  if (!pm.colreds.empty() && pm.desc.shard_world > 1 && pm.fused_kernels.empty()) {
    pm.fused_kernels.resize(1);
    astitch_status s = build_plan_kernel(pm, ROLE_FUSED, pm.fused_kernels[0]);
    std::string e2;
    if (s == ASTITCH_OK && !pm.fused_kernels[0].module && !drv_load(pm, pm.fused_kernels[0], e2))
      s = fail(ASTITCH_ERR_CUDA, e2);
    if (s != ASTITCH_OK) {
      pm.fused_kernels.clear();
      return s;
    }
    Kernel& k = pm.fused_kernels[0];
    k.grid = resident_grid(pm, k);
    if (k.grid < 1) return fail(ASTITCH_ERR_RESOURCE, "kernel cannot be resident");
  }
  auto* x = new astitch_peer_s();
  x->world = p.desc.shard_world;
  x->rank = p.desc.shard_rank;
  x->device = p.device;
  x->bytes = xbuf_bytes(x->world, std::max<size_t>(p.colreds.size(), 1), p.desc.cols);
  std::string err;
  if (!drv_alloc_zero(x->device, x->bytes, &x->local, err)) {
    delete x;
    return fail(ASTITCH_ERR_CUDA, err);
  }
  x->ptrs.assign(x->world, nullptr);
  x->opened.assign(x->world, false);
  x->ptrs[x->rank] = x->local;
  if (ipc_handle) {
    memset(ipc_handle, 0, 64);
    if (!drv_ipc_get(x->local, ipc_handle, err)) {
      drv_free(x->local);
      delete x;
      return fail(ASTITCH_ERR_CUDA, err);
    }
  }
  *out = x;
  return ASTITCH_OK;
}

astitch_status astitch_peer_open(astitch_peer_t x, int32_t rank, const uint8_t ipc_handle[64]) {
  if (!x || !ipc_handle) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL peer or handle");
  if (rank < 0 || rank >= x->world) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "rank out of range");
  if (rank == x->rank) return ASTITCH_OK;
  std::string err;
  void* ptr = nullptr;
  if (!drv_ipc_open(x->device, ipc_handle, &ptr, err)) return fail(ASTITCH_ERR_CUDA, err);
  if (x->opened[rank]) drv_ipc_close(x->ptrs[rank]);
  x->ptrs[rank] = ptr;
  x->opened[rank] = true;
  x->table_dirty = true;
  return ASTITCH_OK;
}

astitch_status astitch_peer_link(astitch_peer_t x, int32_t rank, astitch_peer_t other) {
  if (!x || !other) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL peer");
  if (rank < 0 || rank >= x->world || other->rank != rank || other->world != x->world || other->bytes != x->bytes)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "peer does not match (rank / world / plan)");
  x->ptrs[rank] = other->local;
  x->table_dirty = true;
  return ASTITCH_OK;
}

astitch_status astitch_peer_status(astitch_peer_t x, int32_t* timed_out) {
  if (!x || !timed_out) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL argument");
  uint32_t e = 0;
  std::string err;
  if (!drv_dtoh(&e, static_cast<char*>(x->local) + kXErr, 4, err)) return fail(ASTITCH_ERR_CUDA, err);
  *timed_out = e ? 1 : 0;
  return ASTITCH_OK;
}

astitch_status astitch_peer_destroy(astitch_peer_t x) {
  if (!x) return ASTITCH_OK;
  for (int q = 0; q < x->world; ++q)
    if (x->opened[q]) drv_ipc_close(x->ptrs[q]);
  drv_free(x->local);
  delete x;
  return ASTITCH_OK;
}

astitch_status astitch_run_fused(astitch_plan_t h, astitch_peer_t x, const void* const* inputs,
                                 void* const* outputs, void* ws, void* stream) {
  if (!h) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL plan");
  Plan& p = *h->p;
  if (p.colreds.empty() || p.desc.shard_world <= 1) return astitch_run(h, inputs, outputs, ws, stream);
  if (!x) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "column reduction over shards needs a peer exchange");
  if (x->world != p.desc.shard_world || x->rank != p.desc.shard_rank ||
      x->bytes != xbuf_bytes(x->world, std::max<size_t>(p.colreds.size(), 1), p.desc.cols))
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "peer exchange does not match the plan's shard");
  for (int q = 0; q < x->world; ++q)
    if (!x->ptrs[q]) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "peer " + std::to_string(q) + " not opened / linked");
  astitch_status s = check_io(p, inputs, outputs, ws);
  if (s != ASTITCH_OK) return s;
  std::string err;
  if (p.fused_kernels.empty()) {
    p.fused_kernels.resize(1);
    if ((s = build_plan_kernel(p, ROLE_FUSED, p.fused_kernels[0])) != ASTITCH_OK) {
      p.fused_kernels.clear();
      return s;
    }
    Kernel& k = p.fused_kernels[0];
    if (!k.module && !drv_load(p, k, err)) return fail(ASTITCH_ERR_CUDA, err);
    k.grid = resident_grid(p, k);
    if (k.grid < 1) return fail(ASTITCH_ERR_RESOURCE, "kernel cannot be resident");
  }
  if (x->table_dirty) {  // device addresses of every rank's buffer, read by the kernel
    std::vector<uint64_t> t(x->world);
    for (int q = 0; q < x->world; ++q) t[q] = reinterpret_cast<uint64_t>(x->ptrs[q]);
    if (!drv_htod(x->local, t.data(), 8 * t.size(), err)) return fail(ASTITCH_ERR_CUDA, err);
    x->table_dirty = false;
  }
  KernelParams kp = make_params(p, inputs, outputs, ws);
  kp.xbuf = x->local;
  return launch(p, p.fused_kernels[0], kp, stream);
}

astitch_status astitch_plan_colpart(astitch_plan_t h, size_t* byte_offset, size_t* count) {
  if (!h || !byte_offset || !count) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL argument");
  const Plan& p = *h->p;
  const size_t C = static_cast<size_t>(p.desc.cols);
  *byte_offset = p.ws.colvals + p.post_colvecs.size() * C * 4;
  *count = p.colreds.size() * C;
  return ASTITCH_OK;
}

astitch_status astitch_plan_colpart_ops(astitch_plan_t h, int32_t* ops, size_t cap, size_t* n) {
  if (!h || !n) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL argument");
  const Plan& p = *h->p;
  *n = p.colreds.size();
  if (cap < p.colreds.size() || (!ops && !p.colreds.empty()))
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "ops buffer smaller than the number of column reductions");
  for (size_t q = 0; q < p.colreds.size(); ++q) ops[q] = p.g.nodes[p.colreds[q]].sub == ASTITCH_RMAX ? ASTITCH_RMAX : ASTITCH_SUM;
  return ASTITCH_OK;
}

astitch_status astitch_run_shard_stage(astitch_plan_t h, int32_t stage, const void* const* inputs,
                                       void* const* outputs, void* ws, void* stream) {
  if (!h) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "NULL plan");
  if (stage != 0 && stage != 1) return fail(ASTITCH_ERR_INVALID_ARGUMENT, "stage must be 0 or 1");
  const Plan& p = *h->p;
  if (p.colreds.empty() || p.desc.shard_world <= 1)
    return stage == 0 ? astitch_run(h, inputs, outputs, ws, stream) : ASTITCH_OK;
  if (p.shard_kernels.empty() || !p.shard_kernels[0].function)
    return fail(ASTITCH_ERR_INVALID_ARGUMENT, "plan has no loaded sharded kernels");
  astitch_status s = check_io(p, inputs, outputs, ws);
  if (s != ASTITCH_OK) return s;
  KernelParams kp = make_params(p, inputs, outputs, ws);
  if (stage == 0) return launch(p, p.shard_kernels[0], kp, stream);
  for (size_t i = 1; i < p.shard_kernels.size(); ++i)
    if ((s = launch(p, p.shard_kernels[i], kp, stream)) != ASTITCH_OK) return s;
  return ASTITCH_OK;
}

}  // extern "C"
