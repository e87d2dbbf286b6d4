// CUDA driver API access through dlopen("libcuda.so.1"): module loading,
// occupancy queries and kernel launches (cooperative / cluster attributes) on
// the caller's stream.  Linking no CUDA library keeps libastitch loadable on
// hosts without a GPU (the host-side tests).
#include <cuda.h>
#include <dlfcn.h>

#include <cstring>
#include <mutex>
#include <string>

#include "internal.h"

namespace astitch {

struct Driver {
  void* h = nullptr;
  CUresult (*Init)(unsigned int);
  CUresult (*DeviceGet)(CUdevice*, int);
  CUresult (*DeviceGetAttribute)(int*, CUdevice_attribute, CUdevice);
  CUresult (*PrimaryCtxRetain)(CUcontext*, CUdevice);
  CUresult (*CtxGetCurrent)(CUcontext*);
  CUresult (*CtxSetCurrent)(CUcontext);
  CUresult (*CtxGetDevice)(CUdevice*);
  CUresult (*ModuleLoadData)(CUmodule*, const void*);
  CUresult (*ModuleUnload)(CUmodule);
  CUresult (*ModuleGetFunction)(CUfunction*, CUmodule, const char*);
  CUresult (*FuncSetAttribute)(CUfunction, CUfunction_attribute, int);
  CUresult (*FuncGetAttribute)(int*, CUfunction_attribute, CUfunction);
  CUresult (*Occupancy)(int*, CUfunction, int, size_t);
  CUresult (*OccupancyClusters)(int*, CUfunction, const CUlaunchConfig*);
  CUresult (*LaunchKernelEx)(const CUlaunchConfig*, CUfunction, void**, void**);
  CUresult (*MemsetD8Async)(CUdeviceptr, unsigned char, size_t, CUstream);
  CUresult (*MemcpyAsync)(CUdeviceptr, CUdeviceptr, size_t, CUstream);
  CUresult (*StreamSynchronize)(CUstream);
  CUresult (*GetErrorString)(CUresult, const char**);
  CUresult (*StreamCreate)(CUstream*, unsigned int);
  CUresult (*StreamDestroy)(CUstream);
  CUresult (*EventCreate)(CUevent*, unsigned int);
  CUresult (*EventDestroy)(CUevent);
  CUresult (*EventRecord)(CUevent, CUstream);
  CUresult (*StreamWaitEvent)(CUstream, CUevent, unsigned int);
  CUresult (*MemAlloc)(CUdeviceptr*, size_t);
  CUresult (*MemFree)(CUdeviceptr);
  CUresult (*MemsetD8)(CUdeviceptr, unsigned char, size_t);
  CUresult (*MemcpyHtoD)(CUdeviceptr, const void*, size_t);
  CUresult (*MemcpyDtoH)(void*, CUdeviceptr, size_t);
  CUresult (*IpcGetMemHandle)(CUipcMemHandle*, CUdeviceptr);
  CUresult (*IpcOpenMemHandle)(CUdeviceptr*, CUipcMemHandle, unsigned int);
  CUresult (*IpcCloseMemHandle)(CUdeviceptr);
};

namespace {

std::string cu_err(Driver* d, CUresult r, const char* what) {
  const char* s = nullptr;
  if (d && d->GetErrorString) d->GetErrorString(r, &s);
  return std::string(what) + " failed: " + (s ? s : "unknown CUDA error") + " (" + std::to_string(r) + ")";
}

}  // namespace

Driver* driver(std::string& err) {
  static Driver d;
  static bool tried = false;
  static std::string load_err;
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  if (tried) {
    if (!d.h) err = load_err;
    return d.h ? &d : nullptr;
  }
  tried = true;
  d.h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_LOCAL);
  if (!d.h) {
    load_err = "cannot dlopen libcuda.so.1 (no NVIDIA driver on this host)";
    err = load_err;
    return nullptr;
  }
#define SYM(field, name)                                          \
  *reinterpret_cast<void**>(&d.field) = dlsym(d.h, name);         \
  if (!d.field) {                                                 \
    load_err = std::string("libcuda lacks ") + name;              \
    err = load_err;                                               \
    d.h = nullptr;                                                \
    return nullptr;                                               \
  }
  SYM(Init, "cuInit");
  SYM(DeviceGet, "cuDeviceGet");
  SYM(DeviceGetAttribute, "cuDeviceGetAttribute");
  SYM(PrimaryCtxRetain, "cuDevicePrimaryCtxRetain");
  SYM(CtxGetCurrent, "cuCtxGetCurrent");
  SYM(CtxSetCurrent, "cuCtxSetCurrent");
  SYM(CtxGetDevice, "cuCtxGetDevice");
  SYM(ModuleLoadData, "cuModuleLoadData");
  SYM(ModuleUnload, "cuModuleUnload");
  SYM(ModuleGetFunction, "cuModuleGetFunction");
  SYM(FuncSetAttribute, "cuFuncSetAttribute");
  SYM(FuncGetAttribute, "cuFuncGetAttribute");
  SYM(Occupancy, "cuOccupancyMaxActiveBlocksPerMultiprocessor");
  SYM(OccupancyClusters, "cuOccupancyMaxActiveClusters");
  SYM(LaunchKernelEx, "cuLaunchKernelEx");
  SYM(MemsetD8Async, "cuMemsetD8Async");
  SYM(MemcpyAsync, "cuMemcpyAsync");
  SYM(StreamSynchronize, "cuStreamSynchronize");
  SYM(GetErrorString, "cuGetErrorString");
  SYM(StreamCreate, "cuStreamCreate");
  SYM(StreamDestroy, "cuStreamDestroy_v2");
  SYM(EventCreate, "cuEventCreate");
  SYM(EventDestroy, "cuEventDestroy_v2");
  SYM(EventRecord, "cuEventRecord");
  SYM(StreamWaitEvent, "cuStreamWaitEvent");
  SYM(MemAlloc, "cuMemAlloc_v2");
  SYM(MemFree, "cuMemFree_v2");
  SYM(MemsetD8, "cuMemsetD8_v2");
  SYM(MemcpyHtoD, "cuMemcpyHtoD_v2");
  SYM(MemcpyDtoH, "cuMemcpyDtoH_v2");
  SYM(IpcGetMemHandle, "cuIpcGetMemHandle");
  SYM(IpcOpenMemHandle, "cuIpcOpenMemHandle_v2");
  SYM(IpcCloseMemHandle, "cuIpcCloseMemHandle");
#undef SYM
  CUresult r = d.Init(0);
  if (r != CUDA_SUCCESS) {
    load_err = cu_err(&d, r, "cuInit");
    err = load_err;
    d.h = nullptr;
    return nullptr;
  }
  return &d;
}

namespace {

// Make the device's primary context current on this thread (the one PyTorch
// uses), unless a context is already current.
bool ensure_ctx(Driver* d, int device, std::string& err) {
  CUcontext cur = nullptr;
  d->CtxGetCurrent(&cur);
  if (cur) {
    CUdevice dev;
    if (d->CtxGetDevice(&dev) == CUDA_SUCCESS && static_cast<int>(dev) == device) return true;
  }
  CUdevice dev;
  CUresult r = d->DeviceGet(&dev, device);
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuDeviceGet"); return false; }
  CUcontext ctx;
  r = d->PrimaryCtxRetain(&ctx, dev);
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuDevicePrimaryCtxRetain"); return false; }
  r = d->CtxSetCurrent(ctx);
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuCtxSetCurrent"); return false; }
  return true;
}

}  // namespace

bool drv_device_info(int device, int& sm_count, int& max_smem_optin, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  if (!ensure_ctx(d, device, err)) return false;
  CUdevice dev;
  d->DeviceGet(&dev, device);
  d->DeviceGetAttribute(&sm_count, CU_DEVICE_ATTRIBUTE_MULTIPROCESSOR_COUNT, dev);
  d->DeviceGetAttribute(&max_smem_optin, CU_DEVICE_ATTRIBUTE_MAX_SHARED_MEMORY_PER_BLOCK_OPTIN, dev);
  return true;
}

bool drv_load(Plan& p, Kernel& k, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  if (!ensure_ctx(d, p.device, err)) return false;
  CUmodule mod;
  CUresult r = d->ModuleLoadData(&mod, k.cubin.data());
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuModuleLoadData"); return false; }
  CUfunction fn;
  r = d->ModuleGetFunction(&fn, mod, k.name.c_str());
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuModuleGetFunction"); d->ModuleUnload(mod); return false; }
  if (k.smem > 0) {  // dynamic + static may exceed the 48 KB default even when dynamic alone does not
    r = d->FuncSetAttribute(fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, k.smem);
    if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuFuncSetAttribute(smem)"); d->ModuleUnload(mod); return false; }
  }
  if (k.cluster > 8) {
    // clusters of 9-16 CTAs are non-portable: opt in per function
    r = d->FuncSetAttribute(fn, CU_FUNC_ATTRIBUTE_NON_PORTABLE_CLUSTER_SIZE_ALLOWED, 1);
    if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuFuncSetAttribute(non-portable cluster)"); d->ModuleUnload(mod); return false; }
  }
  k.max_clusters = -1;
  if (k.cluster > 1) {
    CUlaunchConfig cfg{};
    cfg.gridDimX = static_cast<unsigned>(k.grid);
    cfg.gridDimY = cfg.gridDimZ = 1;
    cfg.blockDimX = static_cast<unsigned>(k.threads);
    cfg.blockDimY = cfg.blockDimZ = 1;
    cfg.sharedMemBytes = static_cast<unsigned>(k.smem);
    int nc = 0;
    if (d->OccupancyClusters(&nc, fn, &cfg) == CUDA_SUCCESS) k.max_clusters = nc;
  }
  int regs = -1, local = -1;
  d->FuncGetAttribute(&regs, CU_FUNC_ATTRIBUTE_NUM_REGS, fn);
  d->FuncGetAttribute(&local, CU_FUNC_ATTRIBUTE_LOCAL_SIZE_BYTES, fn);
  k.regs = regs;
  if (k.spill_bytes < 0) k.spill_bytes = local;
  int occ = 0;
  r = d->Occupancy(&occ, fn, k.threads, static_cast<size_t>(k.smem));
  if (r != CUDA_SUCCESS) {
    // cluster kernels may reject the per-block query; only the cooperative
    // (grid-barrier) kernels depend on it for co-residency
    if (k.cooperative) { err = cu_err(d, r, "cuOccupancyMaxActiveBlocksPerMultiprocessor"); d->ModuleUnload(mod); return false; }
    occ = -1;
  }
  k.occupancy = occ;
  k.module = mod;
  k.function = fn;
  return true;
}

bool drv_unload(Kernel& k) {
  std::string err;
  Driver* d = driver(err);
  if (d && k.module) d->ModuleUnload(static_cast<CUmodule>(k.module));
  k.module = nullptr;
  k.function = nullptr;
  return true;
}

bool drv_launch(const Kernel& k, void* params, size_t params_size, void* stream, std::string& err) {
  (void)params_size;
  void* args[] = {params};
  return drv_launch_args(k, args, stream, err);
}

bool drv_launch_args(const Kernel& k, void** args, void* stream, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  CUlaunchConfig cfg{};
  cfg.gridDimX = static_cast<unsigned>(k.grid);
  cfg.gridDimY = 1;
  cfg.gridDimZ = 1;
  cfg.blockDimX = static_cast<unsigned>(k.threads);
  cfg.blockDimY = 1;
  cfg.blockDimZ = 1;
  cfg.sharedMemBytes = static_cast<unsigned>(k.smem);
  cfg.hStream = static_cast<CUstream>(stream);
  CUlaunchAttribute attr[1];
  if (k.cooperative) {
    attr[0].id = CU_LAUNCH_ATTRIBUTE_COOPERATIVE;
    attr[0].value.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
  } else if (k.pdl) {
    // the kernel starts with griddepcontrol.wait, so it may be scheduled
    // before its predecessor in the stream completes (hides launch latency)
    attr[0].id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
    attr[0].value.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
  }
  CUresult r = d->LaunchKernelEx(&cfg, static_cast<CUfunction>(k.function), args, nullptr);
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, ("cuLaunchKernelEx(" + k.name + ")").c_str()); return false; }
  return true;
}

bool drv_memset_async(void* ptr, size_t bytes, void* stream, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  CUresult r = d->MemsetD8Async(reinterpret_cast<CUdeviceptr>(ptr), 0, bytes, static_cast<CUstream>(stream));
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuMemsetD8Async"); return false; }
  return true;
}

bool drv_memcpy_async(void* dst, const void* src, size_t bytes, int kind, void* stream, std::string& err) {
  (void)kind;
  Driver* d = driver(err);
  if (!d) return false;
  CUresult r = d->MemcpyAsync(reinterpret_cast<CUdeviceptr>(dst), reinterpret_cast<CUdeviceptr>(src), bytes,
                              static_cast<CUstream>(stream));
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuMemcpyAsync"); return false; }
  return true;
}

bool drv_stream_create(void** s, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  CUstream st;
  CUresult r = d->StreamCreate(&st, CU_STREAM_NON_BLOCKING);
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuStreamCreate"); return false; }
  *s = st;
  return true;
}

bool drv_event_create(void** e, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  CUevent ev;
  CUresult r = d->EventCreate(&ev, CU_EVENT_DISABLE_TIMING);
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuEventCreate"); return false; }
  *e = ev;
  return true;
}

bool drv_event_record(void* e, void* s, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  CUresult r = d->EventRecord(static_cast<CUevent>(e), static_cast<CUstream>(s));
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuEventRecord"); return false; }
  return true;
}

bool drv_stream_wait(void* s, void* e, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  CUresult r = d->StreamWaitEvent(static_cast<CUstream>(s), static_cast<CUevent>(e), 0);
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuStreamWaitEvent"); return false; }
  return true;
}

void drv_stream_destroy(void* s) {
  std::string err;
  Driver* d = driver(err);
  if (d && s) d->StreamDestroy(static_cast<CUstream>(s));
}

void drv_event_destroy(void* e) {
  std::string err;
  Driver* d = driver(err);
  if (d && e) d->EventDestroy(static_cast<CUevent>(e));
}

// ---- peer exchange buffers of the fused sharded run (comm.cpp)
bool drv_alloc_zero(int device, size_t bytes, void** ptr, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  if (!ensure_ctx(d, device, err)) return false;
  CUdeviceptr p = 0;
  CUresult r = d->MemAlloc(&p, bytes);
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuMemAlloc"); return false; }
  r = d->MemsetD8(p, 0, bytes);
  if (r != CUDA_SUCCESS) { d->MemFree(p); err = cu_err(d, r, "cuMemsetD8"); return false; }
  *ptr = reinterpret_cast<void*>(p);
  return true;
}
void drv_free(void* ptr) {
  std::string err;
  Driver* d = driver(err);
  if (d && ptr) d->MemFree(reinterpret_cast<CUdeviceptr>(ptr));
}
bool drv_htod(void* dst, const void* src, size_t bytes, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  CUresult r = d->MemcpyHtoD(reinterpret_cast<CUdeviceptr>(dst), src, bytes);
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuMemcpyHtoD"); return false; }
  return true;
}
bool drv_dtoh(void* dst, const void* src, size_t bytes, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  CUresult r = d->MemcpyDtoH(dst, reinterpret_cast<CUdeviceptr>(src), bytes);
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuMemcpyDtoH"); return false; }
  return true;
}
bool drv_ipc_get(void* ptr, unsigned char handle[64], std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  CUipcMemHandle h;
  CUresult r = d->IpcGetMemHandle(&h, reinterpret_cast<CUdeviceptr>(ptr));
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuIpcGetMemHandle"); return false; }
  memcpy(handle, h.reserved, 64);
  return true;
}
bool drv_ipc_open(int device, const unsigned char handle[64], void** ptr, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  if (!ensure_ctx(d, device, err)) return false;
  CUipcMemHandle h;
  memcpy(h.reserved, handle, 64);
  CUdeviceptr p = 0;
  CUresult r = d->IpcOpenMemHandle(&p, h, CU_IPC_MEM_LAZY_ENABLE_PEER_ACCESS);
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuIpcOpenMemHandle"); return false; }
  *ptr = reinterpret_cast<void*>(p);
  return true;
}
void drv_ipc_close(void* ptr) {
  std::string err;
  Driver* d = driver(err);
  if (d && ptr) d->IpcCloseMemHandle(reinterpret_cast<CUdeviceptr>(ptr));
}

bool drv_sync(void* stream, std::string& err) {
  Driver* d = driver(err);
  if (!d) return false;
  CUresult r = d->StreamSynchronize(static_cast<CUstream>(stream));
  if (r != CUDA_SUCCESS) { err = cu_err(d, r, "cuStreamSynchronize"); return false; }
  return true;
}

}  // namespace astitch
