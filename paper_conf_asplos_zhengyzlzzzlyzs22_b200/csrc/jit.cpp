// NVRTC just-in-time compilation of generated stitched kernels for sm_100a
// (the paper compiles each stitch op just in time, P:L127 / P:L232; here the
// LLVM backend is replaced by NVRTC + ptxas).  libnvrtc is dlopen'ed so the
// library loads on machines without CUDA libraries on the default path.
#include <dlfcn.h>

#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <unordered_map>
#include <vector>

#include "internal.h"

#include "embedded_device_cuh.h"  // kAstitchDeviceCuh (generated at build time)

namespace astitch {

const char* device_header_source() { return kAstitchDeviceCuh; }

namespace {

typedef int nvrtcResult;
typedef struct _nvrtcProgram* nvrtcProgram;

struct Nvrtc {
  void* h = nullptr;
  nvrtcResult (*create)(nvrtcProgram*, const char*, const char*, int, const char* const*, const char* const*);
  nvrtcResult (*compile)(nvrtcProgram, int, const char* const*);
  nvrtcResult (*cubin_size)(nvrtcProgram, size_t*);
  nvrtcResult (*cubin)(nvrtcProgram, char*);
  nvrtcResult (*log_size)(nvrtcProgram, size_t*);
  nvrtcResult (*log)(nvrtcProgram, char*);
  nvrtcResult (*destroy)(nvrtcProgram*);
  const char* (*errstr)(nvrtcResult);
};

Nvrtc* load_nvrtc(std::string& err) {
  static Nvrtc n;
  static bool tried = false;
  static std::string load_err;
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  if (tried) {
    if (!n.h) err = load_err;
    return n.h ? &n : nullptr;
  }
  tried = true;
  std::vector<std::string> cands;
  if (const char* e = getenv("ASTITCH_NVRTC")) cands.push_back(e);
  cands.push_back("/usr/local/cuda/lib64/libnvrtc.so.12");
  cands.push_back("libnvrtc.so.12");
  cands.push_back("libnvrtc.so");
  for (auto& c : cands) {
    n.h = dlopen(c.c_str(), RTLD_NOW | RTLD_LOCAL);
    if (n.h) break;
  }
  if (!n.h) {
    load_err = "cannot dlopen libnvrtc (set ASTITCH_NVRTC)";
    err = load_err;
    return nullptr;
  }
#define SYM(field, name)                                               \
  *reinterpret_cast<void**>(&n.field) = dlsym(n.h, name);              \
  if (!n.field) {                                                      \
    load_err = std::string("libnvrtc lacks ") + name;                  \
    err = load_err;                                                    \
    n.h = nullptr;                                                     \
    return nullptr;                                                    \
  }
  SYM(create, "nvrtcCreateProgram");
  SYM(compile, "nvrtcCompileProgram");
  SYM(cubin_size, "nvrtcGetCUBINSize");
  SYM(cubin, "nvrtcGetCUBIN");
  SYM(log_size, "nvrtcGetProgramLogSize");
  SYM(log, "nvrtcGetProgramLog");
  SYM(destroy, "nvrtcDestroyProgram");
  SYM(errstr, "nvrtcGetErrorString");
#undef SYM
  return &n;
}

std::mutex g_cache_mu;
std::unordered_map<std::string, std::pair<std::vector<char>, std::string>> g_cache;

}  // namespace

bool nvrtc_compile(const std::string& src, const std::string& name, std::vector<char>& cubin,
                   std::string& log, std::string& err) {
  {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    auto it = g_cache.find(src);
    if (it != g_cache.end()) {
      cubin = it->second.first;
      log = it->second.second;
      return true;
    }
  }
  Nvrtc* n = load_nvrtc(err);
  if (!n) return false;
  nvrtcProgram prog = nullptr;
  const char* hdrs[] = {kAstitchDeviceCuh};
  const char* hdr_names[] = {"astitch_device.cuh"};
  nvrtcResult r = n->create(&prog, src.c_str(), (name + ".cu").c_str(), 1, hdrs, hdr_names);
  if (r != 0) {
    err = std::string("nvrtcCreateProgram: ") + n->errstr(r);
    return false;
  }
  std::vector<const char*> opts = {"--gpu-architecture=sm_100a", "--std=c++17", "-default-device",
                                   "--generate-line-info", "--ptxas-options=-v", "-DASTITCH_JIT=1",
                                   "-diag-suppress=177,550"};
  r = n->compile(prog, static_cast<int>(opts.size()), opts.data());
  size_t ls = 0;
  n->log_size(prog, &ls);
  log.assign(ls, '\0');
  if (ls) n->log(prog, &log[0]);
  if (!log.empty() && log.back() == '\0') log.pop_back();
  if (r != 0) {
    err = std::string("NVRTC compile failed: ") + n->errstr(r) + "\n" + log;
    n->destroy(&prog);
    return false;
  }
  size_t cs = 0;
  n->cubin_size(prog, &cs);
  cubin.resize(cs);
  n->cubin(prog, cubin.data());
  n->destroy(&prog);
  std::lock_guard<std::mutex> lk(g_cache_mu);
  g_cache[src] = {cubin, log};
  return true;
}

}  // namespace astitch
