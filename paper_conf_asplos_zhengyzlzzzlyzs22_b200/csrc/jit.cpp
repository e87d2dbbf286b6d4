// NVRTC just-in-time compilation of generated stitched kernels for sm_100a
// (the paper compiles each stitch op just in time, P:L127 / P:L232; here the
// LLVM backend is replaced by NVRTC + ptxas).  libnvrtc is dlopen'ed so the
// library loads on machines without CUDA libraries on the default path.
#include <dlfcn.h>
#include <sys/stat.h>
#include <unistd.h>

#include <cerrno>
#include <cstdio>
#include <cstdlib>
#include <fstream>
#include <sstream>
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

// ---- on-disk cubin cache (astitch_set_cache_dir): one file per generated
// source, keyed by a 64-bit FNV-1a of (source, device header, NVRTC options);
// the file repeats the source length and hash and is written atomically
// (temp + rename), so concurrent processes and stale files are harmless.
std::mutex g_dir_mu;
bool g_dir_set = false;
std::string g_dir;

uint64_t fnv(const std::string& s, uint64_t h = 1469598103934665603ULL) {
  for (unsigned char c : s) {
    h ^= c;
    h *= 1099511628211ULL;
  }
  return h;
}

std::string cache_dir() {
  std::lock_guard<std::mutex> lk(g_dir_mu);
  if (g_dir_set) return g_dir;
  const char* x = getenv("XDG_CACHE_HOME");
  const char* h = getenv("HOME");
  if (x && *x) return std::string(x) + "/astitch";
  if (h && *h) return std::string(h) + "/.cache/astitch";
  return "";
}

bool mkdirs(const std::string& d) {
  if (d.empty()) return false;
  std::string cur;
  std::stringstream ss(d);
  std::string part;
  if (d[0] == '/') cur = "/";
  while (std::getline(ss, part, '/')) {
    if (part.empty()) continue;
    cur += part + "/";
    if (mkdir(cur.c_str(), 0755) != 0 && errno != EEXIST) return false;
  }
  return true;
}

const char* kMagic = "ASTITCH-CUBIN-3";

bool disk_load(const std::string& path, uint64_t key, const std::string& src, std::vector<char>& cubin,
               std::string& log) {
  const size_t src_len = src.size();
  std::ifstream f(path, std::ios::binary);
  if (!f) return false;
  std::string magic;
  uint64_t k = 0;
  size_t sl = 0, ls = 0, cs = 0;
  if (!std::getline(f, magic) || magic != kMagic) return false;
  if (!(f >> k >> sl >> ls >> cs) || k != key || sl != src_len || cs == 0 || cs > (1u << 30)) return false;
  f.get();  // newline
  std::string stored(sl, '\0');  // the full source: a hash collision can never return a wrong cubin
  if (sl && !f.read(&stored[0], static_cast<std::streamsize>(sl))) return false;
  if (stored != src) return false;
  log.assign(ls, '\0');
  cubin.resize(cs);
  if (ls && !f.read(&log[0], static_cast<std::streamsize>(ls))) return false;
  if (!f.read(cubin.data(), static_cast<std::streamsize>(cs))) return false;
  return true;
}

void disk_store(const std::string& dir, const std::string& path, uint64_t key, const std::string& src,
                const std::vector<char>& cubin, const std::string& log) {
  const size_t src_len = src.size();
  if (!mkdirs(dir)) return;
  const std::string tmp = path + ".tmp" + std::to_string(getpid());
  {
    std::ofstream f(tmp, std::ios::binary);
    if (!f) return;
    f << kMagic << "\n" << key << " " << src_len << " " << log.size() << " " << cubin.size() << "\n";
    f.write(src.data(), static_cast<std::streamsize>(src.size()));
    f.write(log.data(), static_cast<std::streamsize>(log.size()));
    f.write(cubin.data(), static_cast<std::streamsize>(cubin.size()));
    if (!f) { std::remove(tmp.c_str()); return; }
  }
  if (std::rename(tmp.c_str(), path.c_str()) != 0) std::remove(tmp.c_str());
}

}  // namespace

// ASTITCH_LOG=1: one line per plan on stderr (template, grid, registers,
// demotions, plan time).  Diagnostics only: it never changes a plan.
bool log_enabled() {
  static const bool on = [] {
    const char* e = getenv("ASTITCH_LOG");
    return e && *e && *e != '0';
  }();
  return on;
}

void set_cache_dir(const char* dir) {
  std::lock_guard<std::mutex> lk(g_dir_mu);
  g_dir_set = true;
  g_dir = dir ? dir : "";
}

bool nvrtc_compile(const std::string& src, const std::string& name, std::vector<char>& cubin,
                   std::string& log, std::string& err, int* cache_state) {
  if (cache_state) *cache_state = 0;
  {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    auto it = g_cache.find(src);
    if (it != g_cache.end()) {
      cubin = it->second.first;
      log = it->second.second;
      if (cache_state) *cache_state = 1;
      return true;
    }
  }
  static const char* kOpts = "--gpu-architecture=sm_100a --std=c++17 -default-device --generate-line-info "
                             "--ptxas-options=-v -DASTITCH_JIT=1 -diag-suppress=177,550";
  const uint64_t key = fnv(src, fnv(kOpts, fnv(kAstitchDeviceCuh)));
  const std::string dir = cache_dir();
  char hex[32];
  snprintf(hex, sizeof(hex), "%016llx", static_cast<unsigned long long>(key));
  const std::string path = dir.empty() ? "" : dir + "/" + hex + ".cubin";
  if (!path.empty() && disk_load(path, key, src, cubin, log)) {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    g_cache[src] = {cubin, log};
    if (cache_state) *cache_state = 2;
    return true;
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
  if (!path.empty()) disk_store(dir, path, key, src, cubin, log);
  std::lock_guard<std::mutex> lk(g_cache_mu);
  g_cache[src] = {cubin, log};
  return true;
}

}  // namespace astitch
