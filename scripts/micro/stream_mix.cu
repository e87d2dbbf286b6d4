// Microbenchmark: HBM throughput of a 2-read : 1-write bf16 stream (C5's mix,
// z = x + y over 2^30 elements) under different grid structures, to find why
// a persistent row sweep reaches 6.4 TB/s where torch.add reaches 7.1 TB/s.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a stream_mix.cu -o stream_mix
#include <cuda_bf16.h>
#include <cstdio>
#include <cstdint>

struct alignas(16) V4 { uint32_t x, y, z, w; };

__device__ __forceinline__ V4 ld(const V4* p) {
  V4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint32_t add2(uint32_t a, uint32_t b) {
  __nv_bfloat162 x = *reinterpret_cast<__nv_bfloat162*>(&a), y = *reinterpret_cast<__nv_bfloat162*>(&b);
  float2 fx = __bfloat1622float2(x), fy = __bfloat1622float2(y);
  __nv_bfloat162 r = __floats2bfloat162_rn(fx.x + fy.x, fx.y + fy.y);
  return *reinterpret_cast<uint32_t*>(&r);
}
__device__ __forceinline__ V4 addv(V4 a, V4 b) { return V4{add2(a.x, b.x), add2(a.y, b.y), add2(a.z, b.z), add2(a.w, b.w)}; }

// (a) persistent grid-stride, U vectors per thread per step
template <int U>
__global__ void persistent(const V4* __restrict__ x, const V4* __restrict__ y, V4* __restrict__ z, long long n) {
  long long stride = (long long)gridDim.x * blockDim.x * U;
  for (long long base = (long long)blockIdx.x * blockDim.x * U + threadIdx.x; base < n; base += stride) {
    V4 a[U], b[U];
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) { a[u] = ld(x + i); b[u] = ld(y + i); } }
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) z[i] = addv(a[u], b[u]); }
  }
}
// (a') persistent grid-stride recording each CTA's finish time (globaltimer)
template <int U>
__global__ void persistent_t(const V4* __restrict__ x, const V4* __restrict__ y, V4* __restrict__ z, long long n,
                             unsigned long long* t_end, unsigned int* smid) {
  long long stride = (long long)gridDim.x * blockDim.x * U;
  for (long long base = (long long)blockIdx.x * blockDim.x * U + threadIdx.x; base < n; base += stride) {
    V4 a[U], b[U];
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) { a[u] = ld(x + i); b[u] = ld(y + i); } }
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) z[i] = addv(a[u], b[u]); }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    unsigned int s; asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
    t_end[blockIdx.x] = t; smid[blockIdx.x] = s;
  }
}
// (b) one tile per CTA (non-persistent), U vectors per thread
template <int U>
__global__ void tiled(const V4* __restrict__ x, const V4* __restrict__ y, V4* __restrict__ z, long long n) {
  long long base = (long long)blockIdx.x * blockDim.x * U + threadIdx.x;
  V4 a[U], b[U];
#pragma unroll
  for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) { a[u] = ld(x + i); b[u] = ld(y + i); } }
#pragma unroll
  for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) z[i] = addv(a[u], b[u]); }
}
// (c) persistent, but each CTA sweeps ONE contiguous range (blocked, not strided)
template <int U>
__global__ void blocked(const V4* __restrict__ x, const V4* __restrict__ y, V4* __restrict__ z, long long n) {
  long long per = (n + gridDim.x - 1) / gridDim.x;
  long long lo = (long long)blockIdx.x * per, hi = min(n, lo + per);
  for (long long base = lo + threadIdx.x; base < hi; base += (long long)blockDim.x * U) {
    V4 a[U], b[U];
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < hi) { a[u] = ld(x + i); b[u] = ld(y + i); } }
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < hi) z[i] = addv(a[u], b[u]); }
  }
}

// (d) persistent with dynamic tile order: each CTA grabs the next tile from a
// global counter (tiles dispatched in address order, like the hardware
// scheduler does for a non-persistent grid)
template <int U>
__global__ void dynamic_tiles(const V4* __restrict__ x, const V4* __restrict__ y, V4* __restrict__ z, long long n,
                              unsigned long long* counter) {
  __shared__ long long tile;
  const long long per = (long long)blockDim.x * U, ntiles = (n + per - 1) / per;
  for (;;) {
    if (threadIdx.x == 0) tile = (long long)atomicAdd(counter, 1ULL);
    __syncthreads();
    const long long t = tile;
    __syncthreads();
    if (t >= ntiles) break;
    long long base = t * per + threadIdx.x;
    V4 a[U], b[U];
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) { a[u] = ld(x + i); b[u] = ld(y + i); } }
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) z[i] = addv(a[u], b[u]); }
  }
}
// (e) persistent grid-stride with the next step's loads issued before this
// step's stores (software pipeline)
template <int U>
__global__ void persistent_pf(const V4* __restrict__ x, const V4* __restrict__ y, V4* __restrict__ z, long long n) {
  long long stride = (long long)gridDim.x * blockDim.x * U;
  long long base = (long long)blockIdx.x * blockDim.x * U + threadIdx.x;
  V4 a[U], b[U];
#pragma unroll
  for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) { a[u] = ld(x + i); b[u] = ld(y + i); } }
  for (; base < n; base += stride) {
    V4 c[U], d[U];
    const long long nb = base + stride;
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = nb + (long long)u * blockDim.x; if (i < n) { c[u] = ld(x + i); d[u] = ld(y + i); } }
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) z[i] = addv(a[u], b[u]); }
#pragma unroll
    for (int u = 0; u < U; ++u) { a[u] = c[u]; b[u] = d[u]; }
  }
}

// (g) dynamic COARSE tiles: S steps of blockDim x U vectors per grabbed tile,
// swept in order inside the tile (the shape a deterministic per-tile column
// partial needs: C5 rows of 2 KB, 128-row tiles = 256 KB per tensor)
template <int U>
__global__ void dynamic_coarse(const V4* __restrict__ x, const V4* __restrict__ y, V4* __restrict__ z, long long n,
                               unsigned long long* counter, int S) {
  __shared__ long long tq[2];
  const long long step = (long long)blockDim.x * U, per = step * S, ntiles = (n + per - 1) / per;
  if (threadIdx.x == 0) tq[0] = (long long)atomicAdd(counter, 1ULL);
  __syncthreads();
  long long cur = tq[0];
  int k = 1;
  while (cur < ntiles) {
    if (threadIdx.x == 0) tq[k & 1] = (long long)atomicAdd(counter, 1ULL);  // next tile, read after the sweep
    for (int s2 = 0; s2 < S; ++s2) {
      long long base = cur * per + s2 * step + threadIdx.x;
      V4 a[U], b[U];
#pragma unroll
      for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) { a[u] = ld(x + i); b[u] = ld(y + i); } }
#pragma unroll
      for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) z[i] = addv(a[u], b[u]); }
    }
    __syncthreads();
    cur = tq[k & 1];
    __syncthreads();
    ++k;
  }
}
// (f) dynamic tiles + software pipeline: tile i+1's loads are in flight while
// tile i is stored, and the index of tile i+2 is grabbed (atomic) one step
// early, so neither the loads nor the grab sit on the critical path
template <int U>
__global__ void dynamic_pf(const V4* __restrict__ x, const V4* __restrict__ y, V4* __restrict__ z, long long n,
                           unsigned long long* counter) {
  __shared__ long long tq[2];
  const long long per = (long long)blockDim.x * U, ntiles = (n + per - 1) / per;
  if (threadIdx.x == 0) { tq[0] = (long long)atomicAdd(counter, 1ULL); tq[1] = (long long)atomicAdd(counter, 1ULL); }
  __syncthreads();
  long long cur = tq[0], nxt = tq[1];
  V4 a[U], b[U];
  if (cur < ntiles) {
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = cur * per + threadIdx.x + (long long)u * blockDim.x; if (i < n) { a[u] = ld(x + i); b[u] = ld(y + i); } }
  }
  int k = 0;
  while (cur < ntiles) {
    V4 c[U], d[U];
    if (nxt < ntiles) {
#pragma unroll
      for (int u = 0; u < U; ++u) { long long i = nxt * per + threadIdx.x + (long long)u * blockDim.x; if (i < n) { c[u] = ld(x + i); d[u] = ld(y + i); } }
    }
    // grab the tile after next into the slot not read this step
    if (threadIdx.x == 0) tq[k & 1] = (long long)atomicAdd(counter, 1ULL);
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = cur * per + threadIdx.x + (long long)u * blockDim.x; if (i < n) z[i] = addv(a[u], b[u]); }
#pragma unroll
    for (int u = 0; u < U; ++u) { a[u] = c[u]; b[u] = d[u]; }
    __syncthreads();
    cur = nxt;
    nxt = tq[k & 1];
    __syncthreads();
    ++k;
  }
}


// (h) static grid-stride (deterministic ownership) with a drift throttle: a
// CTA may start step k only once every CTA has finished step k - SLACK
// (global step counter, one atomic per CTA per step), so the grid sweeps the
// address space in lock step like counter-ordered tiles do
template <int U>
__global__ void persistent_throttle(const V4* __restrict__ x, const V4* __restrict__ y, V4* __restrict__ z, long long n,
                                    unsigned int* done, int slack) {
  long long stride = (long long)gridDim.x * blockDim.x * U;
  int k = 0;
  for (long long base = (long long)blockIdx.x * blockDim.x * U + threadIdx.x; base < n; base += stride, ++k) {
    if (k >= slack) {
      if (threadIdx.x == 0) {
        const unsigned int need = (unsigned int)(k - slack + 1) * gridDim.x;
        unsigned int v;
        do { asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(done) : "memory"); } while (v < need);
      }
      __syncthreads();
    }
    V4 a[U], b[U];
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) { a[u] = ld(x + i); b[u] = ld(y + i); } }
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) z[i] = addv(a[u], b[u]); }
    __syncthreads();
    if (threadIdx.x == 0) atomicAdd(done, 1u);
  }
}

// (i) static grid-stride with a cheap drift throttle: thread 0 adds 1 to a
// global step counter after every step (fire-and-forget red), and every
// EVERY steps checks (one relaxed load; spins with nanosleep only when
// behind) that every CTA has finished step k - SLACK.  CTAs that run out of
// steps add the steps they will never do, so nobody waits forever; a 20 ms
// guard bounds any spin.  Ownership of rows stays static (deterministic).
template <int U>
__global__ void persistent_throttle2(const V4* __restrict__ x, const V4* __restrict__ y, V4* __restrict__ z, long long n,
                                     unsigned int* done, int slack, int every) {
  const long long stride = (long long)gridDim.x * blockDim.x * U;
  const long long maxsteps = (n + stride - 1) / stride;
  int k = 0;
  for (long long base = (long long)blockIdx.x * blockDim.x * U + threadIdx.x; k < maxsteps; base += stride, ++k) {
    if (k >= slack && (k % every) == 0) {
      if (threadIdx.x == 0) {
        const unsigned int need = (unsigned int)(k - slack + 1) * gridDim.x;
        unsigned int v;
        asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(done) : "memory");
        if (v < need) {
          unsigned long long t0; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
          for (;;) {
            __nanosleep(100);
            asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(done) : "memory");
            if (v >= need) break;
            unsigned long long t1; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
            if (t1 - t0 > 20000000ULL) break;
          }
        }
      }
      __syncthreads();
    }
    if (base < n) {
      V4 a[U], b[U];
#pragma unroll
      for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) { a[u] = ld(x + i); b[u] = ld(y + i); } }
#pragma unroll
      for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) z[i] = addv(a[u], b[u]); }
    }
    if (threadIdx.x == 0) asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" :: "l"(done) : "memory");
  }
}

// (j) static grid-stride with a block barrier every EVERY steps (re-aligns the
// CTA's warps; no global communication)
template <int U>
__global__ void persistent_sync(const V4* __restrict__ x, const V4* __restrict__ y, V4* __restrict__ z, long long n,
                                int every) {
  const long long stride = (long long)gridDim.x * blockDim.x * U;
  int k = 0;
  for (long long base = (long long)blockIdx.x * blockDim.x * U + threadIdx.x; base < n; base += stride, ++k) {
    if ((k % every) == 0) __syncthreads();
    V4 a[U], b[U];
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) { a[u] = ld(x + i); b[u] = ld(y + i); } }
#pragma unroll
    for (int u = 0; u < U; ++u) { long long i = base + (long long)u * blockDim.x; if (i < n) z[i] = addv(a[u], b[u]); }
  }
}

template <typename F>
float timeit(F f) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int i = 0; i < 3; ++i) f();
  cudaDeviceSynchronize();
  float best = 1e30f;
  for (int r = 0; r < 10; ++r) {
    cudaEventRecord(e0); f(); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
  }
  return best;
}

int main(int argc, char** argv) {
  const bool only_throttle = argc > 1;
  const long long elems = 1LL << 30, n = elems / 8;  // V4 = 8 bf16
  V4 *x, *y, *z;
  cudaMalloc(&x, n * 16); cudaMalloc(&y, n * 16); cudaMalloc(&z, n * 16);
  cudaMemset(x, 0, n * 16); cudaMemset(y, 0, n * 16);
  const double bytes = 3.0 * n * 16;
  auto rep = [&](const char* name, float ms) { printf("%-40s %8.1f us %8.1f GB/s\n", name, ms * 1e3, bytes / (ms * 1e-3) / 1e9); };
  int sms = 148;
  if (!only_throttle)
  for (int t : {256, 512}) for (int bps : {1, 2, 4, 8}) {
    if (t * bps > 2048) continue;
    char nm[128];
    snprintf(nm, sizeof nm, "persistent U4 t%d x %d/SM", t, bps);
    rep(nm, timeit([&] { persistent<4><<<sms * bps, t>>>(x, y, z, n); }));
    snprintf(nm, sizeof nm, "blocked U4 t%d x %d/SM", t, bps);
    rep(nm, timeit([&] { blocked<4><<<sms * bps, t>>>(x, y, z, n); }));
  }
  unsigned long long* ctr;
  cudaMalloc(&ctr, 8);
  if (!only_throttle)
  for (int t : {256, 512}) for (int bps : {1, 2, 4}) {
    if (t * bps > 2048) continue;
    char nm[128];
    snprintf(nm, sizeof nm, "dynamic tiles U4 t%d x %d/SM", t, bps);
    rep(nm, timeit([&] { cudaMemsetAsync(ctr, 0, 8); dynamic_tiles<4><<<sms * bps, t>>>(x, y, z, n, ctr); }));
    snprintf(nm, sizeof nm, "dynamic+prefetch U4 t%d x %d/SM", t, bps);
    rep(nm, timeit([&] { cudaMemsetAsync(ctr, 0, 8); dynamic_pf<4><<<sms * bps, t>>>(x, y, z, n, ctr); }));
    snprintf(nm, sizeof nm, "dynamic+prefetch U2 t%d x %d/SM", t, bps);
    rep(nm, timeit([&] { cudaMemsetAsync(ctr, 0, 8); dynamic_pf<2><<<sms * bps, t>>>(x, y, z, n, ctr); }));
    snprintf(nm, sizeof nm, "persistent+prefetch U4 t%d x %d/SM", t, bps);
    rep(nm, timeit([&] { persistent_pf<4><<<sms * bps, t>>>(x, y, z, n); }));
    snprintf(nm, sizeof nm, "persistent+prefetch U2 t%d x %d/SM", t, bps);
    rep(nm, timeit([&] { persistent_pf<2><<<sms * bps, t>>>(x, y, z, n); }));
  }
  if (!only_throttle)
  for (int t : {128, 256, 512}) for (int u : {1, 2, 4}) {
    char nm[128];
    snprintf(nm, sizeof nm, "tiled U%d t%d", u, t);
    long long g = (n + (long long)t * u - 1) / ((long long)t * u);
    if (u == 1) rep(nm, timeit([&] { tiled<1><<<g, t>>>(x, y, z, n); }));
    if (u == 2) rep(nm, timeit([&] { tiled<2><<<g, t>>>(x, y, z, n); }));
    if (u == 4) rep(nm, timeit([&] { tiled<4><<<g, t>>>(x, y, z, n); }));
  }
  if (!only_throttle)
  for (int S : {1, 2, 4, 8, 16}) for (int bps : {1, 2}) {
    char nm[128];
    snprintf(nm, sizeof nm, "dynamic coarse S%d U4 t512 x %d/SM", S, bps);
    rep(nm, timeit([&] { cudaMemsetAsync(ctr, 0, 8); dynamic_coarse<4><<<sms * bps, 512>>>(x, y, z, n, ctr, S); }));
  }
  {
    unsigned int* done;
    cudaMalloc(&done, 4);
    for (int t : {256, 512}) for (int bps : {1, 2}) {
      char nm[128];
      snprintf(nm, sizeof nm, "persistent U4 t%d x %d/SM", t, bps);
      rep(nm, timeit([&] { persistent<4><<<sms * bps, t>>>(x, y, z, n); }));
      for (int ev : {1, 2, 4, 8, 16}) {
        snprintf(nm, sizeof nm, "syncthreads every %d U4 t%d x %d/SM", ev, t, bps);
        rep(nm, timeit([&] { persistent_sync<4><<<sms * bps, t>>>(x, y, z, n, ev); }));
      }
      for (int sl : {8, 32}) for (int ev : {4, 8, 16}) {
        snprintf(nm, sizeof nm, "throttle2 U4 t%d x %d/SM slack %d every %d", t, bps, sl, ev);
        rep(nm, timeit([&] { cudaMemsetAsync(done, 0, 4); persistent_throttle2<4><<<sms * bps, t>>>(x, y, z, n, done, sl, ev); }));
      }
      snprintf(nm, sizeof nm, "dynamic tiles U4 t%d x %d/SM", t, bps);
      rep(nm, timeit([&] { cudaMemsetAsync(ctr, 0, 8); dynamic_tiles<4><<<sms * bps, t>>>(x, y, z, n, ctr); }));
    }
  }
  if (!only_throttle) {  // finish-time spread of the static persistent sweep (tail effect?)
    const int G = sms;
    unsigned long long* t_end; unsigned int* smid;
    cudaMalloc(&t_end, G * 8); cudaMalloc(&smid, G * 4);
    unsigned long long t0h = 0;
    for (int r = 0; r < 3; ++r) persistent_t<4><<<G, 512>>>(x, y, z, n, t_end, smid);
    cudaDeviceSynchronize();
    unsigned long long h[1024]; unsigned int sid[1024];
    cudaMemcpy(h, t_end, G * 8, cudaMemcpyDeviceToHost); cudaMemcpy(sid, smid, G * 4, cudaMemcpyDeviceToHost);
    unsigned long long mn = ~0ULL, mx = 0; double sum = 0;
    for (int i = 0; i < G; ++i) { mn = h[i] < mn ? h[i] : mn; mx = h[i] > mx ? h[i] : mx; }
    for (int i = 0; i < G; ++i) sum += (double)(h[i] - mn);
    printf("static persistent t512 x 1/SM: CTA finish spread %.1f us (mean lag %.1f us)\n", (mx - mn) / 1e3, sum / G / 1e3);
    // finish lag by SM id range (die halves)
    double lo = 0, hi = 0; int nlo = 0, nhi = 0;
    for (int i = 0; i < G; ++i) { if (sid[i] < 74) { lo += (double)(h[i] - mn); ++nlo; } else { hi += (double)(h[i] - mn); ++nhi; } }
    printf("  mean lag SM 0-73: %.1f us, SM 74-147: %.1f us\n", lo / nlo / 1e3, hi / nhi / 1e3);
    (void)t0h;
  }
  cudaError_t e = cudaGetLastError();
  printf("status %s\n", cudaGetErrorString(e));
  return 0;
}
