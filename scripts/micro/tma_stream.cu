// Microbenchmark: the 2-read : 1-write bf16 stream (C5's mix, z = x + y over
// 2^30 elements) with the reads staged by 1D bulk copies (cp.async.bulk,
// UBLKCP) into a ring of shared-memory stages, one persistent CTA per SM and
// STATIC tile ownership (tile t = blockIdx + k * grid: deterministic, as the
// global sweep's column partials need).  Question: does per-CTA bulk staging
// reach the address-ordered 7.0 TB/s of stream_mix.cu's dynamic tiles without
// giving up static ownership?
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a tma_stream.cu -o tma_stream
#include <cuda_bf16.h>
#include <cstdio>
#include <cstdint>

struct alignas(16) V4 { uint32_t x, y, z, w; };

__device__ __forceinline__ uint32_t add2(uint32_t a, uint32_t b) {
  __nv_bfloat162 x = *reinterpret_cast<__nv_bfloat162*>(&a), y = *reinterpret_cast<__nv_bfloat162*>(&b);
  float2 fx = __bfloat1622float2(x), fy = __bfloat1622float2(y);
  __nv_bfloat162 r = __floats2bfloat162_rn(fx.x + fy.x, fx.y + fy.y);
  return *reinterpret_cast<uint32_t*>(&r);
}
__device__ __forceinline__ V4 addv(V4 a, V4 b) { return V4{add2(a.x, b.x), add2(a.y, b.y), add2(a.z, b.z), add2(a.w, b.w)}; }

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(uint64_t* b, int n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void mb_expect(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mb_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sa(b)) : "memory");
}
__device__ __forceinline__ void mb_wait(uint64_t* b, uint32_t par) {
  asm volatile(
      "{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W;\n}\n" ::"r"(sa(b)),
      "r"(par)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* b) {
  asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(sa(dst)),
               "l"(src), "r"(bytes), "r"(sa(b))
               : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(sa(src)), "r"(bytes) : "memory");
}

// TILE V4 per input per stage, S stages, NW consumer warps + 1 producer warp.
// STORE: 0 = STG.128 from registers, 1 = results written back into the x
// stage and stored with one bulk copy (cp.async.bulk.global.shared) per tile.
template <int TILE, int S, int NW, int STORE>
__global__ void __launch_bounds__((NW + 1) * 32, 1)
tma_stream(const V4* __restrict__ x, const V4* __restrict__ y, V4* __restrict__ z, long long n, int dynamic_order,
           unsigned long long* counter) {
  extern __shared__ __align__(128) unsigned char smem[];
  V4* sx = (V4*)smem;                      // [S][TILE]
  V4* sy = sx + S * TILE;                  // [S][TILE]
  uint64_t* full = (uint64_t*)(sy + S * TILE);
  uint64_t* empty = full + S;
  long long* tq = (long long*)(empty + S);  // [S] tile index per stage (dynamic order)
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const long long ntiles = n / TILE;  // n is a multiple of TILE here
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) { mb_init(full + s, 1); mb_init(empty + s, NW); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == NW) {  // producer
    if (lane == 0) {
      long long k = 0;
      for (;; ++k) {
        long long t;
        if (dynamic_order) t = (long long)atomicAdd(counter, 1ULL);
        else t = blockIdx.x + k * gridDim.x;
        const int s = (int)(k % S);
        if (k >= S) mb_wait(empty + s, (uint32_t)(((k / S) - 1) & 1));
        tq[s] = t;
        if (t >= ntiles) { mb_arrive(full + s); break; }
        mb_expect(full + s, 2u * TILE * 16u);
        bulk_g2s(sx + s * TILE, x + t * TILE, TILE * 16u, full + s);
        bulk_g2s(sy + s * TILE, y + t * TILE, TILE * 16u, full + s);
      }
    }
    return;
  }
  const int tid = threadIdx.x;
  for (long long k = 0;; ++k) {
    const int s = (int)(k % S);
    mb_wait(full + s, (uint32_t)((k / S) & 1));
    const long long t = tq[s];
    if (t >= ntiles) break;
    if (STORE == 0) {
#pragma unroll
      for (int i = tid; i < TILE; i += NW * 32) z[t * TILE + i] = addv(sx[s * TILE + i], sy[s * TILE + i]);
      __syncwarp();
      if (lane == 0) mb_arrive(empty + s);
    } else {
#pragma unroll
      for (int i = tid; i < TILE; i += NW * 32) sx[s * TILE + i] = addv(sx[s * TILE + i], sy[s * TILE + i]);
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      asm volatile("bar.sync 1, %0;" ::"n"(NW * 32) : "memory");
      if (tid == 0) {
        bulk_s2g(z + t * TILE, sx + s * TILE, TILE * 16u);
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
      }
      asm volatile("bar.sync 1, %0;" ::"n"(NW * 32) : "memory");
      if (lane == 0) mb_arrive(empty + s);
    }
  }
  if (STORE == 1 && tid == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
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

template <int TILE, int S, int NW, int STORE>
void run(const V4* x, const V4* y, V4* z, long long n, unsigned long long* ctr, double bytes, int bps, int dyn) {
  auto k = tma_stream<TILE, S, NW, STORE>;
  const size_t sm = (size_t)2 * S * TILE * 16 + 2 * S * 8 + S * 8;
  if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm) != cudaSuccess) {
    printf("smem %zu rejected\n", sm); cudaGetLastError(); return;
  }
  const int grid = 148 * bps;
  float ms = timeit([&] { if (dyn) cudaMemsetAsync(ctr, 0, 8); k<<<grid, (NW + 1) * 32, sm>>>(x, y, z, n, dyn, ctr); });
  cudaError_t e = cudaGetLastError();
  printf("tma %s tile %6d B S%d NW%2d %s x %d/SM smem %6zu  %8.1f us %8.1f GB/s %s\n", dyn ? "dyn   " : "static",
         TILE * 16, S, NW, STORE ? "bulkst" : "stg   ", bps, sm, ms * 1e3, bytes / (ms * 1e-3) / 1e9,
         e == cudaSuccess ? "" : cudaGetErrorString(e));
}

__global__ void check(const V4* x, const V4* y, const V4* z, long long n, unsigned int* bad) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    V4 r = addv(x[i], y[i]), g = z[i];
    if (r.x != g.x || r.y != g.y || r.z != g.z || r.w != g.w) atomicAdd(bad, 1u);
  }
}
__global__ void fill(V4* p, long long n, uint32_t seed) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    uint32_t h = (uint32_t)i * 2654435761u + seed;
    h ^= h >> 13; h *= 0x5bd1e995u; h ^= h >> 15;
    uint32_t m = 0x3f803f80u | (h & 0x007f007fu);  // bf16 pairs in [1, 2)
    p[i] = V4{m, m ^ 0x10001u, m ^ 0x20002u, m ^ 0x30003u};
  }
}

int main() {
  const long long elems = 1LL << 30, n = elems / 8;  // V4 = 8 bf16
  V4 *x, *y, *z;
  cudaMalloc(&x, n * 16); cudaMalloc(&y, n * 16); cudaMalloc(&z, n * 16);
  fill<<<1184, 256>>>(x, n, 1); fill<<<1184, 256>>>(y, n, 7);
  unsigned long long* ctr; cudaMalloc(&ctr, 8);
  unsigned int* bad; cudaMalloc(&bad, 4);
  const double bytes = 3.0 * n * 16;
  for (int dyn : {0, 1}) {
    run<1024, 4, 16, 0>(x, y, z, n, ctr, bytes, 1, dyn);   // 16 KB tiles
    run<1024, 6, 16, 0>(x, y, z, n, ctr, bytes, 1, dyn);
    run<2048, 3, 16, 0>(x, y, z, n, ctr, bytes, 1, dyn);   // 32 KB tiles
    run<2048, 4, 16, 0>(x, y, z, n, ctr, bytes, 1, dyn);
    run<2048, 4, 32, 0>(x, y, z, n, ctr, bytes, 1, dyn);
    run<512, 8, 16, 0>(x, y, z, n, ctr, bytes, 1, dyn);    // 8 KB tiles
    run<512, 4, 8, 0>(x, y, z, n, ctr, bytes, 2, dyn);
    run<1024, 3, 8, 0>(x, y, z, n, ctr, bytes, 2, dyn);
    run<1024, 4, 16, 1>(x, y, z, n, ctr, bytes, 1, dyn);
    run<2048, 3, 16, 1>(x, y, z, n, ctr, bytes, 1, dyn);
  }
  cudaMemset(bad, 0, 4);
  check<<<1184, 256>>>(x, y, z, n, bad);
  unsigned int hb = 0; cudaMemcpy(&hb, bad, 4, cudaMemcpyDeviceToHost);
  printf("check (last variant): %u mismatching vectors; status %s\n", hb, cudaGetErrorString(cudaGetLastError()));
  return 0;
}
