// Prototype for the C5 global sweep with address-ordered dynamic tiles:
//   dz = dy * gelu'(z) (bf16 [R, 1024]), db = colsum(dz) (fp32 totals)
// * row tiles of TR rows staged by 1D bulk copies (UBLKCP) into an S-stage
//   shared-memory ring; one producer warp grabs tiles from a global counter
//   (tiles in address order, like a non-persistent grid: 7.0 TB/s for the
//   2R:1W mix in tma_stream.cu, vs 6.5 for static ownership);
// * each compute thread owns 4 columns and TR/2 rows of every tile; its fp32
//   partial over those rows (fixed order) is deposited into an EXACT binned
//   integer accumulator (two 32-bit-aligned int64 bins + a window index), so
//   the column totals do not depend on which CTA took which tile: bitwise
//   deterministic although the tile order is not.
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I../../paper_conf_asplos_zhengyzlzzzlyzs22_b200/csrc/kernels c5_dyn.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cmath>
#include <vector>
#include "astitch_device.cuh"

constexpr int C = 1024;
constexpr int NL = C / 4;  // lanes per row (4 columns each)

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

// ---- exact binned accumulator --------------------------------------------
// |x| = m * 2^(bi - 160), bi = biased exponent + 10 (bit index of m's LSB on
// an absolute scale). Window J: bins lo = bits [32J, 32J+32), hi = [32J+32,
// 32J+64). Each deposit adds the window's 64-bit truncation of |x| (sign
// applied), slice by slice; the window only moves up (drop the lo bin).
// Total = sum over deposits of trunc(x at the final window): independent of
// the deposit order and of how deposits are split across accumulators.
#define BIN_EMPTY (-1000)
struct Bins {
  int J;
  long long hi[4], lo[4];
  float sp[4];  // inf / nan deposits (order-independent: any NaN or +-inf mix gives the same result)
};
__device__ __forceinline__ void bins_init(Bins& b) {
  b.J = BIN_EMPTY;
#pragma unroll
  for (int k = 0; k < 4; ++k) { b.hi[k] = 0; b.lo[k] = 0; b.sp[k] = 0.f; }
}
__device__ __forceinline__ void bins_shift(Bins& b, int need) {
  if (need == b.J + 1) {
#pragma unroll
    for (int k = 0; k < 4; ++k) { b.lo[k] = b.hi[k]; b.hi[k] = 0; }
  } else {
#pragma unroll
    for (int k = 0; k < 4; ++k) { b.lo[k] = 0; b.hi[k] = 0; }
  }
  b.J = need;
}
__device__ __forceinline__ void bins_add4(Bins& b, const float* x) {
  // window needed by the largest of the four (one shared window per thread)
  int need = BIN_EMPTY;
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const uint32_t e = (__float_as_uint(x[k]) >> 23) & 0xffu;
    const int bi = (int)(e ? e : 1u) + 10;
    const int nk = (__float_as_uint(x[k]) & 0x7fffffffu) && e != 0xffu ? ((bi - 40 + 31) >> 5) : BIN_EMPTY;
    need = max(need, nk);
  }
  if (need > b.J) bins_shift(b, need);
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const uint32_t u = __float_as_uint(x[k]);
    const uint32_t e = (u >> 23) & 0xffu;
    if (e == 0xffu) { b.sp[k] += x[k]; continue; }
    const uint32_t m = (u & 0x7fffffu) | (e ? 0x800000u : 0u);
    const int d = (int)(e ? e : 1u) + 10 - 32 * b.J;  // <= 40
    const uint64_t v = d >= 0 ? ((uint64_t)m << d) : (d > -32 ? (uint64_t)(m >> (-d)) : 0ull);
    const long long vl = (long long)(v & 0xffffffffull), vh = (long long)(v >> 32);
    if (u >> 31) { b.lo[k] -= vl; b.hi[k] -= vh; } else { b.lo[k] += vl; b.hi[k] += vh; }
  }
}

struct BinOut { int J; int pad; long long hi, lo; float sp; int pad2; };  // 32 B per column

template <int TR, int S, int NW, int DYN>
__global__ void __launch_bounds__(NW * 32 + 32, 1)
c5_dyn(const uint2* __restrict__ dy, const uint2* __restrict__ z, uint2* __restrict__ dz, int R,
       unsigned long long* counter, BinOut* __restrict__ part) {
  extern __shared__ __align__(128) unsigned char smem[];
  constexpr uint32_t TB = TR * C * 2;  // bytes per input per tile
  unsigned char* sdy = smem;
  unsigned char* sz = smem + S * TB;
  uint64_t* full = (uint64_t*)(smem + 2 * S * TB);
  uint64_t* empty = full + S;
  int* tq = (int*)(empty + S);
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int ntiles = (R + TR - 1) / TR;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) { mb_init(full + s, 1); mb_init(empty + s, NW); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == NW) {
    if (lane == 0) {
      for (int k = 0;; ++k) {
        const int t = DYN ? (int)atomicAdd(counter, 1ULL) : (int)(blockIdx.x + (long long)k * gridDim.x);
        const int s = k % S;
        if (k >= S) mb_wait(empty + s, (uint32_t)(((k / S) - 1) & 1));
        tq[s] = t;
        if (t >= ntiles) { mb_arrive(full + s); break; }
        const int rows = min(TR, R - t * TR);
        mb_expect(full + s, 2u * rows * C * 2u);
        bulk_g2s(sdy + s * TB, (const char*)dy + (size_t)t * TB, rows * C * 2u, full + s);
        bulk_g2s(sz + s * TB, (const char*)z + (size_t)t * TB, rows * C * 2u, full + s);
      }
    }
    return;
  }
  constexpr int TM = NW * 32 / NL;  // teams
  const int l = threadIdx.x % NL, team = threadIdx.x / NL;
  Bins bins;
  bins_init(bins);
  for (int k = 0;; ++k) {
    const int s = k % S;
    mb_wait(full + s, (uint32_t)((k / S) & 1));
    const int t = tq[s];
    if (t >= ntiles) break;
    const int rows = min(TR, R - t * TR);
    float acc[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
    for (int r = 0; r < TR / TM; ++r) {
      const int rr = team + TM * r;
      if (rr < rows) {
        const uint2 a = *(const uint2*)(sdy + s * TB + rr * C * 2 + l * 8);
        const uint2 b = *(const uint2*)(sz + s * TB + rr * C * 2 + l * 8);
        const as::f2 g0 = as::gelu_tanh_grad2(as::f2{as::bf16lo(b.x), as::bf16hi(b.x)});
        const as::f2 g1 = as::gelu_tanh_grad2(as::f2{as::bf16lo(b.y), as::bf16hi(b.y)});
        const as::f2 d0 = as::mul2(as::f2{as::bf16lo(a.x), as::bf16hi(a.x)}, g0);
        const as::f2 d1 = as::mul2(as::f2{as::bf16lo(a.y), as::bf16hi(a.y)}, g1);
        acc[0] += d0.x; acc[1] += d0.y; acc[2] += d1.x; acc[3] += d1.y;
        uint2 o;
        o.x = as::pack_bf16x2(d0.x, d0.y);
        o.y = as::pack_bf16x2(d1.x, d1.y);
        dz[((size_t)t * TR + rr) * NL + l] = o;
      }
    }
    __syncwarp();
    if (lane == 0) mb_arrive(empty + s);
    bins_add4(bins, acc);
  }
  // CTA combine: the two teams' bins of the same columns, aligned to the max
  // window, summed exactly (int64), written as this CTA's partial row
  __shared__ int sJ[NL];
  __shared__ long long shi[NL][4], slo[NL][4];
  __shared__ float ssp[NL][4];
  for (int tt = 1; tt < TM; ++tt) {
    asm volatile("bar.sync 1, %0;" ::"n"(NW * 32) : "memory");
    if (team == tt) {
      sJ[l] = bins.J;
#pragma unroll
      for (int c = 0; c < 4; ++c) { shi[l][c] = bins.hi[c]; slo[l][c] = bins.lo[c]; ssp[l][c] = bins.sp[c]; }
    }
    asm volatile("bar.sync 1, %0;" ::"n"(NW * 32) : "memory");
    if (team == 0) {
      const int J1 = sJ[l], J = max(bins.J, J1);
      if (bins.J != J) bins_shift(bins, J);
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        if (J1 == J) { bins.hi[c] += shi[l][c]; bins.lo[c] += slo[l][c]; } else if (J1 == J - 1) { bins.lo[c] += shi[l][c]; }
        bins.sp[c] += ssp[l][c];
      }
    }
  }
  if (team == 0) {
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      BinOut o; o.J = bins.J; o.pad = 0; o.hi = bins.hi[c]; o.lo = bins.lo[c]; o.sp = bins.sp[c]; o.pad2 = 0;
      part[(size_t)blockIdx.x * C + l * 4 + c] = o;
    }
  }
}

// finalize: one thread per column, all CTA partials aligned to the max window
__global__ void c5_fin(const BinOut* __restrict__ part, int G, float* __restrict__ db) {
  const int col = blockIdx.x * blockDim.x + threadIdx.x;
  if (col >= C) return;
  int J = BIN_EMPTY;
  float sp = 0.f;
  for (int g = 0; g < G; ++g) J = max(J, part[(size_t)g * C + col].J);
  long long H = 0, L = 0;
  for (int g = 0; g < G; ++g) {
    const BinOut o = part[(size_t)g * C + col];
    sp += o.sp;
    if (o.J == J) { H += o.hi; L += o.lo; } else if (o.J == J - 1) { L += o.hi; }
  }
  double v = J == BIN_EMPTY ? 0.0 : ldexp((double)H, 32 * (J + 1) - 160) + ldexp((double)L, 32 * J - 160);
  db[col] = sp != 0.f ? sp : (float)v;
}

// plain static persistent version (register loads) of the same math, fp32 column partials (current kernel shape)
__global__ void fill(uint32_t* p, long long n, uint32_t seed) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    uint32_t h = (uint32_t)i * 2654435761u + seed;
    h ^= h >> 13; h *= 0x5bd1e995u; h ^= h >> 15; h *= 0x27d4eb2fu; h ^= h >> 16;
    // two bf16 in about N(0,1)-ish range: sign, exponent 124..128, random mantissa
    uint32_t lo = ((h & 1u) << 15) | ((124u + ((h >> 1) % 5u)) << 7) | ((h >> 4) & 0x7fu);
    uint32_t hi = (((h >> 11) & 1u) << 15) | ((124u + ((h >> 12) % 5u)) << 7) | ((h >> 16) & 0x7fu);
    p[i] = lo | (hi << 16);
  }
}

static float bf(uint16_t h) { uint32_t u = (uint32_t)h << 16; float f; memcpy(&f, &u, 4); return f; }
static double gelu_grad(double x) {
  const double c = 0.7978845608028654, k = 0.044715;
  double u = c * (x + k * x * x * x), t = tanh(u);
  return 0.5 * (1 + t) + 0.5 * x * (1 - t * t) * c * (1 + 3 * k * x * x);
}

template <int TR, int S, int NW, int DYN>
void run(int bps, const uint2* dy, const uint2* z, uint2* dz, int R, unsigned long long* ctr, BinOut* part, float* db,
         std::vector<float>& out) {
  auto k = c5_dyn<TR, S, NW, DYN>;
  const size_t sm = (size_t)2 * S * TR * C * 2 + 2 * S * 8 + S * 4;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  const int G = 148 * bps;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float best = 1e30f;
  std::vector<float> first(C);
  bool same = true;
  for (int it = 0; it < 13; ++it) {
    cudaMemsetAsync(ctr, 0, 8);
    cudaEventRecord(e0);
    k<<<G, NW * 32 + 32, sm>>>(dy, z, dz, R, ctr, part);
    cudaEventRecord(e1);
    c5_fin<<<(C + 255) / 256, 256>>>(part, G, db);
    cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    if (it >= 3 && ms < best) best = ms;
    cudaMemcpy(out.data(), db, C * 4, cudaMemcpyDeviceToHost);
    if (it == 0) first = out; else if (memcmp(first.data(), out.data(), C * 4)) same = false;
  }
  const double bytes = 3.0 * R * C * 2;
  printf("c5 %s TR %3d S%d NW%2d x%d/SM smem %6zu: %8.1f us %8.1f GB/s  run-to-run bitwise %s  err %s\n", DYN ? "dyn   " : "static", TR,
         S, NW, bps, sm, best * 1e3, bytes / (best * 1e-3) / 1e9, same ? "same" : "DIFF", cudaGetErrorString(cudaGetLastError()));
}

int main(int argc, char** argv) {
  const bool trace = argc > 1;
  const int R = 1 << 20;
  const long long n = (long long)R * C / 2;  // u32 words
  uint32_t *dy, *z, *dz;
  cudaMalloc(&dy, n * 4); cudaMalloc(&z, n * 4); cudaMalloc(&dz, n * 4);
  fill<<<1184, 256>>>(dy, n, 1); fill<<<1184, 256>>>(z, n, 7);
  unsigned long long* ctr; cudaMalloc(&ctr, 8);
  BinOut* part; cudaMalloc(&part, (size_t)148 * 4 * C * sizeof(BinOut));
  float* db; cudaMalloc(&db, C * 4);
  std::vector<float> out(C);
  if (trace) {
    auto k = c5_dyn<16, 3, 16, 1>;
    const size_t sm = (size_t)2 * 3 * 16 * C * 2 + 2 * 3 * 8 + 3 * 4;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    auto ks = c5_dyn<16, 3, 16, 0>;
    cudaFuncSetAttribute(ks, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int it = 0; it < 400; ++it) {
      const bool st = (it / 20) % 2;
      cudaMemsetAsync(ctr, 0, 8);
      cudaEventRecord(e0);
      if (st) ks<<<148, 544, sm>>>((uint2*)dy, (uint2*)z, (uint2*)dz, R, ctr, part);
      else k<<<148, 544, sm>>>((uint2*)dy, (uint2*)z, (uint2*)dz, R, ctr, part);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      printf("%d %s %.1f\n", it, st ? "static" : "dyn", ms * 1e3);
    }
    return 0;
  }
  for (int rep = 0; rep < 3; ++rep) {
    run<16, 3, 16, 1>(1, (uint2*)dy, (uint2*)z, (uint2*)dz, R, ctr, part, db, out);
    run<16, 3, 8, 1>(1, (uint2*)dy, (uint2*)z, (uint2*)dz, R, ctr, part, db, out);
    run<8, 3, 8, 1>(2, (uint2*)dy, (uint2*)z, (uint2*)dz, R, ctr, part, db, out);
    run<8, 4, 8, 1>(1, (uint2*)dy, (uint2*)z, (uint2*)dz, R, ctr, part, db, out);
    run<16, 3, 16, 0>(1, (uint2*)dy, (uint2*)z, (uint2*)dz, R, ctr, part, db, out);
    run<12, 4, 16, 1>(1, (uint2*)dy, (uint2*)z, (uint2*)dz, R, ctr, part, db, out);
    run<4, 6, 8, 1>(2, (uint2*)dy, (uint2*)z, (uint2*)dz, R, ctr, part, db, out);
  }
  run<16, 3, 16, 1>(1, (uint2*)dy, (uint2*)z, (uint2*)dz, R, ctr, part, db, out);
  // accuracy: 8 columns against an fp64 host sum of dy * gelu'(z)
  std::vector<uint32_t> hdy(n), hz(n);
  cudaMemcpy(hdy.data(), dy, n * 4, cudaMemcpyDeviceToHost);
  cudaMemcpy(hz.data(), z, n * 4, cudaMemcpyDeviceToHost);
  double worst = 0, rms = 0;
  for (int col = 0; col < C; col += 129) {
    double s = 0;
    for (long long r = 0; r < R; ++r) {
      const long long w = r * (C / 2) + col / 2;
      const uint16_t a = (col & 1) ? (hdy[w] >> 16) : (hdy[w] & 0xffff), b = (col & 1) ? (hz[w] >> 16) : (hz[w] & 0xffff);
      s += (double)bf(a) * gelu_grad((double)bf(b));
    }
    worst = fmax(worst, fabs(s - out[col]) / fmax(fabs(s), 1.0));
    rms += s * s;
    printf("  col %4d: fp64 %.9g gpu %.9g\n", col, s, out[col]);
  }
  printf("worst rel err %.3g (fp32 output rounding is 6e-8)\n", worst);
  return 0;
}
