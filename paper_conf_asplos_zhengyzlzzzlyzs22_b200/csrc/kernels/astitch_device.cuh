// astitch_device.cuh — hand-written sm_100a device building blocks of the
// stitched kernels.  The planner's code generator (codegen.cpp) instantiates
// one of the scheme templates below per subgraph and fills in the op chain;
// the result is compiled by NVRTC for sm_100a (the paper's JIT).
//
//   memory  : 16/32-byte streaming loads (ld.global.nc.L1::no_allocate),
//             vector stores, bf16/f16 <-> fp32 packing
//   local   : element-wise math in fp32 registers (Table 1 "local")
//   regional: team reductions by warp shuffles / shared memory (Table 1
//             "regional"; block locality)
//   global  : HBM partials + generation-counted grid barrier (Table 1
//             "global")
//   packed  : TMA bulk (cp.async.bulk) row tiles + mbarrier pipeline for
//             many tiny rows (horizontal packing)
//
// No includes: NVRTC compiles this without the CUDA headers.
#pragma once

typedef unsigned int u32;
typedef unsigned long long u64;
typedef unsigned short u16;

#define AS_INF __int_as_float(0x7f800000)

namespace as {

// ------------------------------------------------------------------ raw chunks
template <int NB> struct Raw;
template <> struct Raw<2> { u16 x; };
template <> struct Raw<4> { u32 x; };
template <> struct Raw<8> { u32 x, y; };
template <> struct Raw<16> { u32 x, y, z, w; };
template <> struct Raw<32> { u32 x, y, z, w, a, b, c, d; };
// 32-bit word q of a raw vector (q a compile-time constant after unrolling)
__device__ __forceinline__ u32 word(const Raw<4>& r, int) { return r.x; }
__device__ __forceinline__ u32 word(const Raw<8>& r, int q) { return q == 0 ? r.x : r.y; }
__device__ __forceinline__ u32 word(const Raw<16>& r, int q) { return q == 0 ? r.x : q == 1 ? r.y : q == 2 ? r.z : r.w; }
__device__ __forceinline__ u32 word(const Raw<32>& r, int q) {
  return q == 0 ? r.x : q == 1 ? r.y : q == 2 ? r.z : q == 3 ? r.w : q == 4 ? r.a : q == 5 ? r.b : q == 6 ? r.c : r.d;
}

// streaming (read-once) global loads: no L1 allocation
__device__ __forceinline__ Raw<2> ldg(const Raw<2>* p) {
  Raw<2> r;
  asm volatile("ld.global.nc.L1::no_allocate.b16 %0, [%1];" : "=h"(r.x) : "l"(p));
  return r;
}
__device__ __forceinline__ Raw<4> ldg(const Raw<4>* p) {
  Raw<4> r;
  asm volatile("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(r.x) : "l"(p));
  return r;
}
__device__ __forceinline__ Raw<8> ldg(const Raw<8>* p) {
  Raw<8> r;
  asm volatile("ld.global.nc.L1::no_allocate.v2.b32 {%0,%1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
  return r;
}
// load cache qualifiers of the streaming inputs (experiments: e.g. an L2
// prefetch-size hint), selectable at JIT time like AS_STQ
#ifndef AS_LDQ
#define AS_LDQ ".L1::no_allocate"
#endif
__device__ __forceinline__ Raw<16> ldg(const Raw<16>* p) {
  Raw<16> r;
  asm volatile("ld.global.nc" AS_LDQ ".v4.b32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ Raw<32> ldg(const Raw<32>* p) {
  Raw<32> r;
  asm volatile("ld.global.nc" AS_LDQ ".v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w), "=r"(r.a), "=r"(r.b), "=r"(r.c), "=r"(r.d)
               : "l"(p));
  return r;
}
// L2-coherent (.cg) loads of workspace data written earlier in the same kernel
__device__ __forceinline__ Raw<16> ldg_cg(const Raw<16>* p) {
  Raw<16> r;
  asm volatile("ld.global.cg.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ Raw<8> ldg_cg(const Raw<8>* p) {
  Raw<8> r;
  asm volatile("ld.global.cg.v2.b32 {%0,%1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
  return r;
}
__device__ __forceinline__ Raw<4> ldg_cg(const Raw<4>* p) {
  Raw<4> r;
  asm volatile("ld.global.cg.b32 %0, [%1];" : "=r"(r.x) : "l"(p));
  return r;
}
__device__ __forceinline__ Raw<32> ldg_cg(const Raw<32>* p) {
  Raw<32> r;
  const Raw<16>* q = reinterpret_cast<const Raw<16>*>(p);
  Raw<16> a = ldg_cg(q), b = ldg_cg(q + 1);
  r.x = a.x; r.y = a.y; r.z = a.z; r.w = a.w; r.a = b.x; r.b = b.y; r.c = b.z; r.d = b.w;
  return r;
}
// L1-cached read-only loads for operands re-read every row (COLVEC vectors)
__device__ __forceinline__ Raw<2> ldg_l1(const Raw<2>* p) {
  Raw<2> r; asm volatile("ld.global.nc.b16 %0, [%1];" : "=h"(r.x) : "l"(p)); return r;
}
__device__ __forceinline__ Raw<4> ldg_l1(const Raw<4>* p) {
  Raw<4> r; asm volatile("ld.global.nc.b32 %0, [%1];" : "=r"(r.x) : "l"(p)); return r;
}
__device__ __forceinline__ Raw<8> ldg_l1(const Raw<8>* p) {
  Raw<8> r; asm volatile("ld.global.nc.v2.b32 {%0,%1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p)); return r;
}
__device__ __forceinline__ Raw<16> ldg_l1(const Raw<16>* p) {
  Raw<16> r;
  asm volatile("ld.global.nc.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ Raw<32> ldg_l1(const Raw<32>* p) {
  Raw<32> r;
  asm volatile("ld.global.nc.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w), "=r"(r.a), "=r"(r.b), "=r"(r.c), "=r"(r.d)
               : "l"(p));
  return r;
}

__device__ __forceinline__ void stg(Raw<2>* p, const Raw<2>& r) {
  asm volatile("st.global.b16 [%0], %1;" ::"l"(p), "h"(r.x) : "memory");
}
__device__ __forceinline__ void stg(Raw<4>* p, const Raw<4>& r) {
  asm volatile("st.global.b32 [%0], %1;" ::"l"(p), "r"(r.x) : "memory");
}
__device__ __forceinline__ void stg(Raw<8>* p, const Raw<8>& r) {
  asm volatile("st.global.v2.b32 [%0], {%1,%2};" ::"l"(p), "r"(r.x), "r"(r.y) : "memory");
}
// store cache qualifier for the streaming outputs (empty = default policy;
// e.g. ".cs" evict-first), selectable at JIT time for experiments
#ifndef AS_STQ
#define AS_STQ ""
#endif
__device__ __forceinline__ void stg(Raw<16>* p, const Raw<16>& r) {
  asm volatile("st.global" AS_STQ ".v4.b32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(r.x), "r"(r.y), "r"(r.z), "r"(r.w)
               : "memory");
}
__device__ __forceinline__ void stg(Raw<32>* p, const Raw<32>& r) {
  asm volatile("st.global.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(r.x), "r"(r.y), "r"(r.z),
               "r"(r.w), "r"(r.a), "r"(r.b), "r"(r.c), "r"(r.d)
               : "memory");
}

// shared-memory chunk loads / stores (packed template); saddr = shared window address
__device__ __forceinline__ Raw<2> lds(u32 a) { Raw<2> r; asm volatile("ld.shared.b16 %0, [%1];" : "=h"(r.x) : "r"(a)); return r; }
__device__ __forceinline__ Raw<4> lds4(u32 a) { Raw<4> r; asm volatile("ld.shared.b32 %0, [%1];" : "=r"(r.x) : "r"(a)); return r; }
template <int NB> __device__ __forceinline__ Raw<NB> lds_chunk(u32 a);
template <> __device__ __forceinline__ Raw<2> lds_chunk<2>(u32 a) { return lds(a); }
template <> __device__ __forceinline__ Raw<4> lds_chunk<4>(u32 a) { return lds4(a); }
template <> __device__ __forceinline__ Raw<8> lds_chunk<8>(u32 a) {
  Raw<8> r; asm volatile("ld.shared.v2.b32 {%0,%1}, [%2];" : "=r"(r.x), "=r"(r.y) : "r"(a)); return r;
}
template <> __device__ __forceinline__ Raw<16> lds_chunk<16>(u32 a) {
  Raw<16> r;
  asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "r"(a));
  return r;
}
template <> __device__ __forceinline__ Raw<32> lds_chunk<32>(u32 a) {
  Raw<32> r;
  asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "r"(a));
  asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(r.a), "=r"(r.b), "=r"(r.c), "=r"(r.d) : "r"(a + 16));
  return r;
}
template <int NB> __device__ __forceinline__ void sts_chunk(u32 a, const Raw<NB>& r);
template <> __device__ __forceinline__ void sts_chunk<2>(u32 a, const Raw<2>& r) {
  asm volatile("st.shared.b16 [%0], %1;" ::"r"(a), "h"(r.x) : "memory");
}
template <> __device__ __forceinline__ void sts_chunk<4>(u32 a, const Raw<4>& r) {
  asm volatile("st.shared.b32 [%0], %1;" ::"r"(a), "r"(r.x) : "memory");
}
template <> __device__ __forceinline__ void sts_chunk<8>(u32 a, const Raw<8>& r) {
  asm volatile("st.shared.v2.b32 [%0], {%1,%2};" ::"r"(a), "r"(r.x), "r"(r.y) : "memory");
}
template <> __device__ __forceinline__ void sts_chunk<16>(u32 a, const Raw<16>& r) {
  asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(a), "r"(r.x), "r"(r.y), "r"(r.z), "r"(r.w) : "memory");
}
template <> __device__ __forceinline__ void sts_chunk<32>(u32 a, const Raw<32>& r) {
  asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(a), "r"(r.x), "r"(r.y), "r"(r.z), "r"(r.w) : "memory");
  asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(a + 16), "r"(r.a), "r"(r.b), "r"(r.c), "r"(r.d) : "memory");
}

// ------------------------------------------------------------------ dtype conversion
// DT: 0 = f32, 1 = bf16, 2 = f16
__device__ __forceinline__ float bf16lo(u32 w) { return __int_as_float(w << 16); }
__device__ __forceinline__ float bf16hi(u32 w) { return __int_as_float(w & 0xffff0000u); }
__device__ __forceinline__ u32 pack_bf16x2(float lo, float hi) {
  u32 r;
  asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
}
__device__ __forceinline__ float f16lo(u32 w) {
  float f; asm("{.reg .b16 l, h; mov.b32 {l, h}, %1; cvt.f32.f16 %0, l;}" : "=f"(f) : "r"(w)); return f;
}
__device__ __forceinline__ float f16hi(u32 w) {
  float f; asm("{.reg .b16 l, h; mov.b32 {l, h}, %1; cvt.f32.f16 %0, h;}" : "=f"(f) : "r"(w)); return f;
}
__device__ __forceinline__ u32 pack_f16x2(float lo, float hi) {
  u32 r;
  asm("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
}

__device__ __forceinline__ void words_to_float(int DT, const u32* w, int nwords, float* out) {
  if (DT == 0) {
#pragma unroll
    for (int i = 0; i < nwords; ++i) out[i] = __int_as_float(w[i]);
  } else if (DT == 1) {
#pragma unroll
    for (int i = 0; i < nwords; ++i) { out[2 * i] = bf16lo(w[i]); out[2 * i + 1] = bf16hi(w[i]); }
  } else {
#pragma unroll
    for (int i = 0; i < nwords; ++i) { out[2 * i] = f16lo(w[i]); out[2 * i + 1] = f16hi(w[i]); }
  }
}

template <int DT, int E> struct Conv {
  static constexpr int NB = E * (DT == 0 ? 4 : 2);
  __device__ static __forceinline__ void unpack(const Raw<NB>& r, float* o) {
    if constexpr (NB == 2) {
      u32 w = r.x;
      o[0] = DT == 1 ? bf16lo(w) : f16lo(w);
    } else {
      words_to_float(DT, reinterpret_cast<const u32*>(&r), NB / 4, o);
    }
  }
  __device__ static __forceinline__ Raw<NB> pack(const float* v) {
    Raw<NB> r;
    if constexpr (NB == 2) {
      u32 w = DT == 1 ? pack_bf16x2(v[0], 0.f) : pack_f16x2(v[0], 0.f);
      r.x = static_cast<u16>(w & 0xffffu);
    } else {
      u32* w = reinterpret_cast<u32*>(&r);
      if (DT == 0) {
#pragma unroll
        for (int i = 0; i < NB / 4; ++i) w[i] = __float_as_int(v[i]);
      } else {
#pragma unroll
        for (int i = 0; i < NB / 4; ++i)
          w[i] = DT == 1 ? pack_bf16x2(v[2 * i], v[2 * i + 1]) : pack_f16x2(v[2 * i], v[2 * i + 1]);
      }
    }
    return r;
  }
};

// Packed varlen segments (astitch_graph_segments): the entry {row_start, cols,
// pitch, offset8} of the segment owning `row` = the largest s with
// row_start_s <= row (row_start increasing; empty segments share a start and
// the search lands on the last of them, the one whose range holds the row).
template <int NSEG> __device__ __forceinline__ int seg_find_idx(const int4* __restrict__ sg, int row) {
  int lo = 0, hi = NSEG - 1;
#pragma unroll 1
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (__ldg(&sg[mid].x) <= row) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}
template <int NSEG> __device__ __forceinline__ int4 seg_find(const int4* __restrict__ sg, int row) {
  return __ldg(sg + seg_find_idx<NSEG>(sg, row));
}

// scalar (ROWVEC / COLVEC element) load / store with dtype
template <int DT> __device__ __forceinline__ float ld_scalar(const void* base, long long i) {
  if (DT == 0) return __ldg(reinterpret_cast<const float*>(base) + i);
  u16 h = __ldg(reinterpret_cast<const unsigned short*>(base) + i);
  return DT == 1 ? __int_as_float(static_cast<u32>(h) << 16) : f16lo(h);
}
template <int DT> __device__ __forceinline__ void st_scalar(void* base, long long i, float v) {
  if (DT == 0) { reinterpret_cast<float*>(base)[i] = v; return; }
  u32 w = DT == 1 ? pack_bf16x2(v, 0.f) : pack_f16x2(v, 0.f);
  reinterpret_cast<unsigned short*>(base)[i] = static_cast<unsigned short>(w & 0xffffu);
}

// ------------------------------------------------------------------ local: fp32 math
// MUFU-based with cancellation-free forms (reading R6: no tanh.approx).
__device__ __forceinline__ float ex2(float x) { float r; asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x)); return r; }
__device__ __forceinline__ float rcp(float x) { float r; asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x)); return r; }
// NaN-propagating max / min (reading R12: RMAX propagates NaN, as the oracle's
// numpy max does; fmaxf would drop it).  One FMNMX with the .NaN modifier.
__device__ __forceinline__ float nmax(float a, float b) { float r; asm("max.NaN.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ float nmin(float a, float b) { float r; asm("min.NaN.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b)); return r; }
// Order key of a float for an INTEGER max across ranks (ncclMax on int32):
// monotone in the float order, NaN canonicalised to the largest key, so the
// sharded column RMAX propagates NaN like nmax (an fp32 ncclMax would drop it).
__device__ __forceinline__ int okey(float x) {
  const int b = (x != x) ? 0x7fc00000 : __float_as_int(x);
  return b >= 0 ? b : (b ^ 0x7fffffff);
}
__device__ __forceinline__ float okey_dec(int k) { return __int_as_float(k >= 0 ? k : (k ^ 0x7fffffff)); }
__device__ __forceinline__ double dmaxn(double a, double b) { return (a != a || b != b) ? a + b : fmax(a, b); }
__device__ __forceinline__ double dminn(double a, double b) { return (a != a || b != b) ? a + b : fmin(a, b); }
__device__ __forceinline__ float rsq(float x) { float r; asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x)); return r; }
__device__ __forceinline__ float sqrt_(float x) { float r; asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x)); return r; }
__device__ __forceinline__ float fexp(float x) { return ex2(x * 1.4426950408889634f); }
__device__ __forceinline__ float fdiv(float a, float b) { return a * rcp(b); }
__device__ __forceinline__ float fsigmoid(float x) { return rcp(1.0f + fexp(-x)); }
// tanh for general use: accurate libdevice form (small |x| would cancel in the exp form)
__device__ __forceinline__ float ftanh(float x) { return tanhf(x); }
__device__ __forceinline__ float ferf(float x) { return erff(x); }
__device__ __forceinline__ float flog(float x) { return logf(x); }

#define AS_GELU_C 0.7978845608028654f  /* sqrt(2/pi) */
#define AS_GELU_K 0.044715f
// gelu_tanh(x) = 0.5 x (1 + tanh(u)) = x * sigmoid(2u), u = c (x + k x^3)
__device__ __forceinline__ float gelu_tanh(float x) {
  float u = AS_GELU_C * fmaf(AS_GELU_K * x, x * x, x);
  return x * rcp(1.0f + ex2(-2.8853900817779268f * u));   // exp(-2u) = 2^(-2u log2 e)
}
// d/dx gelu_tanh = sigmoid(2u) + 0.5 x sech^2(u) c (1 + 3 k x^2)
// with e = exp(-2|u|): sigmoid(2u) = u>=0 ? 1/(1+e) : e/(1+e);  sech^2 u = 4e/(1+e)^2
__device__ __forceinline__ float gelu_tanh_grad(float x) {
  float x2 = x * x;
  float u = AS_GELU_C * fmaf(AS_GELU_K * x, x2, x);
  float e = ex2(-2.8853900817779268f * fabsf(u));
  float r = rcp(1.0f + e);
  float sig = u >= 0.f ? r : e * r;
  float sech2 = 4.0f * e * r * r;
  float du = AS_GELU_C * fmaf(3.0f * AS_GELU_K, x2, 1.0f);
  return fmaf(0.5f * x * sech2, du, sig);
}
// exact GELU: x Phi(x) = 0.5 x erfc(-x / sqrt 2) (no cancellation for x << 0)
__device__ __forceinline__ float gelu_erf(float x) { return 0.5f * x * erfcf(-0.7071067811865476f * x); }

__device__ __forceinline__ float fpow(float a, float b) { return powf(a, b); }

// ------------------------------------------------------------------ local: paired fp32 math
// sm_100 executes two fp32 add/mul/fma per instruction (FADD2 / FMUL2 /
// FFMA2 on an aligned register pair).  Element-wise chains are emitted on
// element pairs so the issue slots per element halve; MUFU ops stay scalar.
struct f2 { float x, y; };
__device__ __forceinline__ u64 pk2(f2 a) { u64 r; asm("mov.b64 %0, {%1,%2};" : "=l"(r) : "f"(a.x), "f"(a.y)); return r; }
__device__ __forceinline__ f2 upk2(u64 r) { f2 d; asm("mov.b64 {%0,%1}, %2;" : "=f"(d.x), "=f"(d.y) : "l"(r)); return d; }
__device__ __forceinline__ f2 bc2(float s) { return f2{s, s}; }
__device__ __forceinline__ f2 add2(f2 a, f2 b) { u64 r; asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(pk2(a)), "l"(pk2(b))); return upk2(r); }
__device__ __forceinline__ f2 sub2(f2 a, f2 b) { u64 r; asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(pk2(a)), "l"(pk2(b))); return upk2(r); }
__device__ __forceinline__ f2 mul2(f2 a, f2 b) { u64 r; asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(pk2(a)), "l"(pk2(b))); return upk2(r); }
__device__ __forceinline__ f2 fma2(f2 a, f2 b, f2 c) {
  u64 r; asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(pk2(a)), "l"(pk2(b)), "l"(pk2(c))); return upk2(r);
}
__device__ __forceinline__ f2 abs2(f2 a) { return f2{fabsf(a.x), fabsf(a.y)}; }
// sm_100a mixed-precision adds: fp32 <- (bf16 | f16 element of a packed word) + fp32,
// the 16-bit operand widened exactly inside the FHADD (no separate unpack)
__device__ __forceinline__ f2 hadd2_bf16(u32 w, f2 c) {
  f2 r;
  asm("{ .reg .b16 lo, hi; mov.b32 {lo, hi}, %2;\n add.rn.f32.bf16 %0, lo, %3;\n add.rn.f32.bf16 %1, hi, %4; }"
      : "=f"(r.x), "=f"(r.y) : "r"(w), "f"(c.x), "f"(c.y));
  return r;
}
__device__ __forceinline__ f2 hadd2_f16(u32 w, f2 c) {
  f2 r;
  asm("{ .reg .b16 lo, hi; mov.b32 {lo, hi}, %2;\n add.rn.f32.f16 %0, lo, %3;\n add.rn.f32.f16 %1, hi, %4; }"
      : "=f"(r.x), "=f"(r.y) : "r"(w), "f"(c.x), "f"(c.y));
  return r;
}
__device__ __forceinline__ f2 neg2(f2 a) { return f2{-a.x, -a.y}; }
__device__ __forceinline__ f2 max2(f2 a, f2 b) { return f2{nmax(a.x, b.x), nmax(a.y, b.y)}; }
__device__ __forceinline__ f2 min2(f2 a, f2 b) { return f2{nmin(a.x, b.x), nmin(a.y, b.y)}; }
__device__ __forceinline__ f2 ex2_2(f2 a) { return f2{ex2(a.x), ex2(a.y)}; }
__device__ __forceinline__ f2 rcp_2(f2 a) { return f2{rcp(a.x), rcp(a.y)}; }
__device__ __forceinline__ f2 fexp2(f2 a) { return ex2_2(mul2(a, bc2(1.4426950408889634f))); }
__device__ __forceinline__ f2 fdiv2(f2 a, f2 b) { return mul2(a, rcp_2(b)); }
__device__ __forceinline__ f2 rsq2(f2 a) { return f2{rsq(a.x), rsq(a.y)}; }
__device__ __forceinline__ f2 sqrt2_(f2 a) { return f2{sqrt_(a.x), sqrt_(a.y)}; }
__device__ __forceinline__ f2 flog2_(f2 a) { return f2{flog(a.x), flog(a.y)}; }
__device__ __forceinline__ f2 ftanh2(f2 a) { return f2{ftanh(a.x), ftanh(a.y)}; }
__device__ __forceinline__ f2 ferf2(f2 a) { return f2{ferf(a.x), ferf(a.y)}; }
__device__ __forceinline__ f2 gelu_erf2(f2 a) { return f2{gelu_erf(a.x), gelu_erf(a.y)}; }
__device__ __forceinline__ f2 fpow2(f2 a, f2 b) { return f2{fpow(a.x, b.x), fpow(a.y, b.y)}; }
__device__ __forceinline__ f2 fsigmoid2(f2 a) {
  f2 e = ex2_2(mul2(a, bc2(-1.4426950408889634f)));
  return rcp_2(add2(e, bc2(1.0f)));
}
// gelu_tanh = x * sigmoid(2u), u = x * (c + c k x^2)
// (-2 log2 e) folded into the polynomial's constants: exp(-2u) = 2^(x * t),
// t = -2 log2(e) c (1 + k x^2) -- one paired multiply fewer per element pair
__device__ __forceinline__ f2 gelu_tanh2(f2 x) {
  f2 x2 = mul2(x, x);
  f2 t = fma2(bc2(-2.8853900817779268f * AS_GELU_C * AS_GELU_K), x2, bc2(-2.8853900817779268f * AS_GELU_C));
  f2 e = ex2_2(mul2(x, t));
  return mul2(x, rcp_2(add2(e, bc2(1.0f))));
}
// gelu_tanh' = sigmoid(2u) + (x e r^2) * 2c(1 + 3k x^2),  e = exp(-2|u|), r = 1/(1+e)
// (same cancellation-free form as gelu_tanh_grad, reassociated for FFMA2)
__device__ __forceinline__ f2 gelu_tanh_grad2(f2 x) {
  f2 x2 = mul2(x, x);
  // a = 2 log2(e) u (same sign as u): exp(-2|u|) = 2^(-|a|), the negated
  // absolute value is an operand modifier of the MUFU.EX2
  f2 a = mul2(x, fma2(bc2(2.8853900817779268f * AS_GELU_C * AS_GELU_K), x2, bc2(2.8853900817779268f * AS_GELU_C)));
  f2 e = ex2_2(neg2(abs2(a)));
  f2 r = rcp_2(add2(e, bc2(1.0f)));
  f2 er = mul2(e, r);
  f2 sig = f2{a.x >= 0.f ? r.x : er.x, a.y >= 0.f ? r.y : er.y};
  f2 du2 = fma2(bc2(6.0f * AS_GELU_C * AS_GELU_K), x2, bc2(2.0f * AS_GELU_C));
  return fma2(mul2(mul2(x, er), r), du2, sig);
}
__device__ __forceinline__ f2 gelu_tanh_grad_2(f2 x) { return gelu_tanh_grad2(x); }

// ------------------------------------------------------------------ regional: team reductions
template <int T> __device__ __forceinline__ float team_sum(float v) {
#pragma unroll
  for (int o = (T < 32 ? T : 32) / 2; o > 0; o /= 2) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
template <int T> __device__ __forceinline__ float team_max(float v) {
#pragma unroll
  for (int o = (T < 32 ? T : 32) / 2; o > 0; o /= 2) v = nmax(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
// team larger than a warp == whole block: warp tree, then a fixed-order
// combine of the per-warp values in shared memory (deterministic).
template <int T, bool MAX> __device__ __forceinline__ float block_team_reduce(float v, float* scratch) {
  v = MAX ? team_max<32>(v) : team_sum<32>(v);
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  __syncthreads();  // scratch reuse guard
  if (l == 0) scratch[w] = v;
  __syncthreads();
  constexpr int NW = T / 32;
  float r = (l < NW) ? scratch[l] : (MAX ? -AS_INF : 0.f);
  r = MAX ? team_max<32>(r) : team_sum<32>(r);
  return r;
}

// ------------------------------------------------------------------ regional across a cluster
// Task splitting: one row is split over the K CTAs of a thread-block
// cluster; the block partials are combined through distributed shared memory
// (DSMEM) in a fixed rank order, so every CTA obtains the identical row value
// (replaces the paper's cross-block atomic; deterministic).
__device__ __forceinline__ u32 cluster_rank() { u32 r; asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r)); return r; }
__device__ __forceinline__ u32 cluster_idx() { u32 r; asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(r)); return r; }
__device__ __forceinline__ u32 cluster_count() { u32 r; asm volatile("mov.u32 %0, %%nclusterid.x;" : "=r"(r)); return r; }
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ float ld_dsmem_f32(const float* local, u32 rank) {
  u32 a = static_cast<u32>(__cvta_generic_to_shared(local)), ra;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(a), "r"(rank));
  float v;
  asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(ra) : "memory");
  return v;
}
__device__ __forceinline__ double ld_dsmem_f64(const double* local, u32 rank) {
  u32 a = static_cast<u32>(__cvta_generic_to_shared(local)), ra;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(a), "r"(rank));
  double v;
  asm volatile("ld.shared::cluster.f64 %0, [%1];" : "=d"(v) : "r"(ra) : "memory");
  return v;
}

// fp64 team sum for cancellation-prone row sums (e.g. a mean that is then
// subtracted): the result is carried as a double and split hi+lo in fp32.
template <int T> __device__ __forceinline__ double team_sum_d(double v) {
#pragma unroll
  for (int o = (T < 32 ? T : 32) / 2; o > 0; o /= 2) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
template <int T> __device__ __forceinline__ double block_team_sum_d(double v, double* scratch) {
  v = team_sum_d<32>(v);
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  __syncthreads();
  if (l == 0) scratch[w] = v;
  __syncthreads();
  constexpr int NW = T / 32;
  double r = (l < NW) ? scratch[l] : 0.0;
  return team_sum_d<32>(r);
}
template <int N> struct TreeD {
  __device__ static __forceinline__ double reduce(const float* a) {
    if constexpr (N == 1) {
      return static_cast<double>(a[0]);
    } else {
      constexpr int H = N / 2;
      return TreeD<H>::reduce(a) + TreeD<N - H>::reduce(a + H);
    }
  }
};

// block tree, then the K block partials of the cluster combined via DSMEM
// (slot: a per-reduction __shared__ word; two cluster barriers make the slot
// safe to rewrite by the next row)
template <int NT, int K, bool MAX>
__device__ __forceinline__ float cluster_team_reduce(float v, float* scratch, float* slot) {
  v = block_team_reduce<NT, MAX>(v, scratch);
  if (threadIdx.x == 0) *slot = v;
  cluster_sync_all();
  float r = MAX ? -AS_INF : 0.f;
#pragma unroll
  for (int q = 0; q < K; ++q) {
    const float x = ld_dsmem_f32(slot, static_cast<u32>(q));
    r = MAX ? nmax(r, x) : r + x;
  }
  cluster_sync_all();
  return r;
}
template <int NT, int K>
__device__ __forceinline__ double cluster_team_sum_d(double v, double* scratch, double* slot) {
  v = block_team_sum_d<NT>(v, scratch);
  if (threadIdx.x == 0) *slot = v;
  cluster_sync_all();
  double r = 0.0;
#pragma unroll
  for (int q = 0; q < K; ++q) r += ld_dsmem_f64(slot, static_cast<u32>(q));
  cluster_sync_all();
  return r;
}

// pairwise tree over a register array (fixed order -> deterministic)
template <int N, bool MAX> struct Tree {
  __device__ static __forceinline__ float reduce(const float* a) {
    if constexpr (N == 1) {
      return a[0];
    } else {
      constexpr int H = N / 2;
      float l = Tree<H, MAX>::reduce(a);
      float r = Tree<N - H, MAX>::reduce(a + H);
      return MAX ? nmax(l, r) : l + r;
    }
  }
};

// pairwise tree over f32x2 pairs: (a[0],a[1]), (a[2],a[3]), ... reduced with
// paired FADD2 (half the issue slots of the scalar tree), then x + y.  A fixed
// order, so deterministic (a different order from Tree<N,false>).
template <int M> struct Tree2 {
  __device__ static __forceinline__ f2 reduce(const float* a) {
    if constexpr (M == 1) {
      return f2{a[0], a[1]};
    } else {
      constexpr int H = M / 2;
      return add2(Tree2<H>::reduce(a), Tree2<M - H>::reduce(a + 2 * H));
    }
  }
};
template <int N> struct TreeSum {
  __device__ static __forceinline__ float reduce(const float* a) {
    if constexpr (N >= 4 && (N % 2) == 0) {
      const f2 r = Tree2<N / 2>::reduce(a);
      return r.x + r.y;
    } else {
      return Tree<N, false>::reduce(a);
    }
  }
};

// ------------------------------------------------------------------ fused sharded exchange
// System-scope release / acquire on flags that other GPUs write over NVLink
// (peer memory); the data they guard is published with a system fence.
__device__ __forceinline__ void st_release_sys(unsigned int* p, unsigned int v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned int ld_acquire_sys(const unsigned int* p) {
  unsigned int v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long globaltimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Wait (thread 0 of a block) until every rank's flag holds `gen`; bounded
// (5 s of wall time) so a missing rank cannot hang the GPU: on timeout the
// error word is set and the caller proceeds with whatever the slots hold.
__device__ __forceinline__ void wait_flags(const unsigned int* flags, int world, unsigned int gen,
                                           unsigned int* err) {
  const unsigned long long t0 = globaltimer_ns();
  for (int q = 0; q < world; ++q) {
    // wrap-safe "published at or past this generation": a fast peer may
    // already have moved on to gen + 1 (never to gen + 2: that needs our flag)
    while (static_cast<int>(ld_acquire_sys(flags + q) - gen) < 0) {
      if (globaltimer_ns() - t0 > 5000000000ULL) { atomicOr(err, 1u); return; }
      __nanosleep(200);
    }
  }
}

// ------------------------------------------------------------------ global: grid barrier
// Self-resetting barrier for a co-resident (cooperative) grid on the word
// bar[0] (below).  No memset per run.
__device__ __forceinline__ u32 ld_acquire(const u32* p) {
  u32 v; asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ void st_release(u32* p, u32 v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ u32 atom_add_acqrel(u32* p, u32 v) {
  u32 old; asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory"); return old;
}
// Grid barrier on ONE self-resetting word (round 2): every CTA adds 1 except
// CTA 0, which adds 2^31 - (nb - 1), so the word crosses a multiple of 2^31
// -- its top bit flips -- exactly when the last CTA arrives, whatever the
// arrival order; waiters poll that bit.  Each episode adds exactly 2^31, so
// the word is again a multiple of 2^31 afterwards (no reset, any number of
// barriers and runs; workspace_init zeroes it once).  A CTA already at the
// next barrier cannot flip the bit back before everyone has left this one
// (its partial contribution stays below 2^31).  One atomic per CTA and no
// release store on the critical path: 1.2 us per barrier vs 1.9-2.0 us for
// the round-1 count + generation pair (scripts/micro/barrier_compare.cu).
// __threadfence before the arrival publishes this CTA's writes (ordered
// before it by __syncthreads), the one after the wait acquires the others'.
__device__ __forceinline__ u32 ld_volatile_u32(const u32* p) {
  u32 v; asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ void grid_barrier(u32* bar) {
  __syncthreads();
  if (threadIdx.x == 0) {
    const u32 nb = gridDim.x * gridDim.y * gridDim.z;
    const u32 add = (blockIdx.x == 0 && blockIdx.y == 0 && blockIdx.z == 0) ? (0x80000000u - (nb - 1u)) : 1u;
    __threadfence();
    const u32 old = atomicAdd(bar, add);
#ifdef AS_BARRIER_TIMEOUT_NS
    // debug build of the barrier (ASTITCH_FLAG_DEBUG_BARRIER): a block that
    // never arrives (a non-resident grid, a corrupted workspace) makes the
    // waiters trap after the bound instead of hanging the GPU
    const unsigned long long t0 = globaltimer_ns();
    while (((old ^ ld_volatile_u32(bar)) & 0x80000000u) == 0u) {
      if (globaltimer_ns() - t0 > (unsigned long long)(AS_BARRIER_TIMEOUT_NS)) {
        printf("astitch: grid barrier timeout (block %u of %u, word %08x)\n", blockIdx.x, nb, ld_volatile_u32(bar));
        __trap();
      }
    }
#else
    while (((old ^ ld_volatile_u32(bar)) & 0x80000000u) == 0u) { }
#endif
    __threadfence();
  }
  __syncthreads();
}
// L2-coherent load of data written earlier in the same kernel by other blocks
__device__ __forceinline__ float ld_cg(const float* p) { return __ldcg(p); }

// ------------------------------------------------------------------ global: exact binned column sums
// Order-independent column sums for sweeps whose row tiles are handed out
// dynamically (tma_sweep, reading R23): which CTA sums which tile depends on
// scheduling, so an fp32 accumulator would round differently run to run.
// Instead every deposit x (an fp32 tile partial) is added EXACTLY to two
// int64 bins of a 64-bit fixed-point window aligned to multiples of 32 bits:
// |x| = m * 2^(bi - 160) with m the 24-bit significand and bi = biased
// exponent + 10; window J holds bits [32J, 32J + 64) (lo bin: [32J, 32J+32),
// hi bin: [32J+32, 32J+64)); x contributes its truncation (toward zero) at
// the window's bottom, slice by slice, sign applied.  The window only moves
// up (to fit the largest |x| seen: J = (e + 1) >> 5), dropping the lo bin;
// slices never carry between bins, so the total is
//   sum over deposits of trunc(x at the FINAL window),
// the final window being that of the column's largest |x|: independent of
// the deposit order and of how deposits are split across threads and CTAs.
// One window per column (a column's precision never depends on another's).
// Inf / NaN deposits go to an fp32 side sum (any mix of +-inf / NaN sums to
// the same value in any order).  Precision: >= 32 bits below the largest
// deposit per deposit (fp32 tile partials carry 24).
#define AS_BIN_EMPTY (-1000)
template <int NE>
__device__ __forceinline__ void bins_add(int* J, long long* hi, long long* lo, float* sp, const float* x) {
#pragma unroll
  for (int k = 0; k < NE; ++k) {
    const u32 u = __float_as_uint(x[k]);
    const u32 a = u & 0x7fffffffu;
    if (a >= 0x7f800000u) { sp[k] += x[k]; continue; }  // inf / nan (rare)
    const u32 e = a >> 23;
    // window of this column: J = (e + 1) >> 5 fits |x| (top bit <= 32J + 63);
    // moving up drops the lo bin (one step) or both (more)
    const int need = a ? (int)(max(e, 1u) + 1u) >> 5 : AS_BIN_EMPTY;
    if (need > J[k]) {
      lo[k] = need == J[k] + 1 ? hi[k] : 0;
      hi[k] = 0;
      J[k] = need;
    }
    const u32 m = (u & 0x7fffffu) | (e ? 0x800000u : 0u);
    const int d = min((int)(e ? e : 1u) + 10 - 32 * J[k], 40);  // bit offset of m in the window (<= 40)
    const u64 v = d >= 0 ? ((u64)m << d) : (d > -24 ? (u64)(m >> (-d)) : 0ull);
    const long long vl = (long long)(v & 0xffffffffull), vh = (long long)(v >> 32);
    if (u >> 31) { lo[k] -= vl; hi[k] -= vh; } else { lo[k] += vl; hi[k] += vh; }
  }
}
// merge accumulator (J2, hi2, lo2, sp2) into (J, hi, lo, sp): align both to
// the higher window (dropping whole bins), then add exactly
__device__ __forceinline__ void bins_merge(int& J, long long& hi, long long& lo, float& sp, int J2, long long hi2,
                                           long long lo2, float sp2) {
  sp += sp2;
  if (J2 > J) {
    if (J2 == J + 1) { lo = hi; hi = 0; } else { lo = 0; hi = 0; }
    J = J2;
  }
  if (J2 == J) { hi += hi2; lo += lo2; }
  else if (J2 == J - 1) { lo += hi2; }
}
// the accumulator's value: one fp64 rounding of the exact total, then fp32
__device__ __forceinline__ double bins_value_d(int J, long long hi, long long lo, float sp) {
  if (sp != 0.f) return (double)sp;  // +-inf or NaN deposits decide (finite parts cannot change them)
  if (J == AS_BIN_EMPTY) return 0.0;
  return ldexp((double)hi, 32 * (J + 1) - 160) + ldexp((double)lo, 32 * J - 160);
}
// one accumulator in the workspace (J, sp, hi, lo; slots are 48 bytes apart)
struct BinSlot { int J; float sp; long long hi, lo, pad; };

// Precise variant for fp64 tile partials (column sums whose mean is later
// subtracted, reading R7c): four 16-bit-aligned int64 bins b[0..3] of a
// 64-bit window on the absolute scale 2^-1100 (|x| = m * 2^(bi - 1100),
// bi = biased fp64 exponent + 25); window J holds bits [16J, 16J + 64), so
// the largest deposit keeps >= 48 bits (fp32 bins: >= 32).  Same exactness /
// order independence as the fp32 bins.
struct BinSlotP { int J; float sp; long long b[4]; long long pad; };
__device__ __forceinline__ void binsp_shift(int& J, long long* b, int need) {
  const int t = need - J;
#pragma unroll
  for (int k = 0; k < 4; ++k) b[k] = (k + t < 4) ? b[(k + t) & 3] : 0;
  J = need;
}
template <int NE>
__device__ __forceinline__ void bins_add_p(int* J, long long* b, float* sp, const double* x) {
#pragma unroll
  for (int k = 0; k < NE; ++k) {
    const u64 u = static_cast<u64>(__double_as_longlong(x[k]));
    const u32 e = static_cast<u32>(u >> 52) & 0x7ffu;
    if (e == 0x7ffu) { sp[k] += static_cast<float>(x[k]); continue; }
    const u64 mn = u & 0xfffffffffffffull;
    if (!(mn | e)) continue;
    const int bi = (int)(e ? e : 1u) + 25;
    const int need = (bi + 4) >> 4;
    long long* bk = b + 4 * k;
    if (need > J[k]) {
      if (J[k] == AS_BIN_EMPTY || need - J[k] >= 4) { bk[0] = bk[1] = bk[2] = bk[3] = 0; J[k] = need; }
      else binsp_shift(J[k], bk, need);
    }
    const u64 m = mn | (e ? (1ull << 52) : 0ull);
    const int d = min(bi - 16 * J[k], 11);
    const u64 v = d >= 0 ? (m << d) : (d > -53 ? (m >> (-d)) : 0ull);
    const bool neg = (u >> 63) != 0ull;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const long long sl = static_cast<long long>((v >> (16 * q)) & 0xffffull);
      bk[q] += neg ? -sl : sl;
    }
  }
}
__device__ __forceinline__ void bins_merge_p(int& J, long long* b, float& sp, int J2, const long long* b2, float sp2) {
  sp += sp2;
  if (J2 == AS_BIN_EMPTY) return;
  if (J == AS_BIN_EMPTY || J2 - J >= 4) {
    if (J2 > J) { b[0] = b[1] = b[2] = b[3] = 0; J = J2; }
  } else if (J2 > J) {
    binsp_shift(J, b, J2);
  }
  const int t = J - J2;  // >= 0: drop b2's lowest t bins
#pragma unroll
  for (int k = 0; k < 4; ++k)
    if (k + t < 4) b[k] += b2[(k + t) & 3];
}
__device__ __forceinline__ double bins_value_p(int J, const long long* b, float sp) {
  if (sp != 0.f) return (double)sp;
  if (J == AS_BIN_EMPTY) return 0.0;
  double v = 0.0;
#pragma unroll
  for (int k = 3; k >= 0; --k) v += ldexp((double)b[k], 16 * (J + k) - 1100);
  return v;
}
__device__ __forceinline__ BinSlotP ld_cg_binsp(const BinSlotP* p) {
  const Raw<16> a = ldg_cg(reinterpret_cast<const Raw<16>*>(p));
  const Raw<16> c = ldg_cg(reinterpret_cast<const Raw<16>*>(p) + 1);
  const Raw<8> d = ldg_cg(reinterpret_cast<const Raw<8>*>(p) + 4);
  BinSlotP s;
  s.J = static_cast<int>(a.x);
  s.sp = __uint_as_float(a.y);
  s.b[0] = static_cast<long long>((static_cast<u64>(a.w) << 32) | a.z);
  s.b[1] = static_cast<long long>((static_cast<u64>(c.y) << 32) | c.x);
  s.b[2] = static_cast<long long>((static_cast<u64>(c.w) << 32) | c.z);
  s.b[3] = static_cast<long long>((static_cast<u64>(d.y) << 32) | d.x);
  s.pad = 0;
  return s;
}
// L2-coherent load of a slot written by another CTA earlier in the kernel
__device__ __forceinline__ BinSlot ld_cg_bins(const BinSlot* p) {
  const Raw<16> a = ldg_cg(reinterpret_cast<const Raw<16>*>(p));
  const Raw<8> b = ldg_cg(reinterpret_cast<const Raw<8>*>(p) + 2);
  BinSlot s;
  s.J = static_cast<int>(a.x);
  s.sp = __uint_as_float(a.y);
  s.hi = static_cast<long long>((static_cast<u64>(a.w) << 32) | a.z);
  s.lo = static_cast<long long>((static_cast<u64>(b.y) << 32) | b.x);
  s.pad = 0;
  return s;
}

// ------------------------------------------------------------------ packed: TMA bulk + mbarrier
__device__ __forceinline__ u32 smem_addr(const void* p) {
  return static_cast<u32>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(u32 bar, u32 count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(u32 bar, u32 bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(u32 bar, u32 parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(bar), "r"(parity)
      : "memory");
}
// global -> shared bulk copy completing on an mbarrier (UBLKCP)
__device__ __forceinline__ void bulk_g2s(u32 dst, const void* src, u32 bytes, u32 bar) {
  asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}
// shared -> global bulk copy (bulk-group completion)
__device__ __forceinline__ void bulk_s2g(void* dst, u32 src, u32 bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(src), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N> __device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

}  // namespace as

// ------------------------------------------------------------------ measurement kernels
// Only compiled into the measurement module (and the AOT build check), not
// into the generated stitched kernels.
#if defined(ASTITCH_BENCH_KERNELS) || !defined(ASTITCH_JIT)
// Barrier-only kernel (Table 6 micro-benchmark on B200).
extern "C" __global__ void astitch_barrier_bench(u32* bar, int iters) {
  for (int i = 0; i < iters; ++i) as::grid_barrier(bar);
}
// Copy ceiling with the same streaming 16-byte accesses as the stitched kernels.
extern "C" __global__ void __launch_bounds__(256) astitch_copy_bench(const as::Raw<16>* __restrict__ src,
                                                                     as::Raw<16>* __restrict__ dst,
                                                                     long long n16) {
  long long i = blockIdx.x * 256LL + threadIdx.x;
  const long long stride = gridDim.x * 256LL;
  for (; i + 3 * stride < n16; i += 4 * stride) {
    as::Raw<16> a = as::ldg(src + i), b = as::ldg(src + i + stride), c = as::ldg(src + i + 2 * stride),
                d = as::ldg(src + i + 3 * stride);
    as::stg(dst + i, a); as::stg(dst + i + stride, b); as::stg(dst + i + 2 * stride, c);
    as::stg(dst + i + 3 * stride, d);
  }
  for (; i < n16; i += stride) as::stg(dst + i, as::ldg(src + i));
}
#endif  // ASTITCH_BENCH_KERNELS
