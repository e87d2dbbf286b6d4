// Grid-barrier cost on B200 (the paper's Table 6 /
// P:L432-L442): the library's generation-counted barrier (as::grid_barrier,
// kernels/astitch_device.cuh) vs CUDA cooperative groups' grid.sync(), both in
// cooperative launches of `blocks` x `threads`; per-barrier time from kernels
// with 1 and 101 barriers (CUDA events, best of 20).
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -I ../../paper_conf_asplos_zhengyzlzzzlyzs22_b200/csrc/kernels \
//        barrier_compare.cu -o barrier_compare
#include <cooperative_groups.h>
#include <cstdio>
#include "astitch_device.cuh"

namespace cg = cooperative_groups;

__global__ void gen_barrier(unsigned int* bar, int iters) {
  for (int i = 0; i < iters; ++i) as::grid_barrier(bar);
}
// the same one-word barrier with a nanosleep backoff in the poll loop
__device__ __forceinline__ void grid_barrier_backoff(unsigned int* bar, unsigned ns) {
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned nb = gridDim.x;
    const unsigned add = blockIdx.x == 0 ? (0x80000000u - (nb - 1u)) : 1u;
    __threadfence();
    const unsigned old = atomicAdd(bar, add);
    while (((old ^ as::ld_volatile_u32(bar)) & 0x80000000u) == 0u) __nanosleep(ns);
    __threadfence();
  }
  __syncthreads();
}
__global__ void backoff_barrier(unsigned int* bar, int iters, unsigned ns) {
  for (int i = 0; i < iters; ++i) {
    if (ns == 0) {  // variant: release atomic, relaxed polls, one acq_rel fence after the wait
      __syncthreads();
      if (threadIdx.x == 0) {
        const unsigned nb = gridDim.x;
        const unsigned add = blockIdx.x == 0 ? (0x80000000u - (nb - 1u)) : 1u;
        unsigned old;
        asm volatile("atom.add.release.gpu.global.u32 %0, [%1], %2;" : "=r"(old) : "l"(bar), "r"(add) : "memory");
        while (((old ^ as::ld_volatile_u32(bar)) & 0x80000000u) == 0u) { }
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
      }
      __syncthreads();
    } else {
      grid_barrier_backoff(bar, ns);
    }
  }
}
__global__ void cg_barrier(int iters) {
  cg::grid_group g = cg::this_grid();
  for (int i = 0; i < iters; ++i) g.sync();
}

template <typename L>
float best_ms(L launch) {
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  for (int i = 0; i < 3; ++i) launch();
  cudaDeviceSynchronize();
  float best = 1e30f;
  for (int r = 0; r < 20; ++r) {
    cudaEventRecord(a); launch(); cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); best = ms < best ? ms : best;
  }
  return best;
}

int main() {
  unsigned int* bar;
  cudaMalloc(&bar, 256);
  cudaMemset(bar, 0, 256);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  printf("{\"what\": \"grid barrier: generation-counted (astitch) vs cooperative-groups grid.sync\", \"sms\": %d, \"rows\": [\n", sms);
  const int cfgs[][2] = {{20, 1024}, {80, 1024}, {148, 1024}, {148, 512}, {296, 512}, {296, 256}, {592, 256}, {1184, 256}};
  bool first = true;
  for (auto& c : cfgs) {
    const int blocks = c[0], threads = c[1];
    auto run_gen = [&](int it) {
      void* args[] = {&bar, &it};
      cudaLaunchCooperativeKernel((void*)gen_barrier, blocks, threads, args, 0, 0);
    };
    auto run_cg = [&](int it) {
      void* args[] = {&it};
      cudaLaunchCooperativeKernel((void*)cg_barrier, blocks, threads, args, 0, 0);
    };
    const float g1 = best_ms([&] { run_gen(1); }), g101 = best_ms([&] { run_gen(101); });
    const float c1 = best_ms([&] { run_cg(1); }), c101 = best_ms([&] { run_cg(101); });
    float bo[3];
    const unsigned nss[3] = {0, 20, 100};
    for (int q = 0; q < 3; ++q) {
      unsigned ns = nss[q];
      auto run_bo = [&](int it) {
        void* args[] = {&bar, &it, &ns};
        cudaLaunchCooperativeKernel((void*)backoff_barrier, blocks, threads, args, 0, 0);
      };
      bo[q] = (best_ms([&] { run_bo(101); }) - best_ms([&] { run_bo(1); })) * 10.0f;
    }
    cudaError_t e = cudaGetLastError();
    printf("%s {\"blocks\": %d, \"threads\": %d, \"astitch_us_per_barrier\": %.3f, \"cg_us_per_barrier\": %.3f, "
           "\"astitch_kernel_1_barrier_us\": %.3f, \"cg_kernel_1_barrier_us\": %.3f, \"release_atom_and_backoff_20_100ns_us\": [%.3f, %.3f, %.3f], \"status\": \"%s\"}\n",
           first ? "" : ",", blocks, threads, (g101 - g1) * 10.0f, (c101 - c1) * 10.0f, g1 * 1e3f, c1 * 1e3f,
           bo[0], bo[1], bo[2], cudaGetErrorString(e));
    first = false;
  }
  printf("]}\n");
  return 0;
}
