// tcgen05 MMA issue-rate microbenchmark on CTA pairs (cta_group::2): back-to-back
// 256 x N x K MMAs on fixed shared-memory operands (values irrelevant), every SM busy.
// Variants: kind::mxf8f6f4.block_scale (the prefill GEMM's), kind::f8f6f4, kind::f16.
#include <cstdio>
#include <cuda.h>
#include <cuda_runtime.h>
#include "../../paper_conf_sosp_chenxztwdcylqzo25_b200/csrc/sm100.cuh"
using namespace moe::sm100;

__device__ __forceinline__ void mma_f8_pair(uint32_t d, uint64_t a, uint64_t b, uint32_t id, uint32_t acc) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
               "tcgen05.mma.cta_group::2.kind::f8f6f4 [%0], %1, %2, %3, p;\n\t}" ::"r"(d), "l"(a), "l"(b), "r"(id), "r"(acc)
               : "memory");
}
__host__ __device__ constexpr uint32_t idesc_f8(int M, int N) {
  return (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

template <int KIND, int N, int CP>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1) mma_loop(int iters, unsigned long long *out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t *s = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(sm) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar, bar2[6];
  __shared__ uint32_t tbase;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t crank = cluster_rank();
  if (threadIdx.x == 0) { mbar_init(&bar, 1); for (int i = 0; i < 6; ++i) mbar_init(&bar2[i], 1); fence_barrier_init(); }
  if (warp == 0) tmem_alloc_pair(&tbase, 512);
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  const uint32_t tmem = tbase;
  unsigned long long t0 = 0, t1 = 0;
  if (crank == 0 && warp == 1 && lane == 0) {
    const uint32_t a0 = smem_u32(s), b0 = smem_u32(s + 16384);
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    uint32_t ph = 0;
    for (int it = 0; it < iters; ++it) {
      if (CP && (it & 3) == 0) {       // scale images: 3 x tcgen05.cp per 4 k-blocks (the GEMM's cadence)
        const uint32_t set = ((it >> 2) & 1) * 16;
        tmem_cp_32x128b_x4_pair(tmem + 256 + set, sf_desc(smem_u32(s + 49152)));
        tmem_cp_32x128b_x4_pair(tmem + 264 + set, sf_desc(smem_u32(s + 49152 + 512)));
        tmem_cp_32x128b_x4_pair(tmem + 268 + set, sf_desc(smem_u32(s + 49152 + 1024)));
      }
      if (CP == 2) mma_commit_pair(&bar2[it % 6]);   // per-k-block commit to a 6-deep ring (the GEMM's empty barriers)
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const uint64_t ad = sw128_kmajor_desc(a0 + k * 32), bd = sw128_kmajor_desc(b0 + k * 32);
        if (KIND == 0) mma_mxf8_pair(tmem, ad, bd, idesc_mxf8(256, N, it & 3, it & 3), 1, tmem + 256 + ((it >> 2) & 1) * 16, tmem + 264 + ((it >> 2) & 1) * 16);
        else if (KIND == 1) mma_f8_pair(tmem, ad, bd, idesc_f8(256, N), 1);
        else mma_bf16_pair(tmem, ad, bd, idesc_bf16(256, N), 1);
      }
      if ((it & 7) == 7) {            // bounded run-ahead: wait for the MMAs of 8 iterations ago
        mma_commit_pair(&bar);
        mbar_wait(&bar, ph);
        ph ^= 1;
      }
    }
    mma_commit_pair(&bar);
    mbar_wait(&bar, ph);
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
    out[blockIdx.x] = t1 - t0;
  }
  tc_fence_before();
  cluster_sync();
  if (warp == 0) tmem_dealloc_pair(tmem, 512);
}

template <int KIND, int N, int CP = 0>
void run(const char *name, int sms) {
  const int iters = 20000, grid = sms & ~1;
  unsigned long long *out; cudaMalloc(&out, grid * 8); cudaMemset(out, 0, grid * 8);
  auto k = mma_loop<KIND, N, CP>;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  k<<<grid, 128, 64 * 1024>>>(100, out);
  cudaEventRecord(e0);
  k<<<grid, 128, 64 * 1024>>>(iters, out);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  const double kdim = KIND == 2 ? 16 : 32;
  const double flops = 2.0 * 256 * N * kdim * 4 * iters * (grid / 2);
  printf("%-28s CP=%d N=%3d: %.1f TFLOP/s (%.3f ms)  %s\n", name, CP, N, flops / (ms * 1e-3) / 1e12, ms,
         cudaGetErrorString(cudaGetLastError()));
  cudaFree(out);
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int rep = 0; rep < 2; ++rep) {
    run<0, 256>("mxf8f6f4.block_scale", sms);
    run<0, 256, 1>("mxf8f6f4.block_scale", sms);
    run<0, 256, 2>("mxf8f6f4.block_scale", sms);
    run<0, 176, 2>("mxf8f6f4.block_scale", sms);
    run<0, 128, 2>("mxf8f6f4.block_scale", sms);
    run<0, 64, 2>("mxf8f6f4.block_scale", sms);
    run<0, 16, 2>("mxf8f6f4.block_scale", sms);
  }
  return 0;
}
