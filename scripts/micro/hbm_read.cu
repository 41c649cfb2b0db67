// HBM read microbenchmark: every CTA streams a contiguous slice of a buffer
// into a shared-memory ring with cp.async.bulk (one thread issues, the ring
// slot is recycled as soon as its bytes land).  Sweeps ring depth x chunk size.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void stream_kernel(const uint8_t *src, size_t per_cta, int chunk, int stages, unsigned long long *sink) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar[32];
  if (threadIdx.x != 0) return;
  for (int s = 0; s < stages; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su(&bar[s])));
  asm volatile("fence.mbarrier_init.release.cluster;");
  const uint8_t *base = src + (size_t)blockIdx.x * per_cta;
  const int n = (int)(per_cta / chunk);
  uint32_t ph[32] = {0};
  unsigned long long acc = 0;
  for (int i = 0; i < n + stages; ++i) {
    const int s = i % stages;
    if (i >= stages) {   // wait for chunk i - stages
      asm volatile("{\n.reg .pred P;\nW: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n@!P bra W;\n}" ::"r"(su(&bar[s])), "r"(ph[s]));
      ph[s] ^= 1;
      acc += sm[s * chunk];
    }
    if (i < n) {
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su(&bar[s])), "r"(chunk));
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(su(sm + (size_t)s * chunk)),
                   "l"(base + (size_t)i * chunk), "r"(chunk), "r"(su(&bar[s])) : "memory");
    }
  }
  if (acc == 12345) *sink = acc;
}

int main() {
  const size_t total = (size_t)400 << 20;
  uint8_t *buf; cudaMalloc(&buf, total + (64 << 20));
  cudaMemset(buf, 1, total);
  uint8_t *fl; cudaMalloc(&fl, 512 << 20);
  unsigned long long *sink; cudaMalloc(&sink, 8);
  cudaFuncSetAttribute(stream_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int chunks[] = {16384, 32768, 65536};
  const int stages_[] = {2, 4, 6, 8, 12};
  const int ctas_per_sm[] = {1, 2};
  for (int cps : ctas_per_sm)
  for (int chunk : chunks)
    for (int st : stages_) {
      const size_t smem = (size_t)chunk * st;
      if (smem * cps > 200 * 1024) continue;
      const int grid = sms * cps;
      size_t per = total / grid / chunk * chunk;
      float best = 1e9;
      for (int it = 0; it < 5; ++it) {
        cudaEventRecord(e0);
        stream_kernel<<<grid, 32, smem>>>(buf, per, chunk, st, sink);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
      }
      printf("ctas/SM %d chunk %6d stages %2d inflight/SM %4zu KB : %.3f TB/s (%.1f us)\n", cps, chunk, st,
             smem * cps / 1024, per * grid / (best * 1e-3) / 1e12, best * 1e3);
    }
  cudaError_t e = cudaGetLastError();
  printf("status %s\n", cudaGetErrorString(e));
  return 0;
}
