// Latency of the decode router selection (one warp, one token), passes 1..3.
#define SELECT_PROFILE
#include "../../paper_conf_sosp_chenxztwdcylqzo25_b200/csrc/router.cu"
#include <cstdio>
using namespace moe;
__global__ void bench(RouterArgs r, long long *out, int passes) {
  __shared__ float scratch[512];
  __shared__ int ids[64];
  const int lane = threadIdx.x & 31;
  for (int p = 0; p < passes; ++p) {
    __syncwarp();
    long long t0 = clock64();
    select_token_regs(r, 0, scratch, ids, lane, true);
    __syncwarp();
    long long t1 = clock64();
    if (lane == 0) out[p] = t1 - t0;
  }
}
int main() {
  const int E = 256, k = 8;
  float h[E], b[E];
  for (int i = 0; i < E; ++i) { h[i] = sinf(i * 1.7f) * 2.f; b[i] = cosf(i * 0.3f) * 0.05f; }
  float *lg, *bias, *tw, *sg; int *ti; long long *out;
  cudaMalloc(&lg, E * 4); cudaMalloc(&bias, E * 4); cudaMalloc(&tw, 64 * 4); cudaMalloc(&ti, 64 * 4); cudaMalloc(&sg, 64);
  cudaMalloc(&out, 64);
  cudaMemcpy(lg, h, E * 4, cudaMemcpyHostToDevice); cudaMemcpy(bias, b, E * 4, cudaMemcpyHostToDevice);
  RouterArgs r{};
  r.logits = lg; r.ldl = E; r.bias = bias; r.T = 1; r.E = E; r.k = k; r.n_group = 8; r.topk_group = 4;
  r.group_score = MOE_GROUP_TOP2_SUM; r.score_fn = MOE_SCORE_SIGMOID; r.norm_topk = 1; r.routed_scale = 2.5f;
  r.topk_idx = ti; r.topk_w = tw; r.sgate = sg;
  for (int rep = 0; rep < 3; ++rep) {
    bench<<<1, 32>>>(r, out, 4);
    long long o[4]; cudaMemcpy(o, out, 32, cudaMemcpyDeviceToHost);
    printf("launch %d: passes %lld %lld %lld %lld cycles\n", rep, o[0], o[1], o[2], o[3]);
    long long c[8]; cudaMemcpyFromSymbol(c, g_sel_ck, 64);
    printf("  phases (last pass): loads+scores %lld group %lld localsort %lld butterfly %lld weights %lld\n", c[1]-c[0], c[2]-c[1], c[3]-c[2], c[4]-c[3], c[5]-c[4]);
  }
  int idx[8]; cudaMemcpy(idx, ti, 32, cudaMemcpyDeviceToHost);
  printf("ids %d %d %d %d %d %d %d %d  err %s\n", idx[0], idx[1], idx[2], idx[3], idx[4], idx[5], idx[6], idx[7],
         cudaGetErrorString(cudaGetLastError()));
}
