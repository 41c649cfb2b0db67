// common.cuh -- shared device helpers and the layer's internal state.
// Nothing here is shared with oracle/ (the CPU checker); see DESIGN.md §2.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <cuda_fp8.h>
#include <stdint.h>

#include "../../include/moe.h"

namespace moe {

constexpr int kPadM = 128;       // expert segments of the sorted order are padded to this
constexpr int kChunkTokens = 256; // token chunk of the deterministic permutation

// ---------------------------------------------------------------- conversions
__device__ __forceinline__ float bf2f(__nv_bfloat16 v) { return __bfloat162float(v); }

__device__ __forceinline__ void bf16x8_to_f32(const uint4 &u, float *f) {
  const __nv_bfloat162 *p = reinterpret_cast<const __nv_bfloat162 *>(&u);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    float2 t = __bfloat1622float2(p[i]);
    f[2 * i] = t.x;
    f[2 * i + 1] = t.y;
  }
}

__device__ __forceinline__ void fp8x8_to_f32(const uint2 &u, float *f) {
  const __nv_fp8x2_storage_t *p = reinterpret_cast<const __nv_fp8x2_storage_t *>(&u);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    __half2_raw h = __nv_cvt_fp8x2_to_halfraw2(p[i], __NV_E4M3);
    float2 t = __half22float2(*reinterpret_cast<__half2 *>(&h));
    f[2 * i] = t.x;
    f[2 * i + 1] = t.y;
  }
}

// UE8M0 ceil scale (reading R10): s = 2^ceil(log2(fl32(amax/448))),
// ceil taken from the fp32 bits of the IEEE quotient; s = 1 when amax == 0.
// Returns the unbiased exponent e (s = 2^e).
__device__ __forceinline__ int ue8m0_exponent(float amax) {
  if (!(amax > 0.f)) return 0;
  float q = __fdiv_rn(amax, 448.f);
  uint32_t b = __float_as_uint(q);
  int e = int((b >> 23) & 0xFF) - 127 + ((b & 0x7FFFFF) != 0 ? 1 : 0);
  return e;
}
__device__ __forceinline__ float exp2i(int e) { return __uint_as_float(uint32_t(e + 127) << 23); }

__device__ __forceinline__ uint8_t f32_to_e4m3(float v) {
  return (uint8_t)__nv_cvt_float_to_fp8(v, __NV_SATFINITE, __NV_E4M3);
}

// byte offset of the UE8M0 scale of (row, 128-col block kb) in a scale image:
// per group of 4 k-blocks and 128-row tile, 512 B laid out as the
// tcgen05.cp 32x128b.warpx4 source -- datapath l holds rows l, l+32, l+64,
// l+96 (one 32-bit word each, one byte per k-block of the group).
__device__ __forceinline__ size_t sf_img_off(int64_t row, int kb, int tile_stride) {
  const int64_t tile = row >> 7;
  const int r = (int)(row & 127);
  const int word = (r & 31) * 4 + (r >> 5);
  return ((size_t)((kb >> 2) * (int64_t)tile_stride + tile) * 128 + word) * 4 + (kb & 3);
}

__device__ __forceinline__ float silu_f(float g) { return __fdividef(g, 1.f + __expf(-g)); }

// PDL: wait for the stream predecessor's results / let the successor launch
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// Destinations of one token's activation row in the expert-sorted order.
struct ScatterDst {
  int fp8;
  void *xperm; uint8_t *xperm_img; int xperm_img_stride; float *xperm_s;   // sorted rows (+ scales)
  void *xq; float *xs; uint8_t *xq_img; int xq_img_stride;                // token-order copy (shared expert)
};

// The whole CTA (NT threads) moves token t's row: thread = 8-element chunks
// c = tid + NT i with every load issued up front (H <= 8192); FP8 quantises
// each 1x128 block once (UE8M0 ceil scale of the amax over 16 consecutive
// threads, e4m3 RNE satfinite; R10) and stores the codes to each of
// the token's sorted rows pos[0..k) (< 0 = not local) and to xq; bf16 copies.
template <int NT>
__device__ __forceinline__ void scatter_token_row(const __nv_bfloat16 *__restrict__ xrow, int H, int64_t t, int k,
                                                  const int *pos, const ScatterDst &d) {
  constexpr int MAXI = 8192 / 8 / NT;
  const int th = threadIdx.x, lane = th & 31;
  const int nc = H / 8;
  __shared__ uint8_t exs[8192 / 128];               // FP8: the row's UE8M0 bytes, stored as words below
  uint4 raw[MAXI];
#pragma unroll
  for (int i = 0; i < MAXI; ++i) {
    const int c = th + NT * i;
    if (c < nc) raw[i] = __ldg(reinterpret_cast<const uint4 *>(xrow) + c);
  }
#pragma unroll
  for (int i = 0; i < MAXI; ++i) {
    const int c = th + NT * i;
    if (i * NT >= nc) break;                       // warp-uniform (nc % 32 == 0)
    if (d.fp8) {
      float f[8];
      bf16x8_to_f32(raw[i], f);
      float am = 0.f;
#pragma unroll
      for (int j = 0; j < 8; ++j) am = fmaxf(am, fabsf(f[j]));
#pragma unroll
      for (int o = 8; o > 0; o >>= 1) am = fmaxf(am, __shfl_xor_sync(0xffffffffu, am, o));
      if (c >= nc) continue;
      const int ex = ue8m0_exponent(am);
      const float inv = exp2i(-ex);
      uint2 q;
      q.x = (uint32_t)f32_to_e4m3(f[0] * inv) | ((uint32_t)f32_to_e4m3(f[1] * inv) << 8) |
            ((uint32_t)f32_to_e4m3(f[2] * inv) << 16) | ((uint32_t)f32_to_e4m3(f[3] * inv) << 24);
      q.y = (uint32_t)f32_to_e4m3(f[4] * inv) | ((uint32_t)f32_to_e4m3(f[5] * inv) << 8) |
            ((uint32_t)f32_to_e4m3(f[6] * inv) << 16) | ((uint32_t)f32_to_e4m3(f[7] * inv) << 24);
      const int b = c >> 4;                        // 128-element block
      const bool head = (lane & 15) == 0;
      if (head) exs[b] = (uint8_t)(ex + 127);
      if (d.xq) {
        *reinterpret_cast<uint2 *>(reinterpret_cast<uint8_t *>(d.xq) + t * H + c * 8) = q;
        if (head && d.xs) d.xs[t * (H / 128) + b] = exp2i(ex);
      }
#pragma unroll 1
      for (int j = 0; j < k; ++j) {
        const int rw = pos[j];
        if (rw < 0) continue;
        *reinterpret_cast<uint2 *>(reinterpret_cast<uint8_t *>(d.xperm) + (int64_t)rw * H + c * 8) = q;
        if (head && d.xperm_s) d.xperm_s[(int64_t)rw * (H / 128) + b] = exp2i(ex);
      }
    } else if (c < nc) {
#pragma unroll 1
      for (int j = 0; j < k; ++j) {
        const int rw = pos[j];
        if (rw < 0) continue;
        reinterpret_cast<uint4 *>(reinterpret_cast<__nv_bfloat16 *>(d.xperm) + (int64_t)rw * H)[c] = raw[i];
      }
    }
  }
  if (d.fp8 && (d.xq_img || d.xperm_img)) {
    // scale images: the 4 UE8M0 bytes of k-blocks 4g .. 4g+3 of a row are one
    // 32-bit word of the image (sf_img_off), so each destination row gets H/512
    // word stores instead of H/128 scattered byte stores
    __syncthreads();
    const int nb = H / 128, ng = (nb + 3) / 4;
    for (int idx = th; idx < ng * (k + 1); idx += NT) {
      const int g = idx % ng, dst = idx / ng;      // dst 0: xq (row t), 1..k: the sorted rows
      uint32_t w = 0;
#pragma unroll
      for (int j = 0; j < 4; ++j) w |= (4 * g + j < nb ? (uint32_t)exs[4 * g + j] : 0u) << (8 * j);
      const int64_t row = dst == 0 ? t : (int64_t)pos[dst - 1];
      uint8_t *img = dst == 0 ? d.xq_img : d.xperm_img;
      const int stride = dst == 0 ? d.xq_img_stride : d.xperm_img_stride;
      if (row < 0 || !img || (dst == 0 && !d.xq)) continue;
      *reinterpret_cast<uint32_t *>(img + sf_img_off(row, 4 * g, stride)) = w;
    }
    __syncthreads();                             // exs is reused by the caller's next token
  }
}

}  // namespace moe

// ------------------------------------------------------------------ layer state
struct moe_layer {
  moe_layer_config cfg;
  int E;        // local experts (E / ep_size)
  int E_glob;   // global experts
  int e0;       // first global expert owned by this rank
  int k, H, F, Fs;
  bool fp8, f32w;
  bool fp4 = false;   // 4-bit (e2m1) expert weights: decode streams the packed codes
  bool scale_nonpow2 = false;   // some FP8 block scale is not a power of two (decode-only layer)
  char nonpow2_what[96] = {};
  int act_bytes;  // bytes per activation element fed to the expert GEMMs (1 fp8, 2 bf16)
  int max_tokens;
  int gemv_max_tokens;
  int64_t R_max;  // padded sorted rows capacity

  // ---- weights (library-owned, repacked) ----
  void *gate_w = nullptr;      // [E_glob (+1 shared gate row), H] bf16
  float *gate_bias = nullptr;  // [E_glob] or null
  int gate_rows = 0;
  void *w13 = nullptr;         // [E, 2F, H]  rows interleaved per 128: (W1 blk b, W3 blk b);
                               // tcgen05 path: as 256-row x 128-byte SW128 tiles
  float *w13_s = nullptr;      // [E, 2F/128, H/128]  (same interleave)
  void *w2 = nullptr;          // [E, H, F]
  float *w2_s = nullptr;       // [E, H/128, F/128]
  void *ws13 = nullptr;        // [2Fs, H] interleaved
  float *ws13_s = nullptr;
  void *ws2 = nullptr;         // [H, Fs]
  float *ws2_s = nullptr;
  int64_t weight_bytes = 0;

  // ---- workspace ----
  float *logits = nullptr;      // [maxT, gate_rows]
  int32_t *topk_idx = nullptr;  // [maxT, k]  (global expert ids, canonical order)
  float *topk_w = nullptr;      // [maxT, k]
  float *sgate = nullptr;       // [maxT]  sigmoid(x . w_sg) (Qwen2)
  int32_t *chunk_cnt = nullptr; // [nchunk, E]
  int32_t *chunk_base = nullptr;// [nchunk, E]
  int32_t *counts = nullptr;    // [E]
  int32_t *offs = nullptr;      // [E+1] unpadded
  int32_t *offs_pad = nullptr;  // [E+1] padded to kPadM
  int4 *tiles = nullptr;        // [max_tiles] (expert, row0, row_end, 0)
  int32_t *n_tiles = nullptr;   // [1]
  int32_t *act_list = nullptr;  // [E] active experts (count > 0, any slot), ascending
  int32_t *n_active = nullptr;  // [1]
  int32_t *sched = nullptr;     // [8] work counters of the persistent GEMM launches
  int32_t *row_token = nullptr; // [R_max] token of each padded row (-1 = pad)
  int32_t *pos = nullptr;       // [maxT*k] padded row of (t, j) (local experts only; -1 = remote)
  void *xq = nullptr;           // [maxT, H] e4m3 (FP8 only)
  float *xs = nullptr;          // [maxT, H/128]
  void *xperm = nullptr;        // [R_max, H] act dtype
  float *xperm_s = nullptr;     // [R_max, H/128]
  void *hbuf = nullptr;         // [R_max, F] act dtype
  float *h_s = nullptr;         // [R_max, F/128]
  __nv_bfloat16 *yperm = nullptr; // [R_max, H]
  void *hsh = nullptr;          // [maxT, Fs]
  float *hsh_s = nullptr;       // [maxT, Fs/128]
  __nv_bfloat16 *ysh = nullptr; // [maxT, H]
  // ---- tcgen05 path ----
  bool umma = false;
  uint8_t *w13_img = nullptr, *w2_img = nullptr, *ws13_img = nullptr, *ws2_img = nullptr;  // weight scale images
  uint8_t *xperm_img = nullptr, *h_img = nullptr, *xq_img = nullptr, *hsh_img = nullptr;   // activation images
  int img_tiles_sh = 0;         // ceil(maxT / 128)
  int64_t w13_img_stride = 0, w2_img_stride = 0;
  CUtensorMap map_xperm, map_h, map_xq, map_hsh, map_gate;   // activation rows (box 128), router rows
  CUtensorMap dmap_xperm, dmap_h, dmap_xq, dmap_hsh;           // decode: activation rows (box 16)
  float *dacc = nullptr;        // fused decode: [2][gemv_max_tokens, H] fp32 sums (immediate, deferred), kept zero
  int32_t *zero_i32 = nullptr; // [0] a device 0 (an empty routed list), [1..2] the EP shared launch's work counter
  bool fused_decode = false;
  // chained Expert Deferral (moe_layer_forward_chained): expert lists of the
  // immediate / deferred canonical slots, and what the last chained call left
  int32_t *imm_list = nullptr, *def_list = nullptr;   // [E] ascending local ids
  int32_t *n_lists = nullptr;                          // [2] lengths (immediate, deferred)
  int chain_T = -1, chain_ndef = 0;
  void *xcopy = nullptr;        // BF16 decode: [gemv_max_tokens, H] copy of x (the stream's operand)
  CUtensorMap dmap_xc;          // its tensor map (box 16 rows)
  // tensor parallelism within every expert (config tp_rank / tp_size): this rank's
  // 128-column chunks [c0, c0 + F/128) of the full ffn (F, Fs are the slice sizes)
  int tp_rank = 0, tp_size = 1;
  int F_full = 0, Fs_full = 0;
  void *tp_comm = nullptr;      // ncclComm_t of the TP group (null: in-process group)
  bool pending_use_def = false; // in-process TP group: the last partial forward kept deferred sums
  // fused decode cluster split: resident clusters per size (index = size), peers' partials
  int fd_max_clusters[9] = {};
  // FP4 weights: packed e2m1 codes for the decode stream (W13 rows in the stream's tile order)
  void *w13_f4 = nullptr, *w2_f4 = nullptr, *ws13_f4 = nullptr, *ws2_f4 = nullptr;
  CUtensorMap fmap_w13, fmap_w2, fmap_ws13, fmap_ws2;
  float *cl_scratch = nullptr;
  int n_launch = 0, launches_prefill = 0, launches_decode = 0;   // kernel launches per forward
  unsigned long long *trace = nullptr;   // MOE_DEBUG_TRACE timeline buffer (timing experiments)
  // swap-AB CTA-pair GEMM (umma_swap.cu): tiled weights as 128-byte rows (box 128),
  // token rows (box 32), weight scale images (box 1) and token scale images (box 2)
  CUtensorMap tmap_w13, tmap_w2, tmap_ws13, tmap_ws2;
  CUtensorMap xmap_xperm, xmap_h, xmap_xq, xmap_hsh;
  CUtensorMap x64map_xperm, x64map_h, x64map_xq, x64map_hsh;   // box 64 rows (token boxes split between 2 pairs)
  int swap_clusters4 = 0;       // co-resident clusters of 2 CTA pairs (0: pair kernel only)
  CUtensorMap smap_w13, smap_w2, smap_ws13, smap_ws2, smap_xperm, smap_h, smap_xq, smap_hsh;
  int4 *pairs = nullptr;        // [max_tiles] work list of 256-token tiles (2 x 128-row tiles)
  int32_t *n_pairs = nullptr;
  bool gemv_ok = false;         // decode weight-streaming path usable for T <= gemv_max_tokens
  int num_sms = 148;
  int max_rows = 0;             // routed rows capacity (ep_size * max_tokens)
  // ---- expert parallelism (ep_size > 1) ----
  struct Ep {
    int P = 1, rank = 0;
    void *comm = nullptr;       // ncclComm_t (NCCL transport) or null (in-process group)
    uint8_t *send_x = nullptr;         // [P][Tm] rows of row_bytes: bf16 x, or FP8 codes + exponent bytes
    int row_bytes = 0;
    int32_t *send_idx = nullptr;       // [P][Tm][k]
    float *send_w = nullptr;           // [P][Tm][k]
    int32_t *sendpos = nullptr;        // [Tm][P]
    int32_t *cnt_dev = nullptr;        // [2P] send counts, recv counts
    int32_t *cnt_host = nullptr;       // pinned [2P]
    uint8_t *recv_x = nullptr;         // [P*Tm] rows of row_bytes
    __nv_bfloat16 *partial = nullptr;  // [P*Tm][H] expert-side weighted sums (immediate)
    __nv_bfloat16 *partial_def = nullptr;
    __nv_bfloat16 *back = nullptr;     // [P][Tm][H] partial sums returned to this rank
    __nv_bfloat16 *back_def = nullptr;
    bool fixed = false;                // ep_fixed_capacity: whole [P][Tm] blocks, no host sync
    int R = 0;                         // rows received this step
    int roff[33] = {};                 // receive offsets per source
  } ep;
  int64_t workspace_bytes = 0;
  int max_tiles = 0;
  // ---- stage timing (moe_layer_profile) ----
  static constexpr int kStages = 10;
  bool prof = false;
  cudaEvent_t ev[kStages + 1] = {};
  bool ev_hit[kStages + 1] = {};
  int nchunk_max = 0;
};
