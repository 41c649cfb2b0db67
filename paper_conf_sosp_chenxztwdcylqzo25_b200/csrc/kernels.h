// kernels.h -- internal launch interface between the host layer (moe_api.cu)
// and the kernels.  Not part of the public C ABI (include/moe.h).
#pragma once
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <cstdlib>
#include <utility>

#include "common.cuh"

namespace moe {

// Timing-experiment knobs (stale-smem / loads-only GEMM modes, router phase
// skips, PDL off): compiled in only with -DMOE_EXPERIMENTS (build.py,
// MOE_EXPERIMENTS=1); the default library ignores the environment and every
// knob reads 0, so no stray variable can change a result.
#ifdef MOE_EXPERIMENTS
constexpr bool kExperiments = true;
#else
constexpr bool kExperiments = false;
#endif
int experiment_knob(const char *env);

// cudaFuncSetAttribute acts on the CURRENT device only: remember the
// (kernel, device, attribute) triples already set instead of one process-wide
// flag, so a process that drives several GPUs opts in on each of them.
cudaError_t set_kernel_attr(const void *kernel, cudaFuncAttribute attr, int value);

// Launch with programmatic dependent launch (PDL): the kernel may start while
// its stream predecessor is still running and must execute pdl_wait() before
// touching the predecessor's outputs (CUDA-graph capturable).
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                       Args &&...args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  static const bool no_pdl = experiment_knob("MOE_NO_PDL") == 1;   // A/B experiments (MOE_EXPERIMENTS only)
  cfg.numAttrs = no_pdl ? 0 : 1;
  return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}

enum { WT_BF16 = 0, WT_FP8 = 1, WT_F32 = 2 };
enum { GEMM_LOGITS = 0, GEMM_SWIGLU = 1, GEMM_PLAIN = 2 };

struct SimtGemmArgs {
  const void *A;          // activation rows
  const float *As;        // fp8 A: [rows, K/128] scales
  int64_t lda;            // elements
  int a_fp8;
  const void *B;          // weights of expert 0
  const float *Bs;        // fp8 B scales of expert 0 [N/128, K/128]
  int64_t b_stride;       // elements between experts
  int64_t bs_stride;      // scales between experts
  int b_type;             // WT_*
  int N, K;
  const int4 *tiles;      // routed: (expert, row0, row_end, 0) per 128-row tile; null = dense
  const int32_t *n_tiles; // device count of tiles
  int M;                  // dense rows
  void *C;                // output
  float *Cs;              // fp8 output scales [rows, ldc/128]
  int64_t ldc;
  int out_fp8;
};
cudaError_t launch_simt_gemm(int mode, const SimtGemmArgs &a, int grid_x, cudaStream_t st);

struct RouterArgs {
  const float *logits;    // [T, ldl]
  int ldl;
  const float *bias;      // [E] or null
  int T, E, k, n_group, topk_group, group_score, score_fn, norm_topk;
  float routed_scale;
  int shared_gated;       // logit column E is the shared-expert gate
  int32_t *topk_idx;      // [T, k]
  float *topk_w;          // [T, k]
  float *sgate;           // [T]
};
cudaError_t launch_router_select(const RouterArgs &a, cudaStream_t st);

struct PermuteArgs {
  const int32_t *topk_idx;  // [T, k] global expert ids
  int T, k, E, e0;          // local experts [e0, e0 + E)
  int32_t *chunk_cnt, *chunk_base;  // [nchunk, E]
  int32_t *counts, *offs, *offs_pad;
  int4 *tiles; int32_t *n_tiles;
  int4 *pairs; int32_t *n_pairs;   // 2-CTA work list (null = not needed)
  int32_t *act_list; int32_t *n_active;
  int32_t *row_token;       // [R_max]
  int64_t R_max;
  int32_t *pos;             // [T*k]
  int32_t *dbg_perm;        // [T*k] unpadded token order or null
  int32_t *dbg_counts;      // [E] or null
};
cudaError_t launch_permute(const PermuteArgs &a, cudaStream_t st);

// decode (T <= 16): router logits + selection + permutation in one launch
struct RouteSmallArgs {
  RouterArgs r;
  PermuteArgs p;
  const void *x;                // bf16 [T, H]
  const void *wg;               // bf16 [rows, H]
  int H, rows;
  int *done;                    // zero-initialised CTA counter (re-armed by the kernel)
  int debug;                    // timing experiments only (MOE_EXPERIMENTS builds, MOE_DEBUG_ROUTE)
  // FP8: x quantised in token order (1x128 UE8M0 + e4m3) for the fused decode stream;
  // BF16: x copied into the layer's own buffer (the stream reads it there, so a chained
  // next layer can still read it after the caller reused its x buffer)
  int fp8;
  void *xq; float *xs;
  void *xcopy;
  unsigned long long *trace;     // MOE_DEBUG_TRACE: [0] CTA 0 entry, [1..4] tail start / select / permute / end
  int early_trigger;            // let the decode stream launch at once (it has the previous layer's deferred
                                // units to stream meanwhile); else only when routing is complete
  // The tail writes the active-expert list (p.act_list: any slot) and, for chained
  // Expert Deferral, the experts of the immediate slots [0, n_imm) and of the
  // deferred slots [n_imm, k) (ascending local ids); the full counts and
  // permutation only when dbg_perm / dbg_counts ask for them (parity outputs).
  int n_imm;
  int32_t *imm_list, *n_imm_list, *def_list, *n_def_list;
};
cudaError_t launch_route_small(const RouteSmallArgs &a, cudaStream_t st);



// prefill: each token's row (FP8-quantised or copied) into its k sorted rows and xq
cudaError_t launch_scatter_rows(const void *x, int T, int H, int k, const int32_t *pos, const ScatterDst &d,
                                cudaStream_t st);

struct CombineArgs {
  int T, H, k, n_imm;
  const int32_t *pos;        // [T, k] padded rows
  const float *topk_w;       // [T, k]
  const void *yperm;         // [R, H] bf16
  const void *ysh;           // [T, H] bf16 or null
  const float *sgate;        // [T] or null
  const void *residual;      // [T, H] or null
  const void *deferred_in;   // [T, H] or null
  void *y;                   // [T, H]
  void *deferred_out;        // [T, H] or null
};
cudaError_t launch_combine(const CombineArgs &a, cudaStream_t st);

// ---------------------------------------------------------------- decode GEMV
struct GemvArgs {
  int T, H, F, Fs, fp8, has_shared;
  const int32_t *act_list, *n_active, *counts, *offs_pad, *row_token;
  const void *x;                 // bf16 [T, H] (BF16 weights)
  const void *xq; const float *xs;  // e4m3 [T, H] + [T, H/128] (FP8 weights)
  const void *w13, *w2, *ws13, *ws2;
  const float *w13_s, *w2_s, *ws13_s, *ws2_s;
  void *h, *hsh; float *h_s, *hsh_s;
  __nv_bfloat16 *yperm, *ysh;
};
constexpr int kGemvMaxTokens = 8;
size_t gemv_smem_bytes(int T, int H, int F, int Fs);
// which = 1: W13 + SwiGLU -> h;  which = 2: W2 -> y rows
cudaError_t launch_gemv(const GemvArgs &a, int which, int max_slots, cudaStream_t st);
cudaError_t launch_router_gemv(const void *x, int T, int H, const void *wg, int rows, float *logits,
                               cudaStream_t st);

// ---------------------------------------------------------------- expert parallelism
struct EpCombineArgs {
  int T, H, P, Tm;
  const int32_t *sendpos;        // [T][P]
  const __nv_bfloat16 *back, *back_def;   // [P][Tm][H]
  const __nv_bfloat16 *ysh; const float *sgate;
  const __nv_bfloat16 *residual, *deferred_in;
  __nv_bfloat16 *y, *deferred_out;
};
cudaError_t launch_ep_plan(const int32_t *idx, int T, int k, int E_loc, int P, int32_t *sendpos, int32_t *cnt,
                           cudaStream_t st);
cudaError_t launch_ep_pack(const void *x, int T, int H, int k, const int32_t *idx, const float *w, int E_loc, int P,
                           int Tm, const int32_t *sendpos, void *send_x, int32_t *send_idx, float *send_w,
                           cudaStream_t st);
cudaError_t launch_ep_final_combine(const EpCombineArgs &a, cudaStream_t st);
// FP8 dispatch: rows of [H e4m3 codes | H/128 UE8M0 exponent bytes], row_bytes apart
cudaError_t launch_ep_pack_fp8(const void *xq, const float *xs, int T, int H, int k, const int32_t *idx,
                               const float *w, int E_loc, int P, int Tm, int row_bytes, const int32_t *sendpos,
                               void *send_x, int32_t *send_idx, float *send_w, cudaStream_t st);
cudaError_t launch_ep_scatter_fp8(const void *recv, int R, int H, int k, int row_bytes, const int32_t *pos,
                                  void *xperm, uint8_t *img, int img_stride, cudaStream_t st);
cudaError_t launch_ep_unpack_fp8(const void *recv, int R, int H, int row_bytes, void *xq, float *xs, cudaStream_t st);
int ep_nccl_get_unique_id(void *out128);
int ep_nccl_init(void **comm, int P, int rank, const void *uid128);
void ep_nccl_destroy(void *comm);
const char *ep_nccl_error(void *comm);
int ep_nccl_counts(void *comm, const int32_t *send_cnt, int32_t *recv_cnt, int P, cudaStream_t st);
int ep_nccl_allreduce_f32(void *comm, float *buf, size_t n, cudaStream_t st);   // in place, sum
// dst[i] += sum_j src[j][i], i < n (the in-process TP group's reduction)
cudaError_t launch_sum_f32(float *dst, const float *const *src, int nsrc, int64_t n, cudaStream_t st);
int ep_nccl_rows(void *comm, int P, const int32_t *send_cnt, const int64_t *send_off, const int32_t *recv_cnt,
                 const int64_t *recv_off, int nbuf, const void *const *send, void *const *recv,
                 const int64_t *row_bytes, cudaStream_t st);

// ---------------------------------------------------------------- tcgen05 router logits
struct LogitsParams {
  CUtensorMap a_map;            // x [T, H] bf16, K-major SW128, box 64 x 128 rows
  CUtensorMap b_map;            // router rows [gate_rows, H] bf16, box 64 x 256 rows
  int kblocks;                  // H / 64
  float *out;                   // logits [T, ldc] fp32
  int64_t ldc;
  int n_valid;                  // columns < n_valid are written
  int T;                        // token rows
  int nb;                       // 256-row blocks of router rows
  int *sched;                   // device work counter, zero at launch
};
cudaError_t launch_umma_logits(const LogitsParams &p, int grid, cudaStream_t st);
// Repack row-major weights [rows, K] (es bytes/elem) into 256-row x 128-byte
// tiles, 128B-swizzled (the smem image TMA would produce).  interleave_f > 0:
// rows are W13 [2F, K] and tile rows are ordered (W1 block b, W3 block b) per 128.
cudaError_t launch_tile_weights(const void *src, void *dst, int nexp, int rows, int kbytes, int interleave_f,
                                cudaStream_t st);

// decode, fused per (slot, 128-column FFN chunk) unit (umma_decode_fused.cu):
// W13 tile -> SwiGLU (+ FP8 requant) -> h_c in smem -> W2 column block ->
// weighted fp32 partial sums; decode_finalize writes y / deferred_out
struct FdGroup {                // 0 routed, 1 shared, 2 the previous layer's deferred experts
  CUtensorMap x_map;            // token-order activation rows (xq / bf16 x), K-major SW128, box 16 rows
  CUtensorMap w13_map4, w2_map4;   // FP4 weights (packed e2m1, 16U4_ALIGN16B, box 128 x 256 rows, SW128):
                                   // W13 rows in the tile order [expert][F/128][256], W2 rows [expert][H]
  const uint8_t *w13;           // tiled W13 [expert][F/128][H/128 B][256 x 128 B]
  const float *w13_s;           // FP8: [expert][2F/128][H/128] block scales, rows interleaved per 128 (gate, up)
  const float *xs;              // FP8: [T][H/128] activation scales (token order)
  const uint8_t *w2;            // tiled W2 [expert][H/256][F/128 B][256 x 128 B]
  const float *w2_s;            // FP8: [expert][H/128][F/128]
  int nch;                      // 128-column FFN chunks per expert (F/128, Fs/128)
  // routed groups: expert list (ascending local ids) and the routing that picks the tokens
  const int32_t *list, *n_list;
  const int32_t *topk_idx;      // [T, k] global ids, canonical slot order
  const float *topk_w;          // [T, k]
  int k, e0;
  int a0, a1, a2;               // canonical slots [a0, a1) -> acc_imm, [a1, a2) -> acc_def, others skipped
};
struct DecodeFinalizeArgs {
  int T, H, use_def;
  float *acc_imm, *acc_def;
  const void *residual, *deferred_in;
  void *y, *deferred_out;
  unsigned long long *trace;     // MOE_DEBUG_TRACE: [2000] past the PDL wait, [2001] end (CTA 0)
};
struct FusedDecodeParams {
  FdGroup g[3];
  int H, T, has_shared, has_prev;
  const float *sgate;           // null unless the shared expert is gated (Qwen2)
  float *acc_imm, *acc_def;     // [T, H] fp32 sums, zero on entry (re-zeroed by decode_finalize)
  int *sched, *done;            // work counter + exit ticket, zero on entry (re-armed by the kernel)
  unsigned long long *trace;     // MOE_DEBUG_TRACE: per-CTA globaltimer timeline (timing experiments only)
  int debug;                    // MOE_EXPERIMENTS builds (MOE_DEBUG_FD): 1 no phase-A fold, 2 no phase-A MMAs
  float *cl_scratch;            // cluster split: [clusters][7][128][32] fp32 partials of the peers (L2)
};
// csize > 1: clusters of csize CTAs share each unit (the cluster split)
cudaError_t launch_umma_decode_fused(bool fp8, bool w4, const FusedDecodeParams &p, int grid, int csize,
                                     cudaStream_t st);
int fused_decode_max_clusters(bool fp8, int csize);
cudaError_t launch_decode_finalize(const DecodeFinalizeArgs &a, cudaStream_t st);

bool make_kmajor_map(CUtensorMap *m, const void *base, bool fp8, int64_t rows, int64_t cols, int box_rows);
// packed e2m1 [rows, cols / 2 bytes] -> shared memory unpacked to 16-byte groups (box 128 x box_rows, SW128)
bool make_fp4_map(CUtensorMap *m, const void *base, int64_t rows, int64_t cols, int box_rows);
// FP4 weights at create: e2m1 nibbles -> e4m3 bytes (exact: e2m1 is a subset of e4m3)
cudaError_t launch_fp4_to_e4m3(const void *packed, void *out, int64_t n_bytes_in, cudaStream_t st);
// W13 rows [nexp][2F] (W1 rows then W3 rows) -> the 256-row tile order of the decode stream
// (per tile nb: 128-row halves of [gate | up | gate | up] 32-row quadrants), row_bytes each
cudaError_t launch_permute_w13_rows(const void *src, void *dst, int nexp, int F, int row_bytes, cudaStream_t st);
bool make_rows_map(CUtensorMap *m, const void *base, bool u32, int64_t rows, int row_elems, int box_rows);
bool make_blocks_map(CUtensorMap *m, const void *base, int64_t total_bytes, int row_bytes, int box_rows);
// prefill grouped expert GEMM, swap-AB on CTA pairs (umma_swap.cu): weights are
// the M = 256 operand, an expert's tokens (<= 256, padded to 16) the N operand
struct SwapGroup {              // one operand set: 0 = routed experts, 1 = shared expert
  CUtensorMap w_map;            // tiled weights as 128-byte rows, box 128 rows
  CUtensorMap x_map;            // token rows, K-major SW128, box 32 rows (ragged tails)
  CUtensorMap x_map128;         // the same, box 128 rows (full halves)
  CUtensorMap x_map64;          // the same, box 64 rows (a half split between 2 multicasting pairs)
  CUtensorMap x_map16;          // the same, box 16 rows
  CUtensorMap sfw_map;          // FP8: weight scale images as 512-byte rows, box 1
  CUtensorMap sfx_map;          // FP8: token scale images as 512-byte rows, box 2
  int w_nblk;                   // 256-row weight blocks per expert
  int kblocks;                  // K / 128 bytes
  int sfw_per_cta;              // 1: an image per 128-row CTA half (W2); 0: per 256-row block (W13)
  int sfx_tile_stride;          // 128-row tiles per k-group in the token image
  void *out;                    // h (SWIGLU) or y (PLAIN) rows
  int64_t ldc;                  // elements
  uint8_t *out_sf;              // FP8 SWIGLU: scale image of h
  int out_sf_tile_stride;
};
struct SwapParams {
  SwapGroup g[2];
  const int4 *tiles;            // routed 256-token tiles (expert, row0, row_end, t0 | nt << 16)
  const int32_t *n_tiles;
  int nb_r, nb_s;               // weight blocks per unit group
  int T_shared;                 // shared-expert tokens (0 = none)
  int *sched;                   // device work counter, zero at launch
  int debug_mode;               // 0; (MOE_DEBUG_GEMM) 2 = no epilogue math -- timing experiments
  unsigned long long *trace;     // MOE_DEBUG_TRACE: MMA-warp cycle breakdown per CTA pair (timing experiments)
};
// np = 1: grid = CTAs (pairs of 2); np = 2: grid = clusters of 2 pairs sharing token boxes (multicast)
cudaError_t launch_umma_swap_gemm(bool fp8, int epi, const SwapParams &p, int grid, int np, cudaStream_t st);
int umma_swap_max_clusters4(bool fp8);   // co-resident clusters of 4 CTAs (0: not available)

}  // namespace moe
