/*
 * moe.h -- C ABI of the B200-native MoE routed-expert layer.
 *
 * The operation (PAPER.md = the KTransformers paper, SOSP'25; L<n> = line n):
 *
 *   O_k = I_k + S_k(I_k) + R_k^all(I_k)                               (L219, §4.1)
 *   O_k = I_k + S_k(I_k) + R_{k-1}^def(I_{k-1}) + R_k^imm(I_k)         (L241, §4.1)
 *
 * R_k: routed experts chosen per token by the gate, "top-k or its variants
 * (e.g., grouped top-k in DeepSeek-V3/R1)" (L98, §2.1); S_k: shared experts
 * "activated across all tokens" (L98); deferred experts are the lowest-scoring
 * selected experts, whose output joins one layer later (L215, Fig. 9b).
 * Gate and expert FFN follow the public DeepSeek-V2/V3 and Qwen2-MoE
 * definitions the paper evaluates (reading R1):
 *   s = sigmoid(x Wg^T) | softmax(x Wg^T); sel = s + bias; optional group limit;
 *   idx = top_k(sel); w = s[idx] (/ sum if norm_topk) * routed_scale;
 *   FFN_e(x) = W2_e (silu(W1_e x) * W3_e x).
 *
 * Conventions (all functions):
 *   - Every pointer documented "device" is a CUDA device pointer on
 *     config.device; "host" pointers are ordinary host memory.
 *   - Nothing aborts.  Errors are returned as moe_status; moe_last_error()
 *     gives a thread-local detail string.  Asynchronous device faults surface
 *     at the caller's next synchronisation (normal CUDA convention).
 *   - A handle is not reentrant: one forward at a time per handle (the
 *     workspace is single-stream).
 */
#ifndef MOE_B200_H
#define MOE_B200_H

#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct moe_layer moe_layer; /* opaque, library-owned */

typedef enum {
  MOE_OK = 0,
  MOE_ERR_INVALID_ARG = -1, /* bad pointer / size / enum / n_deferred          */
  MOE_ERR_UNSUPPORTED = -2, /* shape or dtype the kernels do not implement     */
  MOE_ERR_OOM = -3,         /* device allocation failed at create              */
  MOE_ERR_CUDA = -4,        /* a CUDA runtime call or kernel launch failed     */
  MOE_ERR_NCCL = -5,        /* an NCCL call failed (expert parallel)           */
  MOE_ERR_CAPACITY = -6     /* T > max_tokens                                  */
} moe_status;

typedef enum { MOE_SCORE_SOFTMAX = 0, MOE_SCORE_SIGMOID = 1 } moe_score_fn;
/* group score of group-limited routing (n_group > 1):
 * MAX = DeepSeek-V2/V2.5 group_limited_greedy; TOP2_SUM = DeepSeek-V3.       */
typedef enum { MOE_GROUP_MAX = 0, MOE_GROUP_TOP2_SUM = 1 } moe_group_score;
/* weight storage: BF16; e4m3 codes + one fp32 power-of-two scale per 128x128
 * block (reading R10: UE8M0 block scaling, north_star "128x128
 * block-scaled FP8"); F32 (toy config only).                                 */
typedef enum { MOE_W_BF16 = 0, MOE_W_FP8_BLOCK128 = 1, MOE_W_F32 = 2, MOE_W_FP4_BLOCK128 = 3 } moe_wtype;
/* MOE_W_FP4_BLOCK128 ("Int4 tiles are
 * packed into Int8-sized blocks"): OCP FP4 e2m1 codes, two per byte (element 2i
 * in the LOW nibble of byte i) -- w13 [E, 2F, H/2], w2 [E, H, F/2], shared
 * likewise -- with the FP8 path's power-of-two scales per 128x128 block.  The
 * decode stream reads the packed codes (half the bytes of FP8); prefill runs the
 * FP8 kernels on the exact e4m3 expansion made at create.  Activations are
 * e4m3-quantised as for FP8 (R25).                                 */

typedef struct {
  int32_t hidden;            /* H, multiple of 128                                   */
  int32_t ffn;               /* F of one routed expert, multiple of 128              */
  int32_t n_experts;         /* E, global number of routed experts (<= 1024)         */
  int32_t top_k;             /* k, 1 <= k <= 32, k <= E                              */
  int32_t n_group;           /* 1 => plain top-k; else E % n_group == 0, n_group<=32 */
  int32_t topk_group;        /* groups kept (1 <= topk_group <= n_group)             */
  int32_t group_score;       /* moe_group_score                                      */
  int32_t score_fn;          /* moe_score_fn                                         */
  int32_t norm_topk;         /* 1 => w /= sum(w) before routed_scale                 */
  float routed_scale;        /* multiplies the combine weights                      */
  int32_t shared_ffn;        /* Fs (multiple of 128); 0 => no shared expert          */
  int32_t shared_gated;      /* 1 => shared output *= sigmoid(x . w_sg) (Qwen2)      */
  int32_t wtype;             /* moe_wtype                                            */
  int32_t max_tokens;        /* per-rank capacity; every workspace sized at create   */
  int32_t gemv_max_tokens;   /* T <= this => weight-streaming (decode) kernels;
                                0 => library default (the L170 switch) */
  int32_t device;            /* CUDA device ordinal                                  */
  int32_t ep_rank, ep_size;  /* expert parallel group; ep_size 1 => single GPU       */
  const void *nccl_unique_id;/* host, 128 bytes (ncclUniqueId) when ep_size > 1 or
                                tp_size > 1 (the group's communicator)              */
  int32_t tp_rank, tp_size;  /* tensor parallelism within every expert (decode):
                                tp_size 1 => off; see "Tensor parallelism" below    */
  int32_t ep_fixed_capacity; /* ep_size > 1: 1 => fixed-capacity exchange, no host
                                synchronisation (CUDA-Graph capturable); 0 => exact
                                row counts learned on the host (fewer bytes moved) */
} moe_layer_config;

/* Tensor parallelism within every expert (the B200
 * analog of the paper's NUMA-aware TP, Fig. 8b: "each
 * socket stores only its slice ... lightweight reduce-scatter").
 * With tp_size = P > 1 (ep_size must be 1) rank r owns the 128-column FFN
 * chunks [r*n/P, (r+1)*n/P) of every routed expert (n = ffn/128) and of the
 * shared expert (n = shared_ffn/128): ffn and shared_ffn in the config are the
 * FULL sizes, and the weights passed to create are this rank's SLICE only
 *   w13 [E, 2*F_r, H]: rows 0..F_r-1 = W1 rows of the slice, F_r..2F_r-1 = W3 rows
 *   w2  [E, H, F_r]:   the slice's W2 columns        (F_r = 128 x chunks of rank r;
 *   scales [E, 2F_r/128, H/128], [E, H/128, F_r/128]; shared expert alike)
 * so 1/P of the expert bytes are resident per rank.  Routing is replicated (every
 * rank routes every token).  A forward computes this rank's fp32 partial of
 * every token's expert sum; the partials are summed over the P ranks (NCCL
 * all-reduce in fp32 on the layer's own communicator when nccl_unique_id is
 * given; moe_tp_group_forward for an in-process group), then every rank adds
 * residual and deferred_in once and writes the full bf16 y (and deferred_out).
 * Requires P <= ffn/128 (and <= shared_ffn/128) and the decode path: a forward
 * with T > moe_layer_info.gemv_max_tokens returns MOE_ERR_UNSUPPORTED.      */

/* Weights: DEVICE pointers, row-major, read at create and copied + repacked into
 * library-owned memory (the paper's load-time repack, L157); the caller may
 * free them after moe_layer_create returns.  With ep_size = P each rank passes
 * its contiguous slice of E/P experts (rank r owns [r*E/P, (r+1)*E/P)).
 *   gate_w      [E, H]      bf16 (the full router on every rank)
 *   gate_bias   [E]         fp32 or NULL (selection-only bias, DeepSeek-V3)
 *   w13         [E/P, 2F, H]  rows 0..F-1 = W1 (gate_proj), F..2F-1 = W3 (up_proj)
 *   w2          [E/P, H, F]   W2 (down_proj)
 *   *_scale     FP8 only: fp32 powers of two, [.., rows/128, cols/128]
 *   ws13, ws2   shared expert [2Fs, H], [H, Fs] (same dtype/scales as routed)
 *   shared_gate_w [H] bf16 or NULL (required iff shared_gated)               */
typedef struct {
  const void *gate_w;  const float *gate_bias;
  const void *w13;     const float *w13_scale;
  const void *w2;      const float *w2_scale;
  const void *ws13;    const float *ws13_scale;
  const void *ws2;     const float *ws2_scale;
  const void *shared_gate_w;
} moe_layer_weights;

/* Optional DEVICE outputs for parity checks (any member may be NULL):
 *   topk_idx      [T, k] int32  expert ids in canonical slot order
 *                               (combine weight descending, ties -> lower id)
 *   topk_w        [T, k] fp32   combine weights in the same order
 *   expert_counts [E]    int32  tokens routed to each expert (this rank's tokens)
 *   perm          [T*k]  int32  token index of every row of the expert-sorted
 *                               order (stable: by expert, then token)          */
typedef struct {
  int32_t *topk_idx;
  float *topk_w;
  int32_t *expert_counts;
  int32_t *perm;
} moe_routing_out;

/* ncclGetUniqueId for the expert-parallel bootstrap (rank 0 calls it and
 * broadcasts the 128 bytes through the launcher's process group).            */
moe_status moe_get_unique_id(void *out128);

/* Validate the config, allocate all workspaces for max_tokens and copy/repack
 * the weights.  Synchronous (returns after the copies are done).  *out is set
 * to NULL on failure.  With ep_size > 1 and a unique id this initialises the
 * NCCL communicator and is collective over the EP group; with ep_size > 1 and
 * nccl_unique_id == NULL the layer is one rank of an in-process group
 * (moe_ep_group_forward).  Expert-parallel forwards with ep_fixed_capacity = 0
 * synchronise the stream to learn the received row counts and move exactly
 * those rows (not CUDA-Graph capturable).  With ep_fixed_capacity = 1 every
 * (source, destination) transfer moves the whole max_tokens-row block (rows
 * past the source's count carry expert ids -1 and are skipped by the expert
 * side), both ways: no host synchronisation, capturable, at the cost of
 * P * max_tokens rows per direction per rank instead of the routed rows.     */
moe_status moe_layer_create(const moe_layer_config *cfg, const moe_layer_weights *w,
                            moe_layer **out);

/* y = residual + S(x) + R^all(x)   (Eq. L219), stream-ordered on `stream`
 * (a cudaStream_t; NULL = legacy default stream), no host synchronisation and
 * no allocation on the single-GPU path (CUDA-Graph capturable, L193).
 *   x         device [T, H] bf16, 16-byte aligned
 *   residual  device [T, H] bf16 or NULL (NULL => no I_k term, reading R7)
 *   y         device [T, H] bf16; may alias residual, must not alias x
 *   T         0 <= T <= max_tokens (T == 0 is legal and launches nothing)
 *   dbg       NULL or routing outputs (see moe_routing_out)
 * Kernel choice: T <= gemv_max_tokens (default 16) on the tensor-core path runs
 * the decode stream (router, fused per-expert-chunk weight stream, finalize);
 * its expert sums are fp32 atomics, so two calls agree to fp32 rounding, not
 * bitwise (R22).  Larger T runs the grouped-GEMM path, which is
 * deterministic.  The kernels use programmatic dependent launch: the first one
 * may start before the stream's previous kernel ends, but reads nothing the
 * caller wrote on the stream before its own dependency wait.                 */
moe_status moe_layer_forward(moe_layer *layer, const void *x, const void *residual, int32_t T,
                             void *y, moe_routing_out *dbg, void *stream);

/* Expert Deferral (Eq. L241): the last n_deferred slots of each token's
 * canonical order are deferred.
 *   y            = residual + S(x) + R^imm(x) + deferred_in
 *   deferred_out = R^def(x)
 * deferred_in  device [T, H] bf16 or NULL (NULL: first layer, k = 1 case)
 * deferred_out device [T, H] bf16 or NULL (NULL: last layer, k = L case -- all
 *              experts immediate, L215 "not applied at the final layer")
 * 0 <= n_deferred <= k-1, else MOE_ERR_INVALID_ARG.  n_deferred = 0 with both
 * NULL is exactly moe_layer_forward.                                          */
moe_status moe_layer_forward_deferred(moe_layer *layer, const void *x, const void *residual,
                                      int32_t T, int32_t n_deferred, const void *deferred_in,
                                      void *y, void *deferred_out, moe_routing_out *dbg,
                                      void *stream);

/* Expert parallelism inside ONE process: P layers created
 * with ep_size = P, ep_rank = r and nccl_unique_id = NULL form a group; this
 * call runs one forward of every rank -- dispatch of each token row to the
 * ranks owning its experts, expert FFNs there, return of one partial row per
 * (token, rank) -- with device copies (peer copies when the layers live on
 * different GPUs) as the transport.  Arrays are indexed by rank; x[r], y[r],
 * residual[r], deferred_in[r], deferred_out[r] are rank r's device [T[r], H]
 * bf16 buffers (residual/deferred arrays may be NULL).  Synchronises the
 * stream twice (the received row counts size the copies).                    */
moe_status moe_ep_group_forward(moe_layer *const *layers, int32_t P, const void *const *x,
                                const void *const *residual, const int32_t *T, int32_t n_deferred,
                                const void *const *deferred_in, void *const *y, void *const *deferred_out,
                                void *stream);

/* Expert Deferral chained across consecutive layers (§4.1 Eq. 2;
 * §8(f) NEXT-2):
 *   O_k = I_k + S_k(I_k) + R_{k-1}^def(I_{k-1}) + R_k^imm(I_k)
 * The last n_deferred slots of each token's canonical order (the lowest combine
 * weights, L215) are NOT computed by this call: the NEXT layer's chained
 * forward computes them (passing this layer as `prev`) and adds them to its own
 * output.  `prev` (NULL for the first layer, k = 1 case) is the previous layer's
 * handle whose last call was a chained forward with n_deferred > 0 on the same T
 * tokens; its deferred experts stream at the start of this call, before this
 * layer's router has finished -- the overlap the paper's deferral buys.
 *   y = residual + S(x) + R^imm(x) + R^def_prev(x_prev)
 * n_deferred = 0 is the last layer (k = L: all experts immediate).  The caller
 * keeps the chain on one stream (prev's workspace holds x_prev's quantised copy
 * and routing until prev's next forward).  Decode path only (T <= gemv_max_tokens,
 * the paper applies deferral in decode, L245); MOE_ERR_UNSUPPORTED otherwise,
 * MOE_ERR_INVALID_ARG if prev is this layer, has another shape / dtype / device /
 * TP split, or its last call was not a chained forward with n_deferred > 0 on T
 * tokens.                                                                     */
moe_status moe_layer_forward_chained(moe_layer *layer, const void *x, const void *residual, int32_t T,
                                     int32_t n_deferred, moe_layer *prev, void *y, void *stream);

/* Tensor parallelism inside ONE process (the test vehicle of the NCCL path on a
 * single GPU): P layers created with tp_size = P, tp_rank = r and no unique id
 * form a group; this call runs one forward of every rank (rank r's x[r], same
 * T tokens on every rank), sums the P fp32 partials on the devices with peer
 * copies and a reduction kernel (what the NCCL all-reduce does across GPUs), and
 * writes every rank's full y[r] (and deferred_out[r]).  Arrays indexed by rank;
 * residual / deferred_in / deferred_out arrays may be NULL.                   */
moe_status moe_tp_group_forward(moe_layer *const *layers, int32_t P, const void *const *x,
                                const void *const *residual, int32_t T, int32_t n_deferred,
                                const void *const *deferred_in, void *const *y, void *const *deferred_out,
                                void *stream);

/* Timing experiments only: a layer created with the environment variable
 * MOE_DEBUG_TRACE set records globaltimer/clock stamps of its kernels into a
 * 4096-entry u64 device buffer; this synchronises the device, copies
 * min(cap, 4096) entries to `host` and clears the buffer.  MOE_ERR_UNSUPPORTED
 * without MOE_DEBUG_TRACE.  Layout: DESIGN.md §6 / scripts/decode_trace.py.   */
moe_status moe_layer_debug_trace(moe_layer *layer, void *host, int32_t cap);

/* Free every library allocation (and the NCCL communicator).  NULL is a no-op. */
moe_status moe_layer_destroy(moe_layer *layer);

const char *moe_status_string(moe_status s);
const char *moe_last_error(void);

/* Introspection for tests and the bench (host-only, no device work). */
typedef struct {
  int64_t weight_bytes;      /* library-owned weight bytes (after repack)          */
  int64_t workspace_bytes;   /* library-owned workspace bytes                       */
  int32_t gemv_max_tokens;   /* effective decode/prefill switch                     */
  int32_t kernels_per_forward_prefill; /* launches of one forward, GEMM path        */
  int32_t kernels_per_forward_decode;  /* launches of one forward, GEMV path        */
  int32_t local_experts;     /* E / ep_size                                         */
} moe_layer_info;
moe_status moe_layer_get_info(const moe_layer *layer, moe_layer_info *info);

/* Stage timing (instrumentation for the bench's roofline figures; off by
 * default).  When enabled, forward records a CUDA event after every stage on
 * the forward's stream (adds no synchronisation).  moe_layer_stage_times waits
 * for the last recorded forward and writes the elapsed ms of each stage
 * (n_out = number of stages, at most cap; stages not run in that forward give
 * 0).  moe_stage_name(i) names stage i ("router_logits", "gemm1", ...).      */
moe_status moe_layer_profile(moe_layer *layer, int32_t enable);
moe_status moe_layer_stage_times(moe_layer *layer, float *ms_out, int32_t cap, int32_t *n_out);
const char *moe_stage_name(int32_t i);

#ifdef __cplusplus
}
#endif
#endif /* MOE_B200_H */
