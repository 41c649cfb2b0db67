"""CPU oracle for the MoE routed-expert layer -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this module.  The product path
(``paper_conf_sosp_chenxztwdcylqzo25_b200``) never imports it and shares no code,
headers, tables or helpers with it.

What it computes, step by step and in the paper's notation
(PAPER.md = /root/reference/PAPER.md, cited as L<line>):

  O_k = I_k + S_k(I_k) + R_k^all(I_k)                        (§4.1 Eq. 1)
  O_k = I_k + S_k(I_k) + R_{k-1}^def(I_{k-1}) + R_k^imm(I_k)  (§4.1 Eq. 2)

with R_k the routed experts picked by the gate ("top-k or its variants (e.g.
grouped top-k in DeepSeek-V3/R1)", L98 §2.1) and S_k the shared experts that are
"activated across all tokens" (L98).  The paper never writes the gate or the
expert FFN down; the readings used here are the
public model definitions the paper evaluates (DeepSeek-V2/V3 [6,7], Qwen2 [50]):

  router   logits = x Wg^T; s = sigmoid(logits) or softmax(logits)
           sel = s + bias (bias only steers selection)
           optional group limit: keep the topk_group groups with the best group
           score (max of sel, or sum of the top-2 sel in the group), others -inf
           idx = the top_k largest sel (ties -> lower expert id)
           w = s[idx] (unbiased), optional w /= sum(w), w *= routed_scale
           canonical slot order: w descending, ties -> lower expert id
  expert   FFN_e(x) = W2_e ( silu(W1_e x) * (W3_e x) ),   silu(g) = g * sigmoid(g)
  shared   S(x) = FFN_s(x), times sigmoid(x . w_sg) if shared_gated (Qwen2)
  combine  y = residual + S(x) + sum_{imm} w_j FFN_{e_j}(x) + deferred_in
           deferred_out = sum_{def} w_j FFN_{e_j}(x)   (def = last n_def slots)

Arithmetic is float64 (numpy), except where a float decides an integer code:
the FP8 activation quantiser takes its decisions in float32, the precision of the
kernel (the paper fixes none), see ``act_quant_e4m3``.

Parity pins: every function here is pinned by tests in tests/test_oracle_*.py
against things other than itself (hand-computed closed forms, brute force,
invariants, ml_dtypes, torch.nn.functional, HF transformers' DeepSeek-V2/V3 and
Qwen2-MoE blocks).  No function is "parity unpinned".
"""
from __future__ import annotations

import math
from dataclasses import dataclass

import numpy as np

F64 = np.float64
F32 = np.float32

SCORE_SOFTMAX = 0
SCORE_SIGMOID = 1
GROUP_MAX = 0        # DeepSeek-V2/V2.5 group_limited_greedy: group score = max
GROUP_TOP2_SUM = 1   # DeepSeek-V3: group score = sum of the two largest


# --------------------------------------------------------------------------
# Router (§2.1 "top-k or its variants (e.g. grouped top-k)";
# L187 §3.3 "After the GPU's gating network finishes, it knows the routed
# experts for every token").  Gate math: DESIGN.md reading R1.
# --------------------------------------------------------------------------
def router_logits(x: np.ndarray, wg: np.ndarray) -> np.ndarray:
    """logits[t, e] = sum_h x[t, h] * Wg[e, h]   (fp64)."""
    return np.asarray(x, F64) @ np.asarray(wg, F64).T


def sigmoid(z: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):          # exp(-z) -> inf gives exactly 0
        return 1.0 / (1.0 + np.exp(-np.asarray(z, F64)))


def softmax(z: np.ndarray) -> np.ndarray:
    z = np.asarray(z, F64)
    m = z.max(axis=-1, keepdims=True)
    e = np.exp(z - m)
    return e / e.sum(axis=-1, keepdims=True)


def scores(logits: np.ndarray, score_fn: int) -> np.ndarray:
    return sigmoid(logits) if score_fn == SCORE_SIGMOID else softmax(logits)


def _top_indices(v: np.ndarray, k: int) -> list[int]:
    """Indices of the k largest entries of a 1-D vector, larger value first,
    equal values -> lower index first (reading R2)."""
    order = sorted(range(len(v)), key=lambda i: (-v[i], i))
    return order[:k]


def select_experts(s: np.ndarray, bias, n_group: int, topk_group: int, top_k: int,
                   group_score: int) -> np.ndarray:
    """Expert choice per token: returns idx [T, top_k] (selection order).

    sel = s + bias; group limit (if n_group > 1); top_k of sel.
    Experts outside the kept groups get -inf (reading R19)."""
    s = np.asarray(s, F64)
    T, E = s.shape
    sel = s + (np.asarray(bias, F64)[None, :] if bias is not None else 0.0)
    out = np.zeros((T, top_k), np.int64)
    gsize = E // n_group
    for t in range(T):
        row = sel[t].copy()
        if n_group > 1:
            gscore = []
            for g in range(n_group):
                members = row[g * gsize:(g + 1) * gsize]
                if group_score == GROUP_TOP2_SUM:
                    top2 = sorted(members, reverse=True)[:2]
                    gscore.append(top2[0] + top2[1])
                else:
                    gscore.append(max(members))
            keep = set(_top_indices(np.array(gscore), topk_group))
            for g in range(n_group):
                if g not in keep:
                    row[g * gsize:(g + 1) * gsize] = -np.inf
        out[t] = _top_indices(row, top_k)
    return out


def combine_weights(s: np.ndarray, idx: np.ndarray, norm_topk: bool,
                    routed_scale: float) -> np.ndarray:
    """w[t, j] = s[t, idx[t, j]] (unbiased score), optionally normalised to sum
    1 (no epsilon, reading R8), then multiplied by routed_scale."""
    s = np.asarray(s, F64)
    w = np.take_along_axis(s, idx, axis=1)
    if norm_topk:
        w = w / w.sum(axis=1, keepdims=True)
    return w * F64(routed_scale)


def canonical_order(idx: np.ndarray, w: np.ndarray):
    """Sort each token's k slots by (w descending, expert id ascending).
    PAPER.md L215 (Fig. 9): "only the top-2 experts with the highest routing
    score ... are immediate; the remaining ... deferred" -> the deferred experts
    are the LAST n_def slots of this order (reading R4)."""
    idx2 = np.empty_like(idx)
    w2 = np.empty_like(w)
    for t in range(idx.shape[0]):
        order = sorted(range(idx.shape[1]), key=lambda j: (-w[t, j], idx[t, j]))
        idx2[t] = idx[t, order]
        w2[t] = w[t, order]
    return idx2, w2


def route(x, wg, bias, cfg) -> tuple[np.ndarray, np.ndarray, np.ndarray]:
    """Full gate: returns (idx [T,k] canonical order, w [T,k], s [T,E])."""
    s = scores(router_logits(x, wg), cfg.score_fn)
    idx = select_experts(s, bias, cfg.n_group, cfg.topk_group, cfg.top_k, cfg.group_score)
    w = combine_weights(s, idx, cfg.norm_topk, cfg.routed_scale)
    idx, w = canonical_order(idx, w)
    return idx, w, s


# --------------------------------------------------------------------------
# Count / prefix-sum / permutation (§3.2 "dynamic task
# scheduling ... co-scheduling tasks targeting the same expert"; the grouping
# of token rows by expert that the fused MoE operator (L179) consumes).
# --------------------------------------------------------------------------
def count_and_permute(idx: np.ndarray, n_experts: int):
    """counts[e] = #{(t, j): idx[t, j] == e};  offsets = exclusive prefix sum
    (length E+1);  perm = the flattened (t, j) pairs stably ordered by
    (expert, t), stored as the token index t of each sorted row."""
    T, k = idx.shape
    counts = np.zeros(n_experts, np.int64)
    for t in range(T):
        for j in range(k):
            counts[idx[t, j]] += 1
    offsets = np.zeros(n_experts + 1, np.int64)
    for e in range(n_experts):
        offsets[e + 1] = offsets[e] + counts[e]
    pairs = sorted(((int(idx[t, j]), t, j) for t in range(T) for j in range(k)))
    perm_token = np.array([p[1] for p in pairs], np.int64)
    perm_slot = np.array([p[2] for p in pairs], np.int64)
    return counts, offsets, perm_token, perm_slot


# --------------------------------------------------------------------------
# FP8 (e4m3) with power-of-two (UE8M0) block scales -- north_star "128x128
# block-scaled FP8"; PAPER.md L159 only names symmetric group-wise Int8/Int4,
# so the encoding is reading R10.
# --------------------------------------------------------------------------
E4M3_MAX = 448.0


def e4m3_decode(code: np.ndarray) -> np.ndarray:
    """OCP e4m3fn: sign 1, exponent 4 (bias 7), mantissa 3; no inf; 0x7f/0xff NaN."""
    c = np.asarray(code, np.uint8).astype(np.int64)
    sign = np.where(c & 0x80, -1.0, 1.0)
    exp = (c >> 3) & 0xF
    man = c & 0x7
    val = np.where(exp == 0, man / 8.0 * 2.0 ** -6, (1.0 + man / 8.0) * np.exp2(exp - 7.0))
    val = np.where((c & 0x7F) == 0x7F, np.nan, val)
    return sign * val


def e4m3_round(v: np.ndarray) -> np.ndarray:
    """Round float32 values to the nearest e4m3fn value, ties to even, saturating
    at +-448 (satfinite).  Returns the rounded values (float64, exact)."""
    v = np.asarray(v, F32).astype(F64)
    a = np.abs(v)
    out = np.zeros_like(a)
    nz = a > 0
    # spacing of the e4m3 grid around a: normals have 3 mantissa bits, the
    # subnormal range (a < 2^-6) has fixed spacing 2^-9.
    e = np.floor(np.log2(np.where(nz, a, 1.0)))
    # fix possible log2 rounding at exact powers of two
    e = np.where(np.exp2(e) > a, e - 1, e)
    e = np.where(np.exp2(e + 1) <= a, e + 1, e)
    e = np.maximum(e, -6.0)
    ulp = np.exp2(e - 3.0)
    q = a / ulp                      # exact (power-of-two division)
    r = np.floor(q)
    frac = q - r
    r = np.where(frac > 0.5, r + 1, np.where(frac < 0.5, r, r + (r % 2)))
    out = np.where(nz, r * ulp, 0.0)
    out = np.minimum(out, E4M3_MAX)
    return np.sign(v) * out


def ue8m0_ceil_scale(amax: np.ndarray) -> np.ndarray:
    """s = the smallest power of two >= fl32(amax / 448) (IEEE fp32 division),
    s = 1 where amax == 0.  Ceil taken from the fp32 bit pattern: an exact power
    of two keeps its exponent, anything else rounds up one binade."""
    amax = np.asarray(amax, F32)
    q = (amax / F32(E4M3_MAX)).astype(F32)
    bits = q.view(np.uint32).astype(np.int64)
    exp = (bits >> 23) & 0xFF
    man = bits & 0x7FFFFF
    # normals only (q >= 2^-126 always holds for realistic amax > 1e-36)
    e_unbiased = exp - 127 + (man != 0).astype(np.int64)
    s = np.exp2(e_unbiased.astype(F64))
    return np.where(amax > 0, s, 1.0)


def act_quant_e4m3(v: np.ndarray, block: int = 128) -> np.ndarray:
    """Per-row, per-`block`-column activation quantisation (reading R10):
    a = max|v| over the block, s = ue8m0_ceil_scale(a), v <- e4m3(v / s) * s.
    Decisions are taken on float32 values (the kernel's precision)."""
    v32 = np.asarray(v, F64).astype(F32)
    rows, cols = v32.shape
    assert cols % block == 0
    blk = v32.reshape(rows, cols // block, block)
    amax = np.abs(blk).max(axis=2)
    s = ue8m0_ceil_scale(amax)                       # [rows, nblk] float64 powers of 2
    q = e4m3_round((blk.astype(F64) / s[:, :, None]).astype(F32))
    return (q * s[:, :, None]).reshape(rows, cols)


def dequant_block128(codes: np.ndarray, scales: np.ndarray) -> np.ndarray:
    """W[r, c] = e4m3(codes[r, c]) * scales[r // 128, c // 128].
    (e4m3_decode evaluated once per code value as a 256-entry table.)"""
    table = e4m3_decode(np.arange(256, dtype=np.uint8))
    w = table[np.asarray(codes, np.uint8)]
    r, c = w.shape
    w = w.reshape(r // 128, 128, c // 128, 128) * np.asarray(scales, F64)[:, None, :, None]
    return w.reshape(r, c)


# --------------------------------------------------------------------------
# 4-bit expert weights for decode (PAPER.md L159
# "symmetric group-wise linear quantization for Int8 and Int4 ... Int4 tiles
# are packed into Int8-sized blocks").  B200 reading (R25): the
# 4-bit element is OCP FP4 e2m1 -- the type the 5th-gen tensor cores take
# next to e4m3 -- packed two per byte (element 2i in the low nibble of byte i),
# with one power-of-two scale per 128x128 block (the group of R10).
# --------------------------------------------------------------------------
def unpack_fp4(packed: np.ndarray) -> np.ndarray:
    """[..., C/2] bytes -> [..., C] 4-bit codes: element 2i = low nibble of byte i."""
    b = np.asarray(packed, np.uint8)
    out = np.empty(b.shape[:-1] + (2 * b.shape[-1],), np.uint8)
    out[..., 0::2] = b & 0x0F
    out[..., 1::2] = b >> 4
    return out


def e2m1_decode(code: np.ndarray) -> np.ndarray:
    """OCP e2m1: sign bit 3, exponent bits 2-1 (bias 1), mantissa bit 0; no inf/NaN.
    exponent 0 is subnormal (0 or 0.5)."""
    c = np.asarray(code, np.uint8).astype(np.int64)
    sign = np.where(c & 0x8, -1.0, 1.0)
    exp = (c >> 1) & 0x3
    man = c & 0x1
    val = np.where(exp == 0, man * 0.5, (1.0 + man / 2.0) * np.exp2(exp - 1.0))
    return sign * val


def dequant_fp4_block128(packed: np.ndarray, scales: np.ndarray) -> np.ndarray:
    """W[r, c] = e2m1(code[r, c]) * scales[r // 128, c // 128], codes unpacked from
    `packed` [R, C/2] (e2m1_decode evaluated once per code as a 16-entry table)."""
    table = e2m1_decode(np.arange(16, dtype=np.uint8))
    w = table[unpack_fp4(packed)]
    r, c = w.shape
    w = w.reshape(r // 128, 128, c // 128, 128) * np.asarray(scales, F64)[:, None, :, None]
    return w.reshape(r, c)


# --------------------------------------------------------------------------
# Expert FFN (SwiGLU; reading R1 -- HF DeepseekV3MLP / Qwen2MoeMLP) and the
# fused gate+up "one batch" structure of PAPER.md L179 §3.2.
# --------------------------------------------------------------------------
def silu(g: np.ndarray) -> np.ndarray:
    g = np.asarray(g, F64)
    return g * sigmoid(g)


def swiglu_ffn(x: np.ndarray, w1: np.ndarray, w3: np.ndarray, w2: np.ndarray,
               fp8_act: bool = False) -> np.ndarray:
    """FFN(x) = W2 (silu(W1 x) * W3 x).  x [n, H], W1/W3 [F, H], W2 [H, F].
    fp8_act: quantise x and h with act_quant_e4m3 before each GEMM (R10/R11)."""
    x = np.asarray(x, F64)
    if fp8_act:
        x = act_quant_e4m3(x)
    g = x @ np.asarray(w1, F64).T
    u = x @ np.asarray(w3, F64).T
    h = silu(g) * u
    if fp8_act:
        h = act_quant_e4m3(h)
    return h @ np.asarray(w2, F64).T


@dataclass
class OracleConfig:
    hidden: int
    ffn: int
    n_experts: int
    top_k: int
    n_group: int = 1
    topk_group: int = 1
    group_score: int = GROUP_MAX
    score_fn: int = SCORE_SOFTMAX
    norm_topk: bool = False
    routed_scale: float = 1.0
    shared_ffn: int = 0
    shared_gated: bool = False
    fp8: bool = False          # FP8 activation quantisation (FP8 and FP4 weight storage)


class OracleWeights:
    """Dequantised weights.  Expert weights are fetched through callables so
    that FP8 experts are dequantised one expert at a time (host RAM stays small
    for DeepSeek-V3: the fp64 copy of all 256 experts would be 90 GB).

    expert(e) -> (W1 [F,H], W3 [F,H], W2 [H,F]) float64
    shared()  -> (W1s, W3s, W2s) or None
    """

    def __init__(self, gate_w, gate_bias, expert_fn, shared_fn=None, shared_gate_w=None):
        self.gate_w = np.asarray(gate_w, F64)
        self.gate_bias = None if gate_bias is None else np.asarray(gate_bias, F64)
        self.expert = expert_fn
        self.shared = shared_fn
        self.shared_gate_w = None if shared_gate_w is None else np.asarray(shared_gate_w, F64)


def shared_expert(x: np.ndarray, W: OracleWeights, cfg: OracleConfig) -> np.ndarray:
    """S_k(I_k): SwiGLU shared FFN on every token, times
    sigmoid(x . w_sg) for Qwen2 (reading R15)."""
    T, H = x.shape
    if cfg.shared_ffn == 0 or W.shared is None:
        return np.zeros((T, H), F64)
    w1, w3, w2 = W.shared()
    ys = swiglu_ffn(x, w1, w3, w2, fp8_act=cfg.fp8)
    if cfg.shared_gated:
        ys = ys * sigmoid(np.asarray(x, F64) @ W.shared_gate_w)[:, None]
    return ys


def routed_expert_outputs(x, idx, W: OracleWeights, cfg: OracleConfig):
    """Y[t, j, :] = FFN_{idx[t,j]}(x[t]) for every selected (t, j)."""
    T, H = x.shape
    k = idx.shape[1]
    Y = np.zeros((T, k, H), F64)
    for e in sorted(set(int(v) for v in idx.reshape(-1))):
        rows, slots = np.nonzero(idx == e)
        w1, w3, w2 = W.expert(e)
        Y[rows, slots] = swiglu_ffn(np.asarray(x, F64)[rows], w1, w3, w2, fp8_act=cfg.fp8)
    return Y


def moe_layer(x, W: OracleWeights, cfg: OracleConfig, residual=None, n_deferred: int = 0,
              deferred_in=None, forced_routing=None):
    """One MoE layer (PAPER.md L219 / L241).

    Returns dict(y, deferred_out, idx, w, counts, offsets, perm_token).
    `residual` stands for the I_k term of Eq. L219 (None -> not added; reading R7).
    `n_deferred` slots (the lowest-weight ones) go to deferred_out (Eq. L241);
    n_deferred = 0 with deferred_in = None is the standard layer (Eq. L219).
    forced_routing = (idx, w) replaces the gate (used for tie-band tokens)."""
    x = np.asarray(x, F64)
    T, H = x.shape
    if forced_routing is None:
        idx, w, _ = route(x, W.gate_w, W.gate_bias, cfg)
    else:
        idx, w = (np.asarray(a) for a in forced_routing)
        w = np.asarray(w, F64)
    counts, offsets, perm_token, _ = count_and_permute(idx, cfg.n_experts)
    Y = routed_expert_outputs(x, idx, W, cfg)
    k = cfg.top_k
    n_imm = k - n_deferred
    y_imm = np.einsum("tj,tjh->th", w[:, :n_imm], Y[:, :n_imm])
    y_def = np.einsum("tj,tjh->th", w[:, n_imm:], Y[:, n_imm:])
    y = shared_expert(x, W, cfg) + y_imm
    if residual is not None:
        y = y + np.asarray(residual, F64)
    if deferred_in is not None:
        y = y + np.asarray(deferred_in, F64)
    return dict(y=y, deferred_out=y_def, idx=idx, w=w, counts=counts, offsets=offsets,
                perm_token=perm_token, Y=Y)


def token_outputs(x_rows, W: OracleWeights, cfg: OracleConfig, n_deferred: int = 0):
    """Oracle for a SAMPLE of tokens of a large layer (the routing of a token
    depends only on that token), used by the full-size parity
    tests: returns moe_layer() restricted to those rows."""
    return moe_layer(x_rows, W, cfg, n_deferred=n_deferred)


def gap_at(sorted_desc: np.ndarray, pos: int) -> float:
    """Gap between the pos-th and (pos+1)-th largest value (0-based pos-1/pos);
    +inf when pos is out of range.  Used to find tie-band tokens."""
    if pos <= 0 or pos >= len(sorted_desc):
        return math.inf
    return float(sorted_desc[pos - 1] - sorted_desc[pos])


def tie_band_tokens(x, W: OracleWeights, cfg: OracleConfig, n_deferred: int = 0,
                    band: float = 1e-5) -> np.ndarray:
    """Tokens whose routing is not decided by more than `band` (north_star:
    "except where the k-th and (k+1)-th scores differ by less than 1e-5"):
    the gap at the top_k boundary of sel, at the topk_group boundary of the
    group scores, and (deferral) at the k - n_def boundary of w."""
    x = np.asarray(x, F64)
    s = scores(router_logits(x, W.gate_w), cfg.score_fn)
    sel = s + (W.gate_bias[None, :] if W.gate_bias is not None else 0.0)
    idx = select_experts(s, W.gate_bias, cfg.n_group, cfg.topk_group, cfg.top_k, cfg.group_score)
    w = combine_weights(s, idx, cfg.norm_topk, cfg.routed_scale)
    _, w = canonical_order(idx, w)
    E = cfg.n_experts
    gsize = E // cfg.n_group
    flagged = []
    for t in range(x.shape[0]):
        row = sel[t].copy()
        tie = False
        if cfg.n_group > 1:
            gs = []
            for g in range(cfg.n_group):
                m = np.sort(row[g * gsize:(g + 1) * gsize])[::-1]
                gs.append(m[0] + m[1] if cfg.group_score == GROUP_TOP2_SUM else m[0])
            gs_sorted = np.sort(np.array(gs))[::-1]
            tie |= gap_at(gs_sorted, cfg.topk_group) < band
            keep = set(_top_indices(np.array(gs), cfg.topk_group))
            for g in range(cfg.n_group):
                if g not in keep:
                    row[g * gsize:(g + 1) * gsize] = -np.inf
        srt = np.sort(row)[::-1]
        tie |= gap_at(srt, cfg.top_k) < band
        if n_deferred > 0:
            tie |= gap_at(w[t], cfg.top_k - n_deferred) < band
        if tie:
            flagged.append(t)
    return np.array(flagged, np.int64)
