"""Helpers shared by the GPU parity tests: build the oracle's view of the same
seeded weights, merge tie-band routing, and compare GPU results with the oracle.
(Test infrastructure: imports oracle/, never imported by the product path.)"""
from __future__ import annotations

import numpy as np
import torch

from inputs.presets import W_FP4, W_FP8
from oracle import moe_oracle as O

TOL = {0: 5e-3, 1: 2e-2, 2: 5e-3, 3: 2e-2}   # north_star: BF16 rel-L2 <= 5e-3, FP8 <= 2e-2 (F32 toy: BF16 bar;
                                             # FP4 weights: e4m3 activations as FP8, the FP8 bar)


def oracle_cfg(p) -> O.OracleConfig:
    return O.OracleConfig(hidden=p.hidden, ffn=p.ffn, n_experts=p.n_experts, top_k=p.top_k,
                          n_group=p.n_group, topk_group=p.topk_group, group_score=p.group_score,
                          score_fn=p.score_fn, norm_topk=bool(p.norm_topk), routed_scale=p.routed_scale,
                          shared_ffn=p.shared_ffn, shared_gated=bool(p.shared_gated),
                          fp8=p.wtype in (W_FP8, W_FP4))


def _f64(t):
    return t.detach().to("cpu").to(torch.float64).numpy()


def oracle_weights(p, w) -> O.OracleWeights:
    """Dequantised fp64 weights, fetched per expert (works for CPU or GPU tensors)."""
    F, Fs = p.ffn, p.shared_ffn
    fp8 = p.wtype in (W_FP8, W_FP4)

    def deq(codes, scales):
        if p.wtype == W_FP4:
            return O.dequant_fp4_block128(codes.detach().cpu().numpy(), scales.detach().cpu().numpy())
        if fp8:
            return O.dequant_block128(codes.detach().cpu().numpy(), scales.detach().cpu().numpy())
        return _f64(codes)

    def expert(e):
        w13 = deq(w.w13[e], w.w13_scale[e] if fp8 else None)
        return w13[:F], w13[F:], deq(w.w2[e], w.w2_scale[e] if fp8 else None)

    shared = None
    if Fs:
        def shared():
            a = deq(w.ws13, w.ws13_scale)
            return a[:Fs], a[Fs:], deq(w.ws2, w.ws2_scale)
    return O.OracleWeights(_f64(w.gate_w), None if w.gate_bias is None else _f64(w.gate_bias), expert, shared,
                           None if w.shared_gate_w is None else _f64(w.shared_gate_w))


def _valid_in_band(sel_t, gpu_set, orc_set, cfg, band=1e-5):
    """A tie-band token's GPU expert set is a valid choice: every chosen expert is
    within `band` of the oracle's k-th selection score, and (group-limited
    routing) the chosen experts span at most topk_group groups, each within `band`
    of the oracle's topk_group-th group score."""
    kth = np.sort(sel_t[orc_set])[0]
    if not np.all(sel_t[gpu_set] >= kth - band):
        return False
    if cfg.n_group > 1:
        gsize = cfg.n_experts // cfg.n_group
        gs = []
        for g in range(cfg.n_group):
            m = np.sort(sel_t[g * gsize:(g + 1) * gsize])[::-1]
            gs.append(m[0] + m[1] if cfg.group_score == O.GROUP_TOP2_SUM else m[0])
        gs = np.array(gs)
        gth = np.sort(gs)[::-1][cfg.topk_group - 1]
        used = sorted(set(int(e) // gsize for e in gpu_set))
        if len(used) > cfg.topk_group or not np.all(gs[used] >= gth - band):
            return False
    return True


def merged_routing(x64, W, cfg, gpu_idx, ties):
    """Oracle routing for every token, except tie-band tokens which take the
    GPU's expert set (checked valid within the band, group limit included) with
    oracle weights."""
    s = O.scores(O.router_logits(x64, W.gate_w), cfg.score_fn)
    idx = O.select_experts(s, W.gate_bias, cfg.n_group, cfg.topk_group, cfg.top_k, cfg.group_score)
    if len(ties):
        sel = s + (W.gate_bias[None, :] if W.gate_bias is not None else 0.0)
        for t in ties:
            g = np.array(sorted(gpu_idx[t]))
            assert len(set(g.tolist())) == cfg.top_k
            assert _valid_in_band(sel[t], g, idx[t], cfg), f"token {t}: GPU choice outside the tie band"
            idx[t] = g
    w = O.combine_weights(s, idx, cfg.norm_topk, cfg.routed_scale)
    idx, w = O.canonical_order(idx, w)
    return idx, w


MAX_TIE_FRAC = 0.01   # tie-exempt tokens allowed per case (survey measured <= 0.6 %)


def check_tie_fraction(ties, T):
    assert len(ties) <= max(1, MAX_TIE_FRAC * T), f"{len(ties)} of {T} tokens tie-exempt (> 1 %)"


def per_token_max_rel(a, b) -> float:
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    num = np.linalg.norm(a - b, axis=1)
    den = np.maximum(np.linalg.norm(b, axis=1), 1e-30)
    return float((num / den).max()) if len(a) else 0.0


def log_case(name, **kw):
    """Achieved errors of one parity case: one JSON line appended to
    $PARITY_LOG (default gpurun_out/parity_log.jsonl) and printed."""
    import json
    import os
    path = os.environ.get("PARITY_LOG", os.path.join(os.path.dirname(os.path.dirname(__file__)), "gpurun_out",
                                                     "parity_log.jsonl"))
    rec = {"case": name, **{k: (float(v) if isinstance(v, (float, np.floating)) else v) for k, v in kw.items()}}
    print("PARITY", json.dumps(rec))
    try:
        os.makedirs(os.path.dirname(path), exist_ok=True)
        with open(path, "a") as f:
            f.write(json.dumps(rec) + "\n")
    except OSError:
        pass


def check_output(name, y, ref, tol, **extra):
    """rel-L2 over the compared rows (north_star bar) plus the max per-token rel
    error (logged; held to 5x the bar), both recorded with log_case."""
    err = rel_l2(y, ref)
    tok = per_token_max_rel(y, ref)
    log_case(name, rel_l2=err, max_token_rel=tok, tol=tol, rows=int(np.asarray(y).shape[0]), **extra)
    assert err <= tol, f"{name}: rel L2 {err:.3e} > {tol}"
    assert tok <= 5 * tol, f"{name}: max per-token rel error {tok:.3e} > {5 * tol}"
    return err


def rel_l2(a, b) -> float:
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    return float(np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-30))


def check_routing(gpu_idx, gpu_w, orc_idx, orc_w, ties, routed_scale, norm):
    T = gpu_idx.shape[0]
    keep = np.setdiff1d(np.arange(T), ties)
    # bit-exact expert sets outside the tie band
    np.testing.assert_array_equal(np.sort(gpu_idx[keep], 1), np.sort(orc_idx[keep], 1))
    # canonical order on the GPU side: weights non-increasing
    assert np.all(np.diff(gpu_w, axis=1) <= 0)
    # weights per expert
    for t in keep[:4096]:
        og = dict(zip(orc_idx[t].tolist(), orc_w[t].tolist()))
        for e, wv in zip(gpu_idx[t].tolist(), gpu_w[t].tolist()):
            assert abs(wv - og[e]) <= 1e-5 * max(1.0, abs(og[e])), (t, e, wv, og[e])
    if norm:
        np.testing.assert_allclose(gpu_w.sum(1), routed_scale, rtol=1e-5)


def check_permutation(gpu_counts, gpu_perm, idx, n_experts):
    counts, offsets, perm_t, _ = O.count_and_permute(idx, n_experts)
    np.testing.assert_array_equal(gpu_counts, counts)
    np.testing.assert_array_equal(gpu_perm, perm_t)
