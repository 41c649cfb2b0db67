"""Pins for the CPU oracle (oracle/moe_oracle.py) against things other than itself:
closed forms / hand-computed values (tests/golden), brute force on tiny inputs,
invariants, library routines (ml_dtypes, numpy, torch.nn.functional) and the
paper's Expert-Deferral equations."""
import itertools
import json
import math
import os

import ml_dtypes
import numpy as np
import pytest
import torch

from oracle import moe_oracle as O

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _hand_weights(score_fn=O.SCORE_SOFTMAX):
    g = json.load(open(os.path.join(GOLD, "hand_2expert.json")))["setup"]
    W1, W3, W2 = (np.array(g[k], float) for k in ("W1", "W3", "W2"))
    W = O.OracleWeights(np.array(g["Wg"]), None, lambda e: (W1[e], W3[e], W2[e]))
    return np.array([g["x"]]), W


def _cfg(**kw):
    base = dict(hidden=2, ffn=1, n_experts=2, top_k=2)
    base.update(kw)
    return O.OracleConfig(**base)


# ---------------------------------------------------------------- hand example
def test_hand_example_closed_forms_match_fixture():
    """The fixture numbers equal their closed forms (guards a typo in the fixture)."""
    e = math.e
    c = json.load(open(os.path.join(GOLD, "hand_2expert.json")))["cases"]
    y0 = 2 * e ** 3 / ((e + 1) * (e * e + 1))
    y1 = -e / (e + 1) ** 2
    assert c["softmax_k2"]["y"] == pytest.approx([y0, y1], rel=1e-15)
    s0 = e / (e + 1)
    w0, w1 = 2.5 * s0 / (s0 + 0.5), 2.5 * 0.5 / (s0 + 0.5)
    silu = lambda v: v / (1 + math.exp(-v))
    assert c["sigmoid_norm_scale2.5_k2"]["w"] == pytest.approx([w0, w1], rel=1e-15)
    assert c["sigmoid_norm_scale2.5_k2"]["y"] == pytest.approx([w0 * silu(2), -w1 * silu(1)], rel=1e-15)


@pytest.mark.parametrize("case,kw,ndef", [
    ("softmax_k2", dict(top_k=2), 0),
    ("softmax_k1", dict(top_k=1), 0),
    ("sigmoid_norm_scale2.5_k2", dict(top_k=2, score_fn=O.SCORE_SIGMOID, norm_topk=True, routed_scale=2.5), 0),
    ("softmax_k2_ndef1", dict(top_k=2), 1),
])
def test_hand_example(case, kw, ndef):
    want = json.load(open(os.path.join(GOLD, "hand_2expert.json")))["cases"][case]
    x, W = _hand_weights()
    out = O.moe_layer(x, W, _cfg(**kw), n_deferred=ndef)
    np.testing.assert_allclose(out["y"][0], want["y"], rtol=1e-14, atol=1e-15)
    if "w" in want:
        np.testing.assert_allclose(out["w"][0], want["w"], rtol=1e-14)
    if "deferred_out" in want:
        np.testing.assert_allclose(out["deferred_out"][0], want["deferred_out"], rtol=1e-14, atol=1e-15)


def test_fig9_immediate_are_highest_scoring():
    """PAPER.md L215, Fig. 9b: top-2 highest-scoring experts immediate, rest deferred."""
    g = json.load(open(os.path.join(GOLD, "fig9_deferral.json")))
    E = len(g["logits"])
    x = np.array([g["logits"]])
    Z = lambda e: (np.zeros((1, E)), np.zeros((1, E)), np.zeros((E, 1)))
    W = O.OracleWeights(np.eye(E), None, Z)
    cfg = O.OracleConfig(hidden=E, ffn=1, n_experts=E, top_k=g["top_k"])
    idx, w, _ = O.route(x, W.gate_w, None, cfg)
    n_imm = g["top_k"] - g["n_deferred"]
    assert list(idx[0, :n_imm]) == g["immediate"]
    assert list(idx[0, n_imm:]) == g["deferred"]


# ---------------------------------------------------------------- top-k selection
def test_topk_bruteforce_toy():
    """k-subset maximising sum(sel) == oracle selection (C(8,2) = 28 subsets)."""
    rng = np.random.default_rng(0)
    for _ in range(200):
        s = O.softmax(rng.normal(size=(1, 8)))
        idx = O.select_experts(s, None, 1, 1, 2, O.GROUP_MAX)
        best = max(itertools.combinations(range(8), 2), key=lambda c: sum(s[0, list(c)]))
        assert set(idx[0]) == set(best)


@pytest.mark.parametrize("rule", [O.GROUP_MAX, O.GROUP_TOP2_SUM])
def test_group_limited_bruteforce(rule):
    """E=16, 4 groups, keep 2, k=4: enumerate C(4,2) group sets, take the set with
    the best group scores, then all C(8,4) expert sets inside it."""
    rng = np.random.default_rng(1)
    E, G, TG, K = 16, 4, 2, 4
    for _ in range(100):
        s = O.sigmoid(rng.normal(size=(1, E)))
        bias = rng.uniform(-0.05, 0.05, size=E)
        sel = s[0] + bias
        def gscore(g):
            m = sorted(sel[g * 4:(g + 1) * 4], reverse=True)
            return m[0] + m[1] if rule == O.GROUP_TOP2_SUM else m[0]
        gsets = list(itertools.combinations(range(G), TG))
        best_g = max(gsets, key=lambda gs: sum(gscore(g) for g in gs))
        allowed = [e for g in best_g for e in range(g * 4, g * 4 + 4)]
        best = max(itertools.combinations(allowed, K), key=lambda c: sum(sel[list(c)]))
        idx = O.select_experts(s, bias, G, TG, K, rule)
        assert set(idx[0]) == set(best)


def test_topk_matches_numpy_argsort():
    rng = np.random.default_rng(2)
    s = O.softmax(rng.normal(size=(50, 64)))
    idx = O.select_experts(s, None, 1, 1, 6, O.GROUP_MAX)
    ref = np.argsort(-s, axis=1, kind="stable")[:, :6]
    np.testing.assert_array_equal(idx, ref)


def test_tie_break_lower_index():
    s = np.array([[0.25, 0.25, 0.25, 0.25]])
    assert list(O.select_experts(s, None, 1, 1, 2, 0)[0]) == [0, 1]


def test_group_ngroup1_reduces_to_plain_topk():
    rng = np.random.default_rng(3)
    s = O.sigmoid(rng.normal(size=(20, 32)))
    b = rng.uniform(-0.05, 0.05, 32)
    a = O.select_experts(s, b, 1, 1, 8, O.GROUP_TOP2_SUM)
    ref = np.argsort(-(s + b), axis=1, kind="stable")[:, :8]
    np.testing.assert_array_equal(a, ref)


# ---------------------------------------------------------------- weights
def test_weights_normalised_and_ordered():
    rng = np.random.default_rng(4)
    cfg = O.OracleConfig(hidden=32, ffn=8, n_experts=16, top_k=4, n_group=4, topk_group=2,
                         group_score=O.GROUP_TOP2_SUM, score_fn=O.SCORE_SIGMOID, norm_topk=True,
                         routed_scale=2.5)
    x = rng.normal(size=(40, 32))
    wg = rng.normal(size=(16, 32)) / 32 ** 0.5
    idx, w, s = O.route(x, wg, rng.uniform(-0.05, 0.05, 16), cfg)
    np.testing.assert_allclose(w.sum(1), 2.5, rtol=1e-12)
    assert np.all(np.diff(w, axis=1) <= 0)
    # combine weights are the normalised UNBIASED top-k scores (north_star invariant)
    sk = np.take_along_axis(s, idx, 1)
    np.testing.assert_allclose(w, 2.5 * sk / sk.sum(1, keepdims=True), rtol=1e-12)


def test_softmax_no_renorm_sum_le_scale():
    rng = np.random.default_rng(5)
    s = O.softmax(rng.normal(size=(30, 20)))
    idx = O.select_experts(s, None, 1, 1, 6, 0)
    w = O.combine_weights(s, idx, False, 16.0)
    assert np.all(w.sum(1) <= 16.0 + 1e-12)
    np.testing.assert_allclose(O.softmax(np.array([[0.0, math.log(3.0)]])), [[0.25, 0.75]])


# ---------------------------------------------------------------- count / permute
def test_count_permute_invariants():
    rng = np.random.default_rng(6)
    T, E, k = 37, 10, 3
    idx = np.stack([rng.choice(E, k, replace=False) for _ in range(T)])
    counts, offsets, perm_t, perm_s = O.count_and_permute(idx, E)
    assert counts.sum() == T * k
    np.testing.assert_array_equal(np.bincount(idx.ravel(), minlength=E), counts)
    np.testing.assert_array_equal(np.bincount(perm_t, minlength=T), np.full(T, k))
    flat = perm_t * k + perm_s
    assert sorted(flat) == list(range(T * k))            # bijection with [0, T*k)
    for e in range(E):
        seg = perm_t[offsets[e]:offsets[e + 1]]
        assert np.all(np.diff(seg) > 0)                  # sorted by t, contiguous
        assert np.all(idx[seg, perm_s[offsets[e]:offsets[e + 1]]] == e)
    inv = np.empty(T * k, np.int64)
    inv[flat] = np.arange(T * k)
    np.testing.assert_array_equal(flat[inv], np.arange(T * k))


# ---------------------------------------------------------------- FP8 numerics
def test_e4m3_decode_all_codes_match_ml_dtypes():
    codes = np.arange(256, dtype=np.uint8)
    ref = codes.view(ml_dtypes.float8_e4m3fn).astype(np.float64)
    got = O.e4m3_decode(codes)
    np.testing.assert_array_equal(np.isnan(got), np.isnan(ref))
    m = ~np.isnan(ref)
    np.testing.assert_array_equal(got[m], ref[m])


def test_e4m3_round_matches_ml_dtypes_rne():
    rng = np.random.default_rng(7)
    v = np.concatenate([rng.normal(size=20000) * 10 ** rng.uniform(-4, 2.6, 20000),
                        # exact midpoints between neighbouring e4m3 values (ties)
                        (O.e4m3_decode(np.arange(1, 126, dtype=np.uint8)) +
                         O.e4m3_decode(np.arange(2, 127, dtype=np.uint8))) / 2]).astype(np.float32)
    v = v[np.abs(v) <= 448]
    ref = v.astype(ml_dtypes.float8_e4m3fn).astype(np.float64)
    np.testing.assert_array_equal(O.e4m3_round(v), ref)
    # satfinite beyond 448
    np.testing.assert_array_equal(O.e4m3_round(np.array([460.0, 479.0, 1e4, -1e4], np.float32)),
                                  [448.0, 448.0, 448.0, -448.0])


def test_ue8m0_scale_properties():
    rng = np.random.default_rng(8)
    a = (rng.uniform(0, 1, 5000) * 10 ** rng.uniform(-6, 6, 5000)).astype(np.float32)
    a = np.concatenate([a, (448.0 * 2.0 ** np.arange(-10, 10)).astype(np.float32)])
    s = O.ue8m0_ceil_scale(a)
    m, _ = np.frexp(s)
    assert np.all(m == 0.5)                               # powers of two
    q = (a / np.float32(448.0)).astype(np.float32)
    assert np.all(s >= q) and np.all(s / 2 < q)          # smallest such power
    assert O.ue8m0_ceil_scale(np.array([0.0], np.float32))[0] == 1.0
    # exact powers keep their exponent: amax = 448 * 2^n -> s = 2^n
    np.testing.assert_array_equal(O.ue8m0_ceil_scale(np.array([448.0, 896.0, 224.0], np.float32)),
                                  [1.0, 2.0, 0.5])


def test_act_quant_blockwise():
    rng = np.random.default_rng(9)
    x = rng.normal(size=(5, 256))
    q = O.act_quant_e4m3(x)
    for r in range(5):
        for b in range(2):
            blk = x[r, b * 128:(b + 1) * 128].astype(np.float32)
            s = O.ue8m0_ceil_scale(np.abs(blk).max())
            ref = (blk / s).astype(ml_dtypes.float8_e4m3fn).astype(np.float64) * s
            np.testing.assert_array_equal(q[r, b * 128:(b + 1) * 128], ref)


def test_fp8_exact_special_case():
    """Weights and activations already on the e4m3 grid with every block amax =
    448 * 2^n: all quantisation is exact, so the FP8 layer equals the
    unquantised layer up to summation order."""
    rng = np.random.default_rng(10)
    H, F = 256, 128
    grid = O.e4m3_decode(np.arange(0, 126, dtype=np.uint8))
    def on_grid(shape, scale):
        v = rng.choice(grid, size=shape) * rng.choice([-1, 1], size=shape)
        v.reshape(-1)[::128] = 448.0     # every 128-block of a row has amax 448
        return v * scale
    x = on_grid((3, H), 1.0)
    w1, w3 = on_grid((F, H), 2.0 ** -9), on_grid((F, H), 2.0 ** -9)
    w2 = on_grid((H, F), 2.0 ** -9)
    # h = silu(g)*u is NOT on the grid, so compare only the first GEMM exactly
    np.testing.assert_array_equal(O.act_quant_e4m3(x), x)
    y_q = O.swiglu_ffn(x, w1, w3, w2, fp8_act=True)
    y = O.swiglu_ffn(x, w1, w3, w2, fp8_act=False)
    h = O.silu(x @ w1.T) * (x @ w3.T)
    y_hq = O.act_quant_e4m3(h) @ w2.T
    np.testing.assert_allclose(y_q, y_hq, rtol=1e-12)
    assert np.linalg.norm(y_q - y) / np.linalg.norm(y) < 0.05


def test_dequant_block128():
    rng = np.random.default_rng(11)
    codes = rng.integers(0, 126, size=(256, 384), dtype=np.uint8)
    scales = 2.0 ** rng.integers(-10, 3, size=(2, 3))
    w = O.dequant_block128(codes, scales)
    ref = codes.view(ml_dtypes.float8_e4m3fn).astype(np.float64)
    for i in range(2):
        for j in range(3):
            np.testing.assert_array_equal(w[i * 128:(i + 1) * 128, j * 128:(j + 1) * 128],
                                          ref[i * 128:(i + 1) * 128, j * 128:(j + 1) * 128] * scales[i, j])


# ---------------------------------------------------------------- expert FFN
def test_single_expert_is_plain_swiglu_mlp():
    """E=1, k=1, softmax -> w=1: the layer is the textbook SwiGLU MLP
    (torch.nn.functional.silu on CPU as the independent reference)."""
    rng = np.random.default_rng(12)
    H, F = 16, 24
    w1, w3, w2 = rng.normal(size=(F, H)), rng.normal(size=(F, H)), rng.normal(size=(H, F))
    x = rng.normal(size=(7, H))
    W = O.OracleWeights(rng.normal(size=(1, H)), None, lambda e: (w1, w3, w2))
    out = O.moe_layer(x, W, O.OracleConfig(hidden=H, ffn=F, n_experts=1, top_k=1))
    xt = torch.tensor(x)
    ref = (torch.nn.functional.silu(xt @ torch.tensor(w1).T) * (xt @ torch.tensor(w3).T)) @ torch.tensor(w2).T
    np.testing.assert_allclose(out["y"], ref.numpy(), rtol=1e-12, atol=1e-12)


def test_k_equals_E_is_dense_mixture():
    rng = np.random.default_rng(13)
    H, F, E = 8, 6, 4
    Ws = [(rng.normal(size=(F, H)), rng.normal(size=(F, H)), rng.normal(size=(H, F))) for _ in range(E)]
    wg = rng.normal(size=(E, H))
    x = rng.normal(size=(5, H))
    W = O.OracleWeights(wg, None, lambda e: Ws[e])
    out = O.moe_layer(x, W, O.OracleConfig(hidden=H, ffn=F, n_experts=E, top_k=E))
    p = torch.softmax(torch.tensor(x @ wg.T), -1).numpy()
    mix = sum(p[:, e:e + 1] * ((torch.nn.functional.silu(torch.tensor(x @ Ws[e][0].T)).numpy()
                                * (x @ Ws[e][1].T)) @ Ws[e][2].T) for e in range(E))
    np.testing.assert_allclose(out["y"], mix, rtol=1e-11, atol=1e-12)


# ---------------------------------------------------------------- Expert Deferral
def _rand_layer(rng, H=16, F=8, E=8, k=4, shared=6):
    Ws = [(rng.normal(size=(F, H)), rng.normal(size=(F, H)), rng.normal(size=(H, F))) for _ in range(E)]
    Sh = (rng.normal(size=(shared, H)), rng.normal(size=(shared, H)), rng.normal(size=(H, shared)))
    W = O.OracleWeights(rng.normal(size=(E, H)), None, lambda e: Ws[e], lambda: Sh)
    cfg = O.OracleConfig(hidden=H, ffn=F, n_experts=E, top_k=k, shared_ffn=shared)
    return W, cfg


def test_deferral_zero_is_standard_layer():
    rng = np.random.default_rng(14)
    W, cfg = _rand_layer(rng)
    x = rng.normal(size=(9, 16)); r = rng.normal(size=(9, 16))
    a = O.moe_layer(x, W, cfg, residual=r)
    b = O.moe_layer(x, W, cfg, residual=r, n_deferred=0, deferred_in=None)
    np.testing.assert_array_equal(a["y"], b["y"])
    assert np.all(b["deferred_out"] == 0)


@pytest.mark.parametrize("ndef", [1, 2, 3])
def test_deferral_split_sums_to_all(ndef):
    """R^imm + R^def = R^all (PAPER.md L219 vs L241, linearity)."""
    rng = np.random.default_rng(15 + ndef)
    W, cfg = _rand_layer(rng)
    x = rng.normal(size=(9, 16))
    a = O.moe_layer(x, W, cfg)
    b = O.moe_layer(x, W, cfg, n_deferred=ndef)
    np.testing.assert_allclose(b["y"] + b["deferred_out"], a["y"], rtol=1e-12, atol=1e-12)


def test_deferral_three_layer_chain_matches_eq_L241():
    """Three layers chained through deferred_in/deferred_out reproduce the case
    formula of PAPER.md L241: k=1 imm only, 1<k<L adds R_{k-1}^def, k=L uses R^all."""
    rng = np.random.default_rng(20)
    layers = [_rand_layer(rng) for _ in range(3)]
    I = rng.normal(size=(6, 16))
    ndef = 2
    # chained through the API semantics
    carry = None
    inp = I
    outs_api = []
    for li, (W, cfg) in enumerate(layers):
        last = li == len(layers) - 1
        out = O.moe_layer(inp, W, cfg, residual=inp, n_deferred=0 if last else ndef, deferred_in=carry)
        outs_api.append(out["y"])
        carry = None if last else out["deferred_out"]
        inp = out["y"]
    # written out from Eq. L241 with explicit R^imm / R^def / R^all
    def parts(W, cfg, X):
        full = O.moe_layer(X, W, cfg)
        Y, w = full["Y"], full["w"]
        S = O.shared_expert(X, W, cfg)
        n_imm = cfg.top_k - ndef
        Rimm = np.einsum("tj,tjh->th", w[:, :n_imm], Y[:, :n_imm])
        Rdef = np.einsum("tj,tjh->th", w[:, n_imm:], Y[:, n_imm:])
        return S, Rimm, Rdef, Rimm + Rdef
    I1 = I
    S1, Ri1, Rd1, _ = parts(*layers[0], I1)
    O1 = I1 + S1 + Ri1
    S2, Ri2, Rd2, _ = parts(*layers[1], O1)
    O2 = O1 + S2 + Rd1 + Ri2
    S3, _, _, Ra3 = parts(*layers[2], O2)
    O3 = O2 + S3 + Rd2 + Ra3
    for got, want in zip(outs_api, [O1, O2, O3]):
        np.testing.assert_allclose(got, want, rtol=1e-11, atol=1e-11)


# ---------------------------------------------------------------- FP8 x / h quantisation through the FFN
def _fp8_selector_ffn(x_row, c=None):
    """H = F = 128.  W1 routes x[0] = 448 (the block amax, so the x scale is 1)
    into every gate column: g = 64 (silu(64) == 64 in fp64).  Case c is None:
    W3 shifts x by one (u_f = x[f+1]) so y_j = e4m3(x[j+1]); case c given:
    u_f = c_f * x[1] with x[1] = 1 so y_j = e4m3(c_j) (the h quantisation;
    amax(h) = 64 * 448 gives the h scale 64 exactly).  W2 = I / 64."""
    H = F = 128
    w1 = np.zeros((F, H)); w1[:, 0] = 1.0 / 7.0
    w3 = np.zeros((F, H))
    if c is None:
        for f in range(F - 1):
            w3[f, f + 1] = 1.0
    else:
        w3[:len(c), 1] = c
    w2 = np.eye(H) / 64.0
    return O.swiglu_ffn(np.array([x_row]), w1, w3, w2, fp8_act=True)[0], \
        O.swiglu_ffn(np.array([x_row]), w1, w3, w2, fp8_act=False)[0]


def test_fp8_x_quantised_inside_swiglu_ffn_off_grid():
    """Off-grid x through swiglu_ffn(fp8_act=True): every value is rounded to its
    hand-computed e4m3 neighbour (RNE, scale 1 because amax = 448): 1.07 -> 1.125,
    1.0625 -> 1.0 (tie to even), -3.3 -> -3.25, 0.013 -> 7 * 2^-9 (subnormal),
    300 -> 288.  An oracle that skipped the x quantisation returns the raw values."""
    x = np.zeros(128)
    x[0] = 448.0
    x[1:6] = [1.07, 1.0625, -3.3, 0.013, 300.0]
    yq, y = _fp8_selector_ffn(x)
    want = [1.125, 1.0, -3.25, 7 * 2.0 ** -9, 288.0]
    np.testing.assert_allclose(yq[:5], want, rtol=1e-12, atol=0)
    np.testing.assert_allclose(y[:5], x[1:6], rtol=1e-12)           # unquantised: the raw x
    assert np.all(np.abs(yq[:5] - y[:5]) > 1e-4)
    assert np.all(yq[5:] == 0)


def test_fp8_h_quantised_inside_swiglu_ffn_off_grid():
    """x on the grid, h = 64 * c off the grid: y_j = e4m3(c_j) * 64 / 64 with the
    h scale 64 = 2^ceil(log2(64 * 448 / 448)) (exact power of two keeps its exponent)."""
    x = np.zeros(128)
    x[0], x[1] = 448.0, 1.0
    c = [1.07, 1.0625, -3.3, 0.013, 300.0, 448.0]
    yq, y = _fp8_selector_ffn(x, c=c)
    np.testing.assert_allclose(yq[:6], [1.125, 1.0, -3.25, 7 * 2.0 ** -9, 288.0, 448.0], rtol=1e-12, atol=0)
    np.testing.assert_allclose(y[:6], c, rtol=1e-12)
    assert np.all(yq[6:] == 0)


def test_fp8_quantisation_reaches_moe_layer():
    """The same selector expert as the only routed expert (E = 1, k = 1, softmax
    -> w = 1) and as the shared expert: moe_layer(fp8=True) returns 2 x e4m3(x)."""
    H = 128
    x = np.zeros((1, H))
    x[0, 0] = 448.0
    x[0, 1:6] = [1.07, 1.0625, -3.3, 0.013, 300.0]
    w1 = np.zeros((H, H)); w1[:, 0] = 1.0 / 7.0
    w3 = np.zeros((H, H))
    for f in range(H - 1):
        w3[f, f + 1] = 1.0
    w2 = np.eye(H) / 64.0
    W = O.OracleWeights(np.zeros((1, H)), None, lambda e: (w1, w3, w2), lambda: (w1, w3, w2))
    cfg = O.OracleConfig(hidden=H, ffn=H, n_experts=1, top_k=1, shared_ffn=H, fp8=True)
    y = O.moe_layer(x, W, cfg)["y"][0]
    np.testing.assert_allclose(y[:5], 2 * np.array([1.125, 1.0, -3.25, 7 * 2.0 ** -9, 288.0]), rtol=1e-12)


# ---------------------------------------------------------------- tie band (north_star 1e-5)
def test_gap_at():
    v = np.array([5.0, 3.0, 2.5, 2.5])
    assert O.gap_at(v, 1) == 2.0
    assert O.gap_at(v, 2) == 0.5
    assert O.gap_at(v, 3) == 0.0
    assert O.gap_at(v, 0) == math.inf and O.gap_at(v, 4) == math.inf


def _tie_layer(s_rows, bias=None, **kw):
    """Tokens whose sigmoid scores are exactly `s_rows` (Wg = I, x = logit(s))."""
    s = np.array(s_rows, float)
    E = s.shape[1]
    x = np.log(s) - np.log1p(-s)
    W = O.OracleWeights(np.eye(E), None if bias is None else np.array(bias, float),
                        lambda e: (np.zeros((1, E)),) * 2 + (np.zeros((E, 1)),))
    base = dict(hidden=E, ffn=1, n_experts=E, score_fn=O.SCORE_SIGMOID)
    base.update(kw)
    return x, W, O.OracleConfig(**base)


def test_tie_band_tokens_flags_exactly_the_hand_built_ties():
    """E = 8 in 4 groups of 2, keep 2 groups (top-2-sum score), k = 3.
      0: k-boundary sel gap 5e-6 (0.7 vs 0.699995)          -> flagged
      1: k-boundary gap 2e-5                                 -> not flagged
      2: group scores 0.9 vs 0.899996 at the topk_group boundary -> flagged
      3: group gap 1.5e-5                                    -> not flagged
      4: w[1] - w[2] = 4e-6 at k - n_def = 2 (n_def = 1 only) -> flagged iff n_def = 1
      5: every gap large                                     -> never flagged"""
    rows = [
        [0.9, 0.8, 0.7, 0.699995, 0.1, 0.1, 0.05, 0.05],
        [0.9, 0.8, 0.7, 0.69998, 0.1, 0.1, 0.05, 0.05],
        [0.9, 0.8, 0.6, 0.3, 0.5, 0.399996, 0.05, 0.05],
        [0.9, 0.8, 0.6, 0.3, 0.5, 0.399985, 0.05, 0.05],
        [0.9, 0.8, 0.799996, 0.2, 0.05, 0.05, 0.01, 0.01],
        [0.9, 0.5, 0.3, 0.1, 0.2, 0.15, 0.02, 0.01],
    ]
    x, W, cfg = _tie_layer(rows, n_group=4, topk_group=2, group_score=O.GROUP_TOP2_SUM, top_k=3)
    assert list(O.tie_band_tokens(x, W, cfg)) == [0, 2]
    assert list(O.tie_band_tokens(x, W, cfg, n_deferred=1)) == [0, 2, 4]
    # the group gap of token 2 is what flags it: with one group the token is clean
    x1, W1, cfg1 = _tie_layer(rows[2:4], top_k=3)
    assert list(O.tie_band_tokens(x1, W1, cfg1)) == []


def test_tie_band_uses_biased_selection_scores():
    """The k boundary is measured on sel = s + bias, not on s: a bias of 0.099996
    on expert 3 puts it 4e-6 below expert 2's 0.7."""
    rows = [[0.9, 0.8, 0.7, 0.6, 0.1, 0.1, 0.05, 0.05]]
    x, W, cfg = _tie_layer(rows, bias=[0, 0, 0, 0.099996, 0, 0, 0, 0], top_k=3)
    assert list(O.tie_band_tokens(x, W, cfg)) == [0]
    x, W, cfg = _tie_layer(rows, top_k=3)
    assert list(O.tie_band_tokens(x, W, cfg)) == []


def test_tie_band_group_max_rule():
    """DeepSeek-V2.5 group score = max: groups 2 (0.6) and 3 (0.599996) tie at the
    topk_group = 2 boundary."""
    rows = [[0.9, 0.1, 0.6, 0.1, 0.599996, 0.1, 0.05, 0.05],
            [0.9, 0.1, 0.6, 0.1, 0.59, 0.1, 0.05, 0.05]]
    x, W, cfg = _tie_layer(rows, n_group=4, topk_group=2, group_score=O.GROUP_MAX, top_k=2)
    assert list(O.tie_band_tokens(x, W, cfg)) == [0]


# ---------------------------------------------------------------- FP4 (e2m1) weights (NEXT-3)
def test_e2m1_decode_all_codes_match_ml_dtypes():
    codes = np.arange(16, dtype=np.uint8)
    ref = codes.view(ml_dtypes.float4_e2m1fn).astype(np.float64)
    np.testing.assert_array_equal(O.e2m1_decode(codes), ref)
    # the OCP table, by hand: magnitudes 0, 0.5, 1, 1.5, 2, 3, 4, 6 and their negatives
    assert list(O.e2m1_decode(codes[:8])) == [0, 0.5, 1, 1.5, 2, 3, 4, 6]
    assert list(O.e2m1_decode(codes[8:])) == [-0.0, -0.5, -1, -1.5, -2, -3, -4, -6]


def test_unpack_fp4_nibble_order():
    """element 2i is the LOW nibble of byte i: 0x21 -> codes (1, 2) -> (0.5, 1.0)."""
    np.testing.assert_array_equal(O.unpack_fp4(np.array([[0x21, 0xF7]], np.uint8)), [[1, 2, 7, 15]])
    np.testing.assert_array_equal(O.e2m1_decode(O.unpack_fp4(np.array([0x21], np.uint8))), [0.5, 1.0])


def test_dequant_fp4_block128():
    rng = np.random.default_rng(12)
    codes = rng.integers(0, 16, size=(256, 384), dtype=np.uint8)
    packed = (codes[:, 0::2] | (codes[:, 1::2] << 4)).astype(np.uint8)
    scales = 2.0 ** rng.integers(-8, 3, size=(2, 3))
    w = O.dequant_fp4_block128(packed, scales)
    ref = codes.view(ml_dtypes.float4_e2m1fn).astype(np.float64)
    for i in range(2):
        for j in range(3):
            blk = (slice(128 * i, 128 * (i + 1)), slice(128 * j, 128 * (j + 1)))
            np.testing.assert_array_equal(w[blk], ref[blk] * scales[i, j])


def test_fp4_weights_equal_their_e4m3_expansion():
    """e2m1 is a subset of e4m3: the FP4 layer equals the FP8 layer built from the
    same values (the library's prefill path runs on that expansion), exactly."""
    rng = np.random.default_rng(13)
    codes = rng.integers(0, 16, size=(128, 256), dtype=np.uint8)
    packed = (codes[:, 0::2] | (codes[:, 1::2] << 4)).astype(np.uint8)
    vals = O.e2m1_decode(codes)
    e4 = vals.astype(np.float32).astype(ml_dtypes.float8_e4m3fn).view(np.uint8)
    s = np.array([[0.25, 2.0]])
    np.testing.assert_array_equal(O.dequant_fp4_block128(packed, s), O.dequant_block128(e4, s))
