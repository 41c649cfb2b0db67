"""GPU parity: the CUDA path through the C ABI vs the CPU oracle on the same
seeded inputs.  Small presets are compared element by element; the full-size
BASELINE.json presets on sampled tokens plus size-independent invariants."""
import numpy as np
import pytest
import torch

from inputs.presets import PRESETS, SMALL, W_FP8
from inputs.synthetic import make_tokens, make_weights
from oracle import moe_oracle as O
from tests.parity import (TOL, check_permutation, check_routing, merged_routing, oracle_cfg, oracle_weights,
                          rel_l2)

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def lib():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
    return moe


def _run(lib, p, T, n_def=0, with_deferred_in=False, residual=False, max_tokens=None, gemv=0, seed_off=0):
    w_cpu = make_weights(p, "cpu")
    x_cpu, r_cpu = make_tokens(p, T, "cpu", offset=seed_off)
    w = w_cpu.to("cuda")
    layer = lib.MoELayer(p, w, max_tokens=max_tokens or max(T, 1), gemv_max_tokens=gemv)
    x = x_cpu.cuda()
    res = r_cpu.cuda() if residual else None
    din = None
    if with_deferred_in:
        din = (torch.randn(T, p.hidden, generator=torch.Generator().manual_seed(5)) * 0.5).to(torch.bfloat16).cuda()
    routing = {}
    out = layer.forward(x, residual=res, n_deferred=n_def, deferred_in=din,
                        want_deferred_out=n_def > 0, routing=routing)
    torch.cuda.synchronize()
    y, dout = (out if isinstance(out, tuple) else (out, None))
    return dict(w_cpu=w_cpu, x=x_cpu, r=r_cpu, din=din, y=y.float().cpu().numpy(),
                dout=None if dout is None else dout.float().cpu().numpy(),
                routing={k: v.cpu().numpy() for k, v in routing.items()}, layer=layer)


def _oracle(p, res, n_def=0, residual=False):
    cfg = oracle_cfg(p)
    W = oracle_weights(p, res["w_cpu"])
    x64 = res["x"].to(torch.float64).numpy()
    ties = O.tie_band_tokens(x64, W, cfg, n_deferred=n_def)
    g = res["routing"]
    idx, w = merged_routing(x64, W, cfg, g["topk_idx"], ties)
    out = O.moe_layer(x64, W, cfg, residual=res["r"].to(torch.float64).numpy() if residual else None,
                      n_deferred=n_def,
                      deferred_in=None if res["din"] is None else res["din"].cpu().to(torch.float64).numpy(),
                      forced_routing=(idx, w))
    return out, ties, idx, w


@pytest.mark.parametrize("name", list(SMALL))
def test_small_layer_parity(lib, name):
    p = SMALL[name]
    T = p.prefill_tokens
    res = _run(lib, p, T)
    out, ties, idx, w = _oracle(p, res)
    g = res["routing"]
    check_routing(g["topk_idx"], g["topk_w"], idx, w, ties, p.routed_scale, p.norm_topk)
    check_permutation(g["expert_counts"], g["perm"], idx, p.n_experts)
    err = rel_l2(res["y"], out["y"])
    assert err <= TOL[p.wtype], f"{name}: rel L2 {err:.3e} > {TOL[p.wtype]}"


@pytest.mark.parametrize("name", ["toy", "v3_s", "v2lite_s", "v2lite_h384"])
@pytest.mark.parametrize("T", [1, 3, 17])
def test_small_decode_shapes(lib, name, T):
    p = SMALL[name]
    res = _run(lib, p, T, max_tokens=64)
    out, ties, idx, w = _oracle(p, res)
    g = res["routing"]
    check_routing(g["topk_idx"], g["topk_w"], idx, w, ties, p.routed_scale, p.norm_topk)
    assert rel_l2(res["y"], out["y"]) <= TOL[p.wtype]


@pytest.mark.parametrize("name", ["v3_s", "qwen2_s", "v25_s"])
@pytest.mark.parametrize("T,gemv", [(4, 4), (8, 8), (8, 0), (6, 1)])
def test_decode_gemv_vs_gemm_paths(lib, name, T, gemv):
    """Weight-streaming decode path (T <= gemv_max_tokens) and the tcgen05 path
    (T above it) both match the oracle (kernel switch by ARI)."""
    p = SMALL[name]
    res = _run(lib, p, T, max_tokens=16, gemv=gemv)
    out, ties, idx, w = _oracle(p, res)
    g = res["routing"]
    check_routing(g["topk_idx"], g["topk_w"], idx, w, ties, p.routed_scale, p.norm_topk)
    assert rel_l2(res["y"], out["y"]) <= TOL[p.wtype]


@pytest.mark.parametrize("name", ["v3_s", "qwen2_s"])
def test_residual_and_deferral(lib, name):
    """Eq. L241 middle case: y = I + S + R^imm + R^def_{k-1}; deferred_out = R^def."""
    p = SMALL[name]
    T = 64
    n_def = 3
    res = _run(lib, p, T, n_def=n_def, with_deferred_in=True, residual=True)
    out, ties, idx, w = _oracle(p, res, n_def=n_def, residual=True)
    keep = np.setdiff1d(np.arange(T), ties)
    assert rel_l2(res["y"][keep], out["y"][keep]) <= TOL[p.wtype]
    assert rel_l2(res["dout"][keep], out["deferred_out"][keep]) <= TOL[p.wtype]


def test_zero_tokens_and_capacity(lib):
    p = SMALL["toy"]
    w = make_weights(p, "cpu").to("cuda")
    layer = lib.MoELayer(p, w, max_tokens=8)
    x = torch.zeros((0, p.hidden), dtype=torch.bfloat16, device="cuda")
    layer.forward(x)                                    # T == 0 is legal
    with pytest.raises(lib.MoEError) as e:
        layer.forward(torch.zeros((9, p.hidden), dtype=torch.bfloat16, device="cuda"))
    assert e.value.status == -6                          # MOE_ERR_CAPACITY
    with pytest.raises(lib.MoEError) as e:
        layer.forward(torch.zeros((4, p.hidden), dtype=torch.bfloat16, device="cuda"), n_deferred=p.top_k,
                      want_deferred_out=True)
    assert e.value.status == -1


def test_non_pow2_scales_rejected(lib):
    p = SMALL["v3_s"]
    w = make_weights(p, "cpu")
    w.w13_scale[0, 0, 0] = 0.3
    with pytest.raises(lib.MoEError) as e:
        lib.MoELayer(p, w.to("cuda"), max_tokens=8)
    assert e.value.status == -2


def test_deterministic(lib):
    p = SMALL["v3_s"]
    a = _run(lib, p, 200)
    b = _run(lib, p, 200)
    np.testing.assert_array_equal(a["y"], b["y"])
    np.testing.assert_array_equal(a["routing"]["perm"], b["routing"]["perm"])


# ------------------------------------------------------------------ full size
def _full(lib, name, T, n_def=0, sample=6):
    p = PRESETS[name]
    w = make_weights(p, "cuda")
    x, _ = make_tokens(p, T, "cuda")
    layer = lib.MoELayer(p, w, max_tokens=T)
    routing = {}
    out = layer.forward(x, n_deferred=n_def, want_deferred_out=n_def > 0, routing=routing)
    torch.cuda.synchronize()
    y = (out[0] if isinstance(out, tuple) else out).float().cpu().numpy()
    g = {k: v.cpu().numpy() for k, v in routing.items()}
    # ---- size-independent invariants ----
    assert g["expert_counts"].sum() == T * p.top_k
    np.testing.assert_array_equal(np.bincount(g["perm"], minlength=T), np.full(T, p.top_k))
    offs = np.concatenate([[0], np.cumsum(g["expert_counts"])])
    for e in range(p.n_experts):
        seg = g["perm"][offs[e]:offs[e + 1]]
        assert np.all(np.diff(seg) > 0)
        assert np.all(np.any(g["topk_idx"][seg] == e, axis=1))
    if p.norm_topk:
        np.testing.assert_allclose(g["topk_w"].sum(1), p.routed_scale, rtol=1e-5)
    # ---- sampled tokens vs the oracle ----
    rng = np.random.default_rng(0)
    rows = np.sort(rng.choice(T, size=min(sample, T), replace=False))
    cfg = oracle_cfg(p)
    W = oracle_weights(p, w)
    x64 = x[rows].cpu().to(torch.float64).numpy()
    ties = O.tie_band_tokens(x64, W, cfg, n_deferred=n_def)
    idx, wts = merged_routing(x64, W, cfg, g["topk_idx"][rows], ties)
    check_routing(g["topk_idx"][rows], g["topk_w"][rows], idx, wts, ties, p.routed_scale, p.norm_topk)
    out_o = O.moe_layer(x64, W, cfg, n_deferred=n_def, forced_routing=(idx, wts))
    err = rel_l2(y[rows], out_o["y"])
    assert err <= TOL[p.wtype], f"{name} T={T}: rel L2 {err:.3e}"
    return err


@pytest.mark.parametrize("name,T", [("v3", 1), ("v25", 4), ("v2lite", 1), ("v2lite", 512), ("qwen2", 2048),
                                    ("v3", 8192), ("qwen2", 1), ("v3", 16)])
def test_full_size_sampled(lib, name, T):
    _full(lib, name, T, sample=4 if T > 1 else 1)


def test_full_v3_decode_deferral(lib):
    _full(lib, "v3", 1, n_def=3, sample=1)


@pytest.mark.parametrize("name,T", [("qwen2_s", 1100), ("v3_s", 2100), ("v25_s", 1500)])
def test_swap_pair_token_tiles(lib, name, T):
    """Swap-AB CTA-pair grouped GEMM with expert segments above one 256-token
    tile (full 256-token tiles + ragged tails padded to 16) vs the oracle."""
    p = SMALL[name]
    res = _run(lib, p, T)
    out, ties, idx, w = _oracle(p, res)
    assert res["routing"]["expert_counts"].max() > 256
    keep = np.setdiff1d(np.arange(T), ties)
    assert rel_l2(res["y"][keep], out["y"][keep]) <= TOL[p.wtype]


@pytest.mark.parametrize("name", ["v3_s", "qwen2_s", "v2lite_s"])
@pytest.mark.parametrize("T", [1, 5, 16])
def test_fused_decode_residual_deferral(lib, name, T):
    """Fused decode stream (umma_decode_fused.cu): Eq. L241 middle case at decode
    sizes -- y = I + S + R^imm + R^def_{k-1}, deferred_out = R^def -- vs the oracle,
    including T = 16 (the N = 16 token operand full)."""
    p = SMALL[name]
    n_def = min(3, p.top_k - 1)
    res = _run(lib, p, T, n_def=n_def, with_deferred_in=True, residual=True, max_tokens=16)
    out, ties, idx, w = _oracle(p, res, n_def=n_def, residual=True)
    keep = np.setdiff1d(np.arange(T), ties)
    assert rel_l2(res["y"][keep], out["y"][keep]) <= TOL[p.wtype]
    assert rel_l2(res["dout"][keep], out["deferred_out"][keep]) <= TOL[p.wtype]


@pytest.mark.parametrize("name", ["v3_s", "qwen2_s"])
def test_fused_decode_matches_chain_and_repeats(lib, name, monkeypatch):
    """The fused decode stream and the two-launch chain (MOE_DECODE_CHAIN=1, read at
    create) agree; repeated fused forwards agree to fp32-atomic rounding (reading R22:
    the chunk partial sums are added in arrival order)."""
    p = SMALL[name]
    T = 7
    w = make_weights(p, "cpu").to("cuda")
    x, r = make_tokens(p, T, "cuda", offset=3)
    fused = lib.MoELayer(p, w, max_tokens=16)
    monkeypatch.setenv("MOE_DECODE_CHAIN", "1")
    chain = lib.MoELayer(p, w, max_tokens=16)
    monkeypatch.delenv("MOE_DECODE_CHAIN")
    ya = fused.forward(x, residual=r).float()
    yb = fused.forward(x, residual=r).float()
    yc = chain.forward(x, residual=r).float()
    torch.cuda.synchronize()
    assert rel_l2(ya.cpu().numpy(), yc.cpu().numpy()) <= TOL[p.wtype]
    # bf16 outputs of two fused runs: at most a rounding step apart
    d = (ya - yb).abs().max().item()
    assert d <= 2 ** -6 * max(1.0, ya.abs().max().item()), d
    fused.close()
    chain.close()


def _tp_sum(lib, layer, x, r, P, n_def=0, din=None):
    """Sum of the P decode-TP partial outputs of one layer (moe_layer_set_decode_tp),
    fp32, i.e. what the all-reduce over P GPUs returns (before its bf16 cast)."""
    y = d = 0
    for rk in range(P):
        layer.set_decode_tp(rk, P)
        out = layer.forward(x, residual=r, n_deferred=n_def, deferred_in=din, want_deferred_out=n_def > 0)
        yo, do = out if isinstance(out, tuple) else (out, None)
        y = y + yo.float()
        if do is not None:
            d = d + do.float()
    layer.set_decode_tp(0, 1)
    torch.cuda.synchronize()
    return y, d


@pytest.mark.parametrize("name,P", [("v3_s", 2), ("qwen2_s", 2), ("v25_s", 2), ("v2lite_s", 2), ("v2lite_s", 3)])
@pytest.mark.parametrize("T", [1, 6, 16])
def test_decode_tp_partials_sum_to_oracle(lib, name, P, T):
    """Decode TP within every expert:
    rank r streams the 128-column chunks c = r (mod P) of every expert; the sum of
    the P partial outputs (residual, deferred_in on rank 0) is the layer's output
    (Eq. L241 with deferral).  v2lite_s at P = 2 gives ranks 2 and 1 routed chunks
    (F/128 = 3): a ragged split."""
    p = SMALL[name]
    n_def = min(2, p.top_k - 1)
    w_cpu = make_weights(p, "cpu")
    x_cpu, r_cpu = make_tokens(p, T, "cpu", offset=11)
    layer = lib.MoELayer(p, w_cpu.to("cuda"), max_tokens=16)
    din = (torch.randn(T, p.hidden, generator=torch.Generator().manual_seed(7)) * 0.5).to(torch.bfloat16)
    routing = {}
    layer.forward(x_cpu.cuda(), routing=routing)       # this layer's routing, for the oracle's tie band
    y, d = _tp_sum(lib, layer, x_cpu.cuda(), r_cpu.cuda(), P, n_def=n_def, din=din.cuda())
    res = dict(w_cpu=w_cpu, x=x_cpu, r=r_cpu, din=din, routing={k: v.cpu().numpy() for k, v in routing.items()})
    out, ties, idx, w = _oracle(p, res, n_def=n_def, residual=True)
    keep = np.setdiff1d(np.arange(T), ties)
    assert rel_l2(y.cpu().numpy()[keep], out["y"][keep]) <= TOL[p.wtype]
    assert rel_l2(d.cpu().numpy()[keep], out["deferred_out"][keep]) <= TOL[p.wtype]
    layer.close()


def test_decode_tp_errors(lib):
    p = SMALL["v3_s"]                                 # F/128 = Fs/128 = 2
    layer = lib.MoELayer(p, make_weights(p, "cpu").to("cuda"), max_tokens=64)
    for rk, P in [(0, 3), (2, 2), (-1, 2), (0, 0)]:
        with pytest.raises(lib.MoEError):
            layer.set_decode_tp(rk, P)
    layer.set_decode_tp(1, 2)
    x, r = make_tokens(p, 40, "cuda")                 # above the fused decode limit: refused, not silently whole
    with pytest.raises(lib.MoEError):
        layer.forward(x, residual=r)
    layer.set_decode_tp(0, 1)
    layer.forward(x, residual=r)
    torch.cuda.synchronize()
    layer.close()


@pytest.mark.parametrize("name,Ps", [("v3", (2, 4, 8, 16)), ("v25", (5, 8, 12)), ("qwen2", (3, 8, 20))])
def test_full_decode_tp_matches_whole(lib, name, Ps):
    """Full-size layers, T = 1 and 4: the P partials sum to the single-GPU forward up
    to the bf16 rounding of each partial.  V3: F/128 = Fs/128 = 16 chunks; V2.5: 12 routed
    chunks (P = 5, 8 give ranks 2-3 or 1-2 chunks: ragged); Qwen2 (BF16, gated shared
    expert): 20 routed and 160 shared chunks."""
    p = PRESETS[name]
    layer = lib.MoELayer(p, make_weights(p, "cuda"), max_tokens=16)
    for P in Ps:
        for T in (1, 4):
            x, r = make_tokens(p, T, "cuda", offset=P)
            whole = layer.forward(x, residual=r).float()
            y, _ = _tp_sum(lib, layer, x, r, P)
            assert rel_l2(y.cpu().numpy(), whole.cpu().numpy()) <= TOL[p.wtype], (P, T)
    layer.close()
