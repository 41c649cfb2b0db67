"""GPU parity: the CUDA path through the C ABI vs the CPU oracle on the same
seeded inputs.  Small presets are compared element by element; the full-size
BASELINE.json presets on sampled tokens plus size-independent invariants."""
import numpy as np
import pytest
import torch

from inputs.presets import PRESETS, SMALL, W_FP8
from inputs.synthetic import make_tokens, make_weights
from oracle import moe_oracle as O
from tests.parity import (TOL, check_output, check_permutation, check_routing, check_tie_fraction, merged_routing,
                          oracle_cfg, oracle_weights, rel_l2)

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def lib():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
    return moe


def _run(lib, p, T, n_def=0, with_deferred_in=False, residual=False, max_tokens=None, gemv=0, seed_off=0):
    return _run_w(lib, p, make_weights(p, "cpu"), T, n_def, with_deferred_in, residual, max_tokens, gemv, seed_off)


def _run_w(lib, p, w_cpu, T, n_def=0, with_deferred_in=False, residual=False, max_tokens=None, gemv=0, seed_off=0):
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
    check_tie_fraction(ties, T)
    check_output(f"small/{name}/T{T}", res["y"], out["y"], TOL[p.wtype], ties=len(ties))


@pytest.mark.parametrize("name", ["toy", "v3_s", "v2lite_s", "v2lite_h384", "v3_s_fp4", "v3_g32"])
@pytest.mark.parametrize("T", [1, 3, 17])
def test_small_decode_shapes(lib, name, T):
    p = SMALL[name]
    res = _run(lib, p, T, max_tokens=64)
    out, ties, idx, w = _oracle(p, res)
    g = res["routing"]
    check_routing(g["topk_idx"], g["topk_w"], idx, w, ties, p.routed_scale, p.norm_topk)
    check_output(f"decode_shapes/{name}/T{T}", res["y"], out["y"], TOL[p.wtype], ties=len(ties))


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
    check_output(f"kernel_switch/{name}/T{T}/gemv{gemv}", res["y"], out["y"], TOL[p.wtype], ties=len(ties))


@pytest.mark.parametrize("name", ["v3_s", "qwen2_s"])
def test_residual_and_deferral(lib, name):
    """Eq. L241 middle case: y = I + S + R^imm + R^def_{k-1}; deferred_out = R^def."""
    p = SMALL[name]
    T = 64
    n_def = 3
    res = _run(lib, p, T, n_def=n_def, with_deferred_in=True, residual=True)
    out, ties, idx, w = _oracle(p, res, n_def=n_def, residual=True)
    keep = np.setdiff1d(np.arange(T), ties)
    check_output(f"deferral/{name}/y", res["y"][keep], out["y"][keep], TOL[p.wtype])
    check_output(f"deferral/{name}/deferred_out", res["dout"][keep], out["deferred_out"][keep], TOL[p.wtype])


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


def test_non_pow2_scales_prefill_rejected(lib):
    """The prefill GEMMs' block-scaled MMAs take UE8M0 scales only (reading R10): a layer
    that can run prefill (max_tokens > the decode limit) refuses other fp32 scales."""
    p = SMALL["v3_s"]
    w = make_weights(p, "cpu")
    w.w13_scale[0, 0, 0] = 0.3
    with pytest.raises(lib.MoEError) as e:
        lib.MoELayer(p, w.to("cuda"), max_tokens=64)
    assert e.value.status == -2
    w.w13_scale[0, 0, 0] = -1.0
    with pytest.raises(lib.MoEError) as e:
        lib.MoELayer(p, w.to("cuda"), max_tokens=8)
    assert e.value.status == -1


@pytest.mark.parametrize("name", ["v3_s", "v3_m"])
@pytest.mark.parametrize("T", [1, 7, 16])
def test_non_pow2_scales_decode(lib, name, T):
    """Arbitrary fp32 128x128 block scales (the released DeepSeek-V3/V2.5 FP8 checkpoints
    store weight_scale_inv as plain fp32): a decode-only layer (max_tokens <= 16) applies
    them exactly in the stream's epilogues; the oracle dequantises with the same scales."""
    p = SMALL[name]
    w = make_weights(p, "cpu")
    g = torch.Generator().manual_seed(3)
    for t in (w.w13_scale, w.w2_scale, w.ws13_scale, w.ws2_scale):
        t.mul_(1.0 + torch.rand(t.shape, generator=g))            # mantissas in [1, 2)
    res = _run_w(lib, p, w, T, max_tokens=16)
    out, ties, idx, wt = _oracle(p, res)
    check_output(f"nonpow2/{name}/T{T}", res["y"], out["y"], TOL[p.wtype], ties=len(ties))


def test_deterministic(lib):
    p = SMALL["v3_s"]
    a = _run(lib, p, 200)
    b = _run(lib, p, 200)
    np.testing.assert_array_equal(a["y"], b["y"])
    np.testing.assert_array_equal(a["routing"]["perm"], b["routing"]["perm"])


# ------------------------------------------------------------------ full size
def _full(lib, name, T, n_def=0, sample=6, rows=None, min_experts=0):
    """Full-size BASELINE.json layer: routing (expert sets and weights), counts
    and the permutation checked on ALL T tokens against the oracle; outputs on
    `sample` tokens (or the given rows) element by element."""
    p = PRESETS[name]
    w = make_weights(p, "cuda")
    x, _ = make_tokens(p, T, "cuda")
    layer = lib.MoELayer(p, w, max_tokens=T)
    routing = {}
    out = layer.forward(x, n_deferred=n_def, want_deferred_out=n_def > 0, routing=routing)
    torch.cuda.synchronize()
    y = (out[0] if isinstance(out, tuple) else out).float().cpu().numpy()
    g = {k: v.cpu().numpy() for k, v in routing.items()}
    cfg = oracle_cfg(p)
    W = oracle_weights(p, w)
    x64 = x.cpu().to(torch.float64).numpy()
    # ---- routing of every token vs the oracle ----
    ties = O.tie_band_tokens(x64, W, cfg, n_deferred=n_def)
    check_tie_fraction(ties, T)
    idx, wts = merged_routing(x64, W, cfg, g["topk_idx"], ties)
    check_routing(g["topk_idx"], g["topk_w"], idx, wts, ties, p.routed_scale, p.norm_topk)
    check_permutation(g["expert_counts"], g["perm"], idx, p.n_experts)
    # ---- sampled tokens' outputs vs the oracle (forced to the merged routing) ----
    if rows is None:
        rng = np.random.default_rng(0)
        rows = np.sort(rng.choice(T, size=min(sample, T), replace=False))
    elif callable(rows):
        rows = rows(idx)
    out_o = O.moe_layer(x64[rows], W, cfg, n_deferred=n_def, forced_routing=(idx[rows], wts[rows]))
    hit = len(set(idx[rows].reshape(-1).tolist()))
    assert hit >= min_experts, (hit, min_experts)
    return check_output(f"full/{name}/T{T}/ndef{n_def}", y[rows], out_o["y"], TOL[p.wtype], ties=len(ties),
                        experts_compared=hit)


@pytest.mark.parametrize("name,T", [("v3", 1), ("v25", 4), ("v2lite", 1), ("v2lite", 512), ("qwen2", 2048),
                                    ("qwen2", 1), ("v3", 16), ("v3_fp4", 1), ("v3_fp4", 16)])
def test_full_size(lib, name, T):
    _full(lib, name, T, sample=8 if T > 1 else 1)


def _greedy_rows(idx, n=64):
    """n tokens chosen so that they reach as many distinct experts as possible:
    first every token that adds an unseen expert, then the lowest remaining ids."""
    rows, seen = [], set()
    for t in range(idx.shape[0]):
        new = set(idx[t].tolist()) - seen
        if new and len(rows) < n:
            rows.append(t)
            seen |= new
    t = 0
    while len(rows) < n:
        if t not in rows:
            rows.append(t)
        t += 1
    return np.array(sorted(rows))


def test_full_v3_prefill_8k_64_tokens(lib):
    """V3 prefill at T = 8192 (the bench workload): routing of all 8192 tokens
    bit-exact (outside the tie band), outputs of 64 tokens chosen greedily so
    that they reach >= 64 distinct experts, compared element by element."""
    _full(lib, "v3", 8192, rows=_greedy_rows, min_experts=64)


def test_full_v3_decode_deferral(lib):
    _full(lib, "v3", 1, n_def=3, sample=1)


@pytest.mark.parametrize("name", ["v3_m", "v3_m_fp4"])
@pytest.mark.parametrize("T", [1, 16, 300])
def test_mid_size_fp8_elementwise(lib, name, T):
    """Mid-size FP8 preset (H = 2048, F = 1024: 16 W13 k-blocks = 4 scale groups,
    8 W2 k-blocks = 2 groups, so both TMEM scale-column sets of the swap GEMM and
    the fused decode stream are used) compared element by element on all tokens."""
    p = SMALL[name]
    res = _run(lib, p, T, max_tokens=max(T, 16))
    out, ties, idx, w = _oracle(p, res)
    g = res["routing"]
    check_tie_fraction(ties, T)
    check_routing(g["topk_idx"], g["topk_w"], idx, w, ties, p.routed_scale, p.norm_topk)
    check_permutation(g["expert_counts"], g["perm"], idx, p.n_experts)
    check_output(f"mid/{name}/T{T}", res["y"], out["y"], TOL[p.wtype], ties=len(ties))


@pytest.mark.parametrize("name", ["v3_m", "v3_m_fp4"])
@pytest.mark.parametrize("T", [2, 5, 8])
def test_mid_size_decode(lib, name, T):
    """Mid-size decode (v3_m: the routed units fill most of the GPU at T >= 2, one CTA per unit)
    element by element against the oracle."""
    p = SMALL[name]
    res = _run(lib, p, T, max_tokens=16)
    out, ties, idx, w = _oracle(p, res)
    g = res["routing"]
    check_routing(g["topk_idx"], g["topk_w"], idx, w, ties, p.routed_scale, p.norm_topk)
    check_output(f"mid_decode/{name}/T{T}", res["y"], out["y"], TOL[p.wtype], ties=len(ties))


@pytest.mark.parametrize("name", ["v3_s", "qwen2_s", "v3_m"])
def test_skewed_routing(lib, name):
    """Imbalanced expert selection: a Zipf-like hot-expert logit
    offset (inputs/synthetic.py skew) gives the hottest expert several times the
    mean load; routing, permutation and outputs still match the oracle."""
    p = SMALL[name]
    T = 400
    w_cpu = make_weights(p, "cpu", skew=1.0)
    x_cpu, _ = make_tokens(p, T, "cpu", skew=1.0, weights=w_cpu)
    layer = lib.MoELayer(p, w_cpu.to("cuda"), max_tokens=T)
    routing = {}
    y = layer.forward(x_cpu.cuda(), routing=routing)
    torch.cuda.synchronize()
    res = dict(w_cpu=w_cpu, x=x_cpu, r=None, din=None, y=y.float().cpu().numpy(), dout=None,
               routing={k: v.cpu().numpy() for k, v in routing.items()})
    out, ties, idx, w = _oracle(p, res)
    g = res["routing"]
    counts = g["expert_counts"]
    # it is skewed: the hottest expert carries well above the mean load (qwen2_s has 16
    # experts and k = 8, so no expert can exceed 2x the mean there)
    assert counts.max() >= min(2.5, 0.8 * p.n_experts / p.top_k) * counts.mean(), (counts.max(), counts.mean())
    check_tie_fraction(ties, T)
    check_routing(g["topk_idx"], g["topk_w"], idx, w, ties, p.routed_scale, p.norm_topk)
    check_permutation(counts, g["perm"], idx, p.n_experts)
    check_output(f"skew/{name}", res["y"], out["y"], TOL[p.wtype], ties=len(ties),
                 hot_over_mean=float(counts.max() / counts.mean()))
    layer.close()


@pytest.mark.parametrize("name,T", [("qwen2_s", 1100), ("v3_s", 2100), ("v25_s", 1500)])
def test_swap_pair_token_tiles(lib, name, T):
    """Swap-AB CTA-pair grouped GEMM with expert segments above one 256-token
    tile (full 256-token tiles + ragged tails padded to 16) vs the oracle."""
    p = SMALL[name]
    res = _run(lib, p, T)
    out, ties, idx, w = _oracle(p, res)
    assert res["routing"]["expert_counts"].max() > 256
    check_tie_fraction(ties, T)
    keep = np.setdiff1d(np.arange(T), ties)
    check_output(f"pair_tiles/{name}/T{T}", res["y"][keep], out["y"][keep], TOL[p.wtype])


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
    check_output(f"fused_deferral/{name}/T{T}/y", res["y"][keep], out["y"][keep], TOL[p.wtype])
    check_output(f"fused_deferral/{name}/T{T}/deferred_out", res["dout"][keep], out["deferred_out"][keep],
                 TOL[p.wtype])


@pytest.mark.parametrize("name", ["v3_s", "qwen2_s"])
def test_fused_decode_repeats(lib, name):
    """Repeated fused decode forwards agree to fp32-atomic rounding (reading R22: the
    chunk partial sums are added in arrival order), and match the prefill-path
    grouped GEMMs (gemv_max_tokens = 1 forces T = 7 onto them) within tolerance."""
    p = SMALL[name]
    T = 7
    w = make_weights(p, "cpu").to("cuda")
    x, r = make_tokens(p, T, "cuda", offset=3)
    fused = lib.MoELayer(p, w, max_tokens=16)
    gemm = lib.MoELayer(p, w, max_tokens=16, gemv_max_tokens=1)
    ya = fused.forward(x, residual=r).float()
    yb = fused.forward(x, residual=r).float()
    yc = gemm.forward(x, residual=r).float()
    torch.cuda.synchronize()
    assert rel_l2(ya.cpu().numpy(), yc.cpu().numpy()) <= TOL[p.wtype]
    # bf16 outputs of two fused runs: at most a rounding step apart
    d = (ya - yb).abs().max().item()
    assert d <= 2 ** -6 * max(1.0, ya.abs().max().item()), d
    fused.close()
    gemm.close()


def test_full_v3_single_token_decode_calls(lib):
    """T = 1 forwards without routing outputs -- the router's one-token select and its
    active-expert list (router.cu route_one_fast) -- on 4 separate tokens, each against the
    oracle with the residual."""
    p = PRESETS["v3"]
    w = make_weights(p, "cuda")
    x, r = make_tokens(p, 4, "cuda", offset=21)
    layer = lib.MoELayer(p, w, max_tokens=16)
    ys = [layer.forward(x[i:i + 1].contiguous(), residual=r[i:i + 1].contiguous()) for i in range(4)]
    torch.cuda.synchronize()
    y = torch.cat(ys).float().cpu().numpy()
    cfg, W = oracle_cfg(p), oracle_weights(p, w)
    x64 = x.cpu().to(torch.float64).numpy()
    ties = O.tie_band_tokens(x64, W, cfg)
    keep = np.setdiff1d(np.arange(4), ties)
    out = O.moe_layer(x64[keep], W, cfg, residual=r.cpu().to(torch.float64).numpy()[keep])
    check_output("full/v3/T1x4/no_routing_out", y[keep], out["y"], TOL[p.wtype], ties=len(ties))
    layer.close()
