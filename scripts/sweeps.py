"""Two sweeps on the DeepSeek-V3 layer:
(1) decode-stream vs grouped-GEMM crossover over T (the paper's AVX-512 vs AMX kernel switch,
    PAPER.md L170): per-forward time of both paths, L2 flushed, CUDA graph of 1 layer;
(2) prefill under skewed routing (hot experts ~4x the mean load, L413) vs balanced, T = 8192:
    the dynamic unit scheduler (L181) against imbalance.
Writes JSON lines and a markdown summary (argv[1])."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
import bench

fw = torch.empty(64 << 20, device="cuda"); fr = torch.zeros(64 << 20, device="cuda"); sink = torch.zeros((), device="cuda")
flush = (fw, fr, sink)
p = PRESETS["v3"]
out = []


def graph_time(layer, x, reps=12):
    y = torch.empty_like(x)
    s = torch.cuda.Stream(); s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(2):
            layer.forward(x, y=y)
    torch.cuda.current_stream().wait_stream(s)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        layer.forward(x, y=y)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for i in range(reps):
        bench.flush_l2(flush)
        e0.record(); g.replay(); e1.record(); e1.synchronize()
        if i >= 2:
            ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    return ts[len(ts) // 2]


SKIP_CROSSOVER = os.environ.get("SWEEP_SKIP_CROSSOVER") == "1"
w = make_weights(p, "cuda")
dec = moe.MoELayer(p, w, max_tokens=64)                    # decode stream for T <= 16
gem = moe.MoELayer(p, w, max_tokens=64, gemv_max_tokens=1)  # grouped GEMM for T >= 2
for T in (() if SKIP_CROSSOVER else (1, 2, 4, 8, 16, 32, 64)):
    x, _ = make_tokens(p, T, "cuda", offset=21)
    r = {"sweep": "decode_vs_gemm", "T": T}
    if T <= 16:
        r["decode_stream_us"] = graph_time(dec, x)
    if T >= 2:
        r["grouped_gemm_us"] = graph_time(gem, x)
    routing = {}
    dec.forward(x, routing=routing)
    r["distinct_experts"] = int((routing["expert_counts"] > 0).sum())
    print(json.dumps(r), flush=True)
    out.append(r)
dec.close(); gem.close()
del w
torch.cuda.empty_cache()

# (3) tokens per expert {1 .. 512} (SURVEY.md §8(d) E1/E4 analog): the grouped-GEMM layer from
#     T = 32 (1 token per expert at k/E = 1/32) to T = 16384 (512 per expert) -- where the
#     tensor-core path becomes compute-efficient (the paper's ARI switch, L170)
peaks = bench.load_peaks()
w = make_weights(p, "cuda")
big = moe.MoELayer(p, w, max_tokens=16384)
for tpe in (() if os.environ.get("SWEEP_SKIP_TPE") == "1" else (1, 2, 4, 8, 16, 32, 64, 128, 256, 512)):
    T = tpe * p.n_experts // p.top_k
    x, _ = make_tokens(p, T, "cuda", offset=33)
    y = torch.empty_like(x)
    times, stages = bench.timed_steps(big, [x], y, 5, 3, flush, profile=True)
    times.sort()
    ms = times[len(times) // 2]
    routing = {}
    big.forward(x, y=y, routing=routing)
    nd = int((routing["expert_counts"] > 0).sum())
    alg = bench.algorithmic(p, T, nd)
    tf = alg["layer_flops"] / (ms * 1e-3) / 1e12
    r = {"sweep": "tokens_per_expert", "tokens_per_expert": tpe, "T": T, "ms": ms, "tokens_per_s": T / (ms * 1e-3),
         "tflops": tf, "tensor_frac": tf / (2 * peaks["bf16_tflops"]),
         "hbm_frac": alg["layer_bytes"] / (ms * 1e-3) / 1e9 / peaks["hbm_gbs"], "distinct_experts": nd,
         "gemm1_ms": stages.get("gemm1_swiglu"), "gemm2_ms": stages.get("gemm2")}
    print(json.dumps(r), flush=True)
    out.append(r)
big.close()
del w
torch.cuda.empty_cache()

for skew in (() if os.environ.get("SWEEP_SKIP_SKEW") == "1" else (0.0, 1.0)):
    w = make_weights(p, "cuda", skew=skew)
    x, _ = make_tokens(p, 8192, "cuda", skew=skew, weights=w if skew > 0 else None)
    layer = moe.MoELayer(p, w, max_tokens=8192)
    y = torch.empty_like(x)
    times, stages = bench.timed_steps(layer, [x], y, 6, 3, flush, profile=True)
    times.sort()
    routing = {}
    layer.forward(x, y=y, routing=routing)
    c = routing["expert_counts"].float()
    r = {"sweep": "prefill_skew", "skew": skew, "ms": times[len(times) // 2], "max_over_mean_load": float(c.max() / c.mean()),
         "experts_hit": int((c > 0).sum()), "gemm1_ms": stages.get("gemm1_swiglu"), "gemm2_ms": stages.get("gemm2")}
    print(json.dumps(r), flush=True)
    out.append(r)
    layer.close()
    del w
    torch.cuda.empty_cache()

with open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/sweeps.md", "w") as f:
    f.write("Decode stream vs grouped GEMM (V3 layer, one forward, CUDA graph, L2 flushed):\n\n"
            "| T | distinct experts | decode stream | grouped GEMM |\n|---|---|---|---|\n")
    for r in out:
        if r["sweep"] == "decode_vs_gemm":
            f.write(f"| {r['T']} | {r['distinct_experts']} | {r.get('decode_stream_us', float('nan')):.1f} us | "
                    f"{r.get('grouped_gemm_us', float('nan')):.1f} us |\n")
    f.write("\nTokens per expert (grouped-GEMM layer, V3, one forward, L2 flushed; tensor fraction of 2 x burst bf16):\n\n"
            "| tokens/expert | T | layer ms | M tokens/s | TFLOP/s | tensor frac | HBM frac |\n|---|---|---|---|---|---|---|\n")
    for r in out:
        if r["sweep"] == "tokens_per_expert":
            f.write(f"| {r['tokens_per_expert']} | {r['T']} | {r['ms']:.3f} | {r['tokens_per_s'] / 1e6:.3f} | "
                    f"{r['tflops']:.0f} | {r['tensor_frac']:.3f} | {r['hbm_frac']:.3f} |\n")
    f.write("\nPrefill, T = 8192, balanced vs skewed routing:\n\n| skew | max/mean expert load | layer ms | GEMM1 ms | GEMM2 ms |\n|---|---|---|---|---|\n")
    for r in out:
        if r["sweep"] == "prefill_skew":
            f.write(f"| {r['skew']} | {r['max_over_mean_load']:.2f} | {r['ms']:.3f} | {r['gemm1_ms']:.3f} | {r['gemm2_ms']:.3f} |\n")
print(open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/sweeps.md").read())
