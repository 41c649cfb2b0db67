"""Every BASELINE.json configuration on one B200: prefill tokens/s + TFLOP/s and decode
us/layer + GB/s (CUDA graph over a chain of 8 distinct layers, L2 flushed), each against the
measured peaks (tensor: the burst bf16 figure, x 2 for FP8 -- as bench.py); decode also with
chained Expert Deferral (moe_layer_forward_chained) and the V3 layer with 4-bit (e2m1) weights.
Writes one JSON line per measurement and a markdown table (argv[1])."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
import bench

peaks = bench.load_peaks()
fw = torch.empty(64 << 20, device="cuda"); fr = torch.zeros(64 << 20, device="cuda"); sink = torch.zeros((), device="cuda")
flush = (fw, fr, sink)
rows_out = []


def prefill(name, T):
    p = PRESETS[name]
    w = make_weights(p, "cuda")
    x, _ = make_tokens(p, T, "cuda")
    layer = moe.MoELayer(p, w, max_tokens=T)
    y = torch.empty_like(x)
    times, _ = bench.timed_steps(layer, [x], y, 8, 3, flush, profile=False)
    times.sort()
    ms = times[len(times) // 2]
    routing = {}
    layer.forward(x, y=y, routing=routing)
    nd = int((routing["expert_counts"] > 0).sum())
    alg = bench.algorithmic(p, T, nd)
    fp8 = p.wtype in (1, 3)
    peak_tf = (2 if fp8 else 1) * peaks["bf16_tflops"]
    tf = alg["layer_flops"] / (ms * 1e-3) / 1e12
    gbs = alg["layer_bytes"] / (ms * 1e-3) / 1e9
    r = {"config": name, "phase": "prefill", "T": T, "ms": ms, "tokens_per_s": T / (ms * 1e-3), "tflops": tf,
         "tensor_frac": tf / peak_tf, "gbs": gbs, "hbm_frac": gbs / peaks["hbm_gbs"], "distinct_experts": nd,
         "dtype": {0: "bf16", 1: "e4m3", 2: "f32", 3: "e2m1 weights"}[p.wtype]}
    layer.close()
    del w
    torch.cuda.empty_cache()
    return r


def decode(name, T, L=8, n_def=0, cyclic=False):
    p = PRESETS[name]
    w = make_weights(p, "cuda")
    layers = [moe.MoELayer(p, w, max_tokens=16) for _ in range(L)]
    del w
    torch.cuda.empty_cache()
    xs, _ = make_tokens(p, 16 * T, "cuda", offset=11)
    rows = [xs[i * T:(i + 1) * T].contiguous() for i in range(16)]
    bufs = [rows[0].clone(), torch.empty_like(rows[0])]
    dbufs = [torch.zeros_like(rows[0]), torch.zeros_like(rows[0])]

    first = [True]

    def step():
        # cyclic: every layer defers and layer 0 takes the last layer's deferred experts of the
        # previous replay (a deep stack's steady state, no end layers)
        prev = layers[-1] if (cyclic and not first[0]) else None
        for i, l in enumerate(layers):
            a, b = bufs[i % 2], bufs[(i + 1) % 2]
            if n_def:       # Eq. L241 across the chain: layer i computes layer i-1's deferred experts
                l.forward_chained(a, residual=a, n_deferred=n_def if (cyclic or i < L - 1) else 0, prev=prev, y=b)
                prev = l
            else:
                l.forward(a, residual=a, y=b)
        first[0] = False
    s = torch.cuda.Stream(); s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(2):
            bufs[0].copy_(rows[0]); step()
    torch.cuda.current_stream().wait_stream(s)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        step()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for i in range(16):
        bufs[0].copy_(rows[i])
        bench.flush_l2(flush)
        e0.record(); g.replay(); e1.record(); e1.synchronize()
        if i >= 3:
            ts.append(e0.elapsed_time(e1) * 1e3 / L)
    ts.sort()
    us = ts[len(ts) // 2]
    # algorithmic bytes: the distinct experts of EVERY layer of the chain (its tokens drift along
    # x_{i+1} = x_i + moe_i(x_i), so at T > 1 later layers may hit fewer experts than layer 0),
    # from an eager plain pass over the same chain; deferral moves the same union per layer
    nds = []
    for i in (3, 9, 15):                # inputs of timed replays
        a = rows[i].clone()
        for l in layers:
            routing = {}
            b = l.forward(a, residual=a, routing=routing)
            nds.append(int((routing["expert_counts"] > 0).sum()))
            a = b
    nd = sum(nds) / len(nds)
    alg = {"layer_bytes": sum(bench.algorithmic(p, T, n)["layer_bytes"] for n in nds) / len(nds)}
    gbs = alg["layer_bytes"] / (us * 1e-6) / 1e9
    r = {"config": name, "phase": "decode", "T": T, "n_deferred": n_def, "layers_in_graph": L, "us_per_layer": us,
         "gbs": gbs, "hbm_frac": gbs / peaks["hbm_gbs"], "distinct_experts": nd, "layer_bytes": alg["layer_bytes"]}
    for l in layers:
        l.close()
    torch.cuda.empty_cache()
    return r


# decode rows: (n_def, cyclic) -- cyclic = the steady state of a deep stack (every layer defers)
plan = [("prefill", "v2lite", 512, 0), ("decode", "v2lite", 1, 0), ("decode", "v2lite", 1, 3), ("cyc", "v2lite", 1, 3),
        ("prefill", "qwen2", 2048, 0), ("decode", "qwen2", 1, 0), ("decode", "qwen2", 1, 3), ("cyc", "qwen2", 1, 3),
        ("prefill", "v25", 4096, 0), ("decode", "v25", 4, 0), ("decode", "v25", 4, 3), ("cyc", "v25", 4, 3),
        ("prefill", "v3", 8192, 0), ("decode", "v3", 1, 0), ("decode", "v3", 1, 3), ("cyc", "v3", 1, 3),
        ("decode", "v3", 1, 6),
        ("prefill", "v3_fp4", 8192, 0), ("decode", "v3_fp4", 1, 0), ("decode", "v3_fp4", 1, 3), ("cyc", "v3_fp4", 1, 3)]
for kind, name, T, nd_ in plan:
    r = prefill(name, T) if kind == "prefill" else decode(name, T, n_def=nd_, cyclic=kind == "cyc")
    r["cyclic"] = kind == "cyc"
    print(json.dumps(r), flush=True)
    rows_out.append(r)

with open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/all_configs.md", "w") as f:
    f.write("| config | phase | T | time | throughput | roofline |\n|---|---|---|---|---|---|\n")
    for r in rows_out:
        if r["phase"] == "prefill":
            f.write(f"| {r['config']} ({r['dtype']}) | prefill | {r['T']} | {r['ms']:.3f} ms | {r['tokens_per_s']/1e6:.3f} M tok/s, "
                    f"{r['tflops']:.0f} TFLOP/s | {r['tensor_frac']*100:.1f} % of tensor peak, {r['hbm_frac']*100:.1f} % of HBM "
                    f"({r['distinct_experts']} experts hit) |\n")
        else:
            f.write(f"| {r['config']} | decode{' n_def=%d' % r['n_deferred'] if r['n_deferred'] else ''}"
                    f"{' steady state (cyclic chain)' if r.get('cyclic') else ''} | {r['T']} | "
                    f"{r['us_per_layer']:.1f} us/layer | {r['gbs']:.0f} GB/s | {r['hbm_frac']*100:.1f} % of HBM "
                    f"({r['distinct_experts']:.1f} experts/layer, {r['layer_bytes']/1e6:.1f} MB) |\n")
print(open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/all_configs.md").read())
