"""Decode latency per layer: one CUDA graph over a chain of L distinct layers
(x_{i+1} = y_i = x_i + moe_i(x_i)), L2 flushed before each replay -- A/B
experiments (MOE_DECODE_CHAIN=1 selects the two-launch chain).
python scripts/decode_ab.py v3 1,4,16 [L]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe

cfg = sys.argv[1] if len(sys.argv) > 1 else "v3"
Ts = [int(t) for t in (sys.argv[2] if len(sys.argv) > 2 else "1,4,16").split(",")]
L = int(sys.argv[3]) if len(sys.argv) > 3 else 1
p = PRESETS[cfg]
w = make_weights(p, "cuda")
layers = [moe.MoELayer(p, w, max_tokens=16) for _ in range(L)]
del w
torch.cuda.empty_cache()
fw = torch.empty(64 << 20, device="cuda")
fr = torch.zeros(64 << 20, device="cuda")
sink = torch.zeros((), device="cuda")
out = {"config": cfg, "layers": L, "chain": os.environ.get("MOE_DECODE_CHAIN", "0")}
for T in Ts:
    xs, _ = make_tokens(p, 24 * T, "cuda", offset=77)
    rows = [xs[i * T:(i + 1) * T].contiguous() for i in range(24)]
    bufs = [rows[0].clone(), torch.empty_like(rows[0])]
    def fwd():
        for i, l in enumerate(layers):
            a, b = bufs[i % 2], bufs[(i + 1) % 2]
            l.forward(a, residual=a, y=b)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(2):
            bufs[0].copy_(rows[0]); fwd()
    torch.cuda.current_stream().wait_stream(s)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        fwd()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for i in range(24):
        bufs[0].copy_(rows[i])
        fw.zero_(); torch.sum(fr, 0, out=sink)
        e0.record(); g.replay(); e1.record(); e1.synchronize()
        if i >= 4:
            ts.append(e0.elapsed_time(e1) * 1e3 / L)
    ts.sort()
    out[f"T{T}_us_median"] = round(ts[len(ts) // 2], 2)
    out[f"T{T}_us_min"] = round(ts[0], 2)
print(json.dumps(out))
