"""A/B of decode variants on the same GPU, interleaved to cancel clock drift:
the 8-layer chained CUDA graph (distinct V3 layers, L2 flushed before each replay),
  plain     -- moe_layer_forward per layer
  deferral  -- moe_layer_forward_chained, n_def = 3 (last layer 0)
  deferral3_cyclic -- every layer defers; layer 0 takes the last layer's deferred experts of the
              previous replay (the steady state of a deep stack: no end layers)
Prints per-layer µs for each variant and round.  python scripts/decode_ab.py CONFIG ROUNDS [TOKENS]"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe

cfg = sys.argv[1] if len(sys.argv) > 1 else "v3"
NL, ROUNDS, STEPS = 8, int(sys.argv[2]) if len(sys.argv) > 2 else 4, 10
p = PRESETS[cfg]
w = make_weights(p, "cuda")
layers = [moe.MoELayer(p, w, max_tokens=16) for _ in range(NL)]
TOK = int(sys.argv[3]) if len(sys.argv) > 3 else 1          # tokens per decode step
xd, _ = make_tokens(p, max(4, TOK), "cuda", offset=1000)
x0 = xd[:TOK].contiguous()
bufs = [x0.clone(), torch.empty_like(x0)]
flush = (torch.empty(64 << 20, device="cuda"), torch.zeros(64 << 20, device="cuda"), torch.zeros((), device="cuda"))


def make_graph(n_def, cyclic=False):
    # cyclic: every layer defers, and layer 0 takes the last layer's deferred experts from the
    # previous replay -- the steady state of a deep stack, without the chain's two end layers
    first = [True]

    def step():
        prev = layers[-1] if (cyclic and not first[0]) else None
        for i, l in enumerate(layers):
            a_, b_ = bufs[i % 2], bufs[(i + 1) % 2]
            if n_def:
                nd = n_def if (cyclic or i < NL - 1) else 0
                l.forward_chained(a_, residual=a_, n_deferred=nd, prev=prev, y=b_)
                prev = l
            else:
                l.forward(a_, residual=a_, y=b_)
        first[0] = False
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(2):
            step()
    torch.cuda.current_stream().wait_stream(s)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        step()
    return g


graphs = {"plain": make_graph(0), "deferral3": make_graph(3), "deferral3_cyclic": make_graph(3, cyclic=True)}
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
res = {k: [] for k in graphs}
for r in range(ROUNDS):
    for k, g in graphs.items():
        for _ in range(3):
            g.replay()
        tt = []
        for _ in range(STEPS):
            bufs[0].copy_(x0)
            flush[0].zero_(); torch.sum(flush[1], 0, out=flush[2])
            e0.record(); g.replay(); e1.record(); e1.synchronize()
            tt.append(e0.elapsed_time(e1) * 1e3 / NL)
        res[k].append(round(sorted(tt)[len(tt) // 2], 2))
print(json.dumps({"config": cfg, "layers": NL, "us_per_layer_median_per_round": res}))
