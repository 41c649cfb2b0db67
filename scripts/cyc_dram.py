"""DRAM bytes of the fused decode stream per layer, plain vs cyclic-deferral chain (for ncu with
--cache-control none: L2 reuse across the chain's kernels is kept).  argv: config T mode(plain|cyclic)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe

cfg, T, mode = sys.argv[1], int(sys.argv[2]), sys.argv[3]
p = PRESETS[cfg]
w = make_weights(p, "cuda")
layers = [moe.MoELayer(p, w, max_tokens=16) for _ in range(8)]
del w
x = make_tokens(p, T, "cuda", offset=1000)[0]
bufs = [x.clone(), torch.empty_like(x)]
first = [True]


def step():
    prev = layers[-1] if (mode == "cyclic" and not first[0]) else None
    for i, l in enumerate(layers):
        a, b = bufs[i % 2], bufs[(i + 1) % 2]
        if mode == "cyclic":
            l.forward_chained(a, residual=a, n_deferred=3, prev=prev, y=b)
            prev = l
        else:
            l.forward(a, residual=a, y=b)
    first[0] = False


for _ in range(4):
    bufs[0].copy_(x)
    step()
torch.cuda.synchronize()
print("done")
