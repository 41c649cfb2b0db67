"""Run a few forwards of one preset for ncu capture (not a benchmark).

python scripts/profile_layer.py --config v3 --tokens 8192 --iters 3
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="v3")
ap.add_argument("--tokens", type=int, default=8192)
ap.add_argument("--iters", type=int, default=3)
ap.add_argument("--gemv", type=int, default=0)
a = ap.parse_args()
p = PRESETS[a.config]
w = make_weights(p, "cuda")
x, _ = make_tokens(p, a.tokens, "cuda")
layer = moe.MoELayer(p, w, max_tokens=max(a.tokens, 1), gemv_max_tokens=a.gemv)
y = torch.empty_like(x)
torch.cuda.synchronize()
for _ in range(a.iters):
    layer.forward(x, y=y)
torch.cuda.synchronize()
print("done", a.config, a.tokens)
