"""Per-stage device times (library stage events) of a few forwards -- quick experiments."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
cfg = sys.argv[1] if len(sys.argv) > 1 else "v3"
T = int(sys.argv[2]) if len(sys.argv) > 2 else 1
p = PRESETS[cfg]
w = make_weights(p, "cuda")
x, _ = make_tokens(p, max(T, 8), "cuda")
x = x[:T].contiguous()
layer = moe.MoELayer(p, w, max_tokens=max(T, 16))
y = torch.empty_like(x)
for _ in range(3):
    layer.forward(x, y=y)
torch.cuda.synchronize()
layer.profile(True)
acc = {}
for _ in range(10):
    layer.forward(x, y=y)
    for k, v in layer.stage_times().items():
        acc[k] = acc.get(k, 0) + v / 10
print(json.dumps({k: round(v * 1e3, 2) for k, v in acc.items() if v > 0}))
