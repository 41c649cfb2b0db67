"""Sustained-load probe: loop the V3 prefill forward for a few seconds while
sampling nvidia-smi (SM clock, power, throttle reasons) -- experiments only."""
import os, subprocess, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
T = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
secs = float(sys.argv[2]) if len(sys.argv) > 2 else 4.0
p = PRESETS["v3"]
w = make_weights(p, "cuda")
x, _ = make_tokens(p, T, "cuda")
layer = moe.MoELayer(p, w, max_tokens=T)
y = torch.empty_like(x)
for _ in range(3):
    layer.forward(x, y=y)
torch.cuda.synchronize()
smi = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,power.draw,clocks_throttle_reasons.active",
                        "--format=csv,noheader", "-lms", "100"], stdout=subprocess.PIPE, text=True)
t0 = time.time(); n = 0
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
ev0.record()
while time.time() - t0 < secs:
    for _ in range(20):
        layer.forward(x, y=y)
    n += 20
    torch.cuda.synchronize()
ev1.record(); torch.cuda.synchronize()
smi.terminate()
out = smi.stdout.read().strip().splitlines()
print(f"{os.environ.get('MOE_DEBUG_GEMM','0')}: {n} forwards, {ev0.elapsed_time(ev1)/n:.3f} ms/forward")
mid = out[len(out)//4: 3*len(out)//4]
for l in mid[::max(1, len(mid)//6)]:
    print("  ", l)
