"""MMA-warp cycle breakdown of the prefill swap GEMMs (MOE_DEBUG_TRACE, set here)."""
import os, sys, ctypes
os.environ["MOE_DEBUG_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
cfg = sys.argv[1] if len(sys.argv) > 1 else "v3"
T = int(sys.argv[2]) if len(sys.argv) > 2 else 8192
p = PRESETS[cfg]
w = make_weights(p, "cuda")
x, _ = make_tokens(p, T, "cuda")
layer = moe.MoELayer(p, w, max_tokens=T)
lib = layer._lib
lib.moe_layer_debug_trace.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32]
buf = np.zeros(4096, dtype=np.uint64)
y = torch.empty_like(x)
for _ in range(3):
    layer.forward(x, y=y)
    torch.cuda.synchronize()
    lib.moe_layer_debug_trace(layer._h, buf.ctypes.data, 4096)
for name, base in (("gemm1", 0), ("gemm2", 2048)):
    a = buf[base:base + 8 * 74].reshape(74, 8).astype(np.float64)
    a = a[a[:, 6] > 0]
    tot = a[:, 6].mean()
    print(f"{name}: pairs {len(a)}, mean total {tot:.0f} cyc; unit-wait {a[:,0].mean()/tot*100:.1f}% tmem-wait {a[:,1].mean()/tot*100:.1f}% "
          f"full-wait {a[:,2].mean()/tot*100:.1f}% issue {a[:,3].mean()/tot*100:.1f}%; units/pair {a[:,4].mean():.1f} "
          f"(min {a[:,4].min():.0f} max {a[:,4].max():.0f}); mean N {16*a[:,5].sum()/a[:,4].sum():.1f}; total max {a[:,6].max():.0f}")
