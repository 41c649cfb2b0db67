"""Context measurement: cuBLASLt FP8 (e4m3) dense GEMM throughput on this B200.

Not a roofline denominator (bench.py takes the FP8 peak as 2 x the measured bf16 burst,
per the guide's nominal ratio); this says what a vendor library reaches for the same dtype
under the same power/clock conditions, so the prefill GEMMs' fraction can be read against it.
torch._scaled_mm with per-tensor fp32 scales, M = N = K = 8192, best of 10 (burst) and
back-to-back for 3 s (sustained), CUDA events.  Prints one JSON line.
"""
import json
import time

import torch


def main():
    dev = torch.device("cuda:0")
    n = 8192
    a = (torch.randn(n, n, device=dev) * 0.5).to(torch.float8_e4m3fn)
    b = (torch.randn(n, n, device=dev) * 0.5).to(torch.float8_e4m3fn).t()   # column-major B
    sa = torch.ones((), device=dev)
    sb = torch.ones((), device=dev)

    def mm():
        return torch._scaled_mm(a, b, scale_a=sa, scale_b=sb, out_dtype=torch.bfloat16)

    for _ in range(5):
        mm()
    torch.cuda.synchronize()
    flops = 2.0 * n ** 3
    best = 1e9
    for _ in range(10):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); mm(); e1.record(); torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) * 1e-3)
    t_end = time.time() + 3.0
    iters, e0 = 0, torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    while time.time() < t_end:
        for _ in range(20):
            mm()
        iters += 20
    e1.record(); torch.cuda.synchronize()
    sustained = flops * iters / (e0.elapsed_time(e1) * 1e-3) / 1e12
    print(json.dumps({"what": "torch._scaled_mm e4m3 x e4m3 -> bf16, per-tensor scales, 8192^3",
                      "fp8_tflops_burst": round(flops / best / 1e12, 1),
                      "fp8_tflops_sustained": round(sustained, 1)}))


if __name__ == "__main__":
    main()
