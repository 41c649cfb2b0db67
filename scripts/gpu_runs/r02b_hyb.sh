# round 2: hybrid swap launch (clusters of 2 pairs + pairs in piece mode on the leftover SMs) -- parity, A/B per GEMM
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
MOE_SWAP_NP1=3 MOE_SWAP_NP2=3 timeout 600 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py -k "small_layer or swap_pair or skewed or mid_size_fp8 or prefill_8k or deterministic or zero_tokens or residual" > gpurun_out/hyb_parity.log 2>&1; tail -1 gpurun_out/hyb_parity.log
grep -q " passed" gpurun_out/hyb_parity.log && ! grep -q "failed\|error" gpurun_out/hyb_parity.log || exit 3
summ='import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; s=r["stage_ms"]; print(round(d["value"]), round(d["ms_per_step"],4), round(r["kernel_ms"],3), s["gemm2"], round(r["frac"],3), round(r["layer"]["frac"],3), d["clocks"]["sm_mhz"])'
for i in 1 2 3; do
  for np in "1 1" "3 3" "1 3" "3 1"; do
    set -- $np
    echo "np=$1,$2 $(MOE_SWAP_NP1=$1 MOE_SWAP_NP2=$2 timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
  done
done
