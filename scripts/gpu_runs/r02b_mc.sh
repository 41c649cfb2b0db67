# round 2: swap GEMM on clusters of 2 CTA pairs (token boxes multicast) -- parity, then A/B vs the pair kernel
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py -k "small_layer or swap_pair or skewed or mid_size_fp8 or prefill_8k or deterministic or zero_tokens" > gpurun_out/mc_parity.log 2>&1; tail -3 gpurun_out/mc_parity.log
grep -q " passed" gpurun_out/mc_parity.log && ! grep -q "failed\|error" gpurun_out/mc_parity.log || exit 3
for i in 1 2; do
  for np in 1 0; do
    echo "np=$np $(MOE_SWAP_NP=$np timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; print(round(d["value"]), r["kernel_ms"], r["frac"], r["layer"]["frac"], r["stage_ms"]["gemm2"], d["clocks"]["sm_mhz"])')"
  done
done
MOE_DEBUG_TRACE=1 timeout 300 python scripts/gemm_trace.py > gpurun_out/mc_gemm_trace.txt 2>&1; tail -4 gpurun_out/mc_gemm_trace.txt
