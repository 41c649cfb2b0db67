# round 2: stage groups of 2 released by one commit (SW_CE = 2) on the current kernel -- A/B vs HEAD
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
timeout 600 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py -k "small_layer or swap_pair or skewed or mid_size_fp8 or prefill_8k or deterministic or zero_tokens or residual" > gpurun_out/ce2_parity.log 2>&1; tail -3 gpurun_out/ce2_parity.log
grep -q " passed" gpurun_out/ce2_parity.log && ! grep -q "failed\|error" gpurun_out/ce2_parity.log || exit 3
summ='import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; s=r["stage_ms"]; print(round(d["value"]), round(d["ms_per_step"],4), round(r["kernel_ms"],3), s["gemm2"], s["combine"], round(r["frac"],3), round(r["layer"]["frac"],3), d["clocks"]["sm_mhz"])'
for i in 1 2 3; do
  echo "new $(timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
  echo "old $(cd oldref_tmp && timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
done
timeout 300 python scripts/gemm_trace.py > gpurun_out/ce2_gemm_trace.txt 2>&1; tail -2 gpurun_out/ce2_gemm_trace.txt
