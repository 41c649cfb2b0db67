# round 2: dual units in the swap GEMM (a 256-row + a <= 128-row token tile share each weight k-block load) -- parity, A/B (MOE_SWAP_DUAL=0)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py -k "small_layer or swap_pair or skewed or mid_size_fp8 or prefill_8k or deterministic or zero_tokens or residual or full_size" > gpurun_out/dual_parity.log 2>&1; tail -2 gpurun_out/dual_parity.log
grep -q " passed" gpurun_out/dual_parity.log && ! grep -q "failed\|error" gpurun_out/dual_parity.log || exit 3
summ='import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; s=r["stage_ms"]; print(round(d["value"]), round(d["ms_per_step"],4), round(r["kernel_ms"],3), s["gemm2"], round(r["frac"],3), round(r["layer"]["frac"],3), d["clocks"]["sm_mhz"])'
for i in 1 2 3; do for m in 1 0; do
  echo "dual=$m $(MOE_SWAP_DUAL=$m timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
done; done
for c in qwen2 v25 v2lite v3_fp4; do for m in 1 0; do
  echo "$c dual=$m $(MOE_SWAP_DUAL=$m timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
done; done
timeout 300 python scripts/gemm_trace.py > gpurun_out/dual_gemm_trace.txt 2>&1; tail -2 gpurun_out/dual_gemm_trace.txt
