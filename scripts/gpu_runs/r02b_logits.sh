# round 2: router logits GEMM with 128-row router blocks when 256-wide units leave SMs idle -- parity, A/B vs HEAD
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
timeout 900 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py -k "small_layer or prefill_8k or deterministic or skewed or full_size or mid_size_fp8 or swap_pair" > gpurun_out/logits_parity.log 2>&1; tail -2 gpurun_out/logits_parity.log
grep -q " passed" gpurun_out/logits_parity.log && ! grep -q "failed\|error" gpurun_out/logits_parity.log || exit 3
summ='import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; s=r["stage_ms"]; print(round(d["value"]), round(d["ms_per_step"],4), s["router_logits"], s["router_select"], s["permute"], round(r["kernel_ms"],3), s["gemm2"], s["combine"], round(r["layer"]["frac"],3), d["clocks"]["sm_mhz"])'
for i in 1 2 3; do
  echo "new $(timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
  echo "old $(cd oldref_tmp && timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
done
for c in qwen2 v25 v2lite; do
  echo "new $c $(timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
  echo "old $c $(cd oldref_tmp && timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
done
