# BF16 prefill token boxes back to the single-box scheme vs HEAD (oldref_tmp) -- parity, interleaved A/B on the BF16 configs + V3 control
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
timeout 600 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py -k "small_layer or swap_pair or full_size" > gpurun_out/bf16box_parity.log 2>&1; tail -1 gpurun_out/bf16box_parity.log
grep -q " passed" gpurun_out/bf16box_parity.log && ! grep -q "failed\|error" gpurun_out/bf16box_parity.log || exit 3
summ='import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; s=r["stage_ms"]; print(round(d["value"]), round(d["ms_per_step"],4), round(r["kernel_ms"],3), s["gemm2"])'
for c in qwen2 v2lite v3; do for i in 1 2 3; do
  echo "$c new $(timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
  echo "$c old $(cd oldref_tmp && timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
done; done
