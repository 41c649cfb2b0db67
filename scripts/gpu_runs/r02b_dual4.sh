# dual units only for experts of 257 .. 256 + tail tokens (MOE_SWAP_DUAL_TAIL) -- parity, A/B
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py -k "small_layer or swap_pair or skewed or mid_size_fp8 or prefill_8k or deterministic or full_size" > gpurun_out/dual4_parity.log 2>&1; tail -1 gpurun_out/dual4_parity.log
grep -q " passed" gpurun_out/dual4_parity.log && ! grep -q "failed\|error" gpurun_out/dual4_parity.log || exit 3
nvidia-smi --query-gpu=name,power.limit --format=csv,noheader
summ='import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; s=r["stage_ms"]; print(round(d["value"]), round(d["ms_per_step"],4), round(r["kernel_ms"],3), s["gemm2"], round(r["layer"]["frac"],3))'
for c in v3 qwen2; do for i in 1 2 3; do for m in "1 64" "1 32" "0 64"; do
  set -- $m
  echo "$c dual=$1 tail=$2 $(MOE_SWAP_DUAL=$1 MOE_SWAP_DUAL_TAIL=$2 timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
done; done; done
