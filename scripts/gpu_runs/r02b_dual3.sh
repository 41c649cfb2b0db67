# dual units on/off, interleaved, V3 + Qwen2 (box-to-box check)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
nvidia-smi --query-gpu=name,power.limit,clocks.max.sm,temperature.gpu --format=csv,noheader
summ='import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; s=r["stage_ms"]; print(round(d["value"]), round(d["ms_per_step"],4), round(r["kernel_ms"],3), s["gemm2"], round(r["layer"]["frac"],3))'
for i in 1 2 3 4; do for m in 1 0; do
  echo "dual=$m $(MOE_SWAP_DUAL=$m timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
done; done
