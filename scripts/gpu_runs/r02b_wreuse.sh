# timing experiment: upper bound of weight reuse across an expert's token tiles (MOE_DEBUG_GEMM=6: later
# tiles skip the weight loads, stale smem -- timing only) vs normal, same experiments build
cd $GRAFT_REPO_ROOT
MOE_EXPERIMENTS=1 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
summ='import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; s=r["stage_ms"]; print(round(d["value"]), round(d["ms_per_step"],4), round(r["kernel_ms"],3), s["gemm2"])'
for i in 1 2 3; do for m in 0 6; do
  echo "mode=$m $(MOE_EXPERIMENTS=1 MOE_DEBUG_GEMM=$m timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
done; done
