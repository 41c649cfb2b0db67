# round 2 (re-entry) final validation after adaptive dual units: GPU suite, smoke, bench, reference arm, launch list
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_val5.log 2>&1; tail -3 gpurun_out/pytest_gpu_val5.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_val5.log 2>&1; tail -3 gpurun_out/smoke_val5.log
timeout 900 python bench.py > gpurun_out/bench_val5.json 2> gpurun_out/bench_val5.err; tail -1 gpurun_out/bench_val5.json | cut -c1-300
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref_val5.json 2> gpurun_out/bench_ref_val5.err; tail -1 gpurun_out/bench_ref_val5.json | cut -c1-300
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"umma|route|router|combine|scatter|chunk_count|scan_kernel|assign|decode_finalize" -c 400 --csv \
  --log-file gpurun_out/launches_val5.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-decode-tp --no-deferral > gpurun_out/launches_val5.log 2>&1; tail -1 gpurun_out/launches_val5.log | cut -c1-200
summ='import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; s=r["stage_ms"]; print(round(d["value"]), round(d["ms_per_step"],4), round(r["kernel_ms"],3), s["gemm2"], round(r["layer"]["frac"],3))'
for i in 1 2; do for t in 48 64 96; do
  echo "v3 tail=$t $(MOE_SWAP_DUAL_TAIL=$t timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
done; done
