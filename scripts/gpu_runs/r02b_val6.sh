# round 2 (re-entry) last validation on the final code: GPU suite, smoke, bench, reference arm, launch list
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_val6.log 2>&1; tail -3 gpurun_out/pytest_gpu_val6.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_val6.log 2>&1; tail -3 gpurun_out/smoke_val6.log
timeout 900 python bench.py > gpurun_out/bench_val6.json 2> gpurun_out/bench_val6.err; tail -1 gpurun_out/bench_val6.json | cut -c1-300
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref_val6.json 2> gpurun_out/bench_ref_val6.err; tail -1 gpurun_out/bench_ref_val6.json | cut -c1-300
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"umma|route|router|combine|scatter|chunk_count|scan_kernel|assign|decode_finalize" -c 400 --csv \
  --log-file gpurun_out/launches_val6.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-decode-tp --no-deferral > gpurun_out/launches_val6.log 2>&1; tail -1 gpurun_out/launches_val6.log | cut -c1-200
