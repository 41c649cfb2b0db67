# round 2 (re-entry) closing validation: GPU suite, smoke, bench, reference arm, launch list
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
nvidia-smi --query-gpu=name,power.limit --format=csv,noheader
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_val8.log 2>&1; tail -3 gpurun_out/pytest_gpu_val8.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_val8.log 2>&1; tail -3 gpurun_out/smoke_val8.log
timeout 900 python bench.py > gpurun_out/bench_val8.json 2> gpurun_out/bench_val8.err; tail -1 gpurun_out/bench_val8.json | cut -c1-300
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref_val8.json 2> gpurun_out/bench_ref_val8.err; tail -1 gpurun_out/bench_ref_val8.json | cut -c1-200
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"umma|route|router|combine|scatter|chunk_count|scan_kernel|assign|decode_finalize" -c 400 --csv \
  --log-file gpurun_out/launches_val8.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-decode-tp --no-deferral > gpurun_out/launches_val8.log 2>&1; tail -1 gpurun_out/launches_val8.log | cut -c1-120
