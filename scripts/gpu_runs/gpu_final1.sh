cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/f1_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/f1_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f1_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/f1_smoke.log
/usr/bin/time -v timeout 900 python bench.py > gpurun_out/f1_bench.log 2> gpurun_out/f1_bench_time.log
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/f1_bench_ref.log 2>&1
timeout 1200 ncu -k regex:"umma|route|decode|combine|scatter|assign|scan|chunk_count|router" --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/f1_launches_bench.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --decode-layers 2 > gpurun_out/f1_ncu_bench.log 2>&1
