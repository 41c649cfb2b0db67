cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench13.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"umma" -s 2 -c 2 -o gpurun_out/prof_decode13 python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 > gpurun_out/ncu_full.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_decode13.csv python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 >> gpurun_out/ncu_full.log 2>&1
