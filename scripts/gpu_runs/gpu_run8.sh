cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench8.log 2>&1
MOE_DEBUG_GEMM=2 timeout 600 python bench.py --steps 3 --warmup 3 --no-decode --no-e2e --no-cpu > gpurun_out/bench8_2.log 2>&1
