cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "decode or small or deferral" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
MOE_DEBUG_ROUTE=4 timeout 300 python scripts/time_stages.py v3 1 > gpurun_out/time18.log 2>&1
timeout 300 python scripts/time_stages.py v25 4 >> gpurun_out/time18.log 2>&1
