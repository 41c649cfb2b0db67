cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests -m gpu -q -x > gpurun_out/exp13_parity.log 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/exp13_bench.log 2>&1
MOE_DEBUG_ROUTE=4 timeout 300 python scripts/time_stages.py v3 1 > gpurun_out/exp13_route_tail.log 2>&1
timeout 300 python scripts/power_probe.py 8192 4 > gpurun_out/exp13_power.log 2>&1
