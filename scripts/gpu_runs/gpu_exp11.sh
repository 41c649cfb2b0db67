cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests -m gpu -q -x > gpurun_out/exp11_parity.log 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/exp11_bench.log 2>&1
MOE_DEBUG_ROUTE=12 timeout 300 python scripts/time_stages.py v3 1 > gpurun_out/exp11_route_tail.log 2>&1
