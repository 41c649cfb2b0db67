cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/exp4_parity.log 2>&1
MOE_DEBUG_ROUTE=4 timeout 300 python scripts/time_stages.py v3 1 > gpurun_out/exp4_route_tail.log 2>&1
for pair in 0 1; do
 for pf in 0 4 8 16; do
  MOE_PAIR=$pair MOE_PF=$pf timeout 300 python bench.py --steps 5 --warmup 3 --no-decode --no-e2e --no-cpu > gpurun_out/exp4_pair${pair}_pf${pf}.log 2>&1
 done
done
