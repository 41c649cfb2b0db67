cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "swap or small_layer or decode_shapes" > gpurun_out/exp10_parity.log 2>&1
for dbg in 0 1 5; do
  MOE_DEBUG_GEMM=$dbg timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/exp10_dbg${dbg}.log 2>&1
done
MOE_DEBUG_ROUTE=12 timeout 300 python scripts/time_stages.py v3 1 > gpurun_out/exp10_route_tail.log 2>&1
timeout 300 python scripts/power_probe.py 8192 4 > gpurun_out/exp10_power.log 2>&1
