cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for dbg in 0 1 2 3; do
  MOE_DEBUG_GEMM=$dbg timeout 300 python scripts/power_probe.py 8192 4 >> gpurun_out/exp7_power.log 2>&1
done
for dbg in 1 3; do
  MOE_DEBUG_GEMM=$dbg timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu --no-decode > gpurun_out/exp7_dbg${dbg}.log 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"umma_swap" -s 2 -c 2 -o gpurun_out/prof_swap python scripts/profile_layer.py --config v3 --tokens 8192 --iters 2 > gpurun_out/ncu_swap.log 2>&1
