cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for dbg in 0 1; do
  MOE_PAIR=1 MOE_DEBUG_GEMM=$dbg timeout 300 python bench.py --steps 5 --warmup 3 --no-decode --no-e2e --no-cpu > gpurun_out/exp3_pair_dbg${dbg}.log 2>&1
done
MOE_PAIR=1 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "pair or v3" > gpurun_out/exp3_pair_parity.log 2>&1
