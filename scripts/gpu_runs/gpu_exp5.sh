cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "v3 or pair or fp8" > gpurun_out/exp5_parity.log 2>&1
for dbg in 0 2 3 4 6 7; do
  MOE_DEBUG_GEMM=$dbg timeout 300 python bench.py --steps 5 --warmup 3 --no-decode --no-e2e --no-cpu > gpurun_out/exp5_dbg${dbg}.log 2>&1
done
MOE_PAIR=1 timeout 300 python bench.py --steps 5 --warmup 3 --no-decode --no-e2e --no-cpu > gpurun_out/exp5_pair.log 2>&1
