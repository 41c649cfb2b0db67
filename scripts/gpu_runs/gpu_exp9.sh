cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for dbg in 1 4 5 6; do
  MOE_DEBUG_GEMM=$dbg timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu --no-decode > gpurun_out/exp9_dbg${dbg}.log 2>&1
done
