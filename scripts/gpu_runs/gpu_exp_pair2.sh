cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for dbg in 1 5; do
  MOE_PAIR=1 MOE_DEBUG_GEMM=$dbg timeout 300 python bench.py --steps 5 --warmup 3 --no-decode --no-e2e --no-cpu > gpurun_out/exp2_pair_dbg${dbg}.log 2>&1
done
