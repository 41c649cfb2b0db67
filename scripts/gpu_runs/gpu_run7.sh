cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for m in 0 1 2; do
MOE_DEBUG_GEMM=$m timeout 600 python bench.py --steps 3 --warmup 3 --no-decode --no-e2e --no-cpu > gpurun_out/bench7_$m.log 2>&1
done
