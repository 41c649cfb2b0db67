cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
start=$(date +%s)
timeout 900 python bench.py > gpurun_out/f2_bench.log 2>&1
echo "bench wall s: $(( $(date +%s) - start ))" > gpurun_out/f2_bench_time.log
