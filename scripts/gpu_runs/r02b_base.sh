# round 2 re-entry: validate HEAD on a B200 (full GPU suite + bench line)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_base.log 2>&1; tail -3 gpurun_out/pytest_gpu_base.log
timeout 900 python bench.py > gpurun_out/bench_base.json 2> gpurun_out/bench_base.err; tail -1 gpurun_out/bench_base.json | cut -c1-600
