# round 2: sweeps (decode stream vs GEMM, tokens per expert 1..512, skew) and the default bench line
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 1200 python scripts/sweeps.py gpurun_out/sweeps_r02.md > gpurun_out/sweeps_r02.jsonl 2>&1; tail -30 gpurun_out/sweeps_r02.md
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -2 gpurun_out/bench_default.err
