cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 1200 ncu -k regex:"umma|route|decode|combine|scatter|assign|scan|chunk_count|router" --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/fl_launches_bench.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --decode-layers 2 > gpurun_out/fl_ncu_bench.log 2>&1
