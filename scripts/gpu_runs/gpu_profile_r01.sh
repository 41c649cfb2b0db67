cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
# launch list of the bench command itself (prefill leg)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"umma_grouped_gemm|scatter|combine|route|assign|scan_kernel|chunk_count|router_select" -s 9 -c 9 -o gpurun_out/prof_prefill_full python scripts/profile_layer.py --config v3 --tokens 8192 --iters 2 > gpurun_out/ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"umma_decode|route_small|combine" -s 4 -c 4 -o gpurun_out/prof_decode_full python scripts/profile_layer.py --config v3 --tokens 1 --iters 2 >> gpurun_out/ncu_full.log 2>&1
