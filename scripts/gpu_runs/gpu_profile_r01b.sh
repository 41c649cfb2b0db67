cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
# launch list of the bench command itself (prefill + 8-layer decode legs), our kernels only
timeout 1200 ncu -k regex:"moe::|umma|route|decode|combine|scatter|assign|scan|chunk_count|router" --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/p2_launches_bench.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --decode-layers 2 > gpurun_out/p2_ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"umma_swap|scatter|combine|route|assign|scan_kernel|chunk_count|router_select|umma_grouped" -s 9 -c 9 -o gpurun_out/p2_prefill_full python scripts/profile_layer.py --config v3 --tokens 8192 --iters 2 > gpurun_out/p2_ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"umma_decode_fused|route_small|decode_finalize" -s 6 -c 3 -o gpurun_out/p2_decode_full python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 >> gpurun_out/p2_ncu_full.log 2>&1
