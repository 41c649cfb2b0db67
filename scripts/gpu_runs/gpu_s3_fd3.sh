cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
K='regex:route_small|umma_decode|decode_finalize|combine'
timeout 300 ncu -k "$K" --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/fd3_fused_launches.csv python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 > gpurun_out/fd3_ncu1.log 2>&1
MOE_DECODE_CHAIN=1 timeout 300 ncu -k "$K" --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/fd3_chain_launches.csv python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 > gpurun_out/fd3_ncu2.log 2>&1
MOE_DEBUG_ROUTE=4 timeout 120 python scripts/time_stages.py v3 1 > gpurun_out/fd3_route4.log 2>&1
MOE_DEBUG_ROUTE=12 timeout 120 python scripts/time_stages.py v3 1 > gpurun_out/fd3_route12.log 2>&1
MOE_DEBUG_ROUTE=2 timeout 120 python scripts/time_stages.py v3 1 > gpurun_out/fd3_route2.log 2>&1
MOE_DEBUG_ROUTE=1 timeout 120 python scripts/time_stages.py v3 1 > gpurun_out/fd3_route1.log 2>&1
timeout 300 ncu -k regex:umma_decode_fused -s 2 -c 1 --set full --clock-control none --import-source on -o gpurun_out/fd3_fused_full python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 > gpurun_out/fd3_ncu3.log 2>&1
