cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests -m gpu -q -x -k "decode or small or gemv or deferr" > gpurun_out/fd4_parity_decode.log 2>&1; echo "rc=$?" >> gpurun_out/fd4_parity_decode.log
MOE_DEBUG_ROUTE=4 timeout 120 python scripts/time_stages.py v3 1 > gpurun_out/fd4_route4.log 2>&1
timeout 200 python scripts/decode_ab.py v3 1,4,16 > gpurun_out/fd4_ab_fused.log 2>&1
MOE_DECODE_CHAIN=1 timeout 200 python scripts/decode_ab.py v3 1,4,16 > gpurun_out/fd4_ab_chain.log 2>&1
MOE_NO_PDL=1 timeout 200 python scripts/decode_ab.py v3 1 > gpurun_out/fd4_ab_nopdl.log 2>&1
K='regex:route_small|umma_decode|decode_finalize|combine'
timeout 300 ncu -k "$K" --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/fd4_fused_launches.csv python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 > gpurun_out/fd4_ncu1.log 2>&1
