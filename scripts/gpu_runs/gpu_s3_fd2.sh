cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 200 python scripts/decode_ab.py v3 1,4,16 > gpurun_out/fd2_ab_fused.log 2>&1
MOE_DECODE_CHAIN=1 timeout 200 python scripts/decode_ab.py v3 1,4,16 > gpurun_out/fd2_ab_chain.log 2>&1
timeout 400 python bench.py --no-cpu > gpurun_out/fd2_bench.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/fd2_decode_launches.csv python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 > gpurun_out/fd2_ncu.log 2>&1
