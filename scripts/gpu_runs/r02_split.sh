# round 2: split shared expert (cluster-split shared chunks during routing) validation + timing
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "split_shared" > gpurun_out/pytest_split.log 2>&1; tail -2 gpurun_out/pytest_split.log
timeout 600 python -m pytest tests/test_gpu_parity.py -q -rf -k "full_size or decode_shapes or fused or mid" > gpurun_out/pytest_split2.log 2>&1; tail -2 gpurun_out/pytest_split2.log
timeout 600 python -m pytest tests/test_gpu_tp_chain.py -q -rf > gpurun_out/pytest_split3.log 2>&1; tail -2 gpurun_out/pytest_split3.log
timeout 150 python scripts/decode_trace.py v3 1 8 > gpurun_out/split_trace_v3.txt 2>&1; head -4 gpurun_out/split_trace_v3.txt
timeout 300 python scripts/decode_ab.py v3 2 > gpurun_out/split_ab_v3.json 2>&1; tail -1 gpurun_out/split_ab_v3.json
timeout 300 python scripts/decode_ab.py v3_fp4 2 > gpurun_out/split_ab_fp4.json 2>&1; tail -1 gpurun_out/split_ab_fp4.json
MOE_EXPERIMENTS=1 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_exp.log 2>&1 || exit 1
MOE_NO_SPLIT_SHARED=1 timeout 300 python scripts/decode_ab.py v3 2 > gpurun_out/nosplit_ab_v3.json 2>&1; tail -1 gpurun_out/nosplit_ab_v3.json
timeout 300 python scripts/decode_ab.py v3 2 > gpurun_out/split_ab_v3_exp.json 2>&1; tail -1 gpurun_out/split_ab_v3_exp.json
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
