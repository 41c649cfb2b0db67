# round 2: TS-form MMA (weights staged in TMEM by tcgen05.cp) vs SS form; late route trigger
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "decode_shapes or fused or mid or full_size" > gpurun_out/pytest_ts.log 2>&1; tail -2 gpurun_out/pytest_ts.log
timeout 600 python -m pytest tests/test_gpu_tp_chain.py -q -x -rf > gpurun_out/pytest_ts_tpchain.log 2>&1; tail -2 gpurun_out/pytest_ts_tpchain.log
for a in "v3 1 8" "v3 1 8 8" "v3_fp4 1 8" "v3_fp4 1 8 8" "v3 1 8 1 3"; do
  timeout 150 python scripts/decode_trace.py $a > "gpurun_out/ts_trace_$(echo $a | tr ' ' _).txt" 2>&1
done
timeout 300 python scripts/decode_ab.py v3 2 > gpurun_out/ts_ab_v3.json 2>&1; tail -1 gpurun_out/ts_ab_v3.json
timeout 300 python scripts/decode_ab.py v3_fp4 2 > gpurun_out/ts_ab_fp4.json 2>&1; tail -1 gpurun_out/ts_ab_fp4.json
MOE_EXPERIMENTS=1 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_exp.log 2>&1 || exit 1
MOE_FD_SS=1 timeout 150 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/ss_trace_v3_1_8_8.txt 2>&1
MOE_FD_SS=1 MOE_FD_CLUSTER=1 timeout 150 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/ss_trace_v3_tp8_c1.txt 2>&1
MOE_FD_CLUSTER=1 timeout 150 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/ts_trace_v3_tp8_c1.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
