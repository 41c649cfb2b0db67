# round 2: EP FP8 dispatch tests, sanitizers after the barrier cleanup, decode A/B, launch list
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests/test_gpu_ep.py tests/test_gpu_parity.py -q -rf -k "ep or small_layer or decode_shapes or pair" > gpurun_out/pytest_ep.log 2>&1; tail -2 gpurun_out/pytest_ep.log
timeout 300 python scripts/decode_ab.py v3 3 > gpurun_out/ab2_v3.json 2>&1; tail -1 gpurun_out/ab2_v3.json
for tool in racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 10 python -m pytest tests/test_gpu_parity.py -q -x \
    -k "test_small_decode_shapes and v3_s" > gpurun_out/san2_${tool}_decode.log 2>&1; tail -2 gpurun_out/san2_${tool}_decode.log
  timeout 900 compute-sanitizer --tool $tool --print-limit 10 python -m pytest tests/test_gpu_parity.py -q -x \
    -k "test_small_layer_parity and v3_s" > gpurun_out/san2_${tool}_prefill.log 2>&1; tail -2 gpurun_out/san2_${tool}_prefill.log
  timeout 900 compute-sanitizer --tool $tool --print-limit 10 python -m pytest tests/test_gpu_tp_chain.py -q -x \
    -k "test_tp_group_matches_oracle and v3_m and 1-" > gpurun_out/san2_${tool}_tp.log 2>&1; tail -2 gpurun_out/san2_${tool}_tp.log
done
timeout 900 compute-sanitizer --tool memcheck --print-limit 10 python -m pytest tests/test_gpu_tp_chain.py -q -x \
  -k "test_chained_deferral_matches_eq_L241 and v3_s_fp4" > gpurun_out/san2_memcheck_chain_fp4.log 2>&1; tail -2 gpurun_out/san2_memcheck_chain_fp4.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"umma|route|router|combine|scatter|chunk_count|scan_kernel|assign|decode_finalize" -c 400 --csv \
  --log-file gpurun_out/launches_r02.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-decode-tp --no-deferral > gpurun_out/launches_bench.log 2>&1; tail -1 gpurun_out/launches_bench.log
