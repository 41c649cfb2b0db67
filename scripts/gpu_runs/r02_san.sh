# round 2: router warm-up A/B, decode A/B, launch list (libmoe kernels only), compute-sanitizer
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "decode_shapes or fused" > gpurun_out/pytest_warm.log 2>&1; tail -2 gpurun_out/pytest_warm.log
timeout 150 python scripts/decode_trace.py v3 1 8 > gpurun_out/warm_trace_v3_1_8.txt 2>&1
timeout 150 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/warm_trace_v3_1_8_8.txt 2>&1
timeout 300 python scripts/decode_ab.py v3 3 > gpurun_out/warm_ab_v3.json 2>&1; tail -1 gpurun_out/warm_ab_v3.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"umma|route|router|combine|scatter|chunk_count|scan_kernel|assign|decode_finalize" -c 400 --csv \
  --log-file gpurun_out/launches_r02.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-decode-tp --no-deferral > gpurun_out/launches_bench.log 2>&1; tail -1 gpurun_out/launches_bench.log
for tool in racecheck synccheck memcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -x \
    -k "test_small_decode_shapes and v3_s and 3" > gpurun_out/san_${tool}_decode.log 2>&1; tail -3 gpurun_out/san_${tool}_decode.log
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -x \
    -k "test_small_layer_parity and v3_s" > gpurun_out/san_${tool}_prefill.log 2>&1; tail -3 gpurun_out/san_${tool}_prefill.log
done
MOE_EXPERIMENTS=1 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_exp.log 2>&1 || exit 1
MOE_DEBUG_ROUTE=32 timeout 150 python scripts/decode_trace.py v3 1 8 > gpurun_out/cold_trace_v3_1_8.txt 2>&1
MOE_DEBUG_ROUTE=32 timeout 300 python scripts/decode_ab.py v3 3 > gpurun_out/cold_ab_v3.json 2>&1; tail -1 gpurun_out/cold_ab_v3.json
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
