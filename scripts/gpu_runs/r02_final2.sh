# round 2 final: full GPU suite, bench, all configs, sanitizers on the new router paths, ncu launch list + decode capture
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_final.log 2>&1; tail -3 gpurun_out/pytest_gpu_final.log
timeout 900 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err; tail -1 gpurun_out/bench_final.json
timeout 1500 python scripts/all_configs.py gpurun_out/all_configs_final.md > gpurun_out/all_configs_final.jsonl 2>&1; cat gpurun_out/all_configs_final.md
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider \
    -k "test_small_decode_shapes and (v3_g32 or v2lite_s) and 1" > gpurun_out/san_${tool}_router1.log 2>&1; tail -2 gpurun_out/san_${tool}_router1.log
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"umma|route|router|combine|scatter|chunk_count|scan_kernel|assign|decode_finalize" -c 400 --csv \
  --log-file gpurun_out/launches_final.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-decode-tp --no-deferral > gpurun_out/launches_final.log 2>&1; tail -1 gpurun_out/launches_final.log
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"umma_decode_fused|route_small" -c 2 --launch-skip 20 \
  -o gpurun_out/ncu_decode_final python scripts/decode_trace.py v3 1 8 > gpurun_out/ncu_decode_final.log 2>&1; tail -2 gpurun_out/ncu_decode_final.log
timeout 150 python scripts/decode_trace.py v3 1 8 > gpurun_out/trace_final_v3.txt 2>&1
timeout 150 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/trace_final_tp8.txt 2>&1
timeout 150 python scripts/decode_trace.py v3 1 8 1 3 > gpurun_out/trace_final_def3.txt 2>&1
