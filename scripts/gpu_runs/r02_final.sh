# round 2 final validation: full GPU suite, default bench, all configs, FP8 library context peak
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_final.log 2>&1; tail -3 gpurun_out/pytest_gpu_final.log
timeout 600 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err; tail -1 gpurun_out/bench_final.json
timeout 120 python scripts/fp8_peak.py > gpurun_out/fp8_peak.json 2>&1; cat gpurun_out/fp8_peak.json
timeout 1500 python scripts/all_configs.py gpurun_out/all_configs_final.md > gpurun_out/all_configs_final.jsonl 2>&1; cat gpurun_out/all_configs_final.md
timeout 150 python scripts/decode_trace.py v3 1 8 > gpurun_out/trace_final_v3.txt 2>&1; head -4 gpurun_out/trace_final_v3.txt
