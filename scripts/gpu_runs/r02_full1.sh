# round 2: full GPU test suite, bench, launch list, ncu full captures (prefill GEMM1, decode stream)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
rm -f gpurun_out/parity_log.jsonl
timeout 1200 python -m pytest tests -m gpu -q -rf --durations=10 > gpurun_out/pytest_gpu_full.log 2>&1; tail -14 gpurun_out/pytest_gpu_full.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; tail -2 gpurun_out/bench_full.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches_r02.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-decode-tp > gpurun_out/launches_bench.log 2>&1; tail -2 gpurun_out/launches_bench.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:umma_swap_gemm -s 2 -c 2 \
  -o gpurun_out/ncu_prefill_r02 python scripts/profile_layer.py --config v3 --tokens 8192 > gpurun_out/ncu_prefill_r02.log 2>&1; tail -2 gpurun_out/ncu_prefill_r02.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:umma_decode_fused -s 20 -c 1 \
  -o gpurun_out/ncu_decode_r02 python scripts/decode_trace.py v3 1 8 > gpurun_out/ncu_decode_r02.log 2>&1; tail -2 gpurun_out/ncu_decode_r02.log
