# round 2: FP4 decode + DSMEM cluster exchange validation, traces, bench
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -3 gpurun_out/smoke.log
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "fp4" > gpurun_out/pytest_fp4.log 2>&1; tail -3 gpurun_out/pytest_fp4.log
timeout 900 python -m pytest tests/test_gpu_tp_chain.py -q -rf > gpurun_out/pytest_tpchain.log 2>&1; tail -3 gpurun_out/pytest_tpchain.log
timeout 900 python -m pytest tests -m gpu -q -rf --deselect tests/test_gpu_tp_chain.py > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
for a in "v3 1 8" "v3 1 8 8" "v3_fp4 1 8" "v3_fp4 1 8 8"; do
  timeout 150 python scripts/decode_trace.py $a > "gpurun_out/trace_$(echo $a | tr ' ' _).txt" 2>&1
done
timeout 300 python scripts/decode_ab.py v3_fp4 2 > gpurun_out/decode_ab_fp4.json 2>&1; tail -1 gpurun_out/decode_ab_fp4.json
