# round 2: fused decode (unscaled phase A) validation + per-SM rate experiments
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest tests/test_gpu_tp_chain.py -q -rf > gpurun_out/pytest_tpchain.log 2>&1; tail -3 gpurun_out/pytest_tpchain.log
timeout 600 python -m pytest tests/test_gpu_parity.py -q -rf -k "decode or fused or full_size" > gpurun_out/pytest_dec.log 2>&1; tail -3 gpurun_out/pytest_dec.log
for a in "1 8" "1 8 8" "1 8 1 3"; do
  timeout 120 python scripts/decode_trace.py v3 $a > "gpurun_out/trace_v3_$(echo $a | tr ' ' _).txt" 2>&1
done
MOE_EXPERIMENTS=1 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_exp.log 2>&1 || exit 1
for m in 1 2 3; do
  MOE_DEBUG_FD=$m timeout 120 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/trace_v3_tp8_fd$m.txt 2>&1
  MOE_DEBUG_FD=$m timeout 120 python scripts/decode_trace.py v3 1 8 > gpurun_out/trace_v3_fd$m.txt 2>&1
done
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
