# round 2: cluster-split fused decode validation + timing (every command bounded)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -3 gpurun_out/smoke.log
timeout 900 python -m pytest tests/test_gpu_tp_chain.py -q -x -rf > gpurun_out/pytest_tpchain.log 2>&1; tail -3 gpurun_out/pytest_tpchain.log
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "decode or fused or full_size or small" > gpurun_out/pytest_dec.log 2>&1; tail -3 gpurun_out/pytest_dec.log
for a in "1 8" "1 8 8" "1 8 4" "1 8 1 3"; do
  timeout 150 python scripts/decode_trace.py v3 $a > "gpurun_out/trace_v3_$(echo $a | tr ' ' _).txt" 2>&1
done
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -2 gpurun_out/bench.err
MOE_EXPERIMENTS=1 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_exp.log 2>&1 || exit 1
for m in 1 2 3; do
  MOE_DEBUG_FD=$m MOE_FD_CLUSTER=1 timeout 150 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/trace_v3_tp8_c1_fd$m.txt 2>&1
done
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
