# round 2: phase-B epilogue with REDG (was generic ATOM with return) -- traces + A/B; route trigger experiment
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "decode_shapes or fused or mid" > gpurun_out/pytest_red.log 2>&1; tail -2 gpurun_out/pytest_red.log
for a in "v3 1 8" "v3 1 8 8" "v3_fp4 1 8" "v3_fp4 1 8 8" "v3 1 8 1 3"; do
  timeout 150 python scripts/decode_trace.py $a > "gpurun_out/red_trace_$(echo $a | tr ' ' _).txt" 2>&1
done
timeout 300 python scripts/decode_ab.py v3 2 > gpurun_out/red_ab_v3.json 2>&1; tail -1 gpurun_out/red_ab_v3.json
timeout 300 python scripts/decode_ab.py v3_fp4 2 > gpurun_out/red_ab_fp4.json 2>&1; tail -1 gpurun_out/red_ab_fp4.json
MOE_EXPERIMENTS=1 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_exp.log 2>&1 || exit 1
MOE_DEBUG_ROUTE=16 timeout 150 python scripts/decode_trace.py v3 1 8 > gpurun_out/red_trace_late_trigger.txt 2>&1
MOE_DEBUG_ROUTE=16 timeout 300 python scripts/decode_ab.py v3 2 > gpurun_out/red_ab_v3_late.json 2>&1; tail -1 gpurun_out/red_ab_v3_late.json
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
