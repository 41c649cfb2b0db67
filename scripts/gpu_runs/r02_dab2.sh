# round 2: decode A/B (TS code removed, router quantises x from registers) vs ca52008, chain timeline
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "decode_shapes or fused or mid_size" > gpurun_out/pytest_dab2.log 2>&1; tail -1 gpurun_out/pytest_dab2.log
for i in 1 2; do
  timeout 300 python scripts/decode_ab.py v3 2 > gpurun_out/dab2_new_$i.json 2>&1; tail -1 gpurun_out/dab2_new_$i.json
  (cd oldref_tmp && timeout 300 python scripts/decode_ab.py v3 2 > ../gpurun_out/dab2_old_$i.json 2>&1; tail -1 ../gpurun_out/dab2_old_$i.json)
done
timeout 150 python scripts/decode_trace.py v3 1 8 1 3 > gpurun_out/dab2_trace_def.txt 2>&1; head -3 gpurun_out/dab2_trace_def.txt
timeout 150 python scripts/decode_trace.py v3 1 8 > gpurun_out/dab2_trace_plain.txt 2>&1; head -3 gpurun_out/dab2_trace_plain.txt
timeout 150 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/dab2_trace_tp8.txt 2>&1; head -3 gpurun_out/dab2_trace_tp8.txt
