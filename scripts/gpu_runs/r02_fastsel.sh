# round 2: one-token CTA-wide router select (route_one_fast): parity + A/B vs HEAD (oldref_tmp)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
timeout 1200 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py -k "full" tests/test_gpu_tp_chain.py > gpurun_out/pytest_fastsel.log 2>&1; tail -3 gpurun_out/pytest_fastsel.log
timeout 150 python scripts/decode_trace.py v3 1 8 > gpurun_out/fastsel_trace_v3.txt 2>&1; head -3 gpurun_out/fastsel_trace_v3.txt
timeout 150 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/fastsel_trace_tp8.txt 2>&1; head -3 gpurun_out/fastsel_trace_tp8.txt
for i in 1 2; do
  timeout 300 python scripts/decode_ab.py v3 2 > gpurun_out/fs_new_$i.json 2>&1; tail -1 gpurun_out/fs_new_$i.json
  (cd oldref_tmp && timeout 300 python scripts/decode_ab.py v3 2 > ../gpurun_out/fs_old_$i.json 2>&1; tail -1 ../gpurun_out/fs_old_$i.json)
done
