# round 2: decode finalize in the stream's last CTA (A/B vs HEAD) + decode/chain/TP parity
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
timeout 900 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_tp_chain.py tests/test_gpu_parity.py -k "decode or chain or tp or full_size or fused" > gpurun_out/pytest_fin.log 2>&1; tail -2 gpurun_out/pytest_fin.log
for c in v3 v2lite; do for i in 1 2; do
  echo "new $(timeout 300 python scripts/decode_ab.py $c 2 2>&1 | tail -1)"
  echo "old $(cd oldref_tmp && timeout 300 python scripts/decode_ab.py $c 2 2>&1 | tail -1)"
done; done
timeout 150 python scripts/decode_trace.py v3 1 8 > gpurun_out/fin_v3.txt 2>&1; grep "period\|route:\|unit_end\|finalize" gpurun_out/fin_v3.txt
timeout 150 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/fin_tp8.txt 2>&1; grep "period\|route:\|unit_end\|finalize" gpurun_out/fin_tp8.txt
