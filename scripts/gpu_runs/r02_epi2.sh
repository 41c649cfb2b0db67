# round 2: compact SwiGLU epilogue of the decode stream (rolled token loops) -- parity, traces, A/B vs HEAD
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
timeout 300 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py -k "decode_shapes" > gpurun_out/pytest_epi_quick.log 2>&1; tail -2 gpurun_out/pytest_epi_quick.log
grep -q "passed" gpurun_out/pytest_epi_quick.log && ! grep -q "failed" gpurun_out/pytest_epi_quick.log || exit 3
timeout 900 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_tp_chain.py tests/test_gpu_parity.py -k "decode or chain or tp or full_size or fused" > gpurun_out/pytest_epi.log 2>&1; tail -2 gpurun_out/pytest_epi.log
timeout 150 python scripts/decode_trace.py v3 1 8 8 2>&1 | grep -v slowest | tail -8
for c in v3 v3_fp4; do for i in 1 2; do
  echo "new $(timeout 300 python scripts/decode_ab.py $c 2 2>&1 | tail -1)"
  echo "old $(cd oldref_tmp && timeout 300 python scripts/decode_ab.py $c 2 2>&1 | tail -1)"
done; done
for i in 1 2; do
  echo "new tp: $(timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --no-deferral 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["decode"]["us_per_layer"], d["decode"]["tp_rank_us_per_layer"])')"
  echo "old tp: $(cd oldref_tmp && timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --no-deferral 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["decode"]["us_per_layer"], d["decode"]["tp_rank_us_per_layer"])')"
done
