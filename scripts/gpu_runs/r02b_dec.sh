# round 2: fused decode -- one tcgen05.commit per phase-A k-block (epilogue follows the stage ring) -- parity, A/B vs HEAD
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
timeout 900 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_tp_chain.py tests/test_gpu_parity.py -k "decode or chain or tp or full_size or fused or residual" > gpurun_out/dec_parity.log 2>&1; tail -2 gpurun_out/dec_parity.log
grep -q " passed" gpurun_out/dec_parity.log && ! grep -q "failed\|error" gpurun_out/dec_parity.log || exit 3
for c in v3 v3_fp4 v2lite qwen2; do for i in 1 2; do
  echo "new $c $(timeout 300 python scripts/decode_ab.py $c 2 2>&1 | tail -1)"
  echo "old $c $(cd oldref_tmp && timeout 300 python scripts/decode_ab.py $c 2 2>&1 | tail -1)"
done; done
for i in 1 2; do
  echo "new tp: $(timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --no-deferral 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["decode"]["us_per_layer"], d["decode"]["tp_rank_us_per_layer"])')"
  echo "old tp: $(cd oldref_tmp && timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --no-deferral 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["decode"]["us_per_layer"], d["decode"]["tp_rank_us_per_layer"])')"
done
