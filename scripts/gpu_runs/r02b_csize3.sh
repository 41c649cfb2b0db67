# round 2: decode cluster size -- one-wave rule + C = 2 cost model; parity + timings vs C = 1
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py tests/test_gpu_tp_chain.py -k "decode or fused or chain or tp" > gpurun_out/csize3_parity.log 2>&1; tail -1 gpurun_out/csize3_parity.log
grep -q "failed\|error" gpurun_out/csize3_parity.log && exit 3
for cfg in v2lite qwen2 v25 v3; do for c in 0 1; do
  echo "$cfg C=$c $(MOE_FD_CSIZE=$c timeout 300 python scripts/decode_ab.py $cfg 2 2>&1 | tail -1)"
done; done
for i in 1 2; do
  echo "tp: $(timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --no-deferral 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["decode"]["us_per_layer"], d["decode"]["tp_rank_us_per_layer"])')"
done
