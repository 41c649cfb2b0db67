# round 2: fitted decode cluster-size model (post-router units, measured overheads) vs C = 1
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py tests/test_gpu_tp_chain.py -k "decode or fused or chain or tp" > gpurun_out/csize2_parity.log 2>&1; tail -1 gpurun_out/csize2_parity.log
grep -q "failed\|error" gpurun_out/csize2_parity.log && exit 3
for cfg in v2lite qwen2 v25 v3 v3_fp4; do for r in 1 2; do for c in 0 1; do
  echo "$cfg C=$c $(MOE_FD_CSIZE=$c timeout 300 python scripts/decode_ab.py $cfg 1 2>&1 | tail -1)"
done; done; done
timeout 1500 python scripts/all_configs.py gpurun_out/all_configs_cs.md > gpurun_out/all_configs_cs.jsonl 2>&1; cat gpurun_out/all_configs_cs.md
