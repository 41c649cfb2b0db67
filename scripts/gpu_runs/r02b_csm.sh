# refit decode cluster model (overhead 1.5 us, 2 % margin): decode parity + model vs C = 1 at T = 1 and 4
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py tests/test_gpu_tp_chain.py -k "decode or fused or chain or tp" > gpurun_out/csm_parity.log 2>&1; tail -1 gpurun_out/csm_parity.log
grep -q "failed\|error" gpurun_out/csm_parity.log && exit 3
for cfg in "v3 1" "v3 4" "v25 4" "v25 1" "qwen2 1" "v2lite 1" "v3_fp4 1"; do for c in 0 1; do
  set -- $cfg
  echo "$1 T=$2 C=$c $(MOE_FD_CSIZE=$c timeout 300 python scripts/decode_ab.py $1 1 $2 2>&1 | tail -1)"
done; done
