# round 2: fused decode cluster size by cost model, clusters taking several units -- parity with C forced, timings per C
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for c in 2 4 8; do
  MOE_FD_CSIZE=$c timeout 420 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_parity.py -k "decode_shapes or fused_decode or mid_size_decode" > gpurun_out/csize_parity_$c.log 2>&1; echo "C=$c: $(tail -1 gpurun_out/csize_parity_$c.log)"
done
grep -q "failed\|error\|Timeout" gpurun_out/csize_parity_*.log && exit 3
for cfg in v2lite qwen2 v25 v3 v3_fp4; do for c in 0 1 2 4 8; do
  echo "$cfg C=$c $(MOE_FD_CSIZE=$c timeout 300 python scripts/decode_ab.py $cfg 1 2>&1 | tail -1)"
done; done
