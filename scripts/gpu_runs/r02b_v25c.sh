# V2.5 decode at T = 4 (the BASELINE batch): cluster size forced vs the model
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for i in 1 2; do for c in 0 1 2 4; do
  echo "v25 T=4 C=$c $(MOE_FD_CSIZE=$c timeout 300 python scripts/decode_ab.py v25 1 4 2>&1 | tail -1)"
done; done
for i in 1; do for c in 0 1 2; do
  echo "v3 T=4 C=$c $(MOE_FD_CSIZE=$c timeout 300 python scripts/decode_ab.py v3 1 4 2>&1 | tail -1)"
  echo "qwen2 T=4 C=$c $(MOE_FD_CSIZE=$c timeout 300 python scripts/decode_ab.py qwen2 1 4 2>&1 | tail -1)"
done; done
