# EP decode (in-process group on one GPU): fused stream vs grouped GEMMs on the expert side
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for c in "v3 8 1" "v3 2 1" "v25 8 4"; do for m in 0 1; do
  MOE_EP_DECODE_GEMM=$m timeout 600 python scripts/ep_decode_time.py $c 2>&1 | tail -1
done; done
