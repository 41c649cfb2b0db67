# optional on-box comparator: FlashInfer trtllm_fp8_block_scale_moe vs this library (V3, T = 8192)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python scripts/flashinfer_comparator.py 8192 > gpurun_out/fi_cmp.json 2> gpurun_out/fi_cmp.err; tail -1 gpurun_out/fi_cmp.json; tail -5 gpurun_out/fi_cmp.err
