# ncu --set full of the prefill GEMMs (dual units) and the fused decode stream on the final kernels
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:umma_swap_gemm -c 2 --launch-skip 4 \
  -o gpurun_out/ncu_prefill_final2 python scripts/time_stages.py v3 8192 > gpurun_out/ncu_prefill_final2.log 2>&1; tail -2 gpurun_out/ncu_prefill_final2.log
timeout 600 ncu --set full --import-source on --clock-control none -k regex:umma_decode_fused -c 1 --launch-skip 20 \
  -o gpurun_out/ncu_decode_final2 python scripts/decode_trace.py v3 1 8 > gpurun_out/ncu_decode_final2.log 2>&1; tail -2 gpurun_out/ncu_decode_final2.log
python scripts/summarize_ncu.py gpurun_out/ncu_prefill_final2.ncu-rep gpurun_out/ncu_prefill_final2 > /dev/null 2>&1
python scripts/summarize_ncu.py gpurun_out/ncu_decode_final2.ncu-rep gpurun_out/ncu_decode_final2 > /dev/null 2>&1
