# round 2 (re-entry): ncu --set full of the prefill GEMMs (V3, T = 8192) and the fused decode stream on the final kernels; all configs
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:umma_swap_gemm -c 2 --launch-skip 4 \
  -o gpurun_out/ncu_prefill_final python scripts/time_stages.py v3 8192 > gpurun_out/ncu_prefill_final.log 2>&1; tail -2 gpurun_out/ncu_prefill_final.log
timeout 600 ncu --set full --import-source on --clock-control none -k regex:umma_decode_fused -c 1 --launch-skip 20 \
  -o gpurun_out/ncu_decode_final python scripts/decode_trace.py v3 1 8 > gpurun_out/ncu_decode_final.log 2>&1; tail -2 gpurun_out/ncu_decode_final.log
python scripts/summarize_ncu.py gpurun_out/ncu_prefill_final.ncu-rep gpurun_out/ncu_prefill_final > /dev/null 2>&1
python scripts/summarize_ncu.py gpurun_out/ncu_decode_final.ncu-rep gpurun_out/ncu_decode_final > /dev/null 2>&1
timeout 1500 python scripts/all_configs.py gpurun_out/all_configs_final.md > gpurun_out/all_configs_final.jsonl 2>&1; cat gpurun_out/all_configs_final.md
