# round 2: decode A/B (plain vs chained deferral) + ncu source-level capture of the fused decode kernel
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python scripts/decode_ab.py v3 4 > gpurun_out/decode_ab.json 2>&1; tail -1 gpurun_out/decode_ab.json
timeout 600 ncu --set full --import-source on --clock-control none -k regex:umma_decode_fused -c 1 --launch-skip 20 \
  -o gpurun_out/ncu_fd_tp8 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/ncu_fd_tp8.log 2>&1; tail -2 gpurun_out/ncu_fd_tp8.log
timeout 600 ncu --set full --import-source on --clock-control none -k regex:umma_decode_fused -c 1 --launch-skip 20 \
  -o gpurun_out/ncu_fd_v3 python scripts/decode_trace.py v3 1 8 > gpurun_out/ncu_fd_v3.log 2>&1; tail -2 gpurun_out/ncu_fd_v3.log
