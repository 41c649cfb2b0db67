# round 2: where does a decode unit's time go (TP8 rank, cluster split off: 18 units on 18 SMs)
cd $GRAFT_REPO_ROOT
MOE_EXPERIMENTS=1 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_exp.log 2>&1 || exit 1
for m in 0 1 2 4 8 12 15; do
  MOE_DEBUG_FD=$m MOE_FD_CLUSTER=1 timeout 150 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/exp_tp8_c1_fd$m.txt 2>&1
  MOE_DEBUG_FD=$m MOE_FD_CLUSTER=1 timeout 150 python scripts/decode_trace.py v3_fp4 1 8 8 > gpurun_out/exp_fp4_tp8_c1_fd$m.txt 2>&1
done
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
