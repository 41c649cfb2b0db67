cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 200 python scripts/decode_ab.py v3 1,4 > gpurun_out/fd5_ab_fused.log 2>&1
MOE_DECODE_PF=1 timeout 200 python scripts/decode_ab.py v3 1 > gpurun_out/fd5_ab_pf.log 2>&1
MOE_NO_PDL=1 timeout 200 python scripts/decode_ab.py v3 1 > gpurun_out/fd5_ab_nopdl.log 2>&1
MOE_DECODE_CHAIN=1 timeout 200 python scripts/decode_ab.py v3 1 > gpurun_out/fd5_ab_chain.log 2>&1
MOE_DEBUG_DECODE=1 MOE_DEBUG_ROUTE=16 timeout 200 python scripts/decode_trace.py v3 1 > gpurun_out/fd5_trace.log 2>&1
MOE_DEBUG_DECODE=1 MOE_DEBUG_ROUTE=16 MOE_NO_PDL=1 timeout 200 python scripts/decode_trace.py v3 1 > gpurun_out/fd5_trace_nopdl.log 2>&1
MOE_DEBUG_DECODE=1 MOE_DEBUG_ROUTE=20 timeout 200 python scripts/decode_trace.py v3 1 > gpurun_out/fd5_trace_r4.log 2>&1
