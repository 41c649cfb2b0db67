cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python scripts/gemm_trace.py v3 8192 > gpurun_out/gemm_trace0.log 2>&1
MOE_DEBUG_GEMM=3 timeout 300 python scripts/gemm_trace.py v3 8192 > gpurun_out/gemm_trace3.log 2>&1
MOE_DEBUG_GEMM=1 timeout 300 python scripts/gemm_trace.py v3 8192 > gpurun_out/gemm_trace1.log 2>&1
