cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for m in 0 1 2 3 4 5; do echo "mode $m: $(MOE_DEBUG_GEMM=$m timeout 200 python scripts/time_stages.py v3 8192 2>&1 | tail -1)"; done > gpurun_out/gemm_modes.log
