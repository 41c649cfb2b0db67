cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
MOE_DEBUG_ROUTE=8 timeout 200 python scripts/decode_trace.py v3 1 > gpurun_out/fd9_trace.log 2>&1
