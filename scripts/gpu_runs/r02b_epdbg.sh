cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python scripts/ep_decode_debug.py 2>&1 | tail -10
echo "--- C=1"
MOE_FD_CSIZE=1 timeout 300 python scripts/ep_decode_debug.py 2>&1 | tail -10
