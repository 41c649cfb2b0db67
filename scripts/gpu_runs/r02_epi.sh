cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 150 python scripts/decode_trace.py v3 1 8 8 2>&1 | grep -v slowest | tail -6
timeout 150 python scripts/decode_trace.py v3 1 8 4 2>&1 | grep -v slowest | tail -6
