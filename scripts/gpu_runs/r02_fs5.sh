cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for i in 1 2; do timeout 150 python scripts/decode_trace.py v3 1 8 2>&1 | grep "route"; done
timeout 150 python scripts/decode_trace.py v3 1 1 2>&1 | grep "route"
