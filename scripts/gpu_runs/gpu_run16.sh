cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for m in 0 1 2 3; do echo "route=$m $(MOE_DEBUG_ROUTE=$m timeout 300 python scripts/time_stages.py v3 1 2>&1 | tail -1)"; done > gpurun_out/time16.log 2>&1
