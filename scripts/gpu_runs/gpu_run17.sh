cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
MOE_DEBUG_ROUTE=4 timeout 300 python scripts/time_stages.py v3 1 > gpurun_out/time17.log 2>&1
