cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python scripts/dual_diff.py qwen2 2048 2>&1 | tail -4
timeout 300 python scripts/dual_diff.py v3 8192 2>&1 | tail -4
