cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests -m gpu -q -x -k "small or swap or full_size or determin or ep" > gpurun_out/lgt_parity.log 2>&1; echo "rc=$?" >> gpurun_out/lgt_parity.log
for i in 1 2 3; do timeout 300 python scripts/time_stages.py v3 8192 2>&1 | tail -1; done > gpurun_out/lgt_stages.log
