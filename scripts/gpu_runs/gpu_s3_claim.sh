cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests -m gpu -q -x -k "small or swap or full_size or determin or ep" > gpurun_out/claim_parity.log 2>&1; echo "rc=$?" >> gpurun_out/claim_parity.log
for i in 1 2 3; do timeout 300 python scripts/time_stages.py v3 8192 2>&1 | tail -1; done > gpurun_out/claim_stages.log
timeout 300 python scripts/gemm_trace.py v3 8192 > gpurun_out/claim_trace.log 2>&1
