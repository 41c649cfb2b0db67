cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/sel2_parity.log 2>&1; echo "rc=$?" >> gpurun_out/sel2_parity.log
timeout 400 python scripts/decode_ab.py v3 1,4 8 > gpurun_out/sel2_ab_v3.log 2>&1
timeout 400 python scripts/decode_trace.py v3 1 8 > gpurun_out/sel2_trace.log 2>&1
