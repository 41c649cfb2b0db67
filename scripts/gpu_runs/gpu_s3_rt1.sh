cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests -m gpu -q -x -k "decode or small or deferr or full_size" > gpurun_out/rt1_parity.log 2>&1; echo "rc=$?" >> gpurun_out/rt1_parity.log
timeout 400 python scripts/decode_trace.py v3 1 8 > gpurun_out/rt1_trace_L8.log 2>&1
timeout 400 python scripts/decode_ab.py v3 1,4 8 > gpurun_out/rt1_ab_L8.log 2>&1
