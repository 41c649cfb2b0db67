cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests -m gpu -q -x -k "decode or small or deferr or full_size" > gpurun_out/lg_parity.log 2>&1; echo "rc=$?" >> gpurun_out/lg_parity.log
timeout 400 python scripts/decode_ab.py v3 1,4 8 > gpurun_out/lg_ab_v3.log 2>&1
timeout 400 python scripts/decode_ab.py v25 4 8 > gpurun_out/lg_ab_v25.log 2>&1
timeout 400 python scripts/decode_trace.py v25 4 8 > gpurun_out/lg_trace_v25.log 2>&1
