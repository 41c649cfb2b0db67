cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests -m gpu -q -x -k "decode or small or gemv or deferr or full_size" > gpurun_out/fd7_parity.log 2>&1; echo "rc=$?" >> gpurun_out/fd7_parity.log
timeout 200 python scripts/decode_ab.py v3 1,4,16 > gpurun_out/fd7_ab_fused.log 2>&1
MOE_DECODE_PF=1 timeout 200 python scripts/decode_ab.py v3 1 > gpurun_out/fd7_ab_pf.log 2>&1
timeout 200 python scripts/decode_trace.py v3 1 > gpurun_out/fd7_trace.log 2>&1
MOE_DECODE_PF=1 timeout 200 python scripts/decode_trace.py v3 1 > gpurun_out/fd7_trace_pf.log 2>&1
