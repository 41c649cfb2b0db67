cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests -m gpu -q -x -k "decode or small or deferr" > gpurun_out/fd11_parity.log 2>&1; echo "rc=$?" >> gpurun_out/fd11_parity.log
timeout 200 python scripts/decode_ab.py v3 1,4 1 > gpurun_out/fd11_ab_L1.log 2>&1
timeout 400 python scripts/decode_ab.py v3 1,4 8 > gpurun_out/fd11_ab_L8.log 2>&1
MOE_DECODE_CHAIN=1 timeout 400 python scripts/decode_ab.py v3 1 8 > gpurun_out/fd11_ab_L8_chain.log 2>&1
timeout 200 python scripts/decode_trace.py v3 1 > gpurun_out/fd11_trace.log 2>&1
