cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests -m gpu -q -x -k "decode or small or deferr" > gpurun_out/tr_parity.log 2>&1; echo "rc=$?" >> gpurun_out/tr_parity.log
timeout 400 python scripts/decode_ab.py v3 1,4 8 > gpurun_out/tr_ab_early.log 2>&1
MOE_DECODE_LATE_TRIGGER=1 timeout 400 python scripts/decode_ab.py v3 1,4 8 > gpurun_out/tr_ab_late.log 2>&1
timeout 400 python scripts/decode_ab.py v3 1,4 8 > gpurun_out/tr_ab_early2.log 2>&1
timeout 400 python scripts/decode_trace.py v3 1 8 > gpurun_out/tr_trace.log 2>&1
