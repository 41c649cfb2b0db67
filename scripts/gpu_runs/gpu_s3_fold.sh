cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests -m gpu -q -x > gpurun_out/fold_parity.log 2>&1; echo "rc=$?" >> gpurun_out/fold_parity.log
timeout 400 python scripts/decode_ab.py v3 1,2,4 8 > gpurun_out/fold_ab.log 2>&1
MOE_DECODE_FOLD=0 timeout 400 python scripts/decode_ab.py v3 1,2,4 8 > gpurun_out/fold_ab_off.log 2>&1
