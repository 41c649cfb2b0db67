cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests -m gpu -q -x -k "decode or small or gemv or deferr" > gpurun_out/fd1_parity_decode.log 2>&1; echo "rc=$?" >> gpurun_out/fd1_parity_decode.log
timeout 200 python scripts/decode_ab.py v3 1,4,16 > gpurun_out/fd1_ab_fused.log 2>&1
MOE_DECODE_CHAIN=1 timeout 200 python scripts/decode_ab.py v3 1,4,16 > gpurun_out/fd1_ab_chain.log 2>&1
timeout 600 python -m pytest tests -m gpu -q -x > gpurun_out/fd1_parity_all.log 2>&1; echo "rc=$?" >> gpurun_out/fd1_parity_all.log
timeout 400 python bench.py --no-cpu > gpurun_out/fd1_bench.log 2>&1
