cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python scripts/sweeps.py gpurun_out/sweeps.md > gpurun_out/sweeps.log 2>&1
timeout 600 /usr/local/cuda/bin/compute-sanitizer --tool memcheck --target-processes all python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "test_fused_decode_residual_deferral and v3_s and 5" > gpurun_out/memcheck_decode.log 2>&1; echo "rc=$?" >> gpurun_out/memcheck_decode.log
timeout 600 /usr/local/cuda/bin/compute-sanitizer --tool memcheck --target-processes all python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "test_small_layer_parity and v3_s" > gpurun_out/memcheck_prefill.log 2>&1; echo "rc=$?" >> gpurun_out/memcheck_prefill.log
