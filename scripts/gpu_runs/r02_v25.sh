cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_tp_chain.py -k "v25_cyclic or cyclic_chain" > gpurun_out/pytest_v25cyc.log 2>&1; tail -3 gpurun_out/pytest_v25cyc.log
timeout 150 python scripts/decode_trace.py v3 1 8 8 2>&1 | grep -v slowest | tail -12
