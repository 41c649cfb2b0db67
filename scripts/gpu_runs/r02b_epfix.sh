# round 2: fixed-capacity (capturable) expert parallelism -- EP tests incl. graph capture
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest -q -p no:cacheprovider tests/test_gpu_ep.py tests/test_gpu_multidevice.py > gpurun_out/epfix.log 2>&1; tail -15 gpurun_out/epfix.log
