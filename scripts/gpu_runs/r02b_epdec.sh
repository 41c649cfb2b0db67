# round 2: EP expert side at decode sizes through the fused decode stream -- EP tests
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest -q -p no:cacheprovider tests/test_gpu_ep.py > gpurun_out/epdec.log 2>&1; tail -25 gpurun_out/epdec.log
