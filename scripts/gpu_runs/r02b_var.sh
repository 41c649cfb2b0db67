cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 1500 python -m pytest -q -p no:cacheprovider tests/test_gpu_variants.py > gpurun_out/variants.log 2>&1; tail -3 gpurun_out/variants.log
