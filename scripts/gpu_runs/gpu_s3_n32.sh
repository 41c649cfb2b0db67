cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/n32_parity.log 2>&1; echo "rc=$?" >> gpurun_out/n32_parity.log
SWEEP_SKIP_SKEW=1 timeout 900 python scripts/sweeps.py gpurun_out/n32_sweeps.md > gpurun_out/n32_sweeps.log 2>&1
timeout 400 python scripts/decode_ab.py v3 1,4 8 > gpurun_out/n32_ab_v3.log 2>&1
