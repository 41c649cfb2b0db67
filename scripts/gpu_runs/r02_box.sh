# round 2: 16-row token boxes in the prefill GEMMs (A/B against HEAD in oldref_tmp) + MMA-warp diagnostics
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
for i in 1 2 3; do
  echo "new $(timeout 300 python scripts/time_stages.py v3 8192 2>&1 | tail -1)"
  echo "old $(cd oldref_tmp && timeout 300 python scripts/time_stages.py v3 8192 2>&1 | tail -1)"
done
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/pytest_box.log 2>&1; tail -2 gpurun_out/pytest_box.log
MOE_EXPERIMENTS=1 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_exp.log 2>&1 || exit 1
for m in 0 1 2 3; do echo "mode $m $(MOE_DEBUG_GEMM=$m timeout 300 python scripts/time_stages.py v3 8192 2>&1 | tail -1)"; done
for m in 0 3; do echo "trace mode $m"; MOE_DEBUG_GEMM=$m timeout 300 python scripts/gemm_trace.py v3 8192 2>&1 | tail -2; done
