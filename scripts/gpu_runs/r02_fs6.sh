# round 2: one-token select for softmax gates (V2-Lite / Qwen2) + the v3_g32 preset; full GPU suite
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_fs6.log 2>&1; tail -3 gpurun_out/pytest_fs6.log
for c in v2lite qwen2; do
  timeout 300 python scripts/decode_ab.py $c 2 2>&1 | tail -1
  (cd oldref_tmp && timeout 300 python scripts/decode_ab.py $c 2 2>&1 | tail -1)
done
timeout 150 python scripts/decode_trace.py v2lite 1 8 2>&1 | grep "route:"
