cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for c in v3 v3_fp4 v2lite; do timeout 400 python scripts/decode_ab.py $c 2 2>&1 | tail -1; done
