# round 2: router select cycles, cold (first pass) vs warm (second pass in the same tail)
cd $GRAFT_REPO_ROOT
MOE_EXPERIMENTS=1 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_exp.log 2>&1 || exit 1
for i in 1 2; do MOE_DEBUG_ROUTE=8 timeout 150 python scripts/decode_trace.py v3 1 8 2>&1 | grep -i "select\|route:" ; done
MOE_DEBUG_ROUTE=8 timeout 150 python scripts/decode_trace.py v3 4 8 2>&1 | grep -i "select\|route:"
MOE_DEBUG_ROUTE=8 timeout 150 python scripts/decode_trace.py v25 1 8 2>&1 | grep -i "select\|route:"
