cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 150 python scripts/decode_trace.py v3 1 8 1 3 > gpurun_out/deftr_v3.txt 2>&1; cat gpurun_out/deftr_v3.txt | head -30
timeout 150 python scripts/decode_trace.py v3 1 8 > gpurun_out/plaintr_v3.txt 2>&1; head -12 gpurun_out/plaintr_v3.txt
