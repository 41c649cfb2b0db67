# round 2: decode A/B of the current library against the red.global.add commit (ca52008), same box
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
for i in 1 2; do
  timeout 300 python scripts/decode_ab.py v3 2 > gpurun_out/dab_new_$i.json 2>&1; tail -1 gpurun_out/dab_new_$i.json
  (cd oldref_tmp && timeout 300 python scripts/decode_ab.py v3 2 > ../gpurun_out/dab_old_$i.json 2>&1; tail -1 ../gpurun_out/dab_old_$i.json)
done
timeout 150 python scripts/decode_trace.py v3 1 8 1 3 > gpurun_out/dab_trace_new_def.txt 2>&1
(cd oldref_tmp && timeout 150 python scripts/decode_trace.py v3 1 8 1 3 > ../gpurun_out/dab_trace_old_def.txt 2>&1)
timeout 1500 python scripts/all_configs.py gpurun_out/all_configs_r02.md > gpurun_out/all_configs_r02.jsonl 2>&1; tail -20 gpurun_out/all_configs_r02.md
