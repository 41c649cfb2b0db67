cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
for i in 1 2; do timeout 150 python scripts/decode_trace.py v3 1 8 2>&1 | grep "route"; (cd oldref_tmp && timeout 150 python scripts/decode_trace.py v3 1 8 2>&1 | grep "route"); done
for i in 1 2; do
  timeout 300 python scripts/decode_ab.py v3 2 > gpurun_out/fs_new_$i.json 2>&1; tail -1 gpurun_out/fs_new_$i.json
  (cd oldref_tmp && timeout 300 python scripts/decode_ab.py v3 2 > ../gpurun_out/fs_old_$i.json 2>&1; tail -1 ../gpurun_out/fs_old_$i.json)
done
