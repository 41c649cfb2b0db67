cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"umma_decode" -s 2 -c 2 -o gpurun_out/prof_decode12 python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 > gpurun_out/ncu_full.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_decode12.csv python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 >> gpurun_out/ncu_full.log 2>&1
