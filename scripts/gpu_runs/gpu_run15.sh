cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"route_small|quant_gather|combine" -s 3 -c 3 -o gpurun_out/prof_small15 python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 > gpurun_out/ncu_full.log 2>&1
