cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 200 python scripts/decode_trace.py v3 1 > gpurun_out/fd8_trace.log 2>&1
timeout 300 ncu -k regex:route_small -s 2 -c 1 --set full --clock-control none --import-source on -o gpurun_out/fd8_route_full python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 > gpurun_out/fd8_ncu.log 2>&1
