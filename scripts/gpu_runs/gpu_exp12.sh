cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "swap or small_layer or full_size_sampled" > gpurun_out/exp12_parity.log 2>&1
for dbg in 0 2; do
MOE_DEBUG_GEMM=$dbg timeout 300 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu --no-decode > gpurun_out/exp12_dbg$dbg.log 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"route_small" -s 3 -c 1 -o gpurun_out/prof_route python scripts/profile_layer.py --config v3 --tokens 1 --iters 5 > gpurun_out/ncu_route.log 2>&1
