cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "small or full or ep" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-decode --no-e2e --no-cpu > gpurun_out/bench26_pair.log 2>&1
MOE_PAIR=0 timeout 600 python bench.py --steps 5 --warmup 3 --no-decode --no-e2e --no-cpu > gpurun_out/bench26_nopair.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"umma_pair_gemm" -s 2 -c 2 -o gpurun_out/prof_pair26 python scripts/profile_layer.py --config v3 --tokens 8192 --iters 2 > gpurun_out/ncu_full.log 2>&1
