cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "small or full" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-decode --no-e2e --no-cpu > gpurun_out/bench6.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench6.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:umma_grouped_gemm -s 3 -c 3 -o gpurun_out/prof_prefill6 python scripts/profile_layer.py --config v3 --tokens 8192 --iters 2 > gpurun_out/ncu_full.log 2>&1
