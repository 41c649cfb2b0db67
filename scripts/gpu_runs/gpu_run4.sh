cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --warmup 3 --cpu-budget 5 > gpurun_out/bench4.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench4.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_prefill.csv python scripts/profile_layer.py --config v3 --tokens 8192 --iters 3 > gpurun_out/ncu_launch.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_decode.csv python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 >> gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:umma_grouped_gemm -s 3 -c 3 -o gpurun_out/prof_prefill python scripts/profile_layer.py --config v3 --tokens 8192 --iters 2 > gpurun_out/ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemv -s 4 -c 4 -o gpurun_out/prof_decode python scripts/profile_layer.py --config v3 --tokens 1 --iters 3 >> gpurun_out/ncu_full.log 2>&1
ls -la gpurun_out/ >> gpurun_out/ncu_full.log
