cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/f3_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/f3_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f3_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/f3_smoke.log
start=$(date +%s)
timeout 900 python bench.py > gpurun_out/f3_bench.log 2>&1
echo "bench wall s: $(( $(date +%s) - start ))" >> gpurun_out/f3_smoke.log
