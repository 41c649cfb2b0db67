# all BASELINE.json layers on the final code
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
nvidia-smi --query-gpu=name,power.limit --format=csv,noheader
timeout 1500 python scripts/all_configs.py gpurun_out/all_configs_fin.md > gpurun_out/all_configs_fin.jsonl 2>&1; cat gpurun_out/all_configs_fin.md
