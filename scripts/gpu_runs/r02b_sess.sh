# this session net change, final: HEAD vs the session start 2d1588e (oldref_tmp), interleaved, every config (prefill)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
(cd oldref_tmp && python -c "import __graft_entry__ as g; g.build()" > ../gpurun_out/build_old.log 2>&1) || exit 1
nvidia-smi --query-gpu=name,power.limit --format=csv,noheader
summ='import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; s=r["stage_ms"]; print(round(d["value"]), round(d["ms_per_step"],4), round(r["kernel_ms"],3), s["gemm2"], s["combine"])'
for c in v3 v2lite qwen2 v25; do for i in 1 2; do
  echo "$c new $(timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
  echo "$c old $(cd oldref_tmp && timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e --no-decode 2>/dev/null | tail -1 | python -c "$summ")"
done; done
