# round 2: route -> stream hand-off A/B (late vs early trigger) for the TP8 rank and the full layer
cd $GRAFT_REPO_ROOT
MOE_EXPERIMENTS=1 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_exp.log 2>&1 || exit 1
for e in 0 1; do
  MOE_ROUTE_EARLY=$e timeout 150 python scripts/decode_trace.py v3 1 8 8 > gpurun_out/trig${e}_tp8.txt 2>&1; grep chain gpurun_out/trig${e}_tp8.txt
  MOE_ROUTE_EARLY=$e timeout 150 python scripts/decode_trace.py v3 1 8 4 > gpurun_out/trig${e}_tp4.txt 2>&1; grep chain gpurun_out/trig${e}_tp4.txt
  MOE_ROUTE_EARLY=$e timeout 150 python scripts/decode_trace.py v3 1 8 > gpurun_out/trig${e}_v3.txt 2>&1; grep chain gpurun_out/trig${e}_v3.txt
done
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
