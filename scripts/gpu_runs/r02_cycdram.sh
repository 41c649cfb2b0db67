cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for m in plain cyclic; do
  timeout 600 ncu --cache-control none --clock-control none --metrics dram__bytes_read.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum -k regex:umma_decode_fused \
    --launch-skip 24 -c 8 --csv python scripts/cyc_dram.py v25 4 $m > gpurun_out/cycdram_$m.csv 2>&1; grep -E "dram__bytes_read|lts__t_sectors" gpurun_out/cycdram_$m.csv | awk -F'","' '{print $(NF-2), $NF}' | head -20
done
