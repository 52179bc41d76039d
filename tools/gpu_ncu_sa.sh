#!/bin/bash
# ncu --set full of the NEXT-3 SA kernels on full-size C2 (second pass)
TAG=${1:-sa}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:structured -s 2 -c 2 -o $OUT/sa python tools/next_probe.py 1e8 structured > $OUT/ncu.log 2>&1; echo "ncu rc=$?"
ncu -i $OUT/sa.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sectors_srcunit_tex_op_atom.sum,lts__t_sectors_srcunit_tex_op_read.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,lts__t_sector_hit_rate.pct > $OUT/raw.csv 2>&1
cat $OUT/raw.csv | cut -c1-600
