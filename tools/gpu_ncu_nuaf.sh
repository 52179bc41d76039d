#!/bin/bash
TAG=${1:-nn}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
for k in freq_hist_kernel freq_scatter_kernel freq_events_kernel freq_sweep_kernel; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 8 -c 1 -o $OUT/$k python tools/nuaf_prof.py C2 > $OUT/ncu_$k.log 2>&1; echo "$k rc=$?"
done
ls -la $OUT
