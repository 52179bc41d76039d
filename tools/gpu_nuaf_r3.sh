#!/bin/bash
# NEXT-2 A/B (VARIANTS) + ncu source captures of the event kernel and one one-sweep pass on C2.
TAG=${1:-nr3}; OUT=gpurun_out/$TAG; mkdir -p $OUT
VARIANTS="${VARIANTS:-}" bash tools/gpu_ab_nuaf2.sh $TAG/ab
for k in freq_events_kernel freq_onesweep_kernel; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 2 -c 1 -o $OUT/$k \
    python tools/nuaf_prof.py C2 134217728 > $OUT/ncu_$k.log 2>&1; echo "ncu $k rc=$?"
  ncu -i $OUT/$k.ncu-rep --page source --csv --print-source=cuda,sass > $OUT/src_$k.csv 2>/dev/null
  python tools/ncu_srclines.py $OUT/src_$k.csv 30 > $OUT/lines_$k.txt 2>&1; head -32 $OUT/lines_$k.txt
done
