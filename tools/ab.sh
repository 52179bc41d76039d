#!/bin/bash
# A/B timing of prebuilt library variants on one box (same clocks, same HBM).
# usage: bash tools/ab.sh OUTDIR ROUNDS build/ab/<variant> ...   (each dir holds a libdrgpum.so)
OUT=$1; ROUNDS=$2; shift 2
mkdir -p $OUT
for v in "$@"; do
  name=$(basename $v)
  rm -rf /tmp/ab_$name; mkdir -p /tmp/ab_$name
  cp -r bench.py tracegen oracle paper_conf_asplos_linzs23_b200 MEASURED_PEAKS.json profiles /tmp/ab_$name/ 2>/dev/null
  cp $v/libdrgpum.so /tmp/ab_$name/paper_conf_asplos_linzs23_b200/libdrgpum.so
done
for r in $(seq 1 $ROUNDS); do
  for v in "$@"; do
    name=$(basename $v)
    (cd /tmp/ab_$name && timeout 300 python bench.py --no-next --no-cpu-baseline --e2e-steps 1 --steps 40 ${BENCH_ARGS:-}) > $OUT/${name}_$r.json 2> $OUT/${name}_$r.err
    python -c "
import json; d=json.load(open('$OUT/${name}_$r.json'))
print('$name', $r, 'attr_ms %.4f'%d['phases_ms']['attribute'], 'fin_ms %.4f'%d['phases_ms']['finalize'], 'step_ms %.4f'%d['ms_per_step'], 'frac %.4f'%d['roofline']['frac'], 'clk', d['clocks']['sm_mhz'], 'rec', d['counters']['records'], d['counters']['attributed'])" | tee -a $OUT/summary.txt
  done
done
