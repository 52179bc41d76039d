#!/bin/bash
# Warm-cache launch times of the finalize kernels for library variants: bash tools/ncu_fin_list.sh OUT build/ab/<v> ...
OUT=$(realpath -m $1); shift
mkdir -p $OUT
for v in "$@"; do
  name=$(basename $v)
  rm -rf /tmp/nf_$name; mkdir -p /tmp/nf_$name
  cp -r bench.py tracegen oracle paper_conf_asplos_linzs23_b200 MEASURED_PEAKS.json profiles /tmp/nf_$name/ 2>/dev/null
  cp $v/libdrgpum.so /tmp/nf_$name/paper_conf_asplos_linzs23_b200/libdrgpum.so
  (cd /tmp/nf_$name && timeout 600 ncu --metrics gpu__time_duration.sum --cache-control none --clock-control none \
     -k regex:"${KREGEX:-tile_reduce|group_reduce|object_finalize|attribute_kernel|range_expand|reset_kernel}" -s 20 -c 30 --csv --log-file $OUT/$name.csv \
     python bench.py --steps 5 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-next) > $OUT/$name.out 2> $OUT/$name.err
  python - "$OUT/$name.csv" "$name" <<'PY' | tee -a $OUT/summary.txt
import csv, sys, collections
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]; ki = h.index("Kernel Name"); vi = h.index("Metric Value")
d = collections.defaultdict(list)
for r in rows[1:]:
    d[r[ki].split("(")[0][:40]].append(float(r[vi].replace(",", "")))
for k, v in d.items(): print(sys.argv[2], f"{k:40s} n={len(v):3d} mean_us={sum(v)/len(v)/1000 if max(v) > 1e4 else sum(v)/len(v):.2f}")
PY
done
