#!/bin/bash
# ncu --set full of one attribute_kernel launch per config, with the source page exported (per-line
# executed instructions / stall samples) for tools/ncu_lines.py.
TAG=${1:-ns}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
for c in ${CFGS:-C5 C2}; do
  skip=1; [ $c = C5 ] && skip=22
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:attribute_kernel -s $skip -c 1 -o $OUT/attr_$c \
    python tools/ncu_one.py --config $c > $OUT/ncu_attr_$c.log 2>&1; echo "attr $c rc=$?"
  ncu -i $OUT/attr_$c.ncu-rep --page source --csv --print-source cuda > $OUT/src_$c.csv 2>/dev/null
  ncu -i $OUT/attr_$c.ncu-rep --page raw --csv > $OUT/raw_$c.csv 2>/dev/null
  python tools/ncu_lines.py $OUT/src_$c.csv 45 > $OUT/lines_$c.txt 2>&1; head -50 $OUT/lines_$c.txt
done
