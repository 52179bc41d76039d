#!/bin/bash
TAG=${1:-n9}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
for cap in 16777216 134217728; do timeout 600 python tools/nuaf_prof.py C2 $cap > $OUT/nuaf_prof_$cap.txt 2>&1; echo "== cap $cap"; grep -v -i warn $OUT/nuaf_prof_$cap.txt | head -9; done
