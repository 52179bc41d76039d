#!/bin/bash
TAG=${1:-ns}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:freq_scatter_kernel -s 12 -c 1 -o $OUT/scatter python tools/nuaf_prof.py C2 134217728 > $OUT/ncu.log 2>&1; echo rc=$?
