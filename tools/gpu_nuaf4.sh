#!/bin/bash
TAG=${1:-n10}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_frequency.py tests/test_gpu_structured.py -q -x -k "not c2_prefix" > $OUT/pytest_freq.log 2>&1; echo "freq rc=$?"; tail -2 $OUT/pytest_freq.log
for cap in 16777216 134217728; do timeout 600 python tools/nuaf_prof.py C2 $cap > $OUT/nuaf_prof_$cap.txt 2>&1; echo "== cap $cap"; grep -v -i warn $OUT/nuaf_prof_$cap.txt | head -10; done
