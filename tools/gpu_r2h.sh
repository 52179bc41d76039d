#!/bin/bash
TAG=${1:-r2h}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_frequency.py tests/test_gpu_structured.py -q -x -k "not c2_prefix" > $OUT/pytest_freq.log 2>&1; echo "freq rc=$?"; tail -2 $OUT/pytest_freq.log
timeout 600 python tools/nuaf_prof.py C2 > $OUT/nuaf_prof.txt 2>&1; grep -v Warn $OUT/nuaf_prof.txt | head -16
for c in C2 C4 C5; do timeout 600 python tools/kprof.py --config $c --steps 5 2>/dev/null | grep -v "^ " > $OUT/kprof_$c.txt; head -9 $OUT/kprof_$c.txt; done
