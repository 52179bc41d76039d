#!/bin/bash
# NEXT-2 change check: frequency GPU tests, then the C2 per-kernel profile.
TAG=${1:-nc}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_frequency.py tests/test_gpu_structured.py -q -x > $OUT/pytest_freq.log 2>&1; echo "freq tests rc=$?"; tail -3 $OUT/pytest_freq.log
for i in 1 2; do timeout 300 python tools/nuaf_prof.py C2 134217728 > $OUT/prof_$i.txt 2>&1; grep -v -i warn $OUT/prof_$i.txt | head -12; done
