#!/bin/bash
TAG=${1:-vs}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
for P in 2 4 8; do timeout 900 python tools/owned_time_dev.py $P C5 > $OUT/c5_p$P.json 2> $OUT/c5_p$P.err; echo "P=$P rc=$?"; python -c "
import json; d=json.load(open('$OUT/c5_p$P.json')); print(d['P'], d['max_per_rank_ms'], d['owned_equals_single'])" 2>&1 | tail -1; done
