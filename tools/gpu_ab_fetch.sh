#!/bin/bash
TAG=${1:-abf}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
bash tools/build_variant.sh v1 -DDRGPUM_FETCH_V2=0 > /dev/null 2>&1
bash tools/build_variant.sh v2 > /dev/null 2>&1
for c in C2 C5; do
  BENCH_ARGS="--config $c --extra-configs none --no-parity --steps 10" bash tools/ab.sh $OUT/ab_$c 3 build/ab/v1 build/ab/v2 > /dev/null 2>&1
done
cat $OUT/ab_*/summary.txt
