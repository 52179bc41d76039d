#!/bin/bash
# Round-3 session: attribution A/B (base = HEAD before the change, lean = working tree) on C2 / C5,
# attribution parity tests with the working tree, NEXT-2 ranking A/B.
TAG=${1:-ab3}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_small_objects.py tests/test_gpu_configs.py tests/test_gpu_fullsize.py -m gpu -q -x > $OUT/pytest_attr.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_attr.log
tail -3 $OUT/pytest_attr.log
for c in ${CFGS:-C2 C5}; do
  BENCH_ARGS="--config $c --extra-configs none --no-parity --steps ${STEPS:-10}" bash tools/ab.sh $OUT/ab_$c ${ROUNDS:-2} ${VARS:-build/ab/base build/ab/lean} > /dev/null 2>&1
done
cat $OUT/ab_*/summary.txt
[ -n "$NUAF" ] && VARIANTS="$NUAF" bash tools/gpu_ab_nuaf2.sh $TAG/nuaf
exit 0
