#!/bin/bash
# attribution A/B (VARS: build/ab dirs) on C5 / C2 + the tests touched since the last GPU run
TAG=${1:-ab4}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py::test_c1_full tests/test_gpu_frequency.py -q -x > $OUT/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest.log
for c in ${CFGS:-C5 C2}; do
  BENCH_ARGS="--config $c --extra-configs none --no-parity --steps ${STEPS:-10}" bash tools/ab.sh $OUT/ab_$c ${ROUNDS:-2} ${VARS} > /dev/null 2>&1
done
cat $OUT/ab_*/summary.txt
