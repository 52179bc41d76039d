#!/bin/bash
# finalize A/B (VARS) on C5 / C2 + parity tests of finalize, full-size digests and the owned merge
TAG=${1:-ab5}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_small_objects.py tests/test_gpu_merge_peers.py tests/test_gpu_configs.py -q -x > $OUT/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest.log
for c in ${CFGS:-C5 C2}; do
  BENCH_ARGS="--config $c --extra-configs none --no-parity --steps ${STEPS:-10}" bash tools/ab.sh $OUT/ab_$c ${ROUNDS:-2} ${VARS} > /dev/null 2>&1
done
cat $OUT/ab_*/summary.txt
