#!/bin/bash
# GPU parity subset + A/B of finalize / reset variants + per-kernel times (torch profiler) on C5 and C2.
TAG=${1:-abfin}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q -x -k "not c2_prefix" > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -3 $OUT/pytest_gpu.log
bash tools/build_variant.sh trbig -DDRGPUM_TR_SMALL=0 > /dev/null 2>&1
bash tools/build_variant.sh full > /dev/null 2>&1
for c in C5 C2; do
  BENCH_ARGS="--config $c --extra-configs none --no-parity --steps 10" bash tools/ab.sh $OUT/ab_$c 2 build/ab/trbig build/ab/full
done
for c in C5 C2; do timeout 600 python tools/kprof.py --config $c --steps 5 > $OUT/kprof_$c.txt 2>&1; done
cat $OUT/kprof_*.txt
