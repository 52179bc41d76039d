#!/bin/bash
# GPU suite + A/B of attribution / reset variants on C2, C3, C5 (bench.py step).
# usage (from gpurun): bash tools/gpu_ab_r2.sh TAG
TAG=${1:-ab}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q -x --durations=10 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -15 $OUT/pytest_gpu.log
bash tools/build_variant.sh base -DDRGPUM_UNION_SCRATCH=0 -DDRGPUM_SPARSE_RESET=0 > /dev/null 2>&1
bash tools/build_variant.sh union -DDRGPUM_UNION_SCRATCH=1 -DDRGPUM_SPARSE_RESET=0 > /dev/null 2>&1
bash tools/build_variant.sh full > /dev/null 2>&1
for c in C5 C3 C2; do
  BENCH_ARGS="--config $c --extra-configs none --no-parity --steps 10" bash tools/ab.sh $OUT/ab_$c 2 build/ab/base build/ab/union build/ab/full
done
cat $OUT/ab_*/summary.txt
