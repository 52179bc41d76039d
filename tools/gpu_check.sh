#!/bin/bash
# One GPU round trip: build, parity tests, smoke, bench, ncu launch list + full capture.
# usage (from gpurun): bash tools/gpu_check.sh [tag]
set -x
TAG=${1:-r01}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $OUT/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -50 $OUT/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -30 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
tail -3 $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
cat $OUT/bench.json; tail -5 $OUT/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-next > $OUT/ncu_bench.log 2>&1; echo "ncu list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:attribute_kernel -s 3 -c 1 \
    -o $OUT/attr python bench.py --steps 1 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-next > $OUT/ncu_full.log 2>&1; echo "ncu full rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"tile_reduce|object_finalize|range_expand" -s 6 -c 3 \
    -o $OUT/fin python bench.py --steps 1 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-next > $OUT/ncu_fin.log 2>&1; echo "ncu fin rc=$?"
ls -la $OUT
