#!/bin/bash
# Round-2 GPU check: build, GPU tests (incl. full-size digests), smoke, default bench (C5 + extras).
# usage (from gpurun): bash tools/gpu_r2.sh TAG [pytest selection]
TAG=${1:-r2}; shift
SEL=${@:-tests}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $OUT/gpu.txt 2>&1
free -g > $OUT/host_mem.txt; nproc >> $OUT/host_mem.txt
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -50 $OUT/build.log; exit 1; }
timeout 2400 python -m pytest $SEL -m gpu -q -x --durations=15 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -25 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
tail -2 $OUT/smoke.log
timeout 1500 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
tail -c 3000 $OUT/bench.json; tail -5 $OUT/bench.err
