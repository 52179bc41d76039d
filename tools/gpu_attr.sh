#!/bin/bash
# Attribution iteration: build, parity tests of the attribution path, bench (no NEXT rows),
# one ncu --set full capture of attribute_kernel.   usage: bash tools/gpu_attr.sh TAG
TAG=${1:-a}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -50 $OUT/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_configs.py -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -3 $OUT/pytest_gpu.log
timeout 600 python bench.py --no-next ${BENCH_ARGS:-} > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; tail -3 $OUT/bench.err
python -c "
import json; d=json.load(open('$OUT/bench.json'))
print('ms/step', d['ms_per_step'], 'phases', d['phases_ms'], 'frac', d['roofline']['frac'], 'achieved', d['roofline']['achieved'])"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attribute_kernel -s 3 -c 1 \
    -o $OUT/attr python bench.py --steps 1 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-next > $OUT/ncu_attr.log 2>&1; echo "ncu attr rc=$?"
