#!/bin/bash
# Round check on one B200: build, GPU parity tests, smoke, bench (with NEXT rows),
# ncu launch list, ncu full captures of the attribution, finalize and NEXT kernels.
# usage (from gpurun): bash tools/gpu_round.sh [tag]
TAG=${1:-round}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $OUT/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -50 $OUT/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -4 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
tail -2 $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; tail -3 $OUT/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 3 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-next > $OUT/ncu_list.log 2>&1; echo "ncu list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:attribute_kernel -s 3 -c 1 \
    -o $OUT/attr python bench.py --steps 1 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-next > $OUT/ncu_attr.log 2>&1; echo "ncu attr rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"tile_reduce|object_finalize|group_reduce" -s 6 -c 3 \
    -o $OUT/fin python bench.py --steps 1 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-next > $OUT/ncu_fin.log 2>&1; echo "ncu fin rc=$?"
timeout 900 ncu --set full --clock-control none -k regex:"structured_kernel|freq_main_kernel" -c 2 \
    -o $OUT/next python bench.py --steps 1 --warmup 3 --e2e-steps 1 --no-cpu-baseline > $OUT/ncu_next.log 2>&1; echo "ncu next rc=$?"
ls -la $OUT
