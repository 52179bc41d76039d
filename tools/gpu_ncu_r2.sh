#!/bin/bash
# ncu evidence for the round-2 bench: launch list of the default bench (C5),
# --set full captures of attribute_kernel on C2..C5 and of the finalize kernels.
# usage (from gpurun): bash tools/gpu_ncu_r2.sh TAG
TAG=${1:-ncu}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
NCU="ncu --clock-control none"
timeout 1200 $NCU --metrics gpu__time_duration.sum --csv --log-file $OUT/launches_c5.csv \
  python bench.py --steps 2 --warmup 1 --e2e-steps 1 --no-cpu-baseline --extra-configs '' --no-parity > $OUT/ncu_list.log 2>&1
echo "list rc=$?"
for c in C2 C3 C4 C5; do
  skip=1; [ $c = C5 ] && skip=22
  timeout 900 $NCU --set full --import-source on -k regex:attribute_kernel -s $skip -c 1 -o $OUT/attr_$c \
    python tools/ncu_one.py --config $c > $OUT/ncu_attr_$c.log 2>&1
  echo "attr $c rc=$?"
done
for c in C2 C5; do
  timeout 900 $NCU --set full --import-source on -k regex:"tile_reduce|group_reduce|object_finalize|reset_kernel" -s 4 -c 4 \
    -o $OUT/fin_$c python tools/ncu_one.py --config $c > $OUT/ncu_fin_$c.log 2>&1
  echo "fin $c rc=$?"
done
ls -la $OUT
