#!/bin/bash
TAG=${1:-abn}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
cp paper_conf_asplos_linzs23_b200/libdrgpum.so /tmp/lib_default.so
bash tools/build_variant.sh t2048 -DDRGPUM_FQ_TILE=2048 > /dev/null 2>&1
bash tools/build_variant.sh t2048g8 -DDRGPUM_FQ_TILE=2048 -DDRGPUM_FQ_GRID=8 > /dev/null 2>&1
bash tools/build_variant.sh t4096g8 -DDRGPUM_FQ_GRID=8 > /dev/null 2>&1
for v in default t2048 t2048g8 t4096g8; do
  if [ $v = default ]; then cp /tmp/lib_default.so paper_conf_asplos_linzs23_b200/libdrgpum.so; else cp build/ab/$v/libdrgpum.so paper_conf_asplos_linzs23_b200/libdrgpum.so; fi
  timeout 300 python tools/nuaf_prof.py C2 > $OUT/prof_$v.txt 2>&1
  echo "== $v"; grep -v -i warn $OUT/prof_$v.txt | head -5
done
cp /tmp/lib_default.so paper_conf_asplos_linzs23_b200/libdrgpum.so
