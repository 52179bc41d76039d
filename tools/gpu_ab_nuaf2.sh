#!/bin/bash
# A/B of NEXT-2 ranking variants on C2 (tools/nuaf_prof.py, one sub-call per call).
TAG=${1:-abn}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
cp paper_conf_asplos_linzs23_b200/libdrgpum.so /tmp/lib_default.so
VARIANTS=${VARIANTS:-"match:-DDRGPUM_FQ_MATCH=1"}
names="default"
for v in $VARIANTS; do n=${v%%:*}; f=${v#*:}; bash tools/build_variant.sh $n ${f//,/ } > /dev/null 2>&1 || echo "build $n failed"; names="$names $n"; done
for round in 1 2; do
for v in $names; do
  if [ $v = default ]; then cp /tmp/lib_default.so paper_conf_asplos_linzs23_b200/libdrgpum.so; else cp build/ab/$v/libdrgpum.so paper_conf_asplos_linzs23_b200/libdrgpum.so; fi
  timeout 300 python tools/nuaf_prof.py C2 134217728 > $OUT/prof_${v}_$round.txt 2>&1
  echo "== $v round $round"; grep -v -i warn $OUT/prof_${v}_$round.txt | head -8
done
done
cp /tmp/lib_default.so paper_conf_asplos_linzs23_b200/libdrgpum.so
timeout 600 python -m pytest tests/test_gpu_frequency.py -q -x > $OUT/pytest_freq_default.log 2>&1; echo "freq tests default rc=$?"
