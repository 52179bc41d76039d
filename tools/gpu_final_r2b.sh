#!/bin/bash
# Round-2 final (after the late attribution / NEXT-2 changes): full GPU suite, smoke, the default bench
# line, its launch list, ncu --set full of attribution (C5, C2), finalize (C5), NEXT-2's event kernel and
# one one-sweep pass (C2), then compute-sanitizer over the kernel subset.
TAG=${1:-fin2}; OUT=gpurun_out/$TAG; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $OUT/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q -x --durations=8 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -3 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke.log
timeout 1500 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
python -c "
import json; d=json.loads(open('$OUT/bench.json').read().strip().splitlines()[-1])
print('value %.4g'%d['value'], 'ms', d['ms_per_step'], d['phases_ms'], 'frac', d['roofline']['frac'], 'parity', d['parity'].get('ok'), 'clocks', d['clocks'])
for c,v in d.get('other_configs',{}).items(): print(c, v.get('value'), v.get('phases_ms'), v.get('roofline',{}).get('frac'), (v.get('parity') or {}).get('ok'), v.get('error'))
nx=d['other_configs'].get('C2',{}).get('next') or {}
for k,v in nx.items(): print(k, v)
print('cpu', d['cpu_baseline']['value'], 'e2e', d['e2e']['value'])
"
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
  python bench.py --steps 2 --warmup 1 --e2e-steps 1 --no-cpu-baseline --extra-configs none --no-parity > $OUT/ncu_list.log 2>&1; echo "list rc=$?"
for c in C5 C2; do
  skip=1; [ $c = C5 ] && skip=22
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:attribute_kernel -s $skip -c 1 -o $OUT/attr_$c \
    python tools/ncu_one.py --config $c > $OUT/ncu_attr_$c.log 2>&1; echo "attr $c rc=$?"
  ncu -i $OUT/attr_$c.ncu-rep --page raw --csv > $OUT/raw_attr_$c.csv 2>/dev/null
done
timeout 900 ncu --set full --clock-control none -k regex:"tile_reduce|object_finalize|reset_touched" -s 3 -c 3 -o $OUT/fin_C5 \
  python tools/ncu_one.py --config C5 > $OUT/ncu_fin.log 2>&1; echo "fin rc=$?"
for k in freq_events_kernel freq_onesweep_kernel; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 2 -c 1 -o $OUT/$k \
    python tools/nuaf_prof.py C2 134217728 > $OUT/ncu_$k.log 2>&1; echo "ncu $k rc=$?"
done
timeout 300 python tools/nuaf_prof.py C2 134217728 > $OUT/nuaf_prof.txt 2>&1; grep -v -i warn $OUT/nuaf_prof.txt | head -12
if [ -n "$SAN" ]; then bash tools/gpu_sanitize.sh $TAG/san; fi   # (compute-sanitizer is closed on the current pool)
