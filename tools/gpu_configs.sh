#!/bin/bash
# Full-size BASELINE configs C3-C5 on one B200 (device-generated traces):
# generator parity, then one bench line per config.
# usage (from gpurun): bash tools/gpu_configs.sh TAG [STEPS]
TAG=${1:-cfg}; STEPS=${2:-5}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_tracegen.py -x -q > $OUT/pytest_tracegen.log 2>&1; echo "tracegen pytest rc=$?"; tail -2 $OUT/pytest_tracegen.log
for c in C3 C4 C5; do
  timeout 1200 python bench.py --config $c --steps $STEPS --warmup 3 --e2e-steps 2 > $OUT/bench_$c.json 2> $OUT/bench_$c.err
  echo "$c rc=$?"; tail -2 $OUT/bench_$c.err
  python -c "
import json; d=json.load(open('$OUT/bench_$c.json'))
print('$c', 'rec/s %.3e'%d['value'], 'ms/step %.2f'%d['ms_per_step'], 'phases', {k: round(v,3) for k,v in d['phases_ms'].items()}, 'frac %.3f'%d['roofline']['frac'], 'e2e %.3e'%d['e2e']['value'], 'cpu %.3e'%(d['cpu_baseline'] or {}).get('value',0), d['counters'])" 2>&1 | tail -1
done
