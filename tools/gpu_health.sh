#!/bin/bash
# Health check after a re-entry: build, full GPU suite, smoke, default bench line.
TAG=${1:-h}; OUT=gpurun_out/$TAG; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $OUT/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q -x --durations=12 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -16 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $OUT/smoke.log
timeout 1500 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; tail -3 $OUT/bench.err
python -c "
import json; d=json.loads(open('$OUT/bench.json').read().strip().splitlines()[-1])
print('value %.4g'%d['value'], 'ms', d['ms_per_step'], d['phases_ms'], 'frac', d['roofline']['frac'], 'parity', d['parity'].get('ok'), 'clocks', d['clocks'])
for c,v in d.get('other_configs',{}).items(): print(c, v.get('value'), v.get('phases_ms'), v.get('roofline',{}).get('frac'), (v.get('parity') or {}).get('ok'), v.get('error'))
nx=d['other_configs'].get('C2',{}).get('next') or {}
for k,v in nx.items(): print(k, v)
print('cpu', d['cpu_baseline']['value'], 'e2e', d['e2e']['value'])
"
