#!/bin/bash
TAG=${1:-r2g}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 300 python tools/probe_multicast.py > $OUT/multicast.json 2> $OUT/multicast.err; echo "probe rc=$?"; head -c 600 $OUT/multicast.json
timeout 900 python -m pytest tests/test_gpu_frequency.py tests/test_gpu_structured.py -q -x -k "not c2_prefix" > $OUT/pytest_freq.log 2>&1; echo "freq rc=$?"; tail -2 $OUT/pytest_freq.log
timeout 600 python tools/nuaf_prof.py C2 > $OUT/nuaf_prof.txt 2>&1; cat $OUT/nuaf_prof.txt | head -30
timeout 1500 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"; tail -3 $OUT/bench.err
python -c "
import json; d=json.loads(open('$OUT/bench.json').read().strip().splitlines()[-1])
print('value %.4g'%d['value'], 'ms', d['ms_per_step'], d['phases_ms'], 'frac', d['roofline']['frac'], 'parity', d['parity'].get('ok'), d['parity'].get('mismatches'))
for c,v in d.get('other_configs',{}).items(): print(c, v.get('value'), v.get('phases_ms'), v.get('roofline',{}).get('frac'), (v.get('parity') or {}).get('ok'), v.get('error'))
print('next', json.dumps(d['other_configs'].get('C2',{}).get('next'))[:600])
print('cpu', d['cpu_baseline']); print('e2e', d['e2e']['value'])
"
