#!/bin/bash
TAG=${1:-ck}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_small_objects.py tests/test_gpu_merge_peers.py tests/test_gpu_fullsize.py -q -x > $OUT/pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $OUT/pytest.log
timeout 900 python tools/owned_time_dev.py 8 C5 > $OUT/c5_p8.json 2>/dev/null; python -c "
import json; d=json.load(open('$OUT/c5_p8.json')); print(d['P'], d['max_per_rank_ms'], d['owned_equals_single'])"
timeout 900 python bench.py --extra-configs C2 --no-next --no-cpu-baseline --e2e-steps 1 > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
python -c "
import json; d=json.loads(open('$OUT/bench.json').read().strip().splitlines()[-1])
print('C5 value %.4g'%d['value'], {k:round(v,4) for k,v in d['phases_ms'].items()}, 'frac %.4f'%d['roofline']['frac'], 'parity', d['parity'].get('ok'))
c=d['other_configs']['C2']; print('C2 value %.4g'%c['value'], {k:round(v,4) for k,v in c['phases_ms'].items()}, 'frac %.4f'%c['roofline']['frac'], c['parity'].get('ok'))"
