#!/bin/bash
# summarise a gpurun_out/<tag> directory
D=gpurun_out/$1
tail -3 $D/pytest_gpu.log; tail -2 $D/smoke.log
python - "$D" <<'PY'
import json, sys
d = json.load(open(sys.argv[1] + '/bench.json'))
print('value %.3e rec/s  ms/step %.4f' % (d['value'], d['ms_per_step']))
print('phases', {k: round(v, 4) for k, v in d['phases_ms'].items()})
print('roofline achieved %.0f GB/s frac %.3f' % (d['roofline']['achieved'], d['roofline']['frac']))
print('e2e %.3e rec/s (%.1f ms)' % (d['e2e']['value'], d['e2e']['ms_per_step']), 'clocks', d['clocks'], 'launches', d['gpu_launches'])
if d.get('cpu_baseline'): print('cpu', d['cpu_baseline']['value'])
PY
if [ -f $D/attr.ncu-rep ]; then
ncu -i $D/attr.ncu-rep --page details --csv 2>/dev/null | grep -E '"(Duration|DRAM Throughput|Executed Instructions|Registers Per Thread|Achieved Occupancy|Issue Slots Busy|L2 Hit Rate|Compute \(SM\) Throughput)"' | awk -F'","' '{print $(NF-3)" | "$(NF-1)" | "$NF}'
fi
