#!/bin/bash
TAG=${1:-nuaf}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -30 $OUT/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_frequency.py tests/test_gpu_structured.py -q -x -k "not c2_prefix" > $OUT/pytest_freq.log 2>&1; echo "freq rc=$?"; tail -15 $OUT/pytest_freq.log
timeout 600 python - > $OUT/nuaf_time.txt 2>&1 <<'PY'
import bench, torch, time, numpy as np
w = bench.Workload("C2")
from paper_conf_asplos_linzs23_b200 import Session
d = w.d_recs[:16 * w.n_local]
for name, kw in (("plain", {}), ("freq", {"frequency": True})):
    s = Session(w.prog.objects, w.prog.kinds, **kw)
    for _ in range(2):
        s.reset(); s.attribute(d)
        if kw: s.frequency(20)
    torch.cuda.synchronize()
    ms = []
    for _ in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.reset(); e0.record(); s.attribute(d); e1.record(); torch.cuda.synchronize(); ms.append(e0.elapsed_time(e1))
    t0 = time.perf_counter(); r = s.frequency(20) if kw else None; q = (time.perf_counter() - t0) * 1e3
    print(name, "attribute ms", np.median(ms), "query ms", q, "launches", s.launch_count())
    del s; torch.cuda.empty_cache()
PY
cat $OUT/nuaf_time.txt
timeout 1200 python -m pytest tests/test_gpu_frequency.py -q -k "c2_prefix" > $OUT/pytest_c2prefix.log 2>&1; echo "c2prefix rc=$?"; tail -2 $OUT/pytest_c2prefix.log
timeout 1800 python -m pytest tests -m gpu -q -x -k "not c2_prefix and not test_gpu_frequency" > $OUT/pytest_gpu.log 2>&1; echo "gpu rc=$?"; tail -3 $OUT/pytest_gpu.log
