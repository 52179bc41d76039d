"""Per-kernel device times of one NEXT-2 attribute call on C2 (torch profiler)."""
import collections, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch
import bench
from paper_conf_asplos_linzs23_b200 import Session

w = bench.Workload(sys.argv[1] if len(sys.argv) > 1 else "C2")
d = w.d_recs[:16 * w.n_local]
cap = int(sys.argv[2]) if len(sys.argv) > 2 else None
s = Session(w.prog.objects, w.prog.kinds, frequency=True, frequency_capacity=cap)
for _ in range(2):
    s.reset(); s.attribute(d); s.frequency(20)
torch.cuda.synchronize()
ms = []
for _ in range(3):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.reset(); e0.record(); s.attribute(d); e1.record(); torch.cuda.synchronize(); ms.append(e0.elapsed_time(e1))
print("attribute + NUAF pass ms", np.median(ms))
with torch.profiler.profile(activities=[torch.profiler.ProfilerActivity.CUDA]) as prof:
    s.reset(); s.attribute(d); s.frequency(20)
    torch.cuda.synchronize()
agg = collections.defaultdict(list)
for e in prof.events():
    if e.device_type == torch.autograd.DeviceType.CUDA:
        agg[e.name.split("(")[0][:48]].append(e.device_time_total if hasattr(e, "device_time_total") else e.cuda_time_total)
tot = 0
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print(f"{k:50s} n={len(v):4d} mean_us={np.mean(v):9.2f} total_us={sum(v):9.2f}")
    tot += sum(v)
print("sum", tot)
