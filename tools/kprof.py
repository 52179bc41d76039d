"""In-context per-kernel device times of bench.py's step (torch.profiler /
CUPTI activity records: kernels run back to back as in bench.py, no replay).
Uses bench.Workload, so C5 streams its device-generated chunks (the
generator's kernels are listed too; bench.py does not time them).
usage: python tools/kprof.py [--config C5] [--steps 5] [--records N]"""
import argparse, os, sys, collections
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch
import bench

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C5")
ap.add_argument("--steps", type=int, default=5)
ap.add_argument("--records", type=int, default=None)
a = ap.parse_args()
w = bench.Workload(a.config, a.records)
for _ in range(2):
    w.step()
torch.cuda.synchronize()
with torch.profiler.profile(activities=[torch.profiler.ProfilerActivity.CUDA]) as prof:
    for _ in range(a.steps):
        w.step()
    torch.cuda.synchronize()
agg = collections.defaultdict(list)
evs = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA]
for e in evs:
    agg[e.name.split("(")[0][:48]].append(e.device_time_total if hasattr(e, "device_time_total") else e.cuda_time_total)
tot = 0.0
print(f"{a.config}: {w.N} records, {len(w.chunks)} attribute launches per step")
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print(f"{k:50s} n={len(v):4d} mean_us={np.mean(v):9.2f} per_step_us={sum(v)/a.steps:9.2f}")
    tot += sum(v) / a.steps
print(f"{'sum of kernel time per step':50s} {tot:.2f} us")
