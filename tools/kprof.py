"""In-context per-kernel device times of the bench step (torch.profiler /
CUPTI activity records: kernels run back to back as in bench.py, no replay).
usage: python tools/kprof.py [--config C2] [--steps 10]"""
import argparse, os, sys, collections
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch
from paper_conf_asplos_linzs23_b200 import Session
from tracegen import build_config, gen_records

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--steps", type=int, default=10)
ap.add_argument("--records", type=int, default=None)
a = ap.parse_args()
prog = build_config(a.config, **({"n_records": a.records} if a.records else {}))
if a.config in ("C3", "C4", "C5"):   # device generation (tracegen/gen.cu)
    from tracegen.device import DeviceProgram
    d = DeviceProgram(prog).gen(0, prog.n_records)
else:
    recs = gen_records(prog, 0, prog.n_records)
    d = torch.from_numpy(recs.view(np.uint8)).cuda()
s = Session(prog.objects, prog.kinds)
for _ in range(3):
    s.reset(); s.attribute(d); s.finalize()
torch.cuda.synchronize()
with torch.profiler.profile(activities=[torch.profiler.ProfilerActivity.CUDA]) as prof:
    for _ in range(a.steps):
        s.reset(); s.attribute(d); s.finalize()
    torch.cuda.synchronize()
agg = collections.defaultdict(list)
evs = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA]
for e in evs:
    agg[e.name.split("(")[0][:48]].append(e.device_time_total if hasattr(e, "device_time_total") else e.cuda_time_total)
tot = 0.0
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print(f"{k:50s} n={len(v):4d} mean_us={np.mean(v):9.2f} per_step_us={sum(v)/a.steps:9.2f}")
    tot += sum(v) / a.steps
print(f"{'sum of kernel time per step':50s} {tot:.2f} us")
# gaps: first-to-last span per step
ts = sorted((e.time_range.start, e.time_range.end) for e in evs)
if ts:
    print(f"span of all kernels / steps: {(ts[-1][1] - ts[0][0]) / a.steps:.2f} us")
