"""Time the NEXT-2 frequency pass on C2 (extra device time over plain
attribution, CUDA events), and check it against the oracle on a prefix.
usage: python tools/freq_time.py [n_records] [frequency|structured]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_asplos_linzs23_b200 import Session
from tracegen import build_config, gen_records

n = int(float(sys.argv[1])) if len(sys.argv) > 1 else 100_000_000
feat = sys.argv[2] if len(sys.argv) > 2 else "frequency"
p = build_config("C2", n_records=n)
recs = gen_records(p, 0, p.n_records)
d = torch.from_numpy(recs.view(np.uint8)).cuda()
out = {}
for name, kw in (("plain", {}), (feat, {feat: True})):
    s = Session(p.objects, p.kinds, **kw)
    for _ in range(2):
        s.reset(); s.attribute(d)
    torch.cuda.synchronize()
    ms = []
    for _ in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.reset(); e0.record(); s.attribute(d); e1.record(); torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
    out[name] = float(np.median(ms))
    if name == "frequency":
        cnt, first = s.frequency(20)
        out["nuaf_objects"] = int((cnt > 0).sum()); out["nuaf_apis"] = int(cnt.sum())
    if name == "structured":
        sa, ov = s.structured()
        out["sa_match"] = int(sa.sum()); out["sa_overlap"] = int(ov.sum())
    del s
print({"n": n, **out, "pass_ms": out[feat] - out["plain"]})
