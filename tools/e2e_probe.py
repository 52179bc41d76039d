"""Where the e2e step's time goes (C5, 2^28-record host sample): ingest,
finalize+stats D2H, patterns D2H, pageable vs pinned result arrays."""
import json, sys, os, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import bench
from paper_conf_asplos_linzs23_b200 import pinned_array, STATS_DTYPE, REPORT_DTYPE
n = 1 << 28
w = bench.Workload("C5", n)
pinned = torch.empty(16 * n, dtype=torch.uint8, pin_memory=True)
tmp = torch.empty(16 * bench.GEN_CHUNK, dtype=torch.uint8, device="cuda")
for c0 in range(0, n, bench.GEN_CHUNK):
    c1 = min(n, c0 + bench.GEN_CHUNK)
    w.dp.gen(w.lo + c0, w.lo + c1, out=tmp)
    pinned[16 * c0:16 * c1].copy_(tmp[:16 * (c1 - c0)])
torch.cuda.synchronize()
hs, hr = pinned_array(w.prog.n_obj, STATS_DTYPE), pinned_array(w.prog.n_obj, REPORT_DTYPE)
out = {}
def t(name, f, reps=3):
    f(); torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps): f()
    torch.cuda.synchronize()
    out[name] = (time.perf_counter() - t0) / reps * 1e3
t("reset+attribute_host_ms", lambda: (w.s.reset(), w.s.attribute(pinned)))
t("object_stats_pageable_ms", lambda: w.s.object_stats())
t("object_stats_pinned_ms", lambda: w.s.object_stats(out=hs))
t("patterns_pageable_ms", lambda: w.s.patterns())
t("patterns_pinned_ms", lambda: w.s.patterns(out=hr))
a, _ = w.s.object_stats(); b = w.s.patterns()
out["same_stats"] = bool((a.view("u1") == hs.view("u1")).all())
out["same_reports"] = bool((b.view("u1") == hr.view("u1")).all())
print(json.dumps(out))
