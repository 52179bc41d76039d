"""Per-rank device time of the N>1 step's non-attribution parts on ONE GPU
with P virtual peers (local HBM: the merge times are a lower bound of the
NVLink ones): sparse reset, sparse owned merge, owned finalize, gather --
for any config, shards generated on the device chunk by chunk.
usage: python tools/owned_time_dev.py P [config]"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_asplos_linzs23_b200 import Session  # noqa: E402
from paper_conf_asplos_linzs23_b200.parallel import shard_range  # noqa: E402
from tracegen import build_config  # noqa: E402
from tracegen.device import DeviceProgram  # noqa: E402

P = int(sys.argv[1]) if len(sys.argv) > 1 else 8
cfg = sys.argv[2] if len(sys.argv) > 2 else "C5"
prog = build_config(cfg)
N = prog.n_records
dp = DeviceProgram(prog)
CH = 1 << 30
buf = torch.empty(16 * CH, dtype=torch.uint8, device="cuda")
S = [Session(prog.objects, prog.kinds) for _ in range(P)]
ptrs = [s.workspace.data_ptr() for s in S]


def ev():
    return torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)


def timed(fn):
    a, b = ev()
    torch.cuda.synchronize()
    a.record()
    fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b)


def attribute_all():
    for r, s in enumerate(S):
        s.reset()
        lo, hi = shard_range(N, r, P)
        for c0 in range(lo, hi, CH):
            c1 = min(hi, c0 + CH)
            dp.gen(c0, c1, out=buf)
            s.attribute(buf[:16 * (c1 - c0)])
    torch.cuda.synchronize()


def owned_step():
    m = [timed(lambda r=r: S[r].merge_peers_owned(ptrs, r)) for r in range(P)]
    f = [timed(lambda r=r: S[r].finalize()) for r in range(P)]
    g = [timed(lambda r=r: S[r].gather_peers(ptrs, r)) for r in range(P)]
    return m, f, g


out = {"P": P, "config": cfg, "records_per_rank": N // P}
attribute_all()
m, f, g = owned_step()
attribute_all()                       # steady state: the reset after a merged step
m, f, g = owned_step()
rs = [timed(lambda r=r: S[r].reset()) for r in range(P)]
out.update({"merge_owned_ms": m, "finalize_owned_ms": f, "gather_ms": g, "reset_after_step_ms": rs,
            "max_per_rank_ms": {"merge": max(m), "finalize": max(f), "gather": max(g), "reset": max(rs)}})
# correctness: rank 0's gathered stats == a single session over the whole trace
attribute_all()
owned_step()
st_owned, ctr_owned = S[0].object_stats()
one = Session(prog.objects, prog.kinds)
for c0 in range(0, N, CH):
    c1 = min(N, c0 + CH)
    dp.gen(c0, c1, out=buf)
    one.attribute(buf[:16 * (c1 - c0)])
st_one, ctr_one = one.object_stats()
out["owned_equals_single"] = bool(np.array_equal(st_owned.view(np.uint8), st_one.view(np.uint8))
                                  and ctr_owned == ctr_one)
print(json.dumps(out))
