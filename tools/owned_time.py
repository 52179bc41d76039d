"""Per-rank device time of the exchange + finalize on ONE GPU with P virtual
peers (C2 by default): drgpum_merge_peers + full finalize vs
drgpum_merge_peers_owned + owned finalize + drgpum_gather_peers.  Peers are
local HBM here, so the merge times are a lower bound of the NVLink ones; the
finalize times are what each rank does.  usage: python tools/owned_time.py [P] [config]"""
import json
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_asplos_linzs23_b200 import Session  # noqa: E402
from paper_conf_asplos_linzs23_b200.parallel import shard_range  # noqa: E402
from tracegen import build_config, gen_records  # noqa: E402

P = int(sys.argv[1]) if len(sys.argv) > 1 else 8
cfg = sys.argv[2] if len(sys.argv) > 2 else "C2"
prog = build_config(cfg)
N = prog.n_records
S = [Session(prog.objects, prog.kinds) for _ in range(P)]
ptrs = [s.workspace.data_ptr() for s in S]
shards = []
for r in range(P):
    lo, hi = shard_range(N, r, P)
    shards.append(torch.from_numpy(gen_records(prog, lo, hi).view(np.uint8)).cuda())


def ev():
    return torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)


def timed(fn, reps=10):
    a, b = ev()
    torch.cuda.synchronize()
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def attribute_all():
    for s, d in zip(S, shards):
        s.reset()
        s.attribute(d)
    torch.cuda.synchronize()


out = {"P": P, "config": cfg}
attribute_all()
out["attribute_rank0_ms"] = timed(lambda: (S[0].reset(), S[0].attribute(shards[0])))
attribute_all()
out["merge_peers_rank0_ms"] = timed(lambda: S[0].merge_peers(ptrs, 0))
out["finalize_full_ms"] = timed(lambda: S[0].finalize())
attribute_all()
out["merge_owned_rank0_ms"] = timed(lambda: S[0].merge_peers_owned(ptrs, 0))
for r in range(1, P):
    S[r].merge_peers_owned(ptrs, r)
torch.cuda.synchronize()
fin = [timed(lambda: S[r].finalize()) for r in range(P)]
out["finalize_owned_ms_per_rank"] = fin
out["finalize_owned_max_ms"] = max(fin)
out["gather_rank0_ms"] = timed(lambda: S[0].gather_peers(ptrs, 0), reps=1)
for r in range(1, P):
    S[r].gather_peers(ptrs, r)
torch.cuda.synchronize()
st0, _ = S[0].object_stats()
attribute_all()
for r in range(P):
    S[r].merge_peers(ptrs, r)
torch.cuda.synchronize()
st1, _ = S[0].object_stats()
out["owned_stats_equal_full"] = bool(np.array_equal(st0.view(np.uint8), st1.view(np.uint8)))
print(json.dumps(out))
