"""Seeded stream assignments for multi-stream programs (NEXT-4, §5.3).

Like the rest of tracegen this only draws inputs: which stream each GPU API
was dispatched on, and interleavings of independent single-stream programs.
The dependency graph and the timestamps are computed by the oracle and the
library independently.
"""
import numpy as np

from .layout import NEVER


def assign_streams(n_api, n_streams, seed, run_mean=3.0):
    """u32[n_api] stream ids: runs of consecutive APIs on one stream (geometric
    run lengths), the next run on a uniformly drawn stream."""
    rng = np.random.default_rng(seed)
    out = np.zeros(n_api, np.uint32)
    i = 0
    while i < n_api:
        n = int(rng.geometric(1.0 / max(run_mean, 1.0)))
        out[i: i + n] = int(rng.integers(0, n_streams))
        i += n
    return out


def interleave(programs, records, seed, addr_stride=1 << 44):
    """Merge k single-stream programs into one k-stream program: a seeded
    random interleaving of their timelines (each program keeps its own order),
    program p on stream p with its addresses moved by p * addr_stride so no two
    programs share memory.  Returns (objects, kinds, streams, records, pos)
    where pos[p] maps program p's timestamps to the merged ones."""
    rng = np.random.default_rng(seed)
    lens = [len(p.kinds) for p in programs]
    order = np.concatenate([np.full(n, k, np.int64) for k, n in enumerate(lens)])
    rng.shuffle(order)
    pos = [np.zeros(n, np.uint32) for n in lens]
    nxt = [0] * len(programs)
    for t, k in enumerate(order):
        pos[k][nxt[k]] = t
        nxt[k] += 1
    kinds = np.zeros(len(order), np.uint8)
    streams = order.astype(np.uint32)
    objs, recs = [], []
    for k, (p, r) in enumerate(zip(programs, records)):
        kinds[pos[k]] = p.kinds
        o = p.objects.copy()
        o["base"] += np.uint64(k * addr_stride)
        o["t_alloc"] = pos[k][o["t_alloc"]]
        live = o["t_free"] != NEVER
        o["t_free"][live] = pos[k][o["t_free"][live]]
        objs.append(o)
        r = r.copy()
        ts = r["meta"] & np.uint32(0x7FFFFFFF)
        ok = ts < len(p.kinds)                 # out-of-range timestamps stay invalid
        r["addr"] += np.uint64(k * addr_stride)
        r["meta"][ok] = (r["meta"][ok] & np.uint32(0x80000000)) | pos[k][ts[ok]]
        r["meta"][~ok] = (r["meta"][~ok] & np.uint32(0x80000000)) | np.uint32(0x7FFFFFFF)
        recs.append(r)
    return np.concatenate(objs), kinds, streams, np.concatenate(recs), pos
