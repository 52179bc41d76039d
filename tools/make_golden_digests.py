#!/usr/bin/env python
"""Write tests/golden/digests/<CFG>.json: the CPU ORACLE's whole-trace results
for a BASELINE config at its full benchmarked size, reduced to SHA-256
digests (tests/digest_util.py).

Calls only ``oracle/`` (O1, the std::map replay of PAPER.md §5.1-5.2) and
``tracegen/`` (the seeded program + record(i) expansion): no value here comes
from the CUDA path.  Records are generated on the host in chunks by worker
processes (input generation is embarrassingly parallel) and fed to the ONE
single-threaded oracle in record order; chunking cannot change any result
(OR / MIN / MAX are order-free; the oracle replays the timeline per call).

  python tools/make_golden_digests.py C5 [--workers 3] [--records N]
"""
import argparse
import json
import os
import sys
import time
from multiprocessing import get_context, shared_memory

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

CHUNK = 1 << 25          # records per generated chunk (512 MiB)

_prog = None
_shm = {}


def _init(name, n_records):
    global _prog
    from tracegen import build_config
    _prog = build_config(name, **({"n_records": n_records} if n_records else {}))


def _gen(args):
    from tracegen import REC_DTYPE, gen_records
    shm_name, c0, c1 = args
    if shm_name not in _shm:
        _shm[shm_name] = shared_memory.SharedMemory(name=shm_name)
    buf = np.ndarray((CHUNK,), dtype=REC_DTYPE, buffer=_shm[shm_name].buf)
    gen_records(_prog, c0, c1, out=buf)
    return c0, c1


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--workers", type=int, default=3)
    ap.add_argument("--records", type=int, default=None)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    from oracle import Oracle
    from tracegen import REC_DTYPE, build_config
    from tests.digest_util import digest

    prog = build_config(a.config, **({"n_records": a.records} if a.records else {}))
    N = prog.n_records
    chunks = [(c, min(c + CHUNK, N)) for c in range(0, N, CHUNK)]
    nslot = a.workers + 2
    slots = [shared_memory.SharedMemory(create=True, size=CHUNK * 16) for _ in range(nslot)]
    views = [np.ndarray((CHUNK,), dtype=REC_DTYPE, buffer=s.buf) for s in slots]
    t0 = time.time()
    orc = Oracle(prog.objects, prog.kinds)
    t_orc = 0.0
    ctx = get_context("fork")
    with ctx.Pool(a.workers, initializer=_init, initargs=(a.config, a.records)) as pool:
        pend = {}
        for k in range(min(nslot, len(chunks))):
            pend[k] = pool.apply_async(_gen, ((slots[k % nslot].name,) + chunks[k],))
        for k, (c0, c1) in enumerate(chunks):
            pend.pop(k).get()
            w0 = time.time()
            orc.attribute(views[k % nslot][: c1 - c0])
            t_orc += time.time() - w0
            nxt = k + nslot
            if nxt < len(chunks):
                pend[nxt] = pool.apply_async(_gen, ((slots[nxt % nslot].name,) + chunks[nxt],))
            if k % 16 == 0:
                el = time.time() - t0
                print(f"{a.config}: {c1}/{N} records, {el:.0f} s elapsed, oracle {c1 / max(t_orc, 1e-9):.3e} rec/s",
                      flush=True)
    for s in slots:
        s.close()
        s.unlink()
    w0 = time.time()
    stats, ctr = orc.stats()
    reps = orc.patterns()
    t_fin = time.time() - w0

    def bitmap_bytes(o):
        return orc.bitmap_packed(o).tobytes()

    def accesses(lo, hi):
        ob, ts, rw = [], [], []
        for o in range(lo, hi):
            t, f = orc.accesses(o)
            ob.append(np.full(t.shape[0], o, np.uint32))
            ts.append(t)
            rw.append(f)
        cat = lambda xs, dt: np.concatenate(xs).astype(dt) if xs else np.zeros(0, dt)
        return cat(ob, np.uint32), cat(ts, np.uint32), cat(rw, np.uint8)

    d = digest(prog.objects, ctr, stats, reps, bitmap_bytes, accesses)
    d.update({
        "config": a.config, "program": prog.name, "seed": int(prog.seed), "records": N,
        "n_api": prog.n_api, "thresholds": [2, 80, 80],
        "source": "tools/make_golden_digests.py: oracle O1 (oracle/drgpum_oracle.cpp) over "
                  "tracegen records [0, N), host-generated; no CUDA-path value",
        "oracle_seconds": {"attribute": t_orc, "stats_patterns": t_fin, "total": time.time() - t0},
    })
    out = a.out or os.path.join(ROOT, "tests", "golden", "digests", f"{a.config}.json")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    with open(out, "w") as f:
        json.dump(d, f, indent=1)
    print(f"wrote {out}: counters {d['counters']}, {time.time() - t0:.0f} s", flush=True)


if __name__ == "__main__":
    main()
