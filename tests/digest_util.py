"""Canonical digests of a whole-trace result -- TEST INFRASTRUCTURE.

The full-size BASELINE configs (C3: 10^9 records, C4: 4*10^9, C5: 1.6*10^10)
are too large to compare element by element inside a test run, so the
oracle's results are reduced ONCE, on the dev box, to SHA-256 digests
(``tools/make_golden_digests.py``, which calls only ``oracle/`` and
``tracegen/``) and stored under ``tests/golden/digests/``; the GPU tests and
``bench.py`` reduce the CUDA path's results the same way and compare.

Everything hashed is an exact integer output of the method:
  * counters (records / attributed / unattributed / clipped / invalid);
  * per-object stats (accessed, span, largest unaccessed run, t_first,
    t_last, n_access_apis; the padding word zeroed) and pattern reports;
  * per-object bitmaps, one bit per element, packed little-endian
    into ceil(n_elem / 8) bytes -- bit e of byte e // 8 is element e;
  * per-object accessing-API sets (Defs 3.6 / 3.7): for every object in
    load order, its accessing APIs in timestamp order as (object u32,
    timestamp u32, rw u8) with rw bit 0 = read, bit 1 = write.
Objects are split into N_BLOCKS contiguous blocks (object index ranges) and
every block gets its own digests, so a mismatch names the objects to look at.
This module holds no part of the method: it only serialises results.
"""
import hashlib

import numpy as np

N_BLOCKS = 64


def block_bounds(n_obj, n_blocks=N_BLOCKS):
    return [n_obj * b // n_blocks for b in range(n_blocks + 1)]


def _sha(*arrays):
    h = hashlib.sha256()
    for a in arrays:
        h.update(np.ascontiguousarray(a).view(np.uint8).tobytes() if a.size else b"")
    return h.hexdigest()


def _stats_canon(stats):
    s = np.array(stats, copy=True)
    if "_pad" in s.dtype.names:
        s["_pad"] = 0
    return s


def packed_nbytes(objects):
    n_elem = (objects["size"] // objects["elem_size"]).astype(np.uint64)
    return ((n_elem + np.uint64(7)) // np.uint64(8)).astype(np.int64)


def digest(objects, counters, stats, reports, bitmap_bytes, accesses, n_blocks=N_BLOCKS):
    """objects: OBJ_DTYPE[n]; counters: mapping with the five counter names;
    stats / reports: the per-object arrays (load order);
    bitmap_bytes(o) -> a bytes-like of ceil(n_elem_o / 8) bytes;
    accesses(lo, hi) -> (obj u32[], ts u32[], rw u8[]) of objects [lo, hi)
    in (object, timestamp) order.  Returns a JSON-able dict."""
    n = int(objects.shape[0])
    bounds = block_bounds(n, n_blocks)
    st = _stats_canon(stats)
    nbytes = packed_nbytes(objects)
    out = {"n_obj": n, "n_blocks": n_blocks,
           "counters": {k: int(counters[k]) for k in
                        ("records", "attributed", "unattributed", "clipped", "invalid")},
           "stats_sha": [], "reports_sha": [], "bitmap_sha": [], "access_sha": []}
    n_acc = 0
    for lo, hi in zip(bounds, bounds[1:]):
        out["stats_sha"].append(_sha(st[lo:hi]))
        out["reports_sha"].append(_sha(np.ascontiguousarray(reports[lo:hi])))
        h = hashlib.sha256()
        for o in range(lo, hi):
            b = bitmap_bytes(o)
            assert len(b) == nbytes[o], (o, len(b), nbytes[o])
            h.update(b)
        out["bitmap_sha"].append(h.hexdigest())
        ob, ts, rw = accesses(lo, hi)
        n_acc += int(ob.size)
        out["access_sha"].append(_sha(np.asarray(ob, np.uint32), np.asarray(ts, np.uint32),
                                      np.asarray(rw, np.uint8)))
    flags = np.asarray(reports["flags"])
    out["summary"] = {
        "accessed_elements": int(np.asarray(stats["accessed"], np.uint64).sum()),
        "used_objects": int((np.asarray(stats["n_access_apis"]) > 0).sum()),
        "object_api_accesses": n_acc,
        "flag_counts": {name: int(((flags & bit) != 0).sum()) for bit, name in
                        ((1, "EA"), (2, "LD"), (4, "UA"), (8, "ML"), (16, "TI"), (32, "DW"),
                         (64, "OA"), (128, "OA_ACTIONABLE"))},
    }
    return out


def results_digest(objects, counters, stats, reports):
    """The part of ``digest`` that needs no shadow (counters, stats, reports):
    what every rank holds after an owned merge + gather (bench.py at N > 1)."""
    n = int(objects.shape[0])
    bounds = block_bounds(n)
    st = _stats_canon(stats)
    return {"counters": {k: int(counters[k]) for k in
                         ("records", "attributed", "unattributed", "clipped", "invalid")},
            "stats_sha": [_sha(st[lo:hi]) for lo, hi in zip(bounds, bounds[1:])],
            "reports_sha": [_sha(np.ascontiguousarray(reports[lo:hi]))
                            for lo, hi in zip(bounds, bounds[1:])]}


def compare(got, want, keys=("counters", "stats_sha", "reports_sha", "bitmap_sha", "access_sha")):
    """List of human-readable mismatches (empty = identical)."""
    bad = []
    for k in keys:
        if k not in got or k not in want:
            bad.append(f"{k}: missing")
            continue
        if k == "counters":
            for c, v in want[k].items():
                if got[k].get(c) != v:
                    bad.append(f"counter {c}: got {got[k].get(c)} want {v}")
            continue
        bounds = block_bounds(want.get("n_obj", 0), len(want[k])) if "n_obj" in want else None
        for b, (g, w) in enumerate(zip(got[k], want[k])):
            if g != w:
                where = f" (objects {bounds[b]}..{bounds[b + 1] - 1})" if bounds else ""
                bad.append(f"{k} block {b}{where}")
    return bad


# ---------------------------------------------------------------- GPU side
def shadow_accessors(objects, kinds, layout, bitmap_words, or_words_host):
    """bitmap_bytes / accesses callables over a host copy of the library's
    OR-mergeable shadow (u32 words: bitmaps, then hit rows; the layout of
    drgpum_object_layout)."""
    wb = or_words_host.view(np.uint8)
    nbytes = packed_nbytes(objects)
    bw = layout["bitmap_word"].astype(np.int64)
    k = np.asarray(kinds)
    acc_ts = np.flatnonzero((k != 0) & (k != 1)).astype(np.uint32)
    hit = or_words_host[int(bitmap_words):]
    hw = layout["hit_word"].astype(np.int64)
    nh = layout["n_hit_apis"].astype(np.int64)
    r_lo = layout["r_lo"].astype(np.int64)
    shifts = (2 * np.arange(16, dtype=np.uint32))

    def bitmap_bytes(o):
        return memoryview(wb)[4 * bw[o]: 4 * bw[o] + nbytes[o]]

    def accesses(lo, hi):
        if hi <= lo:
            z = np.zeros(0, np.uint32)
            return z, z, np.zeros(0, np.uint8)
        w0 = hw[lo]
        w1 = hw[hi] if hi < len(hw) else hit.shape[0]
        W = hit[w0:w1]
        pairs = ((W[:, None] >> shifts[None, :]) & np.uint32(3)).astype(np.uint8).ravel()
        pos = np.flatnonzero(pairs)
        starts = (hw[lo:hi] - w0) * 16
        ob = np.searchsorted(starts, pos, side="right") - 1
        kk = pos - starts[ob]
        assert np.all(kk < nh[lo + ob]), "hit bits beyond an object's lifetime"
        o_abs = (lo + ob).astype(np.uint32)
        ts = acc_ts[r_lo[lo + ob] + kk]
        return o_abs, ts.astype(np.uint32), pairs[pos]

    return bitmap_bytes, accesses


def session_digest(session):
    """Digest of a Session's current (finalized) results, whole shadow."""
    stats, ctr = session.object_stats()
    reps = session.patterns()
    orw = session.or_words().cpu().numpy().view(np.uint32)
    bb, acc = shadow_accessors(session.objects, session.kinds, session.layout(),
                               int(session.view.bitmap_words), orw)
    return digest(session.objects, ctr, stats, reps, bb, acc)
