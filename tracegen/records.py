"""Expand a program's bursts into 16-byte access records, chunk by chunk.

``record(i)`` is a pure function of the program: record i belongs to burst b
with prefix[b] <= i < prefix[b+1] and is the (i - prefix[b])-th record of that
burst.  Any chunk [i0, i1) can therefore be generated independently (this is
how bench.py and the large parity cases stream traces bigger than RAM).
"""
import numpy as np

from .layout import REC_DTYPE, PAT_AFFINE, PAT_RANDOM, PAT_RANGE, PAT_RAW

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def splitmix64(x):
    """Counter-based 64-bit mixer (Steele et al.'s splitmix64 finaliser)."""
    with np.errstate(over="ignore"):
        z = (x + np.uint64(0x9E3779B97F4A7C15)) & _M64
        z = ((z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)) & _M64
        z = ((z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)) & _M64
        return z ^ (z >> np.uint64(31))


def gen_records(prog, i0, i1, out=None):
    """Records [i0, i1) of ``prog`` as a REC_DTYPE array (or into ``out``)."""
    n = int(i1) - int(i0)
    if out is None:
        out = np.empty(n, dtype=REC_DTYPE)
    assert out.shape[0] >= n
    if n == 0:
        return out[:0]
    bursts, prefix = prog.bursts, prog.prefix
    b_lo = int(np.searchsorted(prefix, i0, side="right")) - 1
    b_hi = int(np.searchsorted(prefix, i1 - 1, side="right")) - 1
    bsel = np.arange(b_lo, b_hi + 1, dtype=np.int64)
    lo = np.maximum(prefix[bsel], np.uint64(i0))
    hi = np.minimum(prefix[bsel + 1], np.uint64(i1))
    cnt = (hi - lo).astype(np.int64)
    b = np.repeat(bsel, cnt)
    i = np.arange(i0, i1, dtype=np.uint64)
    j = i - prefix[b]
    F = {k: bursts[k] for k in ("pattern", "elem", "span", "start", "stride",
                                  "base", "access_size", "ts", "is_write")}
    pat = F["pattern"][b]
    with np.errstate(over="ignore"):
        span = np.maximum(F["span"][b], np.uint64(1))
        start = F["start"][b]
        elem = start + (j * F["stride"][b]) % span
        rnd = pat == PAT_RANDOM
        if rnd.any():
            bid = b[rnd].astype(np.uint64) if prog.burst_id is None else prog.burst_id[b[rnd]]
            h = splitmix64(np.uint64(prog.seed) ^ (bid << np.uint64(32)) ^ j[rnd])
            elem[rnd] = start[rnd] + h % span[rnd]
        base = F["base"][b]
        addr = base + elem * F["elem"][b].astype(np.uint64)
        raw = pat == PAT_RAW
        addr[raw] = base[raw]
    out = out[:n]
    out["addr"] = addr
    out["size"] = F["access_size"][b]
    out["meta"] = F["ts"][b] | (F["is_write"][b].astype(np.uint32) << np.uint32(31))
    return out


def gen_all_records(prog):
    return gen_records(prog, 0, prog.n_records)
