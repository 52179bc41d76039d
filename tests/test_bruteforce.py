"""O1 (C++ memory-map replay) == O0 (literal per-definition brute force) on
seeded tiny programs with address reuse, all element sizes, leaks, unused
objects, memcpy/memset ranges, clipping and every kind of odd record."""
import numpy as np
import pytest

from oracle import FLAG_NAMES, run_oracle as _run
from oracle.bruteforce import bruteforce
from tracegen import build_tiny, gen_all_records

N_PROGRAMS = 240


def _compare(seed, reuse=True):
    p = build_tiny(seed, reuse=reuse)
    r = gen_all_records(p)
    o, st, ctr, rep = _run(p.objects, p.kinds, r)
    bst, brep, bctr, touched, acc = bruteforce(p.objects, list(p.kinds), r)
    assert dict(zip(ctr.dtype.names, (int(x) for x in ctr))) == bctr
    for i in range(p.n_obj):
        for k, v in bst[i].items():
            assert int(st[i][k]) == v, (seed, i, k)
        got = {n for b, n in FLAG_NAMES.items() if rep[i]["flags"] & b}
        assert got == brep[i]["flags"], (seed, i)
        for k in ("ea_distance", "ld_distance", "ti_ranges", "ti_max_idle",
                  "ti_total_idle", "dw_pairs"):
            assert int(rep[i][k]) == brep[i][k], (seed, i, k)
        assert set(np.flatnonzero(o.bitmap(i)).tolist()) == touched[i]
        ts, rw = o.accesses(i)
        assert {int(t): (bool(f & 1), bool(f & 2)) for t, f in zip(ts, rw)} == acc[i]
    return p, ctr


@pytest.mark.parametrize("block", range(8))
def test_o1_equals_o0(block):
    seen_clipped = 0
    for seed in range(block * N_PROGRAMS // 8, (block + 1) * N_PROGRAMS // 8):
        p, ctr = _compare(1000 + seed)
        seen_clipped += ctr["clipped"] > 0
    assert seen_clipped > 0


@pytest.mark.parametrize("seed", range(10))
def test_o1_equals_o0_no_reuse(seed):
    _compare(5000 + seed, reuse=False)


def test_tiny_programs_exercise_every_case():
    """The seeded tiny programs really contain what the cross-check claims."""
    agg = dict(reuse=0, clipped=0, invalid=0, unattributed=0, leaks=0, E=set())
    for seed in range(1000, 1040):
        p = build_tiny(seed)
        r = gen_all_records(p)
        _, _, ctr, rep = _run(p.objects, p.kinds, r)
        agg["clipped"] += int(ctr["clipped"])
        agg["invalid"] += int(ctr["invalid"])
        agg["unattributed"] += int(ctr["unattributed"])
        agg["leaks"] += int((p.objects["t_free"] == 0xFFFFFFFF).sum())
        agg["E"] |= set(p.objects["elem_size"].tolist())
        b = p.objects["base"]
        agg["reuse"] += len(b) - len(np.unique(b)) + int(
            np.any(np.diff(np.sort(b)) < p.objects["size"][np.argsort(b)][:-1]))
    assert agg["E"] == {1, 2, 4, 8, 16}
    assert all(agg[k] > 0 for k in ("reuse", "clipped", "invalid", "unattributed", "leaks"))
