"""Pins for the CPU oracle (O1) -- against the paper and mathematics, not itself.

Each test names the passage of /root/reference/PAPER.md (l.NNN) that fixes the
expected value.  A plausible slip in the oracle (a dropped term, a wrong sign,
an inclusive "between", LD on a leaked object, Frag inverted, a shifted index)
fails at least one of these.
"""
from fractions import Fraction

import numpy as np
import pytest

from oracle import run_oracle, Oracle, validate, FLAG_NAMES, EA, LD, UA, ML, TI, DW, OA, OA_ACTIONABLE
from oracle.bruteforce import bruteforce, validate as bf_validate
from tracegen import (OBJ_DTYPE, REC_DTYPE, NEVER, build_config, build_tiny,
                      gen_all_records)
from tests.golden_util import golden_names, load, to_arrays

FLAG = {v: k for k, v in FLAG_NAMES.items()}


def _flags(f):
    return {n for b, n in FLAG_NAMES.items() if f & b}


def _apis_between(a, b):
    """Count of API invocations strictly between timestamps a and b, by
    enumeration (the definition of 'between')."""
    return len([t for t in range(a + 1, b)])


def _check(expect, names, objs, st, rep, bf_rep=None):
    for name, ex in expect.items():
        i = names[name]
        fl = _flags(int(rep[i]["flags"]))
        for f in ex.get("has", []):
            assert f in fl, (name, f, fl)
            if bf_rep is not None:
                assert f in bf_rep[i]["flags"], (name, f)
        for f in ex.get("not", []):
            assert f not in fl, (name, f, fl)
            if bf_rep is not None:
                assert f not in bf_rep[i]["flags"], (name, f)
        if "apis_between_alloc_and_first" in ex:
            assert _apis_between(int(objs[i]["t_alloc"]), int(st[i]["t_first"])) == \
                ex["apis_between_alloc_and_first"]
            assert rep[i]["ea_distance"] == st[i]["t_first"] - objs[i]["t_alloc"]
        if "apis_between_last_and_free" in ex:
            assert _apis_between(int(st[i]["t_last"]), int(objs[i]["t_free"])) == \
                ex["apis_between_last_and_free"]
            assert rep[i]["ld_distance"] == objs[i]["t_free"] - st[i]["t_last"]
        for k in ("t_first", "t_last", "n_access_apis", "accessed"):
            if k in ex:
                assert int(st[i][k]) == ex[k], (name, k)
        for k in ("ea_distance", "ti_max_idle", "dw_pairs"):
            if k in ex:
                assert int(rep[i][k]) == ex[k], (name, k, rep[i])
        if "accessed_fraction" in ex:
            num, den = ex["accessed_fraction"]
            assert Fraction(int(st[i]["accessed"]), int(st[i]["n_elems"])) == Fraction(num, den)
        if "frag_3sig" in ex:
            unacc = int(st[i]["n_elems"] - st[i]["accessed"])
            frag = 1 - Fraction(int(st[i]["largest_unaccessed_run"]), unacc)   # Eq. (1)
            assert f"{float(frag):.2e}" == ex["frag_3sig"]


@pytest.mark.parametrize("name", golden_names())
def test_paper_worked_examples(name):
    fx = load(name)
    objs, kinds, recs, names = to_arrays(fx)
    _, st, ctr, rep = run_oracle(objs, kinds, recs)
    assert ctr["attributed"] == len(recs) and ctr["invalid"] == 0
    small = int(objs["size"].max()) <= 1 << 16
    bf_rep = bruteforce(objs, kinds, recs)[1] if small else None
    _check(fx.get("expect", {}), names, objs, st, rep, bf_rep)
    if "fixed_variant" in fx:
        v = fx["fixed_variant"]
        objs, kinds, recs, names = to_arrays(fx, v["kinds"], v["records"])
        _, st, _, rep = run_oracle(objs, kinds, recs)
        _check(v["expect"], names, objs, st, rep, bruteforce(objs, kinds, recs)[1])


def test_fig2_C_is_exactly_leak_and_idle():
    """Fig. 2 caption (l.232): C matches ML and TI; C is accessed right after
    its allocation and fully, so nothing else may fire."""
    objs, kinds, recs, names = to_arrays(load("fig2_mental_model"))
    _, _, _, rep = run_oracle(objs, kinds, recs)
    assert _flags(int(rep[names["C"]]["flags"])) == {"ML", "TI"}


# --------------------------------------------------------------------------
# Closed forms of Def 3.8 / Eq. (1) (l.174, l.189-194)
# --------------------------------------------------------------------------
def _one_object(n, E, recs_elems, ts_list=None, t_free=3):
    kinds = np.array([0, 4, 4, 1], dtype=np.uint8)
    objs = np.zeros(1, dtype=OBJ_DTYPE)
    objs[0] = (1 << 20, n * E, E, 0, t_free, 0)
    recs = np.zeros(len(recs_elems), dtype=REC_DTYPE)
    for k, (e, cnt) in enumerate(recs_elems):
        ts = 1 if ts_list is None else ts_list[k]
        recs[k] = ((1 << 20) + e * E, cnt * E, ts)
    return objs, kinds, recs


@pytest.mark.parametrize("n,p", [(1000, 1), (1000, 799), (1000, 800), (1000, 999), (64, 32), (33, 1)])
def test_prefix_closed_form(n, p):
    """Accessed prefix of p elements out of n: accessed = p, largest unaccessed
    chunk = n - p = all of the unaccessed memory, so Frag = 0 (Eq. (1));
    OA iff p/n < 80% strictly (Def 3.8 'less than X%')."""
    objs, kinds, recs = _one_object(n, 4, [(0, p)])
    _, st, _, rep = run_oracle(objs, kinds, recs)
    s = st[0]
    assert (s["accessed"], s["span_lo"], s["span_hi"], s["largest_unaccessed_run"]) == (p, 0, p - 1, n - p)
    fl = _flags(int(rep[0]["flags"]))
    assert ("OA" in fl) == (Fraction(p, n) < Fraction(80, 100))
    if "OA" in fl:
        assert "OA_ACTIONABLE" in fl   # Frag = 0 < 80%


@pytest.mark.parametrize("n,s", [(1024, 2), (1024, 8), (960, 3), (4096, 64)])
def test_strided_closed_form(n, s):
    """Every s-th element touched (aligned, n a multiple of s): accessed = n/s,
    largest unaccessed run = s-1, Frag = 1 - (s-1)/(n - n/s)."""
    objs, kinds, recs = _one_object(n, 4, [(e, 1) for e in range(0, n, s)])
    _, st, _, rep = run_oracle(objs, kinds, recs)
    assert st[0]["accessed"] == n // s
    assert st[0]["largest_unaccessed_run"] == s - 1
    assert (st[0]["span_lo"], st[0]["span_hi"]) == (0, n - s)
    frag = 1 - Fraction(s - 1, n - n // s)
    fl = _flags(int(rep[0]["flags"]))
    assert "OA" in fl                       # n/s <= 50% < 80%
    assert ("OA_ACTIONABLE" in fl) == (frag < Fraction(80, 100))


def test_partial_element_and_clipping():
    """A 1-byte access touches its whole element (l.210 'which element(s) a
    memory instruction touches'); an access running past the object end is
    clipped to the object (reading R3) and counted."""
    objs, kinds, recs = _one_object(10, 8, [])
    recs = np.zeros(3, dtype=REC_DTYPE)
    base = 1 << 20
    recs[0] = (base + 8 * 3 + 7, 1, 1)        # last byte of element 3
    recs[1] = (base + 8 * 9 + 4, 64, 1)       # element 9, runs past the end
    recs[2] = (base + 80, 4, 1)               # first byte after the object
    _, st, ctr, _ = run_oracle(objs, kinds, recs)
    assert st[0]["accessed"] == 2 and (st[0]["span_lo"], st[0]["span_hi"]) == (3, 9)
    assert (ctr["attributed"], ctr["clipped"], ctr["unattributed"]) == (2, 1, 1)


# --------------------------------------------------------------------------
# Object-level rules at their threshold edges (l.244-249; X=2, l.166)
# --------------------------------------------------------------------------
def _timeline(kinds, accesses, t_alloc, t_free):
    """One object (64 elements) accessed fully at each (ts, write) given."""
    kinds = np.array(kinds, dtype=np.uint8)
    objs = np.zeros(1, dtype=OBJ_DTYPE)
    objs[0] = (4096, 256, 4, t_alloc, t_free, 0)
    recs = np.zeros(len(accesses), dtype=REC_DTYPE)
    for k, (ts, w) in enumerate(accesses):
        recs[k] = (4096, 256, ts | (w << 31))
    return objs, kinds, recs


A, F, C, S, K = 0, 1, 2, 3, 4


def test_no_ea_no_ld_when_adjacent():
    """Nothing between alloc and first use / last use and free -> no EA/LD."""
    objs, kinds, recs = _timeline([A, K, K, F], [(1, 0), (2, 0)], 0, 3)
    _, _, _, rep = run_oracle(objs, kinds, recs)
    assert _flags(int(rep[0]["flags"])) == set()


def test_ea_ld_exactly_one_between():
    objs, kinds, recs = _timeline([A, K, K, K, K, F], [(2, 0), (3, 0)], 0, 5)
    _, _, _, rep = run_oracle(objs, kinds, recs)
    assert _flags(int(rep[0]["flags"])) == {"EA", "LD"}
    assert (rep[0]["ea_distance"], rep[0]["ld_distance"]) == (2, 2)


@pytest.mark.parametrize("gap_apis,expect_ti", [(0, False), (1, False), (2, True), (5, True)])
def test_ti_threshold(gap_apis, expect_ti):
    """TI: 'at least two GPU API invocations between two consecutive GPU APIs
    that access O' (l.248, X=2 l.166)."""
    kinds = [A, K] + [K] * gap_apis + [K, F]
    t2 = 2 + gap_apis
    objs, kinds, recs = _timeline(kinds, [(1, 0), (t2, 0)], 0, t2 + 1)
    _, _, _, rep = run_oracle(objs, kinds, recs)
    assert ("TI" in _flags(int(rep[0]["flags"]))) == expect_ti
    if expect_ti:
        assert rep[0]["ti_max_idle"] == gap_apis and rep[0]["ti_ranges"] == 1


def test_dead_write_kinds():
    """Def 3.7: copy/copy, set/set, copy/set, set/copy writes with no
    intervening access -> DW; a kernel write or an intervening read breaks it."""
    for k1, k2, dw in [(C, C, 1), (S, S, 1), (C, S, 1), (S, C, 1), (K, C, 0), (C, K, 0)]:
        objs, kinds, recs = _timeline([A, k1, k2, F], [(1, 1), (2, 1)], 0, 3)
        _, _, _, rep = run_oracle(objs, kinds, recs)
        assert rep[0]["dw_pairs"] == dw, (k1, k2)
    # read in between: copy W, kernel R, copy W -> no DW
    objs, kinds, recs = _timeline([A, C, K, C, F], [(1, 1), (2, 0), (3, 1)], 0, 4)
    assert run_oracle(objs, kinds, recs)[3][0]["dw_pairs"] == 0
    # copy that only reads O (device-to-host) is not a write of O
    objs, kinds, recs = _timeline([A, C, C, F], [(1, 1), (2, 0)], 0, 3)
    assert run_oracle(objs, kinds, recs)[3][0]["dw_pairs"] == 0


def test_leak_never_late_dealloc():
    """Fig. 2 caption (l.232): a never-freed object is ML, and not LD."""
    objs, kinds, recs = _timeline([A, K, K, K, K], [(1, 0)], 0, NEVER)
    _, _, _, rep = run_oracle(objs, kinds, recs)
    assert _flags(int(rep[0]["flags"])) == {"ML"}


def test_alloc_free_do_not_access():
    """Footnote 2 (l.178): allocation/deallocation APIs do not access the
    object -- a record stamped with an ALLOC/FREE timestamp is invalid."""
    objs, kinds, recs = _timeline([A, K, F], [(0, 0), (2, 0)], 0, 2)
    _, st, ctr, rep = run_oracle(objs, kinds, recs)
    assert ctr["invalid"] == 2 and st[0]["accessed"] == 0 and (int(rep[0]["flags"]) & UA)


def test_address_reuse_attributes_to_live_object():
    """M holds only active objects (l.238-240): a later object reusing a freed
    address range receives the accesses made during its own lifetime."""
    kinds = np.array([A, K, F, A, K, F, K], dtype=np.uint8)
    objs = np.zeros(2, dtype=OBJ_DTYPE)
    objs[0] = (4096, 256, 4, 0, 2, 0)
    objs[1] = (4096 + 128, 256, 4, 3, 5, 1)
    recs = np.zeros(3, dtype=REC_DTYPE)
    recs[0] = (4096 + 128, 4, 1)    # object 0, element 32
    recs[1] = (4096 + 128, 4, 4)    # object 1, element 0
    recs[2] = (4096 + 128, 4, 6)    # after both frees: unattributed
    _, st, ctr, _ = run_oracle(objs, kinds, recs)
    assert (st[0]["span_lo"], st[1]["span_lo"]) == (32, 0)
    assert (ctr["attributed"], ctr["unattributed"]) == (2, 1)


# --------------------------------------------------------------------------
# Textbook reductions and invariants on generated programs
# --------------------------------------------------------------------------
@pytest.fixture(scope="module")
def c1_run():
    p = build_config("C1")
    r = gen_all_records(p)
    o, st, ctr, rep = run_oracle(p.objects, p.kinds, r)
    return p, r, o, st, ctr, rep


def test_reductions_match_numpy(c1_run):
    """popcount / span / longest zero run recomputed with numpy primitives."""
    p, _, o, st, _, _ = c1_run
    for i in range(p.n_obj):
        bits = o.bitmap(i)
        nz = np.flatnonzero(bits)
        assert st[i]["accessed"] == np.count_nonzero(bits)
        if nz.size:
            assert (st[i]["span_lo"], st[i]["span_hi"]) == (nz[0], nz[-1])
        z = np.flatnonzero(~bits)
        if z.size:
            breaks = np.flatnonzero(np.diff(z) != 1)
            runs = np.diff(np.concatenate(([-1], breaks, [z.size - 1])))
            assert st[i]["largest_unaccessed_run"] == runs.max()
        else:
            assert st[i]["largest_unaccessed_run"] == 0


def _invariants(p, st, ctr, rep, o):
    n = st["n_elems"]
    assert np.all(st["accessed"] <= n)
    used = st["accessed"] > 0
    assert np.all(used == (st["t_first"] != NEVER))
    assert np.all(used == (st["n_access_apis"] > 0))
    assert np.all(used == ((rep["flags"] & UA) == 0))
    assert np.all(st["span_lo"][used] <= st["span_hi"][used])
    assert np.all(st["span_hi"][used] < n[used])
    assert np.all(st["accessed"][used] <= st["span_hi"][used] - st["span_lo"][used] + 1)
    assert np.all(st["largest_unaccessed_run"] <= n - st["accessed"])
    ta, tf = p.objects["t_alloc"], p.objects["t_free"]
    assert np.all(ta[used] < st["t_first"][used])
    assert np.all(st["t_first"][used] <= st["t_last"][used])
    assert np.all((st["t_last"][used] < tf[used]))
    assert ctr["attributed"] + ctr["unattributed"] + ctr["invalid"] == ctr["records"]
    assert ctr["clipped"] <= ctr["attributed"]
    for i in np.flatnonzero(used)[:200]:
        ts, _ = o.accesses(int(i))
        assert ts[0] == st[i]["t_first"] and ts[-1] == st[i]["t_last"]
        assert np.all(np.diff(ts.astype(np.int64)) > 0)


def test_invariants_c1(c1_run):
    p, _, o, st, ctr, rep = c1_run
    _invariants(p, st, ctr, rep, o)
    assert ctr["records"] == p.n_records


def test_planted_program_facts_c1(c1_run):
    """The generator's plan is visible: unused objects are UA, leaked objects
    ML, dead-write plants DW, prefix-only objects below 80% accessed -> OA."""
    p, _, _, st, _, rep = c1_run
    f = rep["flags"]
    assert np.all(f[p.meta["unused"]] & UA)
    assert np.all(f[p.meta["leaks"]] & ML)
    assert np.all(f[p.meta["dead_write"]] & DW)
    po = np.array(p.meta["prefix_only"])
    assert np.all(st["accessed"][po] * 100 < 60 * st["n_elems"][po] + 100)


@pytest.mark.parametrize("seed", range(12))
def test_invariants_tiny(seed):
    p = build_tiny(seed)
    r = gen_all_records(p)
    o, st, ctr, rep = run_oracle(p.objects, p.kinds, r)
    _invariants(p, st, ctr, rep, o)


def _run_all(p, chunks):
    o = Oracle(p.objects, p.kinds)
    for c in chunks:
        o.attribute(c)
    st, ctr = o.stats()
    rep = o.patterns()
    bms = [o.bitmap_packed(i) for i in range(p.n_obj)]
    return st, ctr, rep, bms


@pytest.mark.parametrize("seed", [3, 7])
def test_permutation_and_chunking_invariance(seed):
    """OR/min/max/set-union are order-free: shuffling the records or feeding
    them in chunks changes nothing."""
    p = build_tiny(seed, n_rec_max=3000)
    r = gen_all_records(p)
    ref = _run_all(p, [r])
    rng = np.random.default_rng(seed)
    perm = r[rng.permutation(len(r))]
    for chunks in ([perm], np.array_split(perm, 3), np.array_split(r, 5)):
        got = _run_all(p, chunks)
        assert np.array_equal(got[0], ref[0]) and got[1] == ref[1]
        assert np.array_equal(got[2], ref[2])
        assert all(np.array_equal(a, b) for a, b in zip(got[3], ref[3]))


# --------------------------------------------------------------------------
# Validation (SURVEY §8(b) error rules; reading R5)
# --------------------------------------------------------------------------
def _objs(rows):
    a = np.zeros(len(rows), dtype=OBJ_DTYPE)
    for i, r in enumerate(rows):
        a[i] = r
    return a


@pytest.mark.parametrize("rows,kinds,status", [
    ([(4096, 64, 4, 0, 2, 0)], [A, K, F], 0),
    ([(4096, 0, 4, 0, 2, 0)], [A, K, F], 1),               # size 0
    ([(4096, 64, 3, 0, 2, 0)], [A, K, F], 1),              # bad element size
    ([(4096, 66, 4, 0, 2, 0)], [A, K, F], 1),              # size % E
    ([(2**64 - 32, 64, 4, 0, 2, 0)], [A, K, F], 1),        # address overflow
    ([(4096, 64, 4, 1, 2, 0)], [A, K, F], 1),              # t_alloc not an ALLOC
    ([(4096, 64, 4, 0, 1, 0)], [A, K, F], 1),              # t_free not a FREE
    ([(4096, 64, 4, 0, 5, 0)], [A, K, F], 1),              # t_free past timeline
    ([(4096, 64, 4, 0, 2, 0)], [A, K, 7], 1),              # unknown API kind
    ([(4096, 64, 4, 0, NEVER, 0), (4096 + 32, 64, 4, 1, NEVER, 1)], [A, A, K], 2),
    ([(4096, 64, 4, 0, 2, 0), (4096 + 32, 64, 4, 3, NEVER, 1)], [A, K, F, A, K], 0),
    ([(4096, 64, 4, 0, 3, 0), (4096 + 64, 64, 4, 1, NEVER, 1)], [A, A, K, F], 0),
    ([(4096, 64, 4, 0, 3, 0), (4096 + 63, 64, 4, 1, NEVER, 1)], [A, A, K, F], 2),
])
def test_validation(rows, kinds, status):
    objs = _objs(rows)
    k = np.array(kinds, dtype=np.uint8)
    assert validate(objs, k)[0] == status
    assert bf_validate(objs, list(kinds)) == status
