"""NEXT-4 (§5.3): pins of the multi-stream oracle (oracle/multistream.py).

  * the Fig. 4 printed facts (T[ALLOC]=0, T[CPY]=3, EA distance 3) and the
    hand-derived edges / levels of our two-stream reconstruction;
  * one stream: T is the invocation index and every time-dependent pattern
    equals the single-stream oracle's (O1, C++);
  * k independent programs interleaved on k streams: T is the position inside
    the own stream, EA / LD distances are the single-stream ones, and the TI
    idle counts follow the closed form sum_s |{v in s: T_a < pos_s(v) < T_b}|;
  * Kahn levels == the longest path from a source (DP, another algorithm);
  * every edge goes forward in T and in invocation order.
"""
import numpy as np
import pytest

from oracle import Oracle, EA, LD, TI, DW
from oracle.multistream import (dependency_edges, kahn_levels, patterns_topo,
                                INTRA, RAW, WAW, WAR)
from tests.golden_util import load, to_arrays
from tracegen import build_tiny, gen_all_records, NEVER
from tracegen.streams import assign_streams, interleave

LABEL = {"INTRA": INTRA, "RAW": RAW, "WAW": WAW, "WAR": WAR}


def access_sets(objs, kinds, recs):
    o = Oracle(objs, kinds)
    o.attribute(recs)
    out = []
    for i in range(len(objs)):
        ts, rw = o.accesses(i)
        out.append({int(t): (bool(f & 1), bool(f & 2)) for t, f in zip(ts, rw)})
    return o, out


def test_fig4_multistream():
    fx = load("fig4_multistream")
    objs, kinds, recs, names = to_arrays(fx)
    _, acc = access_sets(objs, kinds, recs)
    e = dependency_edges(len(kinds), fx["streams"], objs, acc)
    want = {(a, b): sum(LABEL[x] for x in lab.split("|")) for a, b, lab in fx["edges"]}
    assert e == want
    T = kahn_levels(len(kinds), e)
    assert T == fx["T"]
    rep = patterns_topo(kinds, objs, acc, T)
    o1 = rep[names["O1"]]
    ex = fx["expect_topo"]["O1"]
    assert "EA" in o1["flags"] and o1["ea_distance"] == ex["ea_distance"]
    t_a, t_f = T[int(objs["t_alloc"][names["O1"]])], T[4]
    assert (t_a, t_f) == (0, 3)
    assert sum(1 for v in range(len(kinds)) if t_a < T[v] < t_f) == ex["ea_between"]


def _longest_path(n, edges):
    L = [0] * n
    for (a, b) in sorted(edges, key=lambda x: x[1]):   # edges go forward in index
        L[b] = max(L[b], L[a] + 1)
    return L


@pytest.mark.parametrize("seed", range(30))
def test_kahn_is_longest_path(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 60))
    edges = {}
    for _ in range(int(rng.integers(0, 3 * n))):
        a, b = sorted(rng.integers(0, n, 2).tolist())
        if a != b:
            edges[(a, b)] = 1
    T = kahn_levels(n, edges)
    assert T == _longest_path(n, edges)


def test_kahn_rejects_cycle():
    with pytest.raises(ValueError):
        kahn_levels(3, {(0, 1): 1, (1, 2): 1, (2, 0): 1})


def _sorted(recs):
    return recs[np.argsort(recs["meta"] & 0x7FFFFFFF, kind="stable")]


@pytest.mark.parametrize("seed", range(25))
def test_one_stream_reduces_to_single_stream(seed):
    p = build_tiny(9000 + seed)
    r = gen_all_records(p)
    orc, acc = access_sets(p.objects, p.kinds, r)
    n = len(p.kinds)
    e = dependency_edges(n, np.zeros(n, np.uint32), p.objects, acc)
    T = kahn_levels(n, e)
    assert T == list(range(n))
    rep = patterns_topo(p.kinds, p.objects, acc, T)
    orep = orc.patterns()
    for o, (a, b) in enumerate(zip(rep, orep)):
        for flag, name in ((EA, "EA"), (LD, "LD"), (TI, "TI"), (DW, "DW")):
            assert (name in a["flags"]) == bool(int(b["flags"]) & flag), (o, name)
        for k in ("ea_distance", "ld_distance", "ti_ranges", "ti_max_idle", "ti_total_idle", "dw_pairs"):
            assert a[k] == int(b[k]), (o, k)


@pytest.mark.parametrize("seed", range(12))
def test_independent_streams_closed_form(seed):
    k = 2 + seed % 3
    progs = [build_tiny(9100 + 7 * seed + j, n_api_max=60) for j in range(k)]
    recs = [gen_all_records(p) for p in progs]
    objs, kinds, streams, r, pos = interleave(progs, recs, seed)
    _, acc = access_sets(objs, kinds, r)
    e = dependency_edges(len(kinds), streams, objs, acc)
    for (a, b) in e:
        assert streams[a] == streams[b]          # disjoint memory: no cross-stream edge
    T = kahn_levels(len(kinds), e)
    for j in range(k):
        assert [T[t] for t in pos[j]] == list(range(len(progs[j].kinds)))
    rep = patterns_topo(kinds, objs, acc, T)
    lens = [len(p.kinds) for p in progs]
    o0 = 0
    for j, p in enumerate(progs):
        orc, acc_j = access_sets(p.objects, p.kinds, recs[j])
        orep = orc.patterns()
        for o in range(len(p.objects)):
            a, b = rep[o0 + o], orep[o]
            for flag, name, key in ((EA, "EA", "ea_distance"), (LD, "LD", "ld_distance")):
                assert (name in a["flags"]) == bool(int(b["flags"]) & flag)
                assert a[key] == int(b[key])
            # TI: idle APIs between consecutive accesses, counted over every stream
            ts = sorted(acc_j[o])
            gaps = [sum(max(0, min(tb, L) - ta - 1) for L in lens) for ta, tb in zip(ts, ts[1:])]
            big = [g for g in gaps if g >= 2]
            assert a["ti_ranges"] == len(big) and a["ti_total_idle"] == sum(big)
            assert a["dw_pairs"] == int(b["dw_pairs"])
        o0 += len(p.objects)


@pytest.mark.parametrize("seed", range(20))
def test_edges_forward_and_levels_consistent(seed):
    p = build_tiny(9200 + seed)
    r = gen_all_records(p)
    _, acc = access_sets(p.objects, p.kinds, r)
    n = len(p.kinds)
    streams = assign_streams(n, 1 + seed % 4, seed)
    e = dependency_edges(n, streams, p.objects, acc)
    T = kahn_levels(n, e)
    preds = {}
    for (a, b) in e:
        assert a < b and T[a] < T[b]
        preds.setdefault(b, []).append(a)
    for v in range(n):                           # T(v) = 1 + max over predecessors
        assert T[v] == (1 + max(T[a] for a in preds[v]) if v in preds else 0)
    # every write (and free) of an object is ordered after all its earlier accessors
    for o, obj in enumerate(p.objects):
        ev = [int(obj["t_alloc"])] + sorted(acc[o]) + ([int(obj["t_free"])] if obj["t_free"] != NEVER else [])
        for i, v in enumerate(ev[1:], 1):
            writes = v == ev[-1] and obj["t_free"] != NEVER or acc[o].get(v, (0, 0))[1]
            if writes:
                assert all(T[u] < T[v] for u in ev[:i])


@pytest.mark.parametrize("seed", range(20))
def test_library_kahn_levels_host(seed):
    """drgpum_kahn_levels (product, host code) == the literal oracle."""
    from paper_conf_asplos_linzs23_b200 import kahn_levels as lib_kahn
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(1, 300))
    m = int(rng.integers(0, 4 * n))
    a = rng.integers(0, n, m)
    b = rng.integers(0, n, m)
    keep = a != b
    src, dst = np.minimum(a, b)[keep], np.maximum(a, b)[keep]
    perm = rng.permutation(len(src))          # any order, duplicates included
    T = lib_kahn(n, src[perm], dst[perm])
    assert T.tolist() == kahn_levels(n, {(int(x), int(y)): 1 for x, y in zip(src, dst)})


def test_library_kahn_rejects_cycles_and_bad_vertices():
    from paper_conf_asplos_linzs23_b200 import kahn_levels as lib_kahn, DrgpumError
    with pytest.raises(DrgpumError):
        lib_kahn(3, [0, 1, 2], [1, 2, 0])
    with pytest.raises(DrgpumError):
        lib_kahn(3, [0], [3])
    with pytest.raises(DrgpumError):
        lib_kahn(2, [1], [1])
    assert lib_kahn(0, [], []).size == 0
