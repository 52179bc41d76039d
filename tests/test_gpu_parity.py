"""Bit-exact parity of the CUDA path (through the C ABI) with the CPU oracle.

Everything the library produces is an integer function of (objects,
timeline, records), so every comparison is exact: the whole OR-mergeable
shadow (every bitmap word and hit-row word, padding included), first/last,
stats, pattern reports and counters.  Inputs are seeded synthetic programs
(tracegen) and the paper's worked examples (tests/golden).
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from oracle import Oracle  # noqa: E402
from tracegen import (build_config, build_tiny, gen_all_records, gen_records, OBJ_DTYPE,  # noqa: E402
                      REC_DTYPE, NEVER)
from tests.golden_util import golden_names, load, to_arrays  # noqa: E402


def _session(objs, kinds, **kw):
    from paper_conf_asplos_linzs23_b200 import Session
    return Session(objs, kinds, **kw)


def _acc_rank(kinds):
    k = np.asarray(kinds)
    is_acc = (k != 0) & (k != 1)
    before = np.concatenate(([0], np.cumsum(is_acc)))   # access APIs strictly before t
    return before, is_acc


def expected_or_words(s, orc, objs, kinds):
    """The shadow the oracle implies, placed with the library's layout."""
    lay = s.layout()
    v = s.view
    exp = np.zeros(v.or_words, dtype=np.uint32)
    eb = exp.view(np.uint8)
    before, _ = _acc_rank(kinds)
    for o in range(len(objs)):
        pk = orc.bitmap_packed(o)
        off = int(lay["bitmap_word"][o]) * 4
        eb[off: off + pk.size] = pk
        r_lo = int(before[objs["t_alloc"][o]])
        assert lay["r_lo"][o] == r_lo
        tf = int(objs["t_free"][o])
        r_hi = int(before[-1]) if tf == NEVER else int(before[tf])
        assert lay["n_hit_apis"][o] == r_hi - r_lo
        ts, rw = orc.accesses(o)
        for t, f in zip(ts, rw):
            slot = 2 * (int(before[t]) - r_lo)
            for bit, on in ((slot, f & 1), (slot + 1, f & 2)):
                if on:
                    w = int(v.bitmap_words) + int(lay["hit_word"][o]) + (bit >> 5)
                    exp[w] |= np.uint32(1 << (bit & 31))
    return exp


def run_gpu(objs, kinds, recs, chunks=1, host=False, th=None, shuffle_seed=None, session_kw=None):
    s = _session(objs, kinds, **(session_kw or {}))
    r = recs
    if shuffle_seed is not None:
        r = recs[np.random.default_rng(shuffle_seed).permutation(len(recs))]
    if host:
        for part in np.array_split(r, chunks):
            s.attribute(part)
    else:
        d = torch.from_numpy(np.ascontiguousarray(r).view(np.uint8)).cuda()
        bounds = np.linspace(0, len(r), chunks + 1).astype(np.int64)
        for a, b in zip(bounds, bounds[1:]):
            s.attribute(d[a * 16: b * 16])
    st, ctr = s.object_stats()
    rep = s.patterns(th)
    orw = s.or_words().cpu().numpy().view(np.uint32).copy()
    f, l = s.first_last()
    return s, st, ctr, rep, orw, f.cpu().numpy().view(np.uint32), l.cpu().numpy().view(np.uint32)


def check_parity(objs, kinds, recs, th=(2, 80, 80), **kw):
    orc = Oracle(objs, kinds)
    orc.attribute(recs)
    ost, octr = orc.stats()
    orep = orc.patterns(th)
    s, st, ctr, rep, orw, first, last = run_gpu(objs, kinds, recs, th=th, **kw)
    assert s.consistency_errors() == 0
    for name in octr.dtype.names:
        assert int(ctr[name]) == int(octr[name]), name
    for name in ost.dtype.names:
        if name == "_pad":
            continue
        bad = np.flatnonzero(st[name] != ost[name])
        assert bad.size == 0, (name, bad[:5], st[name][bad[:5]], ost[name][bad[:5]])
    for name in orep.dtype.names:
        bad = np.flatnonzero(rep[name] != orep[name])
        assert bad.size == 0, (name, bad[:5], rep[name][bad[:5]], orep[name][bad[:5]])
    assert np.array_equal(first, ost["t_first"]) and np.array_equal(last, ost["t_last"])
    exp = expected_or_words(s, orc, objs, kinds)
    bad = np.flatnonzero(orw != exp)
    assert bad.size == 0, ("shadow words differ", bad[:8], orw[bad[:8]], exp[bad[:8]])
    return s


@pytest.mark.parametrize("name", golden_names())
def test_golden_fixtures(name):
    objs, kinds, recs, _ = to_arrays(load(name))
    check_parity(objs, kinds, recs)


@pytest.mark.parametrize("seed", range(40))
def test_tiny_programs(seed):
    p = build_tiny(2000 + seed)
    check_parity(p.objects, p.kinds, gen_all_records(p))


@pytest.mark.parametrize("seed", range(8))
def test_tiny_programs_no_reuse_chunked(seed):
    p = build_tiny(3000 + seed, reuse=False)
    check_parity(p.objects, p.kinds, gen_all_records(p), chunks=3)


@pytest.fixture(scope="module")
def c1():
    p = build_config("C1")
    return p, gen_all_records(p)


def test_c1_full(c1):
    p, r = c1
    s = check_parity(p.objects, p.kinds, r)
    # diagnostics: every 32-record tile is counted on exactly one path (the
    # fast-tile count is derived from the fast-record count in the kernel);
    # chunks are multiples of 32 records except the launch's last one
    paths = s.path_stats()
    assert sum(paths.values()) == (len(r) + 31) // 32, paths
    assert paths["affine_union"] > 0 and paths["tile_fast"] > 0, paths


def test_c1_shuffled_and_chunked(c1):
    p, r = c1
    check_parity(p.objects, p.kinds, r, chunks=7, shuffle_seed=1)


def test_c1_host_ingest(c1):
    p, r = c1
    check_parity(p.objects, p.kinds, r, host=True, chunks=2)


@pytest.mark.parametrize("th", [(0, 100, 100), (1, 50, 20), (5, 90, 99), (100, 1, 1)])
def test_c1_thresholds(c1, th):
    p, r = c1
    check_parity(p.objects, p.kinds, r, th=th)


def test_reset_gives_a_fresh_trace(c1):
    p, r = c1
    s = _session(p.objects, p.kinds)
    d = torch.from_numpy(r.view(np.uint8)).cuda()
    s.attribute(d)
    st1, c1_ = s.object_stats()
    s.attribute(d[: 16 * 1000])       # more records, then start over
    s.reset()
    s.attribute(d)
    st2, c2_ = s.object_stats()
    assert np.array_equal(st1, st2) and c1_ == c2_


def test_pinned_result_arrays(c1):
    """object_stats / patterns into caller-owned page-locked arrays (the e2e
    leg's form) equal the freshly allocated results, and a wrong out raises."""
    from paper_conf_asplos_linzs23_b200 import pinned_array, STATS_DTYPE, REPORT_DTYPE
    p, r = c1
    s = _session(p.objects, p.kinds)
    s.attribute(torch.from_numpy(r.view(np.uint8)).cuda())
    st, ctr = s.object_stats()
    rep = s.patterns()
    hs, hr = pinned_array(p.n_obj, STATS_DTYPE), pinned_array(p.n_obj, REPORT_DTYPE)
    hs.view(np.uint8)[:] = 0xAB       # stale contents must be overwritten
    st2, ctr2 = s.object_stats(out=hs)
    assert st2 is hs and np.array_equal(st.view(np.uint8), hs.view(np.uint8)) and ctr == ctr2
    assert s.patterns(out=hr) is hr and np.array_equal(rep.view(np.uint8), hr.view(np.uint8))
    with pytest.raises(ValueError):
        s.object_stats(out=np.zeros(p.n_obj + 1, STATS_DTYPE))
    with pytest.raises(ValueError):
        s.patterns(out=np.zeros(p.n_obj, STATS_DTYPE))


def test_empty_and_degenerate():
    # no records at all: every object unused
    p = build_tiny(7)
    check_parity(p.objects, p.kinds, np.zeros(0, dtype=REC_DTYPE))
    # every record invalid or unattributed
    recs = np.zeros(3, dtype=REC_DTYPE)
    recs[0] = (1, 0, 1)
    recs[1] = (2**64 - 8, 16, 1)
    recs[2] = (0x10, 4, 1)
    check_parity(p.objects, p.kinds, recs)


def test_no_objects():
    kinds = np.array([4, 4], dtype=np.uint8)
    recs = np.zeros(2, dtype=REC_DTYPE)
    recs[0] = (4096, 4, 0)
    recs[1] = (4096, 4, 1)
    s = _session(np.zeros(0, dtype=OBJ_DTYPE), kinds)
    s.attribute(torch.from_numpy(recs.view(np.uint8)).cuda())
    _, ctr = s.object_stats()
    assert int(ctr["unattributed"]) == 2 and int(ctr["records"]) == 2


def test_max_range_record():
    """A memset of 2^30 one-byte elements: one record expands to 2^25 words
    through the range queue (A3b), split into 4096-word work items."""
    kinds = np.array([0, 3, 4, 1], dtype=np.uint8)
    objs = np.zeros(1, dtype=OBJ_DTYPE)
    objs[0] = (1 << 40, 1 << 30, 1, 0, 3, 0)
    recs = np.zeros(3, dtype=REC_DTYPE)
    recs[0] = ((1 << 40) + 5, (1 << 30) - 7, 1 | (1 << 31))    # ragged both ends
    recs[1] = ((1 << 40), 0xFFFFFFFF, 2)                        # clipped at the end
    recs[2] = ((1 << 40) + 3, 1, 2)
    check_parity(objs, kinds, recs)


def test_uint32_size_boundary():
    """Largest record (size 2^32-1) over 16-byte elements."""
    kinds = np.array([0, 2, 1], dtype=np.uint8)
    objs = np.zeros(1, dtype=OBJ_DTYPE)
    objs[0] = (1 << 44, 1 << 33, 16, 0, 2, 0)
    recs = np.zeros(1, dtype=REC_DTYPE)
    recs[0] = ((1 << 44) + 16 * 3 + 1, 0xFFFFFFFF, 1 | (1 << 31))
    check_parity(objs, kinds, recs)


@pytest.mark.slow
def test_c2_full_size():
    """BASELINE.json configs[1] at full size (1e8 records), in the launch
    configuration bench.py times: every word of the ~115 MiB shadow compared."""
    p = build_config("C2")
    r = gen_records(p, 0, p.n_records)
    check_parity(p.objects, p.kinds, r)


@pytest.mark.parametrize("name", ["C1", "C2"])
def test_redundant_allocation_end_to_end(name):
    """NEXT-1 on the GPU's first/last (drgpum_redundant_alloc) == the literal
    walk (oracle/ra.py) on the oracle's first/last."""
    from oracle.ra import redundant_allocations
    p = build_config(name, **({"n_records": 1 << 22} if name == "C2" else {}))
    r = gen_records(p, 0, p.n_records)
    s = _session(p.objects, p.kinds)
    s.attribute(torch.from_numpy(r.view(np.uint8)).cuda())
    got = s.redundant_allocations(10)
    orc = Oracle(p.objects, p.kinds)
    orc.attribute(r)
    ost, _ = orc.stats()
    want = redundant_allocations(p.objects["size"], ost["t_first"], ost["t_last"],
                                 ost["n_access_apis"] > 0, 10)
    assert got == want and len(want) > 0


# ---------------------------------------------------------------- queue overflow
@pytest.mark.parametrize("cap", [1, 3])
def test_range_queue_overflow(cap):
    """A3b: with a range queue of `cap` entries, every range record that does
    not fit is expanded in place by the warp that found it (attribute.cu
    enqueue_range's fallback).  Results must still equal the oracle's, and
    the overflow counter must show that the fallback ran."""
    kinds = np.array([0, 0, 3, 2, 3, 4, 2, 1], dtype=np.uint8)
    objs = np.zeros(2, dtype=OBJ_DTYPE)
    objs[0] = (1 << 40, 1 << 26, 4, 0, 7, 0)        # 2^24 elements: 128 range chunks
    objs[1] = ((1 << 40) + (1 << 27), 3 << 20, 1, 1, NEVER, 1)
    recs = np.zeros(8, dtype=REC_DTYPE)
    recs[0] = ((1 << 40) + 4, (1 << 26) - 9, 2 | (1 << 31))        # memset, ragged
    recs[1] = ((1 << 40) + (1 << 27) + 1, (3 << 20) - 2, 2 | (1 << 31))
    recs[2] = ((1 << 40) + 1000, 1 << 20, 3)                        # memcpy read
    recs[3] = ((1 << 40) + (1 << 27) + 5, 777777, 3 | (1 << 31))
    recs[4] = ((1 << 40) + 12345 * 4, 99999, 4 | (1 << 31))         # memset
    recs[5] = ((1 << 40) + 8, 4, 5)                                 # kernel, inline
    recs[6] = ((1 << 40) + (1 << 27), 3 << 20, 6)                   # whole object
    recs[7] = ((1 << 40) + (1 << 26) - 64, 0xFFFF, 6 | (1 << 31))   # clipped
    s = check_parity(objs, kinds, recs, session_kw={"queue_capacity": (cap, 0)})
    assert int(s.raw_counters()[5].item()) > 0, "the overflow path did not run"


def test_range_queue_overflow_c1_and_tiny():
    """The same fallback on generated traces (C1's memcpy/memset ranges and
    tiny programs with ranges running past object ends), queue of one entry."""
    p = build_config("C1")
    check_parity(p.objects, p.kinds, gen_all_records(p), session_kw={"queue_capacity": (1, 0)})
    for seed in range(6):
        t = build_tiny(seed)
        check_parity(t.objects, t.kinds, gen_all_records(t), session_kw={"queue_capacity": (1, 0)})


# ---------------------------------------------------------------- CUDA graphs
@pytest.mark.parametrize("name", ["C1", "C2"])
def test_cuda_graph_replay(name):
    """bench.py times the step (reset, attribute, finalize) as a CUDA-graph
    replay.  Capture it once and replay it three times: every replay must give
    the oracle's results (the host-side call parity that selects the
    range-queue counter slot is frozen into the graph, so consecutive replays
    exercise both slots' reset logic)."""
    p = build_config(name, **({"n_records": 1 << 24} if name == "C2" else {}))
    r = gen_records(p, 0, p.n_records)
    orc = Oracle(p.objects, p.kinds)
    orc.attribute(r)
    ost, octr = orc.stats()
    orep = orc.patterns()
    s = _session(p.objects, p.kinds)
    d = torch.from_numpy(r.view(np.uint8)).cuda()
    # C1: one attribute call per step (as bench.py); C2: two (both slots)
    cuts = [0, p.n_records] if name == "C1" else [0, p.n_records // 2, p.n_records]

    def step():
        s.reset()
        for a, b in zip(cuts, cuts[1:]):
            s.attribute(d[16 * a: 16 * b])
        s.finalize()

    step()                      # warm-up outside the capture
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        step()
    exp = None
    for rep in range(3):
        g.replay()
        torch.cuda.synchronize()
        st, ctr = s.object_stats()
        rp = s.patterns()
        for k in octr.dtype.names:
            assert int(ctr[k]) == int(octr[k]), (rep, k)
        for k in ost.dtype.names:
            assert np.array_equal(st[k], ost[k]), (rep, k)
        for k in orep.dtype.names:
            assert np.array_equal(rp[k], orep[k]), (rep, k)
        assert s.consistency_errors() == 0
        orw = s.or_words().cpu().numpy().view(np.uint32).copy()
        if exp is None:
            exp = expected_or_words(s, orc, p.objects, p.kinds)
        assert np.array_equal(orw, exp), rep


def test_sparse_reset_between_traces():
    """drgpum_reset zeroes only the objects whose first-use word is set (the
    bitmap tiles and hit rows of the touched objects).  Trace A touches one
    half of the objects, trace B the other half plus some of A's: after
    reset, the shadow must be exactly B's (objects only A touched come back
    all zero), including after a reset that follows a merge of a second
    session's shadow (merged bits carry merged first-use words)."""
    p = build_config("C1")
    r = gen_all_records(p)
    orc_any = Oracle(p.objects, p.kinds)
    # which object each record belongs to (oracle-independent: by address range)
    base = p.objects["base"].astype(np.uint64)
    end = base + p.objects["size"].astype(np.uint64)
    order = np.argsort(base)
    k = np.searchsorted(base[order], r["addr"], side="right") - 1
    obj = np.where(k >= 0, order[np.maximum(k, 0)], -1)
    inside = (k >= 0) & (r["addr"] < end[np.maximum(obj, 0)])
    even = inside & (obj % 2 == 0)
    recs_a, recs_b = r[even], r[~even | (np.arange(len(r)) % 7 == 0)]
    s = _session(p.objects, p.kinds)
    dev = lambda x: torch.from_numpy(np.ascontiguousarray(x).view(np.uint8)).cuda()
    for first_trace in (recs_a, recs_b, r):
        s.reset()
        s.attribute(dev(first_trace))
        s.finalize()
        s.reset()
        s.attribute(dev(recs_b))
        orc = Oracle(p.objects, p.kinds)
        orc.attribute(recs_b)
        ost, octr = orc.stats()
        st, ctr = s.object_stats()
        for name in ost.dtype.names:
            assert np.array_equal(st[name], ost[name]), name
        assert np.array_equal(s.or_words().cpu().numpy().view(np.uint32),
                              expected_or_words(s, orc, p.objects, p.kinds))
    # after a merge: OR a second session's shadow (trace A) into s, reset, B
    t = _session(p.objects, p.kinds)
    t.attribute(dev(recs_a))
    s.reset()
    s.attribute(dev(recs_b))
    s.merge_peers([s.workspace.data_ptr(), t.workspace.data_ptr()], 0)
    t.merge_peers([s.workspace.data_ptr(), t.workspace.data_ptr()], 1)
    torch.cuda.synchronize()
    s.reset()
    s.attribute(dev(recs_b))
    orc = Oracle(p.objects, p.kinds)
    orc.attribute(recs_b)
    assert np.array_equal(s.or_words().cpu().numpy().view(np.uint32),
                          expected_or_words(s, orc, p.objects, p.kinds))
    del orc_any


# ---------------------------------------------------------------- reduce-and-clear
@pytest.mark.parametrize("cfg", ["C1", "tiny"])
def test_finalize_consume(cfg, c1):
    """drgpum_set_finalize_consume: finalize zeroes the bitmap words it
    reduces; stats / reports equal the oracle's (also at other thresholds:
    only the classification re-runs), the bitmap part of the shadow reads
    back zero while the hit rows stay, attribution is refused until a reset,
    and the next trace (sparse reset skipping the consumed tiles) is exact."""
    from paper_conf_asplos_linzs23_b200 import DrgpumError
    if cfg == "C1":
        p, r = c1
        objs, kinds, recs = p.objects, p.kinds, r
    else:
        p = build_tiny(7)
        objs, kinds, recs = p.objects, p.kinds, gen_all_records(p)
    orc = Oracle(objs, kinds)
    orc.attribute(recs)
    ost, octr = orc.stats()
    ths = [(2, 80, 80), (5, 50, 90)]
    oreps = [orc.patterns(th) for th in ths]
    s = _session(objs, kinds)
    s.set_finalize_consume(True)
    d = torch.from_numpy(np.ascontiguousarray(recs).view(np.uint8)).cuda()
    for rnd in range(3):
        s.reset()
        s.attribute(d)
        s.finalize(ths[0])
        st, ctr = s.object_stats()
        for name in octr.dtype.names:
            assert int(ctr[name]) == int(octr[name]), (rnd, name)
        for name in ost.dtype.names:
            if name != "_pad":
                assert np.array_equal(st[name], ost[name]), (rnd, name)
        for th, orep in zip(ths, oreps):
            rep = s.patterns(th)
            for name in orep.dtype.names:
                assert np.array_equal(rep[name], orep[name]), (rnd, th, name)
        assert s.consistency_errors() == 0
        orw = s.or_words().cpu().numpy().view(np.uint32)
        nb = int(s.view.bitmap_words)
        assert not orw[:nb].any(), "bitmap words survived a consuming finalize"
        exp = expected_or_words(s, orc, objs, kinds)
        assert np.array_equal(orw[nb:], exp[nb:]), "hit rows changed"
        with pytest.raises(DrgpumError):
            s.attribute(d)
    s.set_finalize_consume(False)   # back to a plain trace: bitmaps kept
    s.reset()
    s.attribute(d)
    s.finalize()
    assert np.array_equal(s.or_words().cpu().numpy().view(np.uint32), expected_or_words(s, orc, objs, kinds))
