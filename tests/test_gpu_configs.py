"""GPU parity on the larger BASELINE shapes (C3-C5) and the merge step.

C3-C5 keep their full object tables and timelines (address reuse, 10^5-10^6
objects, 68 Gbit of C4 bitmaps) with fewer records.  The oracle runs on a
SAMPLED SUBSET of the objects: since no two objects overlap in address and
lifetime (reading R5), dropping objects never changes which object a record
belongs to -- it only turns records of dropped objects into "unattributed" --
so every per-object output of a kept object (bitmap, accessing APIs,
first/last, stats, patterns) must equal the full GPU run's, bit for bit.

The merge test attributes two halves of a trace in two sessions on one GPU
(virtual shards), ORs one shadow into the other with drgpum_merge_or and
MIN/MAX/SUMs first/last/counters -- the exchange step of parallel.py without
NCCL -- and checks the union against the oracle over the whole trace.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from oracle import Oracle  # noqa: E402
from tracegen import build_config, build_tiny, gen_all_records, gen_records, NEVER  # noqa: E402


def _session(objs, kinds):
    from paper_conf_asplos_linzs23_b200 import Session
    return Session(objs, kinds)


def _before(kinds):
    k = np.asarray(kinds)
    return np.concatenate(([0], np.cumsum((k != 0) & (k != 1))))


def check_subset(prog, recs, idx, th=(2, 80, 80)):
    s = _session(prog.objects, prog.kinds)
    d = torch.from_numpy(np.ascontiguousarray(recs).view(np.uint8)).cuda()
    s.attribute(d)
    st, ctr = s.object_stats()
    rep = s.patterns(th)
    assert s.consistency_errors() == 0
    assert int(ctr["records"]) == len(recs)
    assert int(ctr["attributed"] + ctr["unattributed"] + ctr["invalid"]) == len(recs)
    lay = s.layout()
    orw = s.or_words()
    sub = prog.objects[idx]
    orc = Oracle(sub, prog.kinds)
    orc.attribute(recs)
    ost, octr = orc.stats()
    orep = orc.patterns(th)
    assert int(octr["invalid"]) == int(ctr["invalid"])
    before = _before(prog.kinds)
    for j, o in enumerate(idx):
        for name in ost.dtype.names:
            if name != "_pad":
                assert st[o][name] == ost[j][name], (prog.name, o, name)
        for name in orep.dtype.names:
            assert rep[o][name] == orep[j][name], (prog.name, o, name)
        ne = int(sub["size"][j] // sub["elem_size"][j])
        w0 = int(lay["bitmap_word"][o])
        words = orw[w0: w0 + (ne + 31) // 32].cpu().numpy().view(np.uint32)
        got = np.unpackbits(words.view(np.uint8), bitorder="little")
        assert np.array_equal(got[:ne].astype(bool), orc.bitmap(j)), (prog.name, o)
        assert not got[ne:].any()
        # accessing APIs (hit row) of the object
        nh = int(lay["n_hit_apis"][o])
        hw = int(s.view.bitmap_words + lay["hit_word"][o])
        hrow = orw[hw: hw + (2 * nh + 31) // 32].cpu().numpy().view(np.uint32)
        hbits = np.unpackbits(hrow.view(np.uint8), bitorder="little")[: 2 * nh]
        ts, rw = orc.accesses(j)
        exp = np.zeros(2 * nh, dtype=np.uint8)
        r_lo = int(lay["r_lo"][o])
        for t, f in zip(ts, rw):
            k = 2 * (int(before[t]) - r_lo)
            exp[k] |= f & 1
            exp[k + 1] |= (f >> 1) & 1
        assert np.array_equal(hbits, exp), (prog.name, o)


def _sample(prog, n, rng, must=()):
    # prefer small objects so the oracle's bit-by-bit scans stay cheap
    small = np.flatnonzero(prog.objects["size"] <= (64 << 20))
    pick = rng.choice(small, size=min(n, small.size), replace=False)
    return np.unique(np.concatenate([pick, np.asarray(must, dtype=np.int64)])).astype(np.int64)


@pytest.mark.slow
def test_c3_resnet_reuse_subset():
    p = build_config("C3", n_records=1 << 23)
    r = gen_records(p, 0, p.n_records)
    rng = np.random.default_rng(3)
    must = p.meta["saved_activations"][:50] + p.meta["params"][:40]
    idx = _sample(p, 2500, rng, must)
    # the sample must contain address reuse
    b = p.objects["base"][idx]
    assert len(np.unique(b)) < len(b) or len(np.unique(p.objects["base"])) < p.n_obj
    check_subset(p, r, idx)


@pytest.mark.slow
def test_c4_llm_subset():
    p = build_config("C4", n_records=1 << 23)
    r = gen_records(p, 0, p.n_records)
    rng = np.random.default_rng(4)
    kv = np.array(p.meta["kv_blocks"])
    idx = _sample(p, 3000, rng, must=kv[:200])
    check_subset(p, r, idx)


@pytest.mark.slow
def test_c5_million_objects_subset():
    p = build_config("C5", n_records=1 << 23)
    r = gen_records(p, 0, p.n_records)
    rng = np.random.default_rng(5)
    touched = np.unique(p.bursts["obj"])
    idx = np.unique(np.concatenate([rng.choice(touched, 3000, replace=False),
                                    rng.choice(p.n_obj, 2000, replace=False)]))
    check_subset(p, r, idx)


def _merge_into(dst, src):
    """Exchange step between two sessions on one GPU (parallel.py's semantics)."""
    W = int(dst.view.or_words)
    dst.merge_or(src.or_words(), 1, W, 0, W)
    fd, ld = dst.first_last()
    fs, ls = src.first_last()
    f = torch.minimum(fd.to(torch.int64) & 0xFFFFFFFF, fs.to(torch.int64) & 0xFFFFFFFF)
    l = torch.maximum(ld.to(torch.int64) & 0xFFFFFFFF, ls.to(torch.int64) & 0xFFFFFFFF)
    fd.copy_(torch.where(f > 0x7FFFFFFF, f - (1 << 32), f).to(torch.int32))
    ld.copy_(torch.where(l > 0x7FFFFFFF, l - (1 << 32), l).to(torch.int32))
    dst.counters_tensor().add_(src.counters_tensor())


@pytest.mark.parametrize("which", ["C1", "tiny"])
def test_virtual_shards_merge(which):
    p = build_config("C1") if which == "C1" else build_tiny(77)
    r = gen_all_records(p)
    half = len(r) // 2
    a, b = _session(p.objects, p.kinds), _session(p.objects, p.kinds)
    a.attribute(torch.from_numpy(np.ascontiguousarray(r[:half]).view(np.uint8)).cuda())
    b.attribute(torch.from_numpy(np.ascontiguousarray(r[half:]).view(np.uint8)).cuda())
    _merge_into(a, b)
    st, ctr = a.object_stats()
    rep = a.patterns()
    assert a.consistency_errors() == 0
    orc = Oracle(p.objects, p.kinds)
    orc.attribute(r)
    ost, octr = orc.stats()
    orep = orc.patterns()
    for k in octr.dtype.names:
        assert int(ctr[k]) == int(octr[k]), k
    for k in ost.dtype.names:
        if k != "_pad":
            assert np.array_equal(st[k], ost[k]), k
    for k in orep.dtype.names:
        assert np.array_equal(rep[k], orep[k]), k
    for o in range(p.n_obj):
        assert np.array_equal(a.bitmap(o), orc.bitmap(o)), o
