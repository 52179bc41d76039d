"""GPU parity of NEXT-2 (DRGPUM_FEATURE_FREQUENCY) with the oracle."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from oracle import Oracle, nuaf_cv_exceeds  # noqa: E402
from tracegen import build_config, build_tiny, gen_all_records  # noqa: E402


def _sorted(recs):
    return recs[np.argsort(recs["meta"] & 0x7FFFFFFF, kind="stable")]


def _check(objs, kinds, recs, chunks=1, pct=20):
    from paper_conf_asplos_linzs23_b200 import Session
    s = Session(objs, kinds, frequency=True)
    d = torch.from_numpy(np.ascontiguousarray(recs).view(np.uint8)).cuda()
    b = np.linspace(0, len(recs), chunks + 1).astype(np.int64)
    for x, y in zip(b, b[1:]):
        s.attribute(d[x * 16: y * 16])
    slots = s.frequency_slots()
    cnt, first = s.frequency(pct)
    o = Oracle(objs, kinds, frequency=True)
    o.attribute(recs)
    rows = list(zip(*(c.tolist() for c in o.frequency())))
    lay = s.layout()
    k = np.asarray(kinds)
    before = np.concatenate(([0], np.cumsum((k != 0) & (k != 1))))
    sbase = np.concatenate(([0], np.cumsum(lay["n_hit_apis"].astype(np.int64))))
    want = np.zeros_like(slots)
    ocnt = np.zeros(len(objs), np.uint32)
    ofirst = np.full(len(objs), 0xFFFFFFFF, np.uint32)
    for (ob, ts, n, s1, s2) in rows:
        want[sbase[ob] + before[ts] - int(lay["r_lo"][ob])] = (n, s1, s2)
        if nuaf_cv_exceeds(n, s1, s2, pct):
            ocnt[ob] += 1
            ofirst[ob] = min(ofirst[ob], ts)
    assert np.array_equal(slots, want)
    assert np.array_equal(cnt, ocnt) and np.array_equal(first, ofirst)
    return cnt


@pytest.mark.parametrize("seed", range(25))
def test_tiny(seed):
    p = build_tiny(8100 + seed)
    _check(p.objects, p.kinds, _sorted(gen_all_records(p)), chunks=1 + seed % 3)


def test_c1():
    p = build_config("C1")
    cnt = _check(p.objects, p.kinds, _sorted(gen_all_records(p)), chunks=2)
    assert cnt.sum() > 0


def test_c2_prefix():
    from tracegen import gen_records
    p = build_config("C2", n_records=1 << 22)
    _check(p.objects, p.kinds, _sorted(gen_records(p, 0, p.n_records)))


def test_unsorted_trace_is_rejected():
    from paper_conf_asplos_linzs23_b200 import Session, DrgpumError
    p = build_config("C1")
    r = _sorted(gen_all_records(p))[::-1].copy()
    s = Session(p.objects, p.kinds, frequency=True)
    s.attribute(torch.from_numpy(r.view(np.uint8)).cuda())
    with pytest.raises(DrgpumError):
        s.frequency()
