"""GPU parity of NEXT-2 (DRGPUM_FEATURE_FREQUENCY) with the oracle."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from oracle import Oracle, nuaf_cv_exceeds  # noqa: E402
from tracegen import build_config, build_tiny, gen_all_records  # noqa: E402


def _sorted(recs):
    return recs[np.argsort(recs["meta"] & 0x7FFFFFFF, kind="stable")]


def _check(objs, kinds, recs, chunks=1, pct=20, frequency_capacity=None):
    from paper_conf_asplos_linzs23_b200 import Session
    s = Session(objs, kinds, frequency=True, frequency_capacity=frequency_capacity)
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
    bad = np.flatnonzero((slots != want).any(axis=1))
    assert bad.size == 0, ("slots differ", bad[:6].tolist(), slots[bad[:6]].tolist(), want[bad[:6]].tolist())
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


def _chain_program(seed, n_apis=400, n_elem=2048):
    """Every API touches the same object (a chain the kernel must keep in
    order): kernels with repeated random elements, memsets of sub-ranges,
    and a second object touched every few APIs."""
    from tracegen import OBJ_DTYPE, REC_DTYPE
    rng = np.random.default_rng(seed)
    kinds = [0, 0] + [int(rng.choice([4, 4, 4, 3, 2])) for _ in range(n_apis)] + [1, 1]
    objs = np.zeros(2, dtype=OBJ_DTYPE)
    objs[0] = (1 << 20, 4 * n_elem, 4, 0, len(kinds) - 2, 0)
    objs[1] = (1 << 24, 8 * 512, 8, 1, len(kinds) - 1, 1)
    recs = []
    for t in range(2, 2 + n_apis):
        if kinds[t] == 4:
            for _ in range(int(rng.integers(1, 1200))):
                e = int(rng.integers(0, n_elem if rng.random() < 0.7 else 16))
                recs.append(((1 << 20) + 4 * e, int(rng.choice([4, 8, 16])), t | (int(rng.random() < 0.5) << 31)))
            if t % 3 == 0:
                recs.append(((1 << 24) + 8 * int(rng.integers(0, 512)), 8, t))
        else:
            lo = int(rng.integers(0, n_elem - 1))
            recs.append(((1 << 20) + 4 * lo, 4 * int(rng.integers(1, n_elem - lo + 1)), t | (1 << 31)))
            if rng.random() < 0.3:                      # a second record: no closed form
                recs.append(((1 << 20) + 4 * lo, 4 * int(rng.integers(1, 200)), t | (1 << 31)))
    r = np.zeros(len(recs), dtype=REC_DTYPE)
    for i, x in enumerate(recs):
        r[i] = x
    return objs, np.array(kinds, np.uint8), r


@pytest.mark.parametrize("seed,chunks", [(0, 1), (1, 1), (2, 4), (3, 9)])
def test_dependency_chain(seed, chunks):
    objs, kinds, r = _chain_program(seed)
    _check(objs, kinds, r, chunks=chunks)


@pytest.mark.parametrize("seed", range(4))
def test_sub_calls_and_carried_apis(seed):
    """A small key capacity splits every call into many sub-calls: the API
    running across each sub-call boundary is carried (sorted keys moved to
    the other buffer) and completed by the next sub-call or by the query."""
    p = build_tiny(seed)
    _check(p.objects, p.kinds, _sorted(gen_all_records(p)), frequency_capacity=2048, chunks=3)
    c = build_config("C1")
    _check(c.objects, c.kinds, _sorted(gen_all_records(c)), frequency_capacity=1 << 16)
    objs, kinds, r = _chain_program(seed)
    _check(objs, kinds, r, chunks=1 + seed, frequency_capacity=4096)


def test_api_larger_than_capacity_is_refused():
    """One API whose events exceed the key capacity: ENOMEM at the query
    (never a silent partial count)."""
    from paper_conf_asplos_linzs23_b200 import Session, DrgpumError
    c = build_config("C1")
    s = Session(c.objects, c.kinds, frequency=True, frequency_capacity=1024)
    s.attribute(torch.from_numpy(_sorted(gen_all_records(c)).view(np.uint8)).cuda())
    with pytest.raises(DrgpumError, match="ENOMEM|capacity"):
        s.frequency()
