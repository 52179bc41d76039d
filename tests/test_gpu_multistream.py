"""GPU parity of NEXT-4 (drgpum_dependency_graph / drgpum_patterns_topo) with
the literal oracle (oracle/multistream.py) on access sets from O1."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from oracle import Oracle  # noqa: E402
from oracle.multistream import dependency_edges, kahn_levels, patterns_topo  # noqa: E402
from tests.golden_util import load, to_arrays  # noqa: E402
from tracegen import build_config, build_tiny, gen_all_records  # noqa: E402
from tracegen.streams import assign_streams, interleave  # noqa: E402

FLAGS = {"EA": 1, "LD": 2, "TI": 16, "DW": 32}


def _oracle(objs, kinds, recs, streams, th=2):
    o = Oracle(objs, kinds)
    o.attribute(recs)
    acc = []
    for i in range(len(objs)):
        ts, rw = o.accesses(i)
        acc.append({int(t): (bool(f & 1), bool(f & 2)) for t, f in zip(ts, rw)})
    e = dependency_edges(len(kinds), streams, objs, acc)
    T = kahn_levels(len(kinds), e)
    return o, e, T, patterns_topo(kinds, objs, acc, T, th)


def check(objs, kinds, recs, streams, th=(2, 80, 80)):
    from paper_conf_asplos_linzs23_b200 import Session
    s = Session(objs, kinds)
    s.attribute(torch.from_numpy(np.ascontiguousarray(recs).view(np.uint8)).cuda())
    T, src, dst, lab = s.dependency_graph(streams)
    orc, e, oT, orep = _oracle(objs, kinds, recs, streams, th[0])
    got = {(int(a), int(b)): int(c) for a, b, c in zip(src, dst, lab)}
    assert got == e
    assert list(zip(src.tolist(), dst.tolist())) == sorted(e)
    assert T.tolist() == oT
    rep = s.patterns_topo(T, th)
    base = s.patterns(th)
    for o, want in enumerate(orep):
        r = rep[o]
        for name, bit in FLAGS.items():
            assert bool(int(r["flags"]) & bit) == (name in want["flags"]), (o, name)
        for k in ("ea_distance", "ld_distance", "ti_ranges", "ti_max_idle", "ti_total_idle", "dw_pairs"):
            assert int(r[k]) == want[k], (o, k)
        assert int(r["flags"]) & ~0x33 == int(base[o]["flags"]) & ~0x33
        assert int(r["dw_pairs"]) == int(base[o]["dw_pairs"])    # DW is order-invariant
    return s, T, rep


def test_fig4_multistream():
    fx = load("fig4_multistream")
    objs, kinds, recs, names = to_arrays(fx)
    s, T, rep = check(objs, kinds, recs, np.array(fx["streams"], np.uint32))
    assert T.tolist() == fx["T"]
    o1 = rep[names["O1"]]
    assert int(o1["flags"]) & 1 and int(o1["ea_distance"]) == 3


@pytest.mark.parametrize("seed", range(30))
def test_tiny_random_streams(seed):
    p = build_tiny(9300 + seed)
    check(p.objects, p.kinds, gen_all_records(p), assign_streams(len(p.kinds), 1 + seed % 5, seed),
          th=(seed % 4, 80, 80))


@pytest.mark.parametrize("seed", range(6))
def test_interleaved_programs(seed):
    progs = [build_tiny(9400 + 5 * seed + j, n_api_max=80) for j in range(3)]
    recs = [gen_all_records(p) for p in progs]
    objs, kinds, streams, r, _ = interleave(progs, recs, seed)
    check(objs, kinds, r, streams)


@pytest.mark.parametrize("n_streams", [1, 4, 16])
def test_c1(n_streams):
    p = build_config("C1")
    r = gen_all_records(p)
    s, T, rep = check(p.objects, p.kinds, r, assign_streams(len(p.kinds), n_streams, 7))
    if n_streams == 1:
        assert T.tolist() == list(range(len(p.kinds)))
        assert np.array_equal(rep, s.patterns())      # one stream: the single-stream report


def test_patterns_topo_rejects_bad_T():
    from paper_conf_asplos_linzs23_b200 import Session, DrgpumError
    p = build_tiny(1)
    s = Session(p.objects, p.kinds)
    T = np.zeros(len(p.kinds), np.uint32)
    T[0] = len(p.kinds)
    with pytest.raises(DrgpumError):
        s.patterns_topo(T)
