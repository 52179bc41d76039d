"""NEXT-3 structured access (Def 3.10; §5.2 l.270): oracle O1
against the paper's GramSchmidt example and against the per-definition brute
force; GPU parity in tests/test_gpu_structured.py."""
import numpy as np
import pytest

from oracle import Oracle
from oracle.bruteforce import bruteforce_structured
from tracegen import build_tiny, gen_all_records
from tests.golden_util import load, to_arrays


def _o1(objs, kinds, recs):
    o = Oracle(objs, kinds, structured=True)
    o.attribute(recs)
    return o.structured()


def test_gramschmidt_slices():
    fx = load("gramschmidt_structured")
    objs, kinds, recs, names = to_arrays(fx)
    sa, ov = _o1(objs, kinds, recs)
    bsa, _ = bruteforce_structured(objs, list(kinds), recs)
    for name, want in fx["expect_sa"].items():
        assert sa[names[name]] == want and bsa[names[name]] == want, name
    v = fx["overlapping_variant"]
    objs, kinds, recs, names = to_arrays(fx, records=v["records"])
    sa, ov = _o1(objs, kinds, recs)
    assert sa[names["R_gpu"]] == 0 and ov[names["R_gpu"]] == 1


def test_single_api_is_not_structured():
    """One accessing API has nothing to be disjoint from: not reported."""
    fx = load("gramschmidt_structured")
    objs, kinds, recs, names = to_arrays(fx, records=[{"obj": "R_gpu", "elem": 0, "count": 8,
                                                       "ts": 2, "w": True}])
    sa, ov = _o1(objs, kinds, recs)
    assert sa[names["R_gpu"]] == 0 and ov[names["R_gpu"]] == 0


@pytest.mark.parametrize("seed", range(60))
def test_o1_equals_o0(seed):
    p = build_tiny(7000 + seed)
    r = gen_all_records(p)
    sa, ov = _o1(p.objects, p.kinds, r)
    bsa, bov = bruteforce_structured(p.objects, list(p.kinds), r)
    assert sa.tolist() == bsa and ov.tolist() == bov
