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


def test_gramschmidt_polybench_paper_facts():
    """§7.3 l.400 / Fig. 8 on the PolyBench/GPU GramSchmidt structure:
    R_gpu matches structured access AT gramschmidt_kernel3 [R23: over the
    invocations of that kernel], and the coefficient of variation of its
    slices' access frequencies prints as 58% [R22b] -> non-uniform access
    frequency (> 20%, l.198).  Over all accessing APIs (the H2D copy writes
    every element; kernel1/kernel2 touch the diagonal) R_gpu is NOT
    structured, and no single kernel3 instance has a non-uniform per-element
    count -- the two readings the paper's report rules out."""
    from fractions import Fraction
    from oracle import nuaf_cv_exceeds
    from oracle.bruteforce import bruteforce_structured, bruteforce_slice_frequency
    from tests.golden_util import gramschmidt_polybench
    fx = load("gramschmidt_polybench")
    objs, kinds, recs, k3, k3_ts = gramschmidt_polybench(fx)
    o = Oracle(objs, kinds, structured=True, frequency=True)
    o.attribute(recs)
    sa_k3, ov_k3 = o.structured(k3)
    sa_all, ov_all = o.structured()
    assert sa_k3[0] == 1 and ov_k3[0] == 0                      # paper fact
    assert sa_all[0] == 0 and ov_all[0] == 1                    # derived
    (n, s1, s2), = o.slice_frequency(k3)
    N = fx["program"]["N"]
    assert n == N - 1
    cv2 = Fraction(n * s2 - s1 * s1, s1 * s1)
    assert cv2 == Fraction(n - 1, 3 * (n + 1))                  # closed form, F_k = 3(N-1-k)
    assert Fraction(575, 1000) ** 2 <= cv2 < Fraction(585, 1000) ** 2   # prints as 58%
    assert nuaf_cv_exceeds(n, s1, s2, 20)                       # NUAF (X = 20%)
    rows = list(zip(*(c.tolist() for c in o.frequency())))
    k3set = set(k3_ts)
    per_api = [r for r in rows if r[1] in k3set]
    assert len(per_api) == N - 1 and not any(nuaf_cv_exceeds(a, b, c, 20) for (_, _, a, b, c) in per_api)
    # O0 agrees on the grouped results
    bsa, _ = bruteforce_structured(objs, list(kinds), recs, k3)
    assert bsa == [1]
    assert bruteforce_slice_frequency(objs, list(kinds), recs, k3) == [(n, s1, s2)]


@pytest.mark.parametrize("seed", range(30))
def test_grouped_o1_equals_o0(seed):
    """Grouped SA [R23] and slice frequencies [R22b]: O1 == O0 for random
    API groups on tiny programs (address reuse, ranges, clipping)."""
    from oracle.bruteforce import bruteforce_structured, bruteforce_slice_frequency
    p = build_tiny(7700 + seed)
    r = gen_all_records(p)
    g = (np.random.default_rng(seed).random(p.n_api) < 0.5).astype(np.uint8)
    o = Oracle(p.objects, p.kinds, structured=True, frequency=True)
    o.attribute(r)
    for grp in (None, g):
        sa, ov = o.structured(grp)
        bsa, bov = bruteforce_structured(p.objects, list(p.kinds), r, grp)
        assert sa.tolist() == bsa and ov.tolist() == bov
        assert o.slice_frequency(grp) == bruteforce_slice_frequency(p.objects, list(p.kinds), r, grp)
