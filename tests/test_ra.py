"""NEXT-1 redundant allocation (§5.1 l.253-260, Fig. 3): the paper's
worked example, the library's O(n log n) host algorithm against the literal
O(n^2) oracle walk, and the invariants of Def 3.3."""
import numpy as np
import pytest

from oracle import run_oracle
from oracle.ra import redundant_allocations
from paper_conf_asplos_linzs23_b200 import redundant_pairs
from tests.golden_util import load, to_arrays


def test_fig3_worked_example():
    fx = load("fig3_redundant_allocation")
    objs, kinds, recs, names = to_arrays(fx)
    _, st, _, _ = run_oracle(objs, kinds, recs)
    used = st["n_access_apis"] > 0
    o1, o3, o4 = names["O1"], names["O3"], names["O4"]
    # "the last GPU API A5 of O1 is placed after the first GPU API A5 of O3"
    assert st["t_last"][o1] == st["t_first"][o3] == 8
    ent = sorted([(int(st["t_first"][o]), 0, o) for o in range(len(objs))] +
                 [(int(st["t_last"][o]), 1, o) for o in range(len(objs))])
    assert ent.index((8, 0, o3)) < ent.index((8, 1, o1))
    for impl in (redundant_allocations, redundant_pairs):
        pairs = impl(objs["size"], st["t_first"], st["t_last"], used, 10)
        assert pairs[0] == (o4, o1)          # O4 reuses O1's memory


def _check_invariants(pairs, sizes, first, last, used, pct):
    donors = [j for _, j in pairs]
    reusers = [i for i, _ in pairs]
    assert len(set(donors)) == len(donors)               # each donor handed out once
    assert len(set(reusers)) == len(reusers)             # Done happens once per object
    for i, j in pairs:
        assert used[i] and used[j] and i != j
        assert (last[j], 1, j) < (first[i], 0, i)        # donor's last before reuser's first
        assert abs(int(sizes[i]) - int(sizes[j])) * 100 <= pct * max(int(sizes[i]), int(sizes[j]))


@pytest.mark.parametrize("seed", range(60))
def test_library_equals_literal_walk(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 160))
    centers = rng.choice([1000, 4096, 65536, 1 << 20], size=n)
    sizes = (centers * rng.uniform(0.85, 1.15, n)).astype(np.uint64) + 1
    first = rng.integers(0, 300, n).astype(np.uint32)
    last = (first + rng.integers(0, 60, n)).astype(np.uint32)
    used = rng.random(n) < 0.9
    pct = int(rng.choice([0, 5, 10, 25, 100]))
    want = redundant_allocations(sizes, first, last, used, pct)
    got = redundant_pairs(sizes, first, last, used.astype(np.uint8), pct)
    assert got == want
    _check_invariants(got, sizes, first, last, used, pct)


def test_degenerate():
    assert redundant_pairs(np.zeros(0, np.uint64), [], [], np.zeros(0, np.uint8)) == []
    # a single object, or objects that overlap in use, never pair
    assert redundant_pairs([64], [3], [9], [1]) == []
    assert redundant_pairs([64, 64], [3, 4], [9, 9], [1, 1]) == []
    # strictly disjoint uses of equal size pair up; unused objects never take part
    assert redundant_pairs([64, 64, 64], [0, 5, 1], [2, 7, 1], [1, 1, 0]) == [(1, 0)]
