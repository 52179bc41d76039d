"""The seeded generator produces the BASELINE shapes and
valid programs; record expansion is a pure function of the record index."""
import numpy as np
import pytest

from oracle import validate
from tracegen import build_config, build_tiny, gen_records, gen_all_records, NEVER


@pytest.mark.parametrize("name,n_obj,kinds", [
    ("C1", 64, {0: 64, 1: 56, 4: 90}),
    ("C2", 1000, {0: 1000, 1: 950, 2: 500, 4: 3000}),
    ("C3", None, {3: 200, 4: 4800}),
    ("C4", 100_000, {0: 100_000, 1: 90_608, 4: 20_000}),
    ("C5", 1_000_000, {0: 1_000_000, 1: 950_000}),
])
def test_config_shapes(name, n_obj, kinds):
    p = build_config(name, n_records=1 << 19)   # >= one record per burst
    assert p.n_records == 1 << 19
    if n_obj is not None:
        assert p.n_obj == n_obj
    counts = np.bincount(p.kinds, minlength=5)
    for k, v in kinds.items():
        assert counts[k] == v, (name, k, counts)
    assert validate(p.objects, p.kinds)[0] == 0


def test_c3_has_address_reuse_and_pool_bound():
    p = build_config("C3", n_records=1 << 16)
    b = p.objects["base"]
    assert len(np.unique(b)) < len(b)                                  # reuse
    assert (p.objects["t_free"] == NEVER).sum() == 640                 # params leak (ML)
    assert 15 * 2**30 < int(p.objects["size"].sum()) < 18 * 2**30      # ~16 GiB of tensors
    assert int((b + p.objects["size"]).max() - b.min()) <= 12 * 2**30  # 12 GiB pool


def test_c4_footprint():
    p = build_config("C4", n_records=1 << 19)
    assert 120 * 2**30 < int(p.objects["size"].sum()) < 135 * 2**30
    kv = np.array(p.meta["kv_blocks"])
    assert np.all(p.objects["size"][kv] == 2 << 20) and np.all(p.objects["t_free"][kv] == NEVER)


def test_records_are_a_pure_function_of_the_index():
    p = build_config("C2", n_records=1 << 18)
    whole = gen_records(p, 0, p.n_records)
    i0, i1 = 12345, 200001
    assert np.array_equal(gen_records(p, i0, i1), whole[i0:i1])
    parts = np.concatenate([gen_records(p, a, b) for a, b in ((0, 7), (7, 1 << 17), (1 << 17, 1 << 18))])
    assert np.array_equal(parts, whole)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_generation_is_deterministic(seed):
    a, b = build_tiny(seed), build_tiny(seed)
    assert np.array_equal(a.objects, b.objects) and np.array_equal(a.kinds, b.kinds)
    assert np.array_equal(gen_all_records(a), gen_all_records(b))


def test_object_sample_keeps_record_values():
    """object_sample (the bounded CPU-oracle sample of bench.py) emits, for
    the kept bursts, exactly the records the full program emits for them."""
    from tracegen import object_sample
    for name, kw in (("C1", {}), ("C5", {"n_records": 1 << 21})):
        p = build_config(name, **kw)
        full = gen_records(p, 0, p.n_records)
        sub = object_sample(p, 7, 3)
        got = gen_records(sub, 0, sub.n_records)
        owner = np.repeat(np.arange(len(p.bursts)), p.bursts["count"].astype(np.int64))
        keep = np.zeros(len(p.bursts), bool)
        keep[sub.burst_id.astype(np.int64)] = True
        assert np.array_equal(got, full[keep[owner]])
        assert sub.n_obj == len(range(3, p.n_obj, 7))
        assert np.array_equal(sub.objects, p.objects[3::7])


def test_object_sample_oracle_results_equal_full_run():
    """Dropping objects never changes which object a record belongs to (no two
    objects overlap in address and lifetime, reading R5), so the oracle's
    results for a kept object are the same in the sample and the full run."""
    from oracle import run_oracle
    from tracegen import object_sample
    p = build_config("C1")
    _, st, _, rep = run_oracle(p.objects, p.kinds, gen_records(p, 0, p.n_records))
    sub = object_sample(p, 4, 1)
    _, st2, _, rep2 = run_oracle(sub.objects, sub.kinds, gen_records(sub, 0, sub.n_records))
    assert np.array_equal(st2, st[1::4]) and np.array_equal(rep2, rep[1::4])
