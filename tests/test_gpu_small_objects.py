"""GPU parity for the attribution kernel's small-object scratch and its
fast-path clipping (csrc/attribute.cu: per-warp shared-memory bitmap copies
for objects of <= 4096 elements, flushed on object change and at kernel end;
records running past an object's end clipped inside the fast tiers, reading
R3).  Long warp-coalesced bursts over small objects -- the C5 shape -- are
what those paths serve: sequential sweeps that wrap around the object (every
wrap clips a 16-B access), strided sweeps that revisit words, random gathers,
objects on both sides of the 4096-element bound, and bursts of different
objects interleaved so that scratches are bound, flushed and rebound.  Every
output is compared with the oracle bit for bit (check_parity).
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from tracegen import API_KERNEL, API_MEMCPY, ProgramBuilder, gen_all_records  # noqa: E402
from tests.test_gpu_parity import check_parity  # noqa: E402


def _program(seed, n_obj, sizes_elems, E, bursts_per_api, n_api, count, free_some=True):
    pb = ProgramBuilder(f"small{seed}", seed)
    rng = pb.rng
    oids = [pb.alloc(int(n) * E, E) for n in sizes_elems[:n_obj]]
    for _ in range(n_api):
        ts = pb.api(API_KERNEL if rng.random() < 0.85 else API_MEMCPY)
        for o in rng.choice(len(oids), size=min(bursts_per_api, len(oids)), replace=False):
            o = oids[int(o)]
            n = pb.n_elem(o)
            acc = int(rng.choice([4, 8, 16]))
            w = bool(rng.random() < 0.3)
            r = rng.random()
            if r < 0.4:     # sequential sweep wrapping around the object
                pb.affine(ts, o, int(rng.integers(0, n)), max(1, acc // E), n, count, acc, w)
            elif r < 0.75:  # strided sweep, revisits words after wrapping
                pb.affine(ts, o, int(rng.integers(0, 64)), int(rng.integers(2, 300)), n, count, acc, w)
            else:           # random gather
                pb.random(ts, o, 0, n, count, acc, w)
    if free_some:
        for o in oids[: len(oids) // 3]:
            pb.free(o)
    return pb.build()


@pytest.mark.parametrize("seed", range(6))
def test_small_objects_wrapping_bursts(seed):
    rng = np.random.default_rng(seed)
    # sizes straddle the 4096-element scratch bound (and tiny objects)
    sizes = np.concatenate([rng.integers(40, 4097, 10), [4096, 4097, 4095, 33, 8192], rng.integers(4097, 20000, 3)])
    p = _program(seed, len(sizes), sizes, 4, 4, 30, 5000)
    check_parity(p.objects, p.kinds, gen_all_records(p))


@pytest.mark.parametrize("E", [1, 2, 8, 16])
def test_small_objects_element_sizes(E):
    rng = np.random.default_rng(100 + E)
    sizes = rng.integers(16, 4200, 12)
    p = _program(100 + E, len(sizes), sizes, E, 3, 20, 3000)
    check_parity(p.objects, p.kinds, gen_all_records(p))


def test_small_objects_chunked_calls():
    """The scratch is flushed at the end of every launch: chunked calls give the same shadow."""
    rng = np.random.default_rng(7)
    sizes = rng.integers(100, 4000, 16)
    p = _program(7, len(sizes), sizes, 4, 4, 24, 4000)
    check_parity(p.objects, p.kinds, gen_all_records(p), chunks=5)


def test_c5_shape_subset():
    """C5's program (1M small objects, long wrapping bursts) at 2^22 records."""
    from tracegen import build_config
    p = build_config("C5", n_records=1 << 22)
    from oracle import Oracle
    recs = gen_all_records(p)
    orc = Oracle(p.objects, p.kinds)
    orc.attribute(recs)
    ost, octr = orc.stats()
    from tests.test_gpu_parity import run_gpu
    s, st, ctr, rep, orw, first, last = run_gpu(p.objects, p.kinds, recs)
    assert s.consistency_errors() == 0
    for name in octr.dtype.names:
        assert int(ctr[name]) == int(octr[name]), name
    assert int(ctr["clipped"]) > 0   # the wrapping 16-B accesses do clip
    for name in ("accessed", "span_lo", "span_hi", "largest_unaccessed_run", "t_first", "t_last", "n_access_apis"):
        assert np.array_equal(st[name], ost[name]), name
