"""Full-size parity of the benchmarked configs, through bench.py's own step.

tests/golden/digests/<CFG>.json holds the ORACLE's whole-trace results for
BASELINE configs C3 (10^9 records), C4 (4*10^9: one attribute launch of more
than 2^32 records) and C5 (1.6*10^10: streamed in 2^30-record chunks generated
on the device), reduced to per-block SHA-256 digests of every object's bitmap,
accessing-API set, stats and pattern report plus the counters
(tools/make_golden_digests.py: oracle/ + tracegen/ only).  Here the CUDA path
runs exactly what bench.py times -- bench.Workload's step, replayed from its
CUDA graph when the trace is resident -- and its results are reduced the same
way (tests/digest_util.py) and compared.

The digest pipeline itself is pinned on C1 and a C2 prefix, where the oracle
runs inline: same digest from both sides, and a one-bit change in the GPU's
shadow must change a bitmap digest.
"""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from tests.digest_util import compare, digest, session_digest  # noqa: E402


def _oracle_digest(prog, recs):
    from oracle import Oracle
    o = Oracle(prog.objects, prog.kinds)
    o.attribute(recs)
    st, ctr = o.stats()
    rep = o.patterns()

    def acc(lo, hi):
        ob, ts, rw = [], [], []
        for k in range(lo, hi):
            t, f = o.accesses(k)
            ob.append(np.full(t.shape[0], k, np.uint32)); ts.append(t); rw.append(f)
        cat = lambda xs, dt: np.concatenate(xs).astype(dt) if xs else np.zeros(0, dt)
        return cat(ob, np.uint32), cat(ts, np.uint32), cat(rw, np.uint8)

    return digest(prog.objects, ctr, st, rep, lambda k: o.bitmap_packed(k).tobytes(), acc)


@pytest.mark.parametrize("name,n", [("C1", None), ("C2", 1 << 24), ("C5", 1 << 24)])
def test_digest_pipeline(name, n):
    import bench
    from tracegen import gen_records
    w = bench.Workload(name, n)
    w.step()
    torch.cuda.synchronize()
    got = session_digest(w.s)
    want = _oracle_digest(w.prog, gen_records(w.prog, 0, w.N))
    assert compare(got, want) == []
    assert got["summary"] == want["summary"]
    # a single flipped bit in one bitmap must show up in exactly one block
    lay = w.s.layout()
    o = int(np.flatnonzero(w.prog.objects["size"] >= 64)[0])
    orw = w.s.or_words()
    orw[int(lay["bitmap_word"][o])] ^= 1
    bad = compare(session_digest(w.s), want, keys=("bitmap_sha",))
    assert len(bad) == 1
    w.close()


def _golden(name):
    import bench
    from tracegen import build_config
    g, path = bench.golden(name, build_config(name).n_records)
    if g is None:
        pytest.skip(f"{path} missing (tools/make_golden_digests.py {name})")
    return g


@pytest.mark.slow
@pytest.mark.parametrize("name", ["C3", "C4", "C5"])
def test_full_size_against_oracle_digest(name):
    """bench.py's step at the benchmarked size (device generation; C4's
    single >2^32-record launch; C5's 15 streamed chunks), from its CUDA graph
    where bench.py uses one, twice in a row: every bitmap, accessing-API set,
    stats row, report and counter equals the oracle's."""
    import bench
    want = _golden(name)
    w = bench.Workload(name)
    assert (name == "C5") == w.chunked
    if name == "C4":
        assert w.chunks == [(0, 4_000_000_000)]     # one launch, n > 2^32
    w.step()
    graphed = w.capture(1)
    assert graphed == (not w.chunked)
    for _ in range(2):
        w.run()
    torch.cuda.synchronize()
    got = session_digest(w.s)
    assert w.s.consistency_errors() == 0
    bad = compare(got, want)
    assert bad == [], bad[:10]
    assert got["summary"] == want["summary"]
    w.close()


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_owned_step_cuda_graph_single_rank():
    """bench.py at N>1 captures the whole owned step (reset, attribute,
    symmetric-memory barrier, merge_peers_owned, barrier, finalize, barrier,
    gather_peers, barrier) in one CUDA graph.  With one rank on this GPU the
    same capture must replay to the oracle's results."""
    import torch.distributed as dist
    import bench
    from tracegen import gen_records
    if not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ["MASTER_PORT"] = str(_free_port())
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        w = bench.Workload("C1", world=1)
        from paper_conf_asplos_linzs23_b200 import Session
        from paper_conf_asplos_linzs23_b200.parallel import SymmetricMerge
        try:
            w.sm = SymmetricMerge()
            w.s = Session(w.prog.objects, w.prog.kinds, workspace_alloc=w.sm.alloc)
        except Exception as e:   # symmetric memory unavailable in this torch / driver
            pytest.skip(f"torch symmetric memory unavailable: {e}")
        w.owned = True                    # finalize is followed by gather_peers
        w.do_merge = lambda: w.sm.merge_owned(w.s)
        w.step()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            w.step()
        want = _oracle_digest(w.prog, gen_records(w.prog, 0, w.N))
        for _ in range(3):
            g.replay()
            torch.cuda.synchronize()
            st, ctr = w.s.object_stats()
            from tests.digest_util import results_digest
            got = results_digest(w.s.objects, ctr, st, w.s.patterns())
            assert compare(got, want, ("counters", "stats_sha", "reports_sha")) == []
        w.close()
    finally:
        dist.destroy_process_group()
