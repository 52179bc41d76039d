"""drgpum_merge_peers -- the exchange step as one kernel per rank over peer
pointers -- checked on one GPU with VIRTUAL peers: P sessions
of the same program on cuda:0 each attribute one record-range shard, then
every rank's merge kernel runs over the P workspaces (the pointers a
symmetric-memory rendezvous would hand out on an NVLink box).  Afterwards
EVERY session must hold the single-GPU shadow: stats, patterns, counters and
bitmaps equal to the oracle over the whole trace, bit for bit.  The slices of
different ranks are disjoint, so running the P kernels one after the other on
one device is the same computation as running them concurrently on P GPUs.
"""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from oracle import Oracle  # noqa: E402
from tracegen import build_config, build_tiny, gen_all_records  # noqa: E402
from tests.test_gpu_parity import expected_or_words  # noqa: E402


def _check_against_oracle(s, objs, kinds, recs, orc=None):
    if orc is None:
        orc = Oracle(objs, kinds)
        orc.attribute(recs)
    ost, octr = orc.stats()
    orep = orc.patterns()
    st, ctr = s.object_stats()
    rep = s.patterns()
    assert s.consistency_errors() == 0
    for k in octr.dtype.names:
        assert int(ctr[k]) == int(octr[k]), k
    for k in ost.dtype.names:
        if k != "_pad":
            assert np.array_equal(st[k], ost[k]), k
    for k in orep.dtype.names:
        assert np.array_equal(rep[k], orep[k]), k
    orw = s.or_words().cpu().numpy().view(np.uint32)
    assert np.array_equal(orw, expected_or_words(s, orc, objs, kinds))
    return orc


def _virtual_peers(objs, kinds, recs, P):
    from paper_conf_asplos_linzs23_b200 import Session
    from paper_conf_asplos_linzs23_b200.parallel import shard_range
    sessions = [Session(objs, kinds) for _ in range(P)]
    d = torch.from_numpy(np.ascontiguousarray(recs).view(np.uint8)).cuda()
    for r, s in enumerate(sessions):
        lo, hi = shard_range(len(recs), r, P)
        s.attribute(d[16 * lo: 16 * hi])
    torch.cuda.synchronize()
    ptrs = [s.workspace.data_ptr() for s in sessions]
    for r, s in enumerate(sessions):
        s.merge_peers(ptrs, r)
    torch.cuda.synchronize()
    return sessions


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_virtual_peers_c1(P):
    p = build_config("C1")
    recs = gen_all_records(p)
    orc = None
    for s in _virtual_peers(p.objects, p.kinds, recs, P):
        orc = _check_against_oracle(s, p.objects, p.kinds, recs, orc)


@pytest.mark.parametrize("seed", range(6))
def test_virtual_peers_tiny_reuse(seed):
    p = build_tiny(4100 + seed)
    recs = gen_all_records(p)
    P = 2 + seed % 5
    orc = None
    for s in _virtual_peers(p.objects, p.kinds, recs, P):
        orc = _check_against_oracle(s, p.objects, p.kinds, recs, orc)


def test_merge_peers_rejects_bad_arguments():
    from paper_conf_asplos_linzs23_b200 import Session
    from paper_conf_asplos_linzs23_b200._lib import DrgpumError
    p = build_tiny(4200)
    a, b = Session(p.objects, p.kinds), Session(p.objects, p.kinds)
    ptrs = [a.workspace.data_ptr(), b.workspace.data_ptr()]
    with pytest.raises(DrgpumError):
        a.merge_peers(ptrs, 1)          # ptrs[1] is not a's workspace
    with pytest.raises(DrgpumError):
        a.merge_peers(ptrs, 2)          # rank out of range
    with pytest.raises(DrgpumError):
        a.merge_peers([], 0)
    with pytest.raises(DrgpumError):
        a.merge_peers([ptrs[0], ptrs[1] + 16], 0)   # unaligned peer


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_symmetric_memory_single_rank():
    """The torch symmetric-memory plumbing (allocation, rendezvous, device
    barrier, peer pointers) around drgpum_merge_peers, with one rank."""
    import torch.distributed as dist
    from paper_conf_asplos_linzs23_b200 import Session
    from paper_conf_asplos_linzs23_b200.parallel import SymmetricMerge
    if not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ["MASTER_PORT"] = str(_free_port())
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        sm = SymmetricMerge()
        p = build_config("C1")
        recs = gen_all_records(p)
        try:
            s = Session(p.objects, p.kinds, workspace_alloc=sm.alloc)
        except Exception as e:   # symmetric memory unavailable in this torch / driver
            pytest.skip(f"torch symmetric memory unavailable: {e}")
        s.attribute(torch.from_numpy(recs.view(np.uint8)).cuda())
        sm.merge(s)
        torch.cuda.synchronize()
        assert sm.peer_ptrs() == [s.workspace.data_ptr()]
        _check_against_oracle(s, p.objects, p.kinds, recs)
        # the owned path through the same plumbing (bench.py's N>1 default)
        s.reset()
        s.attribute(torch.from_numpy(recs.view(np.uint8)).cuda())
        sm.merge_owned(s)
        s.finalize()
        sm.gather(s)
        torch.cuda.synchronize()
        _check_against_oracle(s, p.objects, p.kinds, recs)
    finally:
        dist.destroy_process_group()


# ---------------------------------------------------------------- owned merge
def _virtual_peers_owned(objs, kinds, recs, P, th=None):
    """drgpum_merge_peers_owned + finalize + drgpum_gather_peers over P virtual
    peers on cuda:0 (each phase for every rank, then a device sync = the
    barrier between phases on P GPUs)."""
    from paper_conf_asplos_linzs23_b200 import Session
    from paper_conf_asplos_linzs23_b200.parallel import shard_range
    sessions = [Session(objs, kinds) for _ in range(P)]
    d = torch.from_numpy(np.ascontiguousarray(recs).view(np.uint8)).cuda()
    for r, s in enumerate(sessions):
        lo, hi = shard_range(len(recs), r, P)
        s.attribute(d[16 * lo: 16 * hi])
    torch.cuda.synchronize()
    ptrs = [s.workspace.data_ptr() for s in sessions]
    for r, s in enumerate(sessions):
        s.merge_peers_owned(ptrs, r)
    torch.cuda.synchronize()
    for s in sessions:
        s.finalize(th)
    torch.cuda.synchronize()
    for r, s in enumerate(sessions):
        s.gather_peers(ptrs, r)
    torch.cuda.synchronize()
    return sessions, ptrs


def _check_owned(sessions, objs, kinds, recs):
    orc = Oracle(objs, kinds)
    orc.attribute(recs)
    ost, octr = orc.stats()
    orep = orc.patterns()
    for s in sessions:
        st, ctr = s.object_stats()
        rep = s.patterns()
        assert s.consistency_errors() == 0
        for k in octr.dtype.names:
            assert int(ctr[k]) == int(octr[k]), k
        for k in ost.dtype.names:
            if k != "_pad":
                assert np.array_equal(st[k], ost[k]), k
        for k in orep.dtype.names:
            assert np.array_equal(rep[k], orep[k]), k
    # every object's bitmap is merged on (at least) its owner
    exp = expected_or_words(sessions[0], orc, objs, kinds)
    lay = sessions[0].layout()
    have = [s.or_words().cpu().numpy().view(np.uint32) for s in sessions]
    for o in range(len(objs)):
        w0 = int(lay["bitmap_word"][o])
        nw = (int(objs["size"][o] // objs["elem_size"][o]) + 31) // 32
        assert any(np.array_equal(h[w0:w0 + nw], exp[w0:w0 + nw]) for h in have), o


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_virtual_peers_owned_c1(P):
    p = build_config("C1")
    recs = gen_all_records(p)
    sessions, _ = _virtual_peers_owned(p.objects, p.kinds, recs, P)
    _check_owned(sessions, p.objects, p.kinds, recs)


@pytest.mark.parametrize("seed", range(6))
def test_virtual_peers_owned_tiny_reuse(seed):
    p = build_tiny(4300 + seed)
    recs = gen_all_records(p)
    P = 2 + seed % 7            # up to 8 ranks: some own no object at all
    sessions, _ = _virtual_peers_owned(p.objects, p.kinds, recs, P)
    _check_owned(sessions, p.objects, p.kinds, recs)


def test_owned_state_rules():
    """object_stats before the gather, patterns with other thresholds, and a
    gather without an owned merge are refused (ESTATE), not answered from a
    partially merged shadow."""
    from paper_conf_asplos_linzs23_b200 import Session
    from paper_conf_asplos_linzs23_b200._lib import DrgpumError
    p = build_tiny(4400)
    recs = gen_all_records(p)
    a, b = Session(p.objects, p.kinds), Session(p.objects, p.kinds)
    ptrs = [a.workspace.data_ptr(), b.workspace.data_ptr()]
    with pytest.raises(DrgpumError):
        a.gather_peers(ptrs, 0)                     # no owned merge yet
    d = torch.from_numpy(np.ascontiguousarray(recs).view(np.uint8)).cuda()
    a.attribute(d[: 16 * (len(recs) // 2)])
    b.attribute(d[16 * (len(recs) // 2):])
    torch.cuda.synchronize()
    a.merge_peers_owned(ptrs, 0)
    b.merge_peers_owned(ptrs, 1)
    torch.cuda.synchronize()
    with pytest.raises(DrgpumError):
        a.object_stats()                            # not finalized + gathered
    a.finalize(); b.finalize()
    torch.cuda.synchronize()
    with pytest.raises(DrgpumError):
        a.gather_peers(ptrs[::-1], 1)               # rank differs from the merge's
    a.gather_peers(ptrs, 0); b.gather_peers(ptrs, 1)
    torch.cuda.synchronize()
    a.object_stats()
    with pytest.raises(DrgpumError):
        a.patterns((3, 80, 80))
    # NEXT-4 reads every object's hit row: refused after an owned merge
    streams = np.zeros(p.n_api, np.uint32)
    with pytest.raises(DrgpumError):
        a.dependency_graph(streams)
    with pytest.raises(DrgpumError):
        a.patterns_topo(np.arange(p.n_api, dtype=np.uint32))
    # re-finalize + re-gather (the flow the header prescribes for new
    # thresholds) replaces each rank's consistency count instead of adding it
    assert a.consistency_errors() == 0 and b.consistency_errors() == 0
    a.first_last()[0].fill_(0)     # corrupt rank 0's first-use words: its objects now disagree
    counts = []
    for _ in range(2):
        a.finalize((3, 80, 80)); b.finalize((3, 80, 80))
        torch.cuda.synchronize()
        a.gather_peers(ptrs, 0); b.gather_peers(ptrs, 1)
        torch.cuda.synchronize()
        counts.append((a.consistency_errors(), b.consistency_errors()))
    a.patterns((3, 80, 80))
    assert counts[0][0] > 0 and counts[0][0] == counts[0][1] and counts[1] == counts[0], counts
    a.reset()                                       # a new trace: ordinary rules again
    a.attribute(d)
    a.patterns((3, 80, 80))
    a.dependency_graph(streams)
