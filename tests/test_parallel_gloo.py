"""World-size-2 (gloo, CPU) test of the multi-GPU exchange step.

Each rank takes its record range (shard_range), builds its partial shadow --
here with the CPU oracle standing in for the GPU attribution, since this box
has no GPU -- and runs parallel.merge_shadow, the same collective
choreography the GPU path uses (all_to_all of word slices, OR of the owned
slice, all_gather; MIN/MAX/SUM all-reduces).  The OR step is injected (the
library's merge_or kernel on GPU).  After the merge every rank must hold the
single-process shadow bit for bit (BJ: "the union of per-GPU bitmaps equals
the single-GPU bitmap").
"""
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_asplos_linzs23_b200.parallel import merge_shadow, shard_range, slice_words


def _shadow(prog, recs):
    """Partial shadow of a record subset: bitmaps (+accessing-API bits) packed
    into one int32 array, first/last as int32 bit patterns, 5 counters."""
    from oracle import Oracle
    o = Oracle(prog.objects, prog.kinds)
    o.attribute(recs)
    st, ctr = o.stats()
    parts = []
    for i in range(prog.n_obj):
        b = o.bitmap_packed(i)
        b = np.concatenate([b, np.zeros((-len(b)) % 4, np.uint8)])
        parts.append(b.view(np.uint32))
        row = np.zeros((prog.n_api * 2 + 31) // 32, np.uint32)
        ts, rw = o.accesses(i)
        for t, f in zip(ts, rw):
            for k, on in ((0, f & 1), (1, f & 2)):
                if on:
                    bit = 2 * int(t) + k
                    row[bit >> 5] |= np.uint32(1 << (bit & 31))
        parts.append(row)
    words = np.concatenate(parts).view(np.int32)
    first = st["t_first"].view(np.int32).copy()
    last = st["t_last"].view(np.int32).copy()
    counters = np.array([int(ctr[k]) for k in ctr.dtype.names], dtype=np.int64)
    return words, first, last, counters


def _worker(rank, world, port, seed, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from tracegen import build_tiny, gen_all_records
        prog = build_tiny(seed)
        recs = gen_all_records(prog)
        lo, hi = shard_range(len(recs), rank, world)
        w, f, l, c = _shadow(prog, recs[lo:hi])
        orw = torch.from_numpy(w.copy())
        first, last = torch.from_numpy(f), torch.from_numpy(l)
        ctr = torch.from_numpy(c)
        S = slice_words(orw.numel(), world)

        def or_reduce(recv, a, b):       # stand-in for the merge_or kernel
            if b > a:
                acc = orw[a:b].clone()
                for s in range(recv.shape[0]):
                    acc |= recv[s, : b - a]
                orw[a:b] = acc

        merge_shadow(orw, first, last, ctr, None, or_reduce)
        q.put((rank, orw.numpy().copy(), first.numpy().copy(), last.numpy().copy(),
               ctr.numpy().copy(), S))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("seed,world", [(11, 2), (12, 2), (13, 3)])
def test_merge_equals_single_process(seed, world):
    from tracegen import build_tiny, gen_all_records
    prog = build_tiny(seed)
    recs = gen_all_records(prog)
    ref = _shadow(prog, recs)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + (os.getpid() + seed * 7 + world) % 2000
    procs = [ctx.Process(target=_worker, args=(r, world, port, seed, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, w, f, l, c, _ in res:
        assert np.array_equal(w, ref[0]), rank
        assert np.array_equal(f, ref[1]) and np.array_equal(l, ref[2]), rank
        assert np.array_equal(c, ref[3]), rank


def test_shard_range_partitions():
    for n in (0, 1, 7, 1000, 10**9 + 7):
        for world in (1, 2, 3, 8):
            rs = [shard_range(n, r, world) for r in range(world)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(rs, rs[1:]))
            assert max(b - a for a, b in rs) - min(b - a for a, b in rs) <= 1


def test_symmetric_merge_call_order():
    """SymmetricMerge's host sequencing (no GPU): every library call of the
    exchange sits between two device barriers of the symmetric-memory
    handle, with this rank's index and every rank's workspace pointer."""
    from paper_conf_asplos_linzs23_b200.parallel import SymmetricMerge
    log = []

    class Handle:
        rank = 1
        buffer_ptrs = [4096, 8192, 12288]

        def barrier(self, channel=0):
            log.append(("barrier", channel))

    class Sess:
        def merge_peers(self, ptrs, rank, stream=None):
            log.append(("merge_peers", tuple(ptrs), rank))

        def merge_peers_owned(self, ptrs, rank, stream=None):
            log.append(("merge_peers_owned", tuple(ptrs), rank))

        def gather_peers(self, ptrs, rank, stream=None):
            log.append(("gather_peers", tuple(ptrs), rank))

    sm = SymmetricMerge.__new__(SymmetricMerge)
    sm.handle = Handle()
    s = Sess()
    ptrs = (4096, 8192, 12288)
    sm.merge(s)
    assert log == [("barrier", 0), ("merge_peers", ptrs, 1), ("barrier", 0)]
    log.clear()
    sm.merge_owned(s)
    sm.gather(s)
    assert log == [("barrier", 0), ("merge_peers_owned", ptrs, 1), ("barrier", 0),
                   ("barrier", 0), ("gather_peers", ptrs, 1), ("barrier", 0)]
