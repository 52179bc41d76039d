"""Record-range sharding and the one exchange step.

Records are independent and every merge operator is associative,
commutative and idempotent (OR for bitmap / hit-row words, MIN for first, MAX
for last, SUM for counters), so rank r attributes records
[r*N/P, (r+1)*N/P) into its own shadow and one exchange makes every rank's
shadow equal to the single-GPU one, bit for bit.

NCCL has no bitwise-OR reduction, so the OR reduce-scatter is an
all_to_all of equal word slices followed by the library's merge_or kernel on
the owned slice; the merged slices are then all-gathered.  first/last/counters
are small: all_reduce MIN / MAX / SUM.

The collective choreography (``merge_shadow``) takes the OR step as a
callable so the same code is exercised with gloo on CPU tensors in the tests;
on the GPU path ``Session`` passes its merge_or kernel.

``SymmetricMerge`` is the NVLink-native alternative: every rank's workspace
lives in torch symmetric memory, and ONE library kernel per rank
(``drgpum_merge_peers``) reads its owned slice from every peer, combines it
and stores the result into every peer -- no NCCL staging buffers, no second
pass.  Barriers before and after it (the symmetric-memory handle's device
barrier) order it against the peers' attribution and finalize.
"""
import torch
import torch.distributed as dist

U32_MASK = 0xFFFFFFFF


def shard_range(n, rank, world):
    """Contiguous record range of one rank (time-local shards)."""
    return n * rank // world, n * (rank + 1) // world


def slice_words(n_words, world):
    """Equal owned-slice length S (the shadow is padded to world*S words)."""
    return (n_words + world - 1) // world if world else n_words


def merge_shadow(orw, first, last, counters, group, or_reduce):
    """Merge per-rank shadows in place.

    orw:      int32 tensor [W], the OR-mergeable words of this rank.
    first/last: int32 tensors [n_obj] (u32 bit patterns).
    counters: int64 tensor [5].
    or_reduce(recv [P, S] int32, lo, hi): OR the P received slices into
        orw[lo:hi] (the owned slice) -- the library's merge_or kernel on GPU.
    """
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    if world == 1:
        return
    W = orw.numel()
    S = slice_words(W, world)
    padded = torch.zeros(world * S, dtype=torch.int32, device=orw.device)
    padded[:W] = orw
    recv = torch.empty_like(padded)
    dist.all_to_all_single(recv, padded, group=group)
    lo, hi = min(rank * S, W), min((rank + 1) * S, W)
    own = torch.zeros(S, dtype=torch.int32, device=orw.device)
    or_reduce(recv.view(world, S), lo, hi)
    if hi > lo:
        own[: hi - lo] = orw[lo:hi]
    gathered = torch.empty(world * S, dtype=torch.int32, device=orw.device)
    dist.all_gather_into_tensor(gathered, own, group=group)
    orw.copy_(gathered[:W])
    # liveness: u32 values -> int64 so MIN/MAX are unsigned-correct
    f = first.to(torch.int64) & U32_MASK
    l = last.to(torch.int64) & U32_MASK
    dist.all_reduce(f, op=dist.ReduceOp.MIN, group=group)
    dist.all_reduce(l, op=dist.ReduceOp.MAX, group=group)
    first.copy_(torch.where(f > 0x7FFFFFFF, f - (1 << 32), f).to(torch.int32))
    last.copy_(torch.where(l > 0x7FFFFFFF, l - (1 << 32), l).to(torch.int32))
    dist.all_reduce(counters, op=dist.ReduceOp.SUM, group=group)


def merge_session(session, group=None):
    """GPU path: merge a Session's shadow across the ranks of ``group``."""
    orw = session.or_words()
    first, last = session.first_last()
    ctr = session.counters_tensor()
    world = dist.get_world_size(group)
    S = slice_words(orw.numel(), world)

    def or_reduce(recv, lo, hi):
        session.merge_or(recv, recv.shape[0], S, lo, hi)

    merge_shadow(orw, first, last, ctr, group, or_reduce)


class SymmetricMerge:
    """Workspace allocator + merge over torch symmetric memory (NVLink P2P).

    usage:  sm = SymmetricMerge(group); s = Session(objs, kinds, workspace_alloc=sm.alloc)
            ... s.attribute(...) ...; sm.merge(s)
    """

    def __init__(self, group=None):
        self.group = group if group is not None else dist.group.WORLD
        self.handle = None

    def alloc(self, nbytes, device):
        import torch.distributed._symmetric_memory as symm_mem
        buf = symm_mem.empty(nbytes, dtype=torch.uint8, device=device)
        self.handle = symm_mem.rendezvous(buf, self.group)
        self.buf = buf
        return buf

    def peer_ptrs(self):
        return [int(p) for p in self.handle.buffer_ptrs]

    def merge(self, session, stream=None):
        h = self.handle
        h.barrier(channel=0)            # every rank's attribution is done
        session.merge_peers(self.peer_ptrs(), h.rank, stream)
        h.barrier(channel=0)            # every slice is merged everywhere

    def multicast_ptr(self):
        """The NVSwitch multicast mapping of the workspaces (0 if none)."""
        return int(getattr(self.handle, "multicast_ptr", 0) or 0)

    def merge_owned(self, session, stream=None, nvls=False):
        """Owned merge: afterwards this rank holds the merged shadow of its
        objects only; follow with session.finalize() and gather().  nvls:
        objects several ranks touched are read through the multicast mapping
        (NVLS in-switch OR) when the box provides one."""
        h = self.handle
        h.barrier(channel=0)            # every rank's attribution is done
        mc = self.multicast_ptr() if nvls else 0
        if mc:
            session.merge_peers_owned_nvls(self.peer_ptrs(), h.rank, mc, stream)
        else:
            session.merge_peers_owned(self.peer_ptrs(), h.rank, stream)
        h.barrier(channel=0)            # every rank's objects are merged

    def gather(self, session, stream=None):
        h = self.handle
        h.barrier(channel=0)            # every rank's finalize is done
        session.gather_peers(self.peer_ptrs(), h.rank, stream)
        h.barrier(channel=0)            # every rank holds all stats / reports
