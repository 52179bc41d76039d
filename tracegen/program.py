"""Seeded synthetic programs: objects + GPU-API timeline + access bursts.

A *program* is what DrGPUM's collector would have produced for one run
(§5.1 l.238-240: every GPU API gets a timestamp aligned with its
invocation order; allocation APIs give each object's lifetime, start address
and size; §5.2 l.264: each instrumented access gives a start address and a
size).  The builder below fabricates such runs with the shapes of
BASELINE.json's configs; DESIGN.md §"Input recipe" states each recipe.

Nothing here decides attribution or patterns.  The builder only records the
*plan* (e.g. "object 7 is swept over its first 20% only") in ``Program.meta``
so tests can check that the plan is visible in the oracle's answer.
"""
from dataclasses import dataclass, field
import bisect
import math

import numpy as np

from .layout import (OBJ_DTYPE, BURST_DTYPE, API_ALLOC, API_FREE, API_MEMCPY,
                     API_MEMSET, API_KERNEL, NEVER, PAT_AFFINE, PAT_RANDOM,
                     PAT_RANGE, PAT_RAW)

MAX_REC_SIZE = 0xFFFFFFFF  # record size is u32 (ambiguity #13)
CONFIG_SEED_BASE = 0xD46A0000


@dataclass
class Program:
    name: str
    seed: int
    objects: np.ndarray          # OBJ_DTYPE[n_obj]
    kinds: np.ndarray            # u8[n_api]
    bursts: np.ndarray           # BURST_DTYPE[n_burst]
    prefix: np.ndarray           # u64[n_burst+1], record prefix counts
    meta: dict = field(default_factory=dict)
    # burst ids for record(i)'s hash when the bursts are a subset of another
    # program's (object_sample); None = the bursts' own indices
    burst_id: np.ndarray = None

    @property
    def n_records(self):
        return int(self.prefix[-1])

    @property
    def n_obj(self):
        return int(self.objects.shape[0])

    @property
    def n_api(self):
        return int(self.kinds.shape[0])


# --------------------------------------------------------------------------
# Address allocators (they model cudaMalloc / a caching pool; not the method)
# --------------------------------------------------------------------------
class BumpAllocator:
    """Never reuses addresses: base_k = previous end + random 256-B-aligned gap."""

    def __init__(self, rng, base=0x7F0000000000, align=256, max_gap=4096):
        self.rng, self.cur, self.align, self.max_gap = rng, base, align, max_gap

    def alloc(self, size):
        gap = int(self.rng.integers(0, self.max_gap // self.align + 1)) * self.align
        b = self.cur + gap
        self.cur = (b + size + self.align - 1) // self.align * self.align
        return b

    def free(self, base, size):
        pass


class BestFitPool:
    """Best-fit caching pool over one arena: freed blocks are reused, which
    produces address reuse across object lifetimes (PyTorch-style pools,
    PAPER.md §5.4 l.301)."""

    def __init__(self, base, size, align=512):
        self.align = align
        self.free_blocks = [(base, size)]  # sorted by address
        self.base, self.size = base, size

    def alloc(self, size):
        size = (size + self.align - 1) // self.align * self.align
        best = None
        for k, (b, s) in enumerate(self.free_blocks):
            if s >= size and (best is None or s < self.free_blocks[best][1]):
                best = k
                if s == size:
                    break
        if best is None:
            raise MemoryError("pool exhausted")
        b, s = self.free_blocks[best]
        if s == size:
            del self.free_blocks[best]
        else:
            self.free_blocks[best] = (b + size, s - size)
        return b

    def free(self, base, size):
        size = (size + self.align - 1) // self.align * self.align
        fb = self.free_blocks
        k = bisect.bisect_left(fb, (base, 0))
        fb.insert(k, (base, size))
        if k + 1 < len(fb) and fb[k][0] + fb[k][1] == fb[k + 1][0]:
            fb[k] = (fb[k][0], fb[k][1] + fb[k + 1][1])
            del fb[k + 1]
        if k > 0 and fb[k - 1][0] + fb[k - 1][1] == fb[k][0]:
            fb[k - 1] = (fb[k - 1][0], fb[k - 1][1] + fb[k][1])
            del fb[k]


# --------------------------------------------------------------------------
# Builder
# --------------------------------------------------------------------------
class ProgramBuilder:
    def __init__(self, name, seed, allocator=None):
        self.name, self.seed = name, seed
        self.rng = np.random.default_rng(seed)
        self.alloc_impl = allocator or BumpAllocator(self.rng)
        self.kinds = []
        self.objs = []      # [base, size, E, t_alloc, t_free]
        self.bursts = []    # tuples in BURST_DTYPE field order
        self.meta = {}

    # -- timeline -----------------------------------------------------------
    def api(self, kind):
        self.kinds.append(kind)
        return len(self.kinds) - 1

    def alloc(self, size, elem=4, base=None):
        assert size > 0 and size % elem == 0
        ts = self.api(API_ALLOC)
        if base is None:
            base = self.alloc_impl.alloc(size)
        self.objs.append([base, size, elem, ts, NEVER])
        return len(self.objs) - 1

    def free(self, oid):
        ts = self.api(API_FREE)
        o = self.objs[oid]
        assert o[4] == NEVER
        o[4] = ts
        self.alloc_impl.free(o[0], o[1])
        return ts

    def n_elem(self, oid):
        return self.objs[oid][1] // self.objs[oid][2]

    # -- bursts -------------------------------------------------------------
    def _burst(self, base, start, stride, span, count, ts, elem, access_size,
               obj, pattern, is_write):
        self.bursts.append((base, start, stride, span, count, ts, elem,
                            access_size, obj, pattern, int(bool(is_write)),
                            (0,) * 6))

    def affine(self, ts, oid, start, stride, span, count, access_size, w):
        base, _, E = self.objs[oid][:3]
        self._burst(base, start, stride, span, count, ts, E, access_size, oid,
                    PAT_AFFINE, w)

    def random(self, ts, oid, start, span, count, access_size, w):
        base, _, E = self.objs[oid][:3]
        self._burst(base, start, 0, span, count, ts, E, access_size, oid,
                    PAT_RANDOM, w)

    def range_(self, ts, oid, start_elem, nbytes, w):
        """memcpy/memset touching nbytes from element start_elem: split into
        records of at most 2^32-1 bytes (record size is u32)."""
        base, _, E = self.objs[oid][:3]
        off = 0
        while off < nbytes:
            n = min(nbytes - off, (MAX_REC_SIZE // E) * E)
            self._burst(base, start_elem + off // E, 0, 1, 1, ts, E, n, oid,
                        PAT_RANGE, w)
            off += n

    def raw(self, ts, addr, size, w, tag=0xFFFFFFFF):
        self._burst(addr, 0, 0, 1, 1, ts, 1, size, tag, PAT_RAW, w)

    # -- finish -------------------------------------------------------------
    def build(self, n_records=None):
        objs = np.zeros(len(self.objs), dtype=OBJ_DTYPE)
        if self.objs:
            a = np.array(self.objs, dtype=np.uint64)
            objs["base"], objs["size"], objs["elem_size"] = a[:, 0], a[:, 1], a[:, 2]
            objs["t_alloc"], objs["t_free"] = a[:, 3], a[:, 4]
        objs["user_id"] = np.arange(len(self.objs), dtype=np.uint32)
        bursts = np.array(self.bursts, dtype=BURST_DTYPE) if self.bursts else \
            np.zeros(0, dtype=BURST_DTYPE)
        if n_records is not None:
            _rescale_counts(bursts, n_records)
        prefix = np.zeros(len(bursts) + 1, dtype=np.uint64)
        np.cumsum(bursts["count"], out=prefix[1:])
        return Program(self.name, self.seed, objs,
                       np.array(self.kinds, dtype=np.uint8), bursts, prefix,
                       self.meta)


def _rescale_counts(bursts, n_records):
    """Scale AFFINE/RANDOM burst counts (used as weights) so that the total
    record count is exactly n_records (largest-remainder rounding)."""
    var = (bursts["pattern"] == PAT_AFFINE) | (bursts["pattern"] == PAT_RANDOM)
    fixed = int(bursts["count"][~var].sum())
    budget = n_records - fixed
    assert budget >= var.sum(), "record budget too small for the program"
    w = bursts["count"][var].astype(np.float64)
    ideal = w / w.sum() * (budget - var.sum())
    base = np.floor(ideal).astype(np.uint64) + np.uint64(1)
    rem = budget - int(base.sum())
    order = np.argsort(-(ideal - np.floor(ideal)), kind="stable")
    base[order[:rem]] += np.uint64(1)
    bursts["count"][var] = base


# --------------------------------------------------------------------------
# Sizes
# --------------------------------------------------------------------------
def _lognormal_sizes(rng, n, total, sigma, min_size, align):
    s = rng.lognormal(0.0, sigma, n)
    s = s / s.sum() * total
    s = np.maximum(s, min_size)
    s = (np.round(s / align) * align).astype(np.int64)
    return np.maximum(s, align)


def _loguniform_sizes(rng, n, lo, hi, total, align):
    s = np.exp(rng.uniform(math.log(lo), math.log(hi), n))
    s = s / s.sum() * total
    s = np.clip(s, lo, hi)
    return np.maximum((np.round(s / align) * align).astype(np.int64), align)


# --------------------------------------------------------------------------
# HPC-style phase (Rodinia / PolyBench shaped; C1, C2, C5)
# --------------------------------------------------------------------------
def _hpc_phase(pb, sizes, elems, *, n_kernels, n_cpy, n_set, n_leak,
               n_prefix, n_unused, n_dw, n_eald, objs_per_kernel, pat_mix,
               access_sizes, lazy, stride_range=(2, 1024), window=8):
    """One application run: allocate, copy in, launch kernels, copy out, free.

    lazy=False: allocate all objects up front and free them all at the end
    (the batch style PAPER.md §3.1 l.152 calls prevalent).  lazy=True: each
    object is allocated just before its first use and freed right after its
    last use, except n_eald planted early/late ones.
    """
    rng = pb.rng
    n = len(sizes)
    perm = rng.permutation(n)
    unused = set(perm[:n_unused].tolist())
    prefix_only = set(perm[n_unused:n_unused + n_prefix].tolist())
    used = [i for i in range(n) if i not in unused]
    # plan access APIs: SETs and half the CPYs (H2D) first, kernels, CPYs (D2H)
    n_h2d = (n_cpy + 1) // 2
    plan = [("set", None)] * n_set + [("h2d", None)] * n_h2d + \
           [("k", None)] * n_kernels + [("d2h", None)] * (n_cpy - n_h2d)
    # which objects each access API touches: kernels use a sliding window over
    # the used objects so that objects have bounded active ranges
    touches = []
    order = list(used)
    rng.shuffle(order)
    nu = max(1, len(order))
    k_idx = 0
    for kind, _ in plan:
        if kind == "k":
            c = int(np.clip(round(k_idx / max(1, n_kernels) * nu), 0, nu - 1))
            lo, hi = max(0, c - window), min(nu, c + window + 1)
            kk = int(rng.integers(objs_per_kernel[0], objs_per_kernel[1] + 1))
            kk = min(kk, hi - lo)
            sel = rng.choice(np.arange(lo, hi), size=kk, replace=False)
            touches.append([order[s] for s in sel])
            k_idx += 1
        else:
            touches.append([order[int(rng.integers(0, nu))]])
    # make sure every used object is touched at least once by a kernel
    kpos = [p for p, (kind, _) in enumerate(plan) if kind == "k"]
    seen = set(o for t in touches for o in t)
    for o in used:
        if o not in seen:
            touches[kpos[int(rng.integers(0, len(kpos)))]].append(o)
    first = {}
    last = {}
    for p, t in enumerate(touches):
        for o in t:
            first.setdefault(o, p)
            last[o] = p
    # allocation/free positions (relative to access API positions)
    leaks = set(rng.permutation(used)[:n_leak].tolist()) if used else set()
    eald = set(rng.permutation(used)[:n_eald].tolist()) if used else set()
    wr_first = [touches[p][0] for p, (kind, _) in enumerate(plan) if kind in ("set", "h2d")]
    cand = sorted(set(o for o in wr_first if o not in prefix_only))
    dw = [int(x) for x in rng.permutation(cand)[:n_dw]] if cand else []
    alloc_at, free_at = {}, {}
    P = len(plan)
    for o in range(n):
        if o in unused:
            p = int(rng.integers(0, P))
            alloc_at[o], free_at[o] = p, p
            continue
        if lazy:
            a, f = first[o], last[o]
            if o in eald:
                a = max(0, a - int(rng.integers(2, 6)))
                f = min(P - 1, f + int(rng.integers(2, 6)))
        else:
            a, f = 0, P - 1
        alloc_at[o], free_at[o] = a, f
    dw_plan = list(dw)
    by_alloc, by_free = {}, {}
    for o in range(n):
        by_alloc.setdefault(alloc_at[o], []).append(o)
        by_free.setdefault(free_at[o], []).append(o)
    oid = {}
    written = set()
    for p, (kind, _) in enumerate(plan):
        for o in by_alloc.get(p, []):
            oid[o] = pb.alloc(int(sizes[o]), int(elems[o]))
        if kind == "k":
            ts = pb.api(API_KERNEL)
            t = touches[p]
            wo = t[int(rng.integers(0, len(t)))]
            for o in t:
                _kernel_burst(pb, ts, oid[o], o in prefix_only, o == wo,
                              pat_mix, access_sizes, stride_range)
                if o == wo:
                    written.add(o)
        else:
            o = touches[p][0]
            api_kind = API_MEMSET if kind == "set" else API_MEMCPY
            if o in dw and kind in ("set", "h2d"):
                # dead write (Def 3.7): an extra full-object write right before
                ts0 = pb.api(API_MEMSET)
                pb.range_(ts0, oid[o], 0, int(sizes[o]), True)
                dw.remove(o)
            ts = pb.api(api_kind)
            nb = int(sizes[o])
            if o in prefix_only:
                nb = max(int(elems[o]), int(pb.meta_prefix[oid[o]]) * int(elems[o]))
            pb.range_(ts, oid[o], 0, nb, kind != "d2h")
        for o in by_free.get(p, []):
            if o not in leaks:
                pb.free(oid[o])
    # record the plan (global object ids) so tests can look for it
    m = pb.meta
    m.setdefault("prefix_only", []).extend(int(oid[o]) for o in sorted(prefix_only))
    m.setdefault("unused", []).extend(int(oid[o]) for o in sorted(unused))
    m.setdefault("leaks", []).extend(int(oid[o]) for o in sorted(leaks))
    m.setdefault("dead_write", []).extend(int(oid[o]) for o in dw_plan if o not in dw)
    return oid


def _kernel_burst(pb, ts, o, prefix_only, is_write, pat_mix, access_sizes,
                  stride_range):
    rng = pb.rng
    E = pb.objs[o][2]
    n = pb.n_elem(o)
    limit = n
    if prefix_only:
        limit = int(pb.meta_prefix[o])
    acc = int(access_sizes[int(rng.integers(0, len(access_sizes)))])
    weight = int(rng.integers(1, 1000))
    r = rng.random()
    if r < pat_mix[0]:                      # sequential sweep
        stride = max(1, acc // E)
        start = int(rng.integers(0, max(1, limit // 4)))
        pb.affine(ts, o, start, stride, max(1, limit - start), weight, acc, is_write)
    elif r < pat_mix[0] + pat_mix[1]:       # strided (row/column sweeps)
        lo, hi = stride_range
        stride = int(round(math.exp(rng.uniform(math.log(lo), math.log(hi)))))
        start = int(rng.integers(0, stride))
        pb.affine(ts, o, start, stride, max(1, limit - start), weight, acc, is_write)
    else:                                   # random gather/scatter
        pb.random(ts, o, 0, max(1, limit), weight, acc, is_write)


# --------------------------------------------------------------------------
# Configs (BASELINE.json configs[0..4]); C3..C5 added in configs_dl.py
# --------------------------------------------------------------------------
def _inject_odd_records(pb, n_odd):
    """Injected records the method must count but not attribute (A1/A5):
    size 0, ts of an ALLOC, ts past the timeline, address overflow, gaps."""
    rng = pb.rng
    n_api = len(pb.kinds)
    allocs = [t for t, k in enumerate(pb.kinds) if k == API_ALLOC]
    acc = [t for t, k in enumerate(pb.kinds) if k not in (API_ALLOC, API_FREE)]
    for k in range(n_odd):
        c = k % 5
        t = acc[int(rng.integers(0, len(acc)))]
        if c == 0:
            pb.raw(t, 0x7F0000000000 + int(rng.integers(0, 1 << 20)), 0, False)
        elif c == 1:
            pb.raw(allocs[int(rng.integers(0, len(allocs)))], pb.objs[0][0], 4, False)
        elif c == 2:
            pb.raw(n_api + int(rng.integers(0, 100)), pb.objs[0][0], 4, True)
        elif c == 3:
            pb.raw(t, 0xFFFFFFFFFFFFFFF8, 16, False)
        else:
            pb.raw(t, 0x1000 + int(rng.integers(0, 1 << 16)) * 4, 4, False)


def _hpc_config(name, seed, n_records, *, n_obj, total_bytes, sizes_fn,
                e8_byte_frac, n_phases, n_kernels, n_cpy, n_set, n_leak,
                n_prefix, n_unused, n_dw, n_eald, objs_per_kernel, pat_mix,
                access_sizes, lazy, n_odd):
    pb = ProgramBuilder(name, seed)
    rng = pb.rng
    sizes = sizes_fn(rng)
    elems = np.full(n_obj, 4, dtype=np.int64)
    if e8_byte_frac > 0:
        order = rng.permutation(n_obj)
        acc = 0
        for o in order:
            if acc >= e8_byte_frac * sizes.sum():
                break
            elems[o] = 8
            acc += sizes[o]
    sizes = (sizes + elems - 1) // elems * elems
    pb.meta_prefix = {}
    per = [n_obj // n_phases + (1 if p < n_obj % n_phases else 0) for p in range(n_phases)]
    split = lambda x, p: x // n_phases + (1 if p < x % n_phases else 0)
    o0 = 0
    for p in range(n_phases):
        idx = np.arange(o0, o0 + per[p])
        o0 += per[p]
        local_sizes, local_elems = sizes[idx], elems[idx]
        _hpc_phase_with_prefix(
            pb, local_sizes, local_elems, n_kernels=split(n_kernels, p),
            n_cpy=split(n_cpy, p), n_set=split(n_set, p),
            n_leak=split(n_leak, p), n_prefix=split(n_prefix, p),
            n_unused=split(n_unused, p), n_dw=split(n_dw, p),
            n_eald=split(n_eald, p), objs_per_kernel=objs_per_kernel,
            pat_mix=pat_mix, access_sizes=access_sizes, lazy=lazy)
    if n_odd:
        _inject_odd_records(pb, n_odd)
        _sort_bursts_by_ts(pb)
    return pb.build(n_records)


def _sort_bursts_by_ts(pb):
    pb.bursts.sort(key=lambda b: b[5])


def _hpc_phase_with_prefix(pb, sizes, elems, **kw):
    """Wrap _hpc_phase so prefix-only objects get their prefix length recorded
    (keyed by global object id) before their bursts are drawn."""
    rng = pb.rng
    n = len(sizes)
    # _hpc_phase draws its own permutation; we mirror the prefix choice by
    # intercepting alloc: prefix length is drawn when the object is created.
    orig_alloc = pb.alloc

    def alloc(size, elem=4, base=None):
        g = orig_alloc(size, elem, base)
        f = rng.uniform(0.05, 0.60)
        pb.meta_prefix[g] = max(1, int((size // elem) * f))
        return g

    pb.alloc = alloc
    try:
        oid = _hpc_phase(pb, sizes, elems, **kw)
    finally:
        pb.alloc = orig_alloc
    return oid


def build_c1(seed=CONFIG_SEED_BASE + 1, n_records=1 << 20):
    """C1: 1M 4-8 B records over 64 objects (16 MiB), ~100 access APIs."""
    return _hpc_config(
        "C1-synthetic", seed, n_records, n_obj=64, total_bytes=16 << 20,
        sizes_fn=lambda rng: _loguniform_sizes(rng, 64, 16 << 10, 1 << 20, 16 << 20, 256),
        e8_byte_frac=0.0, n_phases=1, n_kernels=90, n_cpy=6, n_set=4,
        n_leak=8, n_prefix=8, n_unused=4, n_dw=2, n_eald=4,
        objs_per_kernel=(1, 4), pat_mix=(0.80, 0.15), access_sizes=(4, 8),
        lazy=True, n_odd=64)


def build_c2(seed=CONFIG_SEED_BASE + 2, n_records=100_000_000):
    """C2: Rodinia-style, 100M records over 1K objects (4 GiB)."""
    return _hpc_config(
        "C2-rodinia", seed, n_records, n_obj=1000, total_bytes=4 << 30,
        sizes_fn=lambda rng: _lognormal_sizes(rng, 1000, 4 << 30, 1.5, 4096, 256),
        e8_byte_frac=0.2, n_phases=20, n_kernels=3000, n_cpy=500, n_set=200,
        n_leak=50, n_prefix=100, n_unused=20, n_dw=20, n_eald=0,
        objs_per_kernel=(2, 6), pat_mix=(0.60, 0.30), access_sizes=(4, 8, 16),
        lazy=False, n_odd=1000)


def build_tiny(seed, n_obj_max=48, n_api_max=200, n_rec_max=4000, reuse=True):
    """Small adversarial program for brute-force cross-checks: address reuse,
    every element size, leaks, unused objects, memcpy/memset ranges, clipping,
    multi-word records, and every kind of invalid/unattributed record."""
    rng = np.random.default_rng(seed)
    arena = 0x10000
    alloc = BestFitPool(arena, 1 << 16, align=16) if reuse else BumpAllocator(rng, arena, 16, 64)
    pb = ProgramBuilder(f"tiny-{seed}", seed, alloc)
    rng = pb.rng
    live = []
    n_api_target = int(rng.integers(8, n_api_max + 1))
    recs_left = int(rng.integers(1, n_rec_max + 1))
    while len(pb.kinds) < n_api_target:
        r = rng.random()
        if (r < 0.25 or not live) and len(pb.objs) < n_obj_max:
            E = int(rng.choice([1, 2, 4, 8, 16]))
            ne = int(rng.integers(1, 300))
            try:
                o = pb.alloc(ne * E, E)
            except MemoryError:
                continue
            live.append(o)
        elif r < 0.40 and live:
            o = live.pop(int(rng.integers(0, len(live))))
            pb.free(o)
        else:
            kind = int(rng.choice([API_KERNEL, API_KERNEL, API_MEMCPY, API_MEMSET]))
            ts = pb.api(kind)
            nb = int(rng.integers(0, 4))
            for _ in range(nb):
                if not live or recs_left <= 0:
                    break
                o = live[int(rng.integers(0, len(live)))]
                E, n = pb.objs[o][2], pb.n_elem(o)
                w = bool(rng.random() < 0.5)
                q = rng.random()
                if kind != API_KERNEL or q < 0.15:
                    s = int(rng.integers(0, n))
                    nbytes = int(rng.integers(1, (n - s) * E + 1 + 2 * E))
                    pb.range_(ts, o, s, nbytes, w)   # may run past the end: clipped
                    recs_left -= 1
                    continue
                cnt = int(min(recs_left, rng.integers(1, 200)))
                recs_left -= cnt
                acc = int(rng.choice([1, 2, 4, 8, 16, 32, 100]))
                if q < 0.6:
                    stride = int(rng.integers(1, 5))
                    start = int(rng.integers(0, n))
                    pb.affine(ts, o, start, stride, max(1, n - start), cnt, acc, w)
                elif q < 0.8:
                    pb.affine(ts, o, int(rng.integers(0, n)), int(rng.integers(2, 70)),
                              n, cnt, acc, w)
                else:
                    pb.random(ts, o, 0, n, cnt, acc, w)
            if rng.random() < 0.3:
                # odd records: gaps, freed objects, alloc ts, past end of timeline
                c = int(rng.integers(0, 6))
                if c == 0:
                    pb.raw(ts, arena + int(rng.integers(0, 1 << 16)), int(rng.integers(1, 64)), False)
                elif c == 1 and pb.objs:
                    o = int(rng.integers(0, len(pb.objs)))
                    pb.raw(ts, pb.objs[o][0] + int(rng.integers(0, pb.objs[o][1])), 4, True)
                elif c == 2:
                    pb.raw(ts, arena, 0, False)
                elif c == 3:
                    pb.raw(int(rng.integers(0, len(pb.kinds))), arena + 64, 4, False)
                elif c == 4:
                    pb.raw(ts, 0xFFFFFFFFFFFFFFF0, 0x20, False)
                else:
                    pb.raw(len(pb.kinds) + 5, arena, 4, False)
    for o in live:
        if rng.random() < 0.7:
            pb.free(o)
    return pb.build()


CONFIGS = {"C1": build_c1, "C2": build_c2}


def object_sample(prog, k, offset=0):
    """The sub-program of objects o with o % k == offset and every burst that
    targets them (plus every k-th injected odd-record burst), over the SAME
    timeline: a proportional 1/k slice of the workload, used to time the CPU
    oracle on a bounded sample whose per-object fixed costs (bitmaps, scans)
    scale with the records like the full trace's.  Records keep the values
    they have in the full program (bursts keep their burst ids for the RANDOM
    hash).  Host generation only (tracegen/gen.cu has no burst ids)."""
    k = max(1, int(k))
    n = prog.n_obj
    keep_obj = (np.arange(n) % k) == offset
    new_idx = np.full(n + 1, 0xFFFFFFFF, np.uint64)
    new_idx[:n][keep_obj] = np.arange(int(keep_obj.sum()), dtype=np.uint64)
    bo = prog.bursts["obj"].astype(np.int64)
    is_obj = bo < n
    bid_all = np.arange(len(prog.bursts), dtype=np.uint64) if prog.burst_id is None else prog.burst_id
    keep_b = np.where(is_obj, keep_obj[np.minimum(bo, n - 1)], (bid_all % np.uint64(k)) == np.uint64(offset))
    bursts = prog.bursts[keep_b].copy()
    ob = bursts["obj"].astype(np.int64)
    bursts["obj"] = np.where(ob < n, new_idx[np.minimum(ob, n)], bursts["obj"]).astype(np.uint32)
    counts = bursts["count"].astype(np.uint64)
    prefix = np.zeros(len(bursts) + 1, np.uint64)
    np.cumsum(counts, out=prefix[1:])
    objs = prog.objects[keep_obj].copy()
    return Program(f"{prog.name}/objects%{k}=={offset}", prog.seed, objs, prog.kinds, bursts, prefix,
                   dict(prog.meta, sample_of=prog.name, sample_k=k, sample_offset=offset),
                   burst_id=bid_all[keep_b])


def build_config(name, **kw):
    if name not in CONFIGS:
        from . import configs_dl  # noqa: F401  (registers C3..C5)
    return CONFIGS[name](**kw)
