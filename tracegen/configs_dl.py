"""C3-C5 program builders (BASELINE.json configs[2..4]).

  C3  ResNet-50 training iteration: 20,000 tensors in a 12 GiB best-fit caching
      pool (address reuse), 640 long-lived parameters / gradients / optimizer
      state (never freed), forward activations saved for backward (temporary
      idleness), short-lived workspaces.
  C4  LLM inference: 1,200 weights (100 GiB, read-only, never freed), 8,192 KV
      blocks of 2 MiB (filled prefixes -> overallocation), 90,608 activations in
      a 4 GiB reused arena; bursts pick weights / KV blocks Zipf(1.1).
  C5  scaling sweep: 10^6 objects (log-normal, median 8 KiB, 32 GiB), 10^5
      access APIs, C2-like bursts over objects picked Zipf(0.8) among the live
      ones, mean lifetime ~10^3 access APIs.

Record counts default to the BASELINE sizes; the parity tests pass smaller
``n_records`` (same objects, timeline and burst structure, fewer records per
burst).
"""
import math

import numpy as np

from .layout import API_KERNEL, API_MEMSET
from .program import (CONFIG_SEED_BASE, CONFIGS, BestFitPool, BumpAllocator, ProgramBuilder,
                      _inject_odd_records, _loguniform_sizes)

GiB, MiB, KiB = 1 << 30, 1 << 20, 1 << 10


def _zipf_pick(rng, n, s, size):
    """Indices in [0, n) with P(i) ~ 1/(i+1)^s."""
    w = 1.0 / np.power(np.arange(1, n + 1, dtype=np.float64), s)
    return rng.choice(n, size=size, p=w / w.sum())


def _seq(pb, ts, o, acc, w, weight, frac=1.0, start_frac=0.0):
    E = pb.objs[o][2]
    n = pb.n_elem(o)
    lim = max(1, int(n * frac))
    start = min(lim - 1, int(n * start_frac))
    pb.affine(ts, o, start, max(1, acc // E), max(1, lim - start), weight, acc, w)


def _mixed(pb, ts, o, acc, w, weight, p_seq, p_str):
    rng = pb.rng
    E = pb.objs[o][2]
    n = pb.n_elem(o)
    r = rng.random()
    if r < p_seq:
        _seq(pb, ts, o, acc, w, weight)
    elif r < p_seq + p_str:
        stride = int(rng.integers(2, 65))
        pb.affine(ts, o, int(rng.integers(0, stride)), stride, max(1, n), weight, acc, w)
    else:
        pb.random(ts, o, 0, max(1, n), weight, acc, w)


# --------------------------------------------------------------------------- C3
def build_c3(seed=CONFIG_SEED_BASE + 3, n_records=1_000_000_000, layers=160):
    pool = BestFitPool(0x7E0000000000, 12 * GiB, align=512)
    pb = ProgramBuilder("C3-resnet50-train", seed, pool)
    rng = pb.rng
    # 640 long-lived tensors: weight, grad, momentum, bn-stat per layer
    psize = _loguniform_sizes(rng, layers, 4 * KiB, 9 * MiB, 100 * MiB, 256)
    params = []
    for l in range(layers):
        E = 8 if rng.random() < 0.02 else 4
        sz = int(psize[l]) // E * E
        params.append([pb.alloc(sz, E) for _ in range(4)])  # w, g, m, bn
    meta_ti, saved = [], []
    n_fwd = 1600
    per_layer = n_fwd // layers
    act = None
    # forward: every kernel allocates its output right before it (+ workspaces)
    for k in range(n_fwd):
        l = k // per_layer
        out_sz = int(math.exp(rng.uniform(math.log(512 * KiB), math.log(8 * MiB)))) // 16 * 16
        out = pb.alloc(out_sz, 4)
        ws = [pb.alloc(int(rng.integers(1, 16)) * 64 * KiB, 4) for _ in range(int(rng.integers(2, 6)))]
        ts = pb.api(API_KERNEL)
        if act is not None:
            _seq(pb, ts, act, 16, False, 400)
        _seq(pb, ts, params[l][0], 16, False, 200)
        _seq(pb, ts, out, 16, True, 400)
        for wsp in ws:
            _mixed(pb, ts, wsp, 4, True, 100, 0.7, 0.2)
        for wsp in ws:
            pb.free(wsp)
        saved.append((l, out))
        act = out
    # backward: zero grads, then re-read saved activations (idle since forward)
    for l in range(layers):
        ts = pb.api(API_MEMSET)
        pb.range_(ts, params[l][1], 0, pb.objs[params[l][1]][1], True)
    grad = pb.alloc(pb.objs[act][1], 4)
    ts = pb.api(API_KERNEL)
    _seq(pb, ts, act, 16, False, 200)
    _seq(pb, ts, grad, 16, True, 200)
    n_bwd = 3000 - 1
    k = 0
    for i, (l, a) in enumerate(reversed(saved)):
        per_saved = n_bwd // len(saved) + (1 if i < n_bwd % len(saved) else 0)
        for j in range(per_saved):
            new_grad = pb.alloc(pb.objs[a][1], 4) if j == per_saved - 1 else None
            ws = [pb.alloc(int(rng.integers(1, 16)) * 64 * KiB, 4) for _ in range(int(rng.integers(2, 6)))]
            ts = pb.api(API_KERNEL)
            _seq(pb, ts, a, 16, False, 300)                   # saved activation (TI)
            _seq(pb, ts, grad, 16, False, 300)
            _seq(pb, ts, params[l][0], 16, False, 150)
            _mixed(pb, ts, params[l][1], 4, True, 150, 0.8, 0.15)  # accumulate weight grad
            if new_grad is not None:
                _seq(pb, ts, new_grad, 16, True, 300)
            for wsp in ws:
                _mixed(pb, ts, wsp, 4, True, 80, 0.7, 0.2)
            for wsp in ws:
                pb.free(wsp)
            k += 1
            if new_grad is not None:
                pb.free(grad)
                grad = new_grad
        pb.free(a)
        meta_ti.append(a)
    pb.free(grad)
    # optimizer: R grad, R/W weight and momentum
    n_opt = 5000 - 200 - n_fwd - 1 - n_bwd
    for k in range(max(0, n_opt)):
        ts = pb.api(API_KERNEL)
        for l in rng.choice(layers, size=min(layers, 3), replace=False):
            w, g, m, _ = params[l]
            _seq(pb, ts, g, 16, False, 50)
            _seq(pb, ts, w, 16, True, 50)
            _seq(pb, ts, m, 16, True, 50)
    for _ in range(200 - layers):
        ts = pb.api(API_MEMSET)
        o = params[int(rng.integers(0, layers))][3]
        pb.range_(ts, o, 0, pb.objs[o][1], True)
    pb.meta["saved_activations"] = meta_ti
    pb.meta["params"] = [o for p in params for o in p]
    _inject_odd_records(pb, 256)
    pb.bursts.sort(key=lambda b: b[5])
    return pb.build(n_records)


# --------------------------------------------------------------------------- C4
def build_c4(seed=CONFIG_SEED_BASE + 4, n_records=4_000_000_000, n_kernels=20_000,
             n_weights=1_200, n_kv=8_192, n_act=90_608, weight_bytes=100 * GiB):
    rng0 = np.random.default_rng(seed)
    pb = ProgramBuilder("C4-llm-inference", seed,
                        BumpAllocator(rng0, base=0x700000000000, align=2 * MiB, max_gap=0))
    rng = pb.rng
    wsz = _loguniform_sizes(rng, n_weights, 8 * MiB, 400 * MiB, weight_bytes, 2 * MiB)
    weights = [pb.alloc(int(s), 2) for s in wsz]
    kv = [pb.alloc(2 * MiB, 2) for _ in range(n_kv)]
    kv_fill = np.zeros(n_kv, dtype=np.int64)      # elements appended so far
    arena = BestFitPool(0x7D0000000000, 4 * GiB, align=512)
    pb.alloc_impl = arena
    hot = _zipf_pick(rng, n_weights + n_kv, 1.1, size=n_kernels * 2)
    acts_per_kernel = n_act / n_kernels
    live = []
    made = 0
    for k in range(n_kernels):
        want = int(acts_per_kernel * (k + 1)) - made
        new = [pb.alloc(int(rng.integers(1, 16)) * 16 * KiB, 2) for _ in range(want)]
        made += want
        ts = pb.api(API_KERNEL)
        for h in hot[2 * k: 2 * k + 2]:
            if h < n_weights:
                _seq(pb, ts, weights[h], 16, False, 600, frac=float(rng.uniform(0.05, 1.0)))
            else:
                b = h - n_weights
                n = pb.n_elem(kv[b])
                if kv_fill[b] < n:                         # append to the KV block
                    app = int(rng.integers(64, 4096))
                    pb.affine(ts, kv[b], int(kv_fill[b]), 8, max(1, n - int(kv_fill[b])), app // 8 + 1, 16, True)
                    kv_fill[b] = min(n, kv_fill[b] + app)
                if kv_fill[b] > 0:
                    _seq(pb, ts, kv[b], 16, False, 300, frac=kv_fill[b] / n)
        for a in new:
            _seq(pb, ts, a, 16, True, 40)
        for a in live[: max(0, len(live) - 8)]:
            _seq(pb, ts, a, 16, False, 20)
        # activations live 1-3 kernels
        keep = []
        for a in live:
            if rng.random() < 0.5:
                pb.free(a)
            else:
                keep.append(a)
        live = keep + new
    for a in live:                       # every activation is freed within the trace
        pb.free(a)
    pb.meta["weights"] = list(range(n_weights))
    pb.meta["kv_blocks"] = list(range(n_weights, n_weights + n_kv))
    _inject_odd_records(pb, 512)
    pb.bursts.sort(key=lambda b: b[5])
    return pb.build(n_records)


# --------------------------------------------------------------------------- C5
def build_c5(seed=CONFIG_SEED_BASE + 5, n_records=16_000_000_000, n_obj=1_000_000,
             n_access=100_000, n_free=950_000, total_bytes=32 * GiB, mean_life=1_000):
    """Vectorised timeline: objects are born at a uniform access-API index and
    live ~Exp(mean_life) access APIs; each access API touches 1-4 live objects
    picked Zipf(0.8) by age rank."""
    rng = np.random.default_rng(seed)
    s = rng.lognormal(math.log(8 * KiB), 1.5, n_obj)
    s = s / s.sum() * total_bytes
    sizes = np.maximum(256, (s // 256) * 256).astype(np.int64)
    birth = np.sort(rng.integers(0, n_access, n_obj))
    life = np.maximum(1, rng.exponential(mean_life, n_obj).astype(np.int64))
    death = birth + life
    freed = np.zeros(n_obj, dtype=bool)
    freed[rng.permutation(n_obj)[:n_free]] = True
    # events: (access index, order, kind, obj): allocs before access a, frees after
    ev_a = np.concatenate([birth, np.where(freed, np.minimum(death, n_access - 1), -1)])
    ev_k = np.concatenate([np.zeros(n_obj, np.int64), np.ones(n_obj, np.int64)])
    ev_o = np.concatenate([np.arange(n_obj), np.arange(n_obj)])
    keep = ev_a >= 0
    ev_a, ev_k, ev_o = ev_a[keep], ev_k[keep], ev_o[keep]
    # per access API a: [allocs of a] [API a] [frees of a]
    order = np.lexsort((ev_o, ev_k, ev_a))
    ev_a, ev_k, ev_o = ev_a[order], ev_k[order], ev_o[order]
    n_api = len(ev_a) + n_access
    kinds = np.full(n_api, API_KERNEL, dtype=np.uint8)
    # position of each event / access API in the timeline
    allocs_upto = np.searchsorted(ev_a * 2 + ev_k, np.arange(n_access) * 2, side="right")
    pos_api = allocs_upto + np.arange(n_access)          # API a sits after all events with key < 2a
    is_api = np.zeros(n_api, dtype=bool)
    is_api[pos_api] = True
    ev_pos = np.flatnonzero(~is_api)
    kinds[ev_pos] = np.where(ev_k == 0, 0, 1).astype(np.uint8)
    t_alloc = np.empty(n_obj, np.int64)
    t_free = np.full(n_obj, 0xFFFFFFFF, np.int64)
    t_alloc[ev_o[ev_k == 0]] = ev_pos[ev_k == 0]
    t_free[ev_o[ev_k == 1]] = ev_pos[ev_k == 1]
    # 10% of the access APIs are memcpy/memset
    cs = rng.random(n_access) < 0.1
    kinds[pos_api[cs]] = np.where(rng.random(cs.sum()) < 0.7, 2, 3).astype(np.uint8)
    base = np.cumsum(np.concatenate([[0x600000000000], sizes[:-1] + 256]))
    from .layout import OBJ_DTYPE, BURST_DTYPE, PAT_AFFINE, PAT_RANDOM
    objs = np.zeros(n_obj, dtype=OBJ_DTYPE)
    objs["base"], objs["size"], objs["elem_size"] = base, sizes, 4
    objs["t_alloc"], objs["t_free"] = t_alloc, t_free
    objs["user_id"] = np.arange(n_obj)
    # bursts: each access API touches 1-4 objects live at it (alive: birth <= a < death or never freed)
    n_touch = rng.integers(1, 5, n_access)
    a_of = np.repeat(np.arange(n_access), n_touch)
    # candidates: objects born at or before a, by recency rank r ~ Zipf(0.8) truncated
    born_upto = np.searchsorted(birth, a_of, side="right")          # objects with birth <= a
    u = rng.random(len(a_of))
    r = np.floor(np.power(u, 1 / 0.2) * mean_life * 2).astype(np.int64)  # heavy head on recent
    cand = np.clip(born_upto - 1 - r, 0, n_obj - 1)
    alive = (birth[cand] <= a_of) & ((~freed[cand]) | (death[cand] > a_of)) & (born_upto > 0)
    a_of, cand = a_of[alive], cand[alive]
    nb = len(a_of)
    bursts = np.zeros(nb, dtype=BURST_DTYPE)
    E = 4
    n_el = sizes[cand] // E
    pat = rng.random(nb)
    acc = rng.choice(np.array([4, 8, 16]), nb)
    bursts["base"] = base[cand]
    bursts["ts"] = pos_api[a_of]
    bursts["elem"] = E
    bursts["access_size"] = acc
    bursts["obj"] = cand
    bursts["is_write"] = rng.random(nb) < 0.4
    seq = pat < 0.6
    strd = (pat >= 0.6) & (pat < 0.9)
    rnd = pat >= 0.9
    bursts["pattern"] = np.where(rnd, PAT_RANDOM, PAT_AFFINE)
    bursts["stride"] = np.where(seq, np.maximum(1, acc // E),
                                np.where(strd, rng.integers(2, 1025, nb), 0))
    bursts["start"] = np.where(strd, rng.integers(0, 2, nb), 0)
    bursts["span"] = np.maximum(1, n_el - bursts["start"].astype(np.int64))
    bursts["count"] = rng.integers(1, 1000, nb)
    from .program import Program, _rescale_counts
    _rescale_counts(bursts, n_records)
    prefix = np.zeros(nb + 1, dtype=np.uint64)
    np.cumsum(bursts["count"], out=prefix[1:])
    return Program("C5-scaling-sweep", seed, objs, kinds, bursts, prefix,
                   {"freed": int(freed.sum())})


CONFIGS.update({"C3": build_c3, "C4": build_c4, "C5": build_c5})
