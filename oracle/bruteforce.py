"""O0: a literal, per-definition brute force of the oracle -- TEST INFRASTRUCTURE.

Independent of O1 (oracle/drgpum_oracle.cpp) in algorithm, not just in
language:
  * attribution scans EVERY object for "contains the address and is live at
    the record's timestamp" (no memory map, no replay) and asserts that at most
    one matches (the uniqueness SURVEY §8(a) A2 relies on);
  * touched elements are found byte by byte: byte b of the clipped range
    belongs to element (b - base) // E ("which element(s) ... a
    memory instruction touches");
  * "GPU API invocations between" is COUNTED by walking the timeline
    (Defs 3.1, 3.2, 3.6 at l.124-166; rules l.244-248), not computed as a
    timestamp difference;
  * percentages use exact fractions (Def 3.8 l.174; Eq. (1) l.191);
  * the largest unaccessed chunk uses itertools.groupby.
Tiny inputs only (every record is expanded byte-wise).
"""
from fractions import Fraction
from itertools import groupby

ALLOC, FREE, MEMCPY, MEMSET, KERNEL = 0, 1, 2, 3, 4
NEVER = 0xFFFFFFFF
U64_MAX = (1 << 64) - 1


def bruteforce(objects, kinds, records, thresholds=(2, 80, 80)):
    x_ti, x_oa, x_frag = thresholds
    n_api = len(kinds)
    objs = [dict(base=int(o["base"]), size=int(o["size"]), E=int(o["elem_size"]),
                 ta=int(o["t_alloc"]), tf=int(o["t_free"])) for o in objects]
    touched = [set() for _ in objs]
    acc = [dict() for _ in objs]        # ts -> [read, write]
    ctr = dict(records=0, attributed=0, unattributed=0, clipped=0, invalid=0)
    for r in records:
        addr, size, meta = int(r["addr"]), int(r["size"]), int(r["meta"])
        ts, w = meta & 0x7FFFFFFF, meta >> 31
        ctr["records"] += 1
        if size == 0 or ts >= n_api or kinds[ts] in (ALLOC, FREE) or addr + size > U64_MAX:
            ctr["invalid"] += 1
            continue

        def live(o):
            return o["ta"] < ts and (o["tf"] == NEVER or ts < o["tf"])
        hits = [i for i, o in enumerate(objs)
                if o["base"] <= addr < o["base"] + o["size"] and live(o)]
        assert len(hits) <= 1, "two live objects contain one address"
        if not hits:
            ctr["unattributed"] += 1
            continue
        i = hits[0]
        o = objs[i]
        ctr["attributed"] += 1
        end = addr + size
        if end > o["base"] + o["size"]:
            ctr["clipped"] += 1
            end = o["base"] + o["size"]
        for b in range(addr, end):
            touched[i].add((b - o["base"]) // o["E"])
        f = acc[i].setdefault(ts, [False, False])
        f[1 if w else 0] = True

    stats, reports = [], []
    for i, o in enumerate(objs):
        n = o["size"] // o["E"]
        bits = [e in touched[i] for e in range(n)]
        accessed = sum(bits)
        zero_runs = [len(list(g)) for k, g in groupby(bits) if not k]
        run = max(zero_runs, default=0)
        apis = sorted(acc[i])
        stats.append(dict(
            n_elems=n, accessed=accessed,
            span_lo=min(touched[i]) if touched[i] else U64_MAX,
            span_hi=max(touched[i]) if touched[i] else U64_MAX,
            largest_unaccessed_run=run,
            t_first=apis[0] if apis else NEVER, t_last=apis[-1] if apis else 0,
            n_access_apis=len(apis)))

        def between(a, b):   # number of GPU API invocations strictly between
            return sum(1 for t in range(n_api) if a < t < b)
        rep = dict(flags=set(), ea_distance=0, ld_distance=0, ti_ranges=0,
                   ti_max_idle=0, ti_total_idle=0, dw_pairs=0)
        if not apis:
            rep["flags"].add("UA")                                  # Def 3.4
        if o["tf"] == NEVER:
            rep["flags"].add("ML")                                  # Def 3.5
        if apis:
            if between(o["ta"], apis[0]) >= 1:                      # Def 3.1 / l.244
                rep["flags"].add("EA")
                rep["ea_distance"] = apis[0] - o["ta"]
            if o["tf"] != NEVER and between(apis[-1], o["tf"]) >= 1:  # Def 3.2 / l.245
                rep["flags"].add("LD")
                rep["ld_distance"] = o["tf"] - apis[-1]
            for a, b in zip(apis, apis[1:]):
                g = between(a, b)                                   # Def 3.6 / l.248
                if g >= x_ti:
                    rep["ti_ranges"] += 1
                    rep["ti_max_idle"] = max(rep["ti_max_idle"], g)
                    rep["ti_total_idle"] += g
                cs = (MEMCPY, MEMSET)                               # Def 3.7 / l.249
                if kinds[a] in cs and kinds[b] in cs and acc[i][a][1] and acc[i][b][1]:
                    rep["dw_pairs"] += 1
            if rep["ti_ranges"]:
                rep["flags"].add("TI")
            if rep["dw_pairs"]:
                rep["flags"].add("DW")
        if Fraction(accessed, n) < Fraction(x_oa, 100):             # Def 3.8
            rep["flags"].add("OA")
            unacc = n - accessed
            frag = Fraction(0) if unacc == 0 else 1 - Fraction(run, unacc)   # Eq. (1)
            if frag < Fraction(x_frag, 100):                        # l.194
                rep["flags"].add("OA_ACTIONABLE")
        reports.append(rep)
    access_sets = [{t: (f[0], f[1]) for t, f in a.items()} for a in acc]
    return stats, reports, ctr, touched, access_sets


def validate(objects, kinds):
    """Status per SURVEY §8(b): 0 ok, 1 EINVAL, 2 EOVERLAP (pairwise check)."""
    n_api = len(kinds)
    if n_api >= 1 << 31 or any(k > KERNEL for k in kinds):
        return 1
    objs = list(objects)
    for o in objs:
        b, s, E, ta, tf = (int(o["base"]), int(o["size"]), int(o["elem_size"]),
                           int(o["t_alloc"]), int(o["t_free"]))
        if s == 0 or E not in (1, 2, 4, 8, 16) or s % E or b + s > U64_MAX:
            return 1
        if ta >= n_api or kinds[ta] != ALLOC:
            return 1
        if tf != NEVER and (tf >= n_api or tf <= ta or kinds[tf] != FREE):
            return 1
    for i, p in enumerate(objs):
        for q in objs[i + 1:]:
            pb, pe = int(p["base"]), int(p["base"]) + int(p["size"])
            qb, qe = int(q["base"]), int(q["base"]) + int(q["size"])
            ptf = float("inf") if int(p["t_free"]) == NEVER else int(p["t_free"])
            qtf = float("inf") if int(q["t_free"]) == NEVER else int(q["t_free"])
            if pb < qe and qb < pe and max(int(p["t_alloc"]), int(q["t_alloc"])) < min(ptf, qtf):
                return 2
    return 0


def bruteforce_structured(objects, kinds, records, group=None):
    """NEXT-3 structured access by definition (Def 3.10, l.200): per object,
    the set of elements each accessing GPU API touches; SA iff at least two
    APIs access O and their slices are pairwise disjoint.  Only the APIs t
    with group[t] count (None = all) [R23].  Returns (sa, overlap) lists of
    0/1."""
    n_api = len(kinds)
    objs = [dict(base=int(o["base"]), size=int(o["size"]), E=int(o["elem_size"]),
                 ta=int(o["t_alloc"]), tf=int(o["t_free"])) for o in objects]
    slices = [dict() for _ in objs]          # ts -> set of elements
    for r in records:
        addr, size, meta = int(r["addr"]), int(r["size"]), int(r["meta"])
        ts = meta & 0x7FFFFFFF
        if size == 0 or ts >= n_api or kinds[ts] in (ALLOC, FREE) or addr + size > U64_MAX:
            continue
        for i, o in enumerate(objs):
            if o["base"] <= addr < o["base"] + o["size"] and o["ta"] < ts and \
                    (o["tf"] == NEVER or ts < o["tf"]):
                end = min(addr + size, o["base"] + o["size"])
                s = slices[i].setdefault(ts, set())
                for b in range(addr, end):
                    s.add((b - o["base"]) // o["E"])
                break
    sa, ov = [], []
    for sl in slices:
        sets = [v for t, v in sl.items() if group is None or group[t]]
        overlap = any(sets[a] & sets[b] for a in range(len(sets)) for b in range(a + 1, len(sets)))
        ov.append(int(overlap))
        sa.append(int(len(sets) >= 2 and not overlap))
    return sa, ov


def bruteforce_frequency(objects, kinds, records):
    """NEXT-2 by definition (Def 3.9 l.196, §5.2 l.271): for every (object,
    accessing API), the access frequency of each element that API touches
    (byte-wise expansion); rows (obj, ts, n, S1, S2) sorted by (obj, ts)."""
    n_api = len(kinds)
    objs = [dict(base=int(o["base"]), size=int(o["size"]), E=int(o["elem_size"]),
                 ta=int(o["t_alloc"]), tf=int(o["t_free"])) for o in objects]
    hm = {}
    for r in records:
        addr, size, meta = int(r["addr"]), int(r["size"]), int(r["meta"])
        ts = meta & 0x7FFFFFFF
        if size == 0 or ts >= n_api or kinds[ts] in (ALLOC, FREE) or addr + size > U64_MAX:
            continue
        for i, o in enumerate(objs):
            if o["base"] <= addr < o["base"] + o["size"] and o["ta"] < ts and \
                    (o["tf"] == NEVER or ts < o["tf"]):
                end = min(addr + size, o["base"] + o["size"])
                elems = {(b - o["base"]) // o["E"] for b in range(addr, end)}
                d = hm.setdefault((i, ts), {})
                for e in elems:
                    d[e] = d.get(e, 0) + 1
                break
    rows = []
    for (i, ts) in sorted(hm):
        f = list(hm[(i, ts)].values())
        rows.append((i, ts, len(f), sum(f), sum(c * c for c in f)))
    return rows


def bruteforce_slice_frequency(objects, kinds, records, group=None):
    """Slice-level NUAF [R22b] by definition: for every object, over the APIs
    t with group[t] (None = all) that access it, F_t = number of (record,
    element) touches of t on the object (byte-wise expansion, an element
    counted once per record); returns per object (n, sum F, sum F^2)."""
    rows = bruteforce_frequency(objects, kinds, records)
    out = [[0, 0, 0] for _ in objects]
    for (i, ts, n, s1, s2) in rows:
        if group is None or group[ts]:
            out[i][0] += 1
            out[i][1] += s1
            out[i][2] += s1 * s1
    return [tuple(x) for x in out]
