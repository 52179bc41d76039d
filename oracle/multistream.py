"""NEXT-4 oracle: multi-stream dependency graph and Kahn timestamps -- TEST
INFRASTRUCTURE (only tests/, smoke() and bench.py's CPU legs may import it).

Follows PAPER.md §5.3 literally:
  * ``dependency_edges``   -- Definition 5.1 (l.277-286): intra-stream
    immediate successors, and RAW / WAW / WAR over every ordered pair of
    events on an object, each "no v_k ... following v_i and before v_j"
    checked by scanning the events in between;
  * ``kahn_levels``        -- the algorithm of l.295, steps (1)-(5): all
    in-degree-zero vertices of a round get the same T;
  * ``patterns_topo``      -- the time-dependent patterns (EA Def 3.1, LD Def
    3.2, TI Def 3.6, DW Def 3.7) with "between" counted over all APIs whose T
    lies strictly between (R26) and distances as T differences
    (l.297 "computing the difference between their timestamps").

Readings (R24-R27): vertices are the APIs in invocation order (the
index the records carry); an object's events are its ALLOC (a write that
"allocates"), its accessing APIs with the read/write flags the attribution
found, and its FREE (a "free"); "following v_i and before v_j" is invocation
order.  Pure Python, tiny inputs (cubic in an object's event count).
"""
NEVER = 0xFFFFFFFF
ALLOC, FREE, MEMCPY, MEMSET, KERNEL = 0, 1, 2, 3, 4
INTRA, RAW, WAW, WAR = 1, 2, 4, 8


def dependency_edges(n_api, streams, objects, access_sets):
    """{(i, j): label bits} per Def 5.1.  access_sets[o] = {ts: (read, write)}."""
    edges = {}

    def add(i, j, lab):
        edges[(i, j)] = edges.get((i, j), 0) | lab

    last = {}
    for v in range(n_api):                      # l.281 intra-stream successor
        s = int(streams[v])
        if s in last:
            add(last[s], v, INTRA)
        last[s] = v
    for o, obj in enumerate(objects):
        # event = (api, allocates, reads, writes, frees)
        ev = [(int(obj["t_alloc"]), True, False, False, False)]
        for t in sorted(access_sets[o]):
            r, w = access_sets[o][t]
            ev.append((int(t), False, bool(r), bool(w), False))
        if int(obj["t_free"]) != NEVER:
            ev.append((int(obj["t_free"]), False, False, False, True))
        for a in range(len(ev)):
            vi, al_i, r_i, w_i, _ = ev[a]
            for b in range(a + 1, len(ev)):
                vj, _, r_j, w_j, f_j = ev[b]
                mid = ev[a + 1:b]
                no_write_between = not any(e[3] for e in mid)
                if (al_i or w_i) and r_j and no_write_between:          # RAW l.283
                    add(vi, vj, RAW)
                if (al_i or w_i) and (f_j or w_j) and not mid:          # WAW l.284
                    add(vi, vj, WAW)
                if r_i and (f_j or w_j) and no_write_between:           # WAR l.285
                    add(vi, vj, WAR)
    return edges


def kahn_levels(n_api, edges):
    """l.295: (1) T = 0; (2) every vertex of in-degree zero gets T and is
    deleted with its outgoing edges; (3) in-degrees of its successors are
    updated; (4) T += 1; (5) repeat until the graph is empty."""
    succ = {v: [] for v in range(n_api)}
    indeg = [0] * n_api
    for (i, j) in edges:
        succ[i].append(j)
        indeg[j] += 1
    T = [None] * n_api
    remaining = set(range(n_api))
    t = 0                                                    # (1)
    while remaining:                                         # (5)
        zero = [v for v in sorted(remaining) if indeg[v] == 0]
        if not zero:
            raise ValueError("dependency graph has a cycle")
        for v in zero:                                       # (2)
            T[v] = t
            remaining.discard(v)
        for v in zero:                                       # (3)
            for j in succ[v]:
                indeg[j] -= 1
        t += 1                                               # (4)
    return T


def patterns_topo(kinds, objects, access_sets, T, ti_min_idle=2):
    """EA / LD / TI / DW of every object on the topological timestamps."""
    n_api = len(kinds)

    def between(a, b):               # APIs whose T lies strictly between
        return sum(1 for v in range(n_api) if T[a] < T[v] < T[b])
    out = []
    for o, obj in enumerate(objects):
        ta, tf = int(obj["t_alloc"]), int(obj["t_free"])
        acc = sorted(access_sets[o], key=lambda t: (T[t], t))
        rep = dict(flags=set(), ea_distance=0, ld_distance=0, ti_ranges=0,
                   ti_max_idle=0, ti_total_idle=0, dw_pairs=0)
        if acc:
            f, l = acc[0], acc[-1]
            if between(ta, f) >= 1:                                   # Def 3.1
                rep["flags"].add("EA")
                rep["ea_distance"] = T[f] - T[ta]
            if tf != NEVER and between(l, tf) >= 1:                   # Def 3.2
                rep["flags"].add("LD")
                rep["ld_distance"] = T[tf] - T[l]
            for a, b in zip(acc, acc[1:]):
                g = between(a, b)                                     # Def 3.6
                if g >= ti_min_idle:
                    rep["ti_ranges"] += 1
                    rep["ti_max_idle"] = max(rep["ti_max_idle"], g)
                    rep["ti_total_idle"] += g
                cs = (MEMCPY, MEMSET)                                 # Def 3.7
                if kinds[a] in cs and kinds[b] in cs and access_sets[o][a][1] and access_sets[o][b][1]:
                    rep["dw_pairs"] += 1
            if rep["ti_ranges"]:
                rep["flags"].add("TI")
            if rep["dw_pairs"]:
                rep["flags"].add("DW")
        out.append(rep)
    return out
