"""CPU oracle for DrGPUM's per-access attribution -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product package ``paper_conf_asplos_linzs23_b200`` never imports it, and the
two share no code (see oracle/drgpum_oracle.cpp's header for the citations of
what it computes).

``run_oracle`` is O1 (the C++ std::map replay of PAPER.md §5.1/§5.2);
``oracle.bruteforce`` is O0 (literal per-definition Python, tiny inputs).
"""
import ctypes
import os
import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")

STATS_DTYPE = np.dtype([
    ("n_elems", "<u8"), ("accessed", "<u8"), ("span_lo", "<u8"),
    ("span_hi", "<u8"), ("largest_unaccessed_run", "<u8"),
    ("t_first", "<u4"), ("t_last", "<u4"), ("n_access_apis", "<u4"), ("_pad", "<u4"),
])
REPORT_DTYPE = np.dtype([
    ("flags", "<u4"), ("ea_distance", "<u4"), ("ld_distance", "<u4"),
    ("ti_ranges", "<u4"), ("ti_max_idle", "<u4"), ("dw_pairs", "<u4"),
    ("ti_total_idle", "<u8"),
])
COUNTERS_DTYPE = np.dtype([("records", "<u8"), ("attributed", "<u8"),
                           ("unattributed", "<u8"), ("clipped", "<u8"),
                           ("invalid", "<u8")])
EA, LD, UA, ML, TI, DW, OA, OA_ACTIONABLE = 1, 2, 4, 8, 16, 32, 64, 128
FLAG_NAMES = {EA: "EA", LD: "LD", UA: "UA", ML: "ML", TI: "TI", DW: "DW",
              OA: "OA", OA_ACTIONABLE: "OA_ACTIONABLE"}
DEFAULT_THRESHOLDS = (2, 80, 80)  # TI X=2, OA 80%, Frag 80%

_lib = None


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `make -C {os.path.dirname(_HERE)} oracle`")
        L = ctypes.CDLL(_LIB_PATH)
        P, U64, U32, I = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
        L.oracle_validate.argtypes = [P, U64, P, U32, ctypes.POINTER(U64)]
        L.oracle_validate.restype = I
        L.oracle_new.argtypes = [P, U64, P, U32, ctypes.POINTER(I)]
        L.oracle_new.restype = P
        L.oracle_free.argtypes = [P]
        L.oracle_attribute.argtypes = [P, P, U64]
        L.oracle_stats.argtypes = [P, P, P]
        L.oracle_patterns.argtypes = [P, P, P]
        L.oracle_get_bitmap.argtypes = [P, U64, P]
        L.oracle_get_accesses.argtypes = [P, U64, P, P, U64]
        L.oracle_get_accesses.restype = U64
        L.oracle_track_structured.argtypes = [P]
        L.oracle_structured.argtypes = [P, P, P]
        L.oracle_structured_group.argtypes = [P, P, P, P]
        L.oracle_slice_frequency.argtypes = [P, P, P]
        L.oracle_track_frequency.argtypes = [P]
        L.oracle_frequency.argtypes = [P, P, P, P, P, P, U64]
        L.oracle_frequency.restype = U64
        _lib = L
    return _lib


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def validate(objects, kinds):
    L = _load()
    objects = np.ascontiguousarray(objects)
    kinds = np.ascontiguousarray(kinds, dtype=np.uint8)
    bad = ctypes.c_uint64(0)
    st = L.oracle_validate(_ptr(objects), objects.shape[0], _ptr(kinds),
                           kinds.shape[0], ctypes.byref(bad))
    return st, bad.value


class Oracle:
    """One oracle run over (objects, kinds); feed records with attribute()."""

    def __init__(self, objects, kinds, structured=False, frequency=False):
        L = _load()
        self.objects = np.ascontiguousarray(objects)
        self.kinds = np.ascontiguousarray(kinds, dtype=np.uint8)
        st = ctypes.c_int(0)
        self._h = L.oracle_new(_ptr(self.objects), self.objects.shape[0],
                               _ptr(self.kinds), self.kinds.shape[0], ctypes.byref(st))
        self.status = st.value
        if not self._h:
            raise ValueError(f"oracle: objects rejected with status {st.value}")
        if structured:
            L.oracle_track_structured(self._h)
        if frequency:
            L.oracle_track_frequency(self._h)

    def __del__(self):
        if getattr(self, "_h", None):
            _load().oracle_free(self._h)
            self._h = None

    def attribute(self, records):
        records = np.ascontiguousarray(records)
        _load().oracle_attribute(self._h, _ptr(records), records.shape[0])

    def stats(self):
        n = self.objects.shape[0]
        out = np.zeros(n, dtype=STATS_DTYPE)
        ctr = np.zeros(1, dtype=COUNTERS_DTYPE)
        _load().oracle_stats(self._h, _ptr(out), _ptr(ctr))
        return out, ctr[0]

    def patterns(self, thresholds=DEFAULT_THRESHOLDS):
        n = self.objects.shape[0]
        out = np.zeros(n, dtype=REPORT_DTYPE)
        th = np.array(thresholds, dtype=np.uint32)
        _load().oracle_patterns(self._h, _ptr(th), _ptr(out))
        return out

    def structured(self, group=None):
        """NEXT-3: (sa u8[n_obj], overlap u8[n_obj]) over the APIs t with
        group[t] != 0 (None = all APIs) [R23]; needs structured=True."""
        n = self.objects.shape[0]
        sa = np.zeros(n, np.uint8)
        ov = np.zeros(n, np.uint8)
        g = None if group is None else np.ascontiguousarray(group, dtype=np.uint8)
        _load().oracle_structured_group(self._h, None if g is None else _ptr(g), _ptr(sa), _ptr(ov))
        return sa, ov

    def slice_frequency(self, group=None):
        """Slice-level NUAF moments [R22b] over the APIs t with group[t] != 0:
        per object (n, sum F, sum F^2) as Python ints, F = total access
        frequency of one API's slice; needs frequency=True."""
        n = self.objects.shape[0]
        out = np.zeros(4 * n, np.uint64)
        g = None if group is None else np.ascontiguousarray(group, dtype=np.uint8)
        _load().oracle_slice_frequency(self._h, None if g is None else _ptr(g), _ptr(out))
        q = out.reshape(n, 4)
        return [(int(a), int(b), int(c) | (int(d) << 64)) for a, b, c, d in q]

    def frequency(self):
        """NEXT-2 rows (obj, ts, n, s1, s2) in (object, ts) order; needs frequency=True."""
        L = _load()
        k = L.oracle_frequency(self._h, None, None, None, None, None, 0)
        cols = [np.zeros(k, np.uint32), np.zeros(k, np.uint32)] + [np.zeros(k, np.uint64) for _ in range(3)]
        L.oracle_frequency(self._h, *[_ptr(c) for c in cols], k)
        return tuple(cols)

    def bitmap(self, o):
        """Object o's bitmap as a bool array of n_elem entries."""
        ne = int(self.objects["size"][o] // self.objects["elem_size"][o])
        buf = np.zeros((ne + 7) // 8, dtype=np.uint8)
        _load().oracle_get_bitmap(self._h, o, _ptr(buf))
        return np.unpackbits(buf, bitorder="little")[:ne].astype(bool)

    def bitmap_packed(self, o):
        ne = int(self.objects["size"][o] // self.objects["elem_size"][o])
        buf = np.zeros((ne + 7) // 8, dtype=np.uint8)
        _load().oracle_get_bitmap(self._h, o, _ptr(buf))
        return buf

    def accesses(self, o):
        """(timestamps u32[k], flags u8[k]) with flags bit0 = read, bit1 = write."""
        L = _load()
        k = L.oracle_get_accesses(self._h, o, None, None, 0)
        ts = np.zeros(k, dtype=np.uint32)
        rw = np.zeros(k, dtype=np.uint8)
        L.oracle_get_accesses(self._h, o, _ptr(ts), _ptr(rw), k)
        return ts, rw


def run_oracle(objects, kinds, records, thresholds=DEFAULT_THRESHOLDS):
    """Convenience: one pass; returns (oracle, stats, counters, reports)."""
    o = Oracle(objects, kinds)
    o.attribute(records)
    st, ctr = o.stats()
    return o, st, ctr, o.patterns(thresholds)


def nuaf_cv_exceeds(n, s1, s2, pct=20):
    """Def 3.9 / fn 3: coefficient of variation (population) of the n touched
    elements' frequencies > pct%, exactly: pct^2 is compared in integers,
    CV^2 = (n*S2 - S1^2) / S1^2 > (pct/100)^2."""
    n, s1, s2 = int(n), int(s1), int(s2)
    return s1 > 0 and (n * s2 - s1 * s1) * 100 * 100 > pct * pct * s1 * s1
