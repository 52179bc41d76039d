"""ctypes binding of libdrgpum.so (include/drgpum.h).  Argument marshalling
only: every step of the hot path runs in the library's sm_100a kernels.
There is no fallback: if the library is missing, importing the binding fails.
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libdrgpum.so")

# Layouts of include/drgpum.h (retyped here; the oracle has its own copy).
OBJECT_DTYPE = np.dtype([("base", "<u8"), ("size", "<u8"), ("elem_size", "<u4"),
                         ("t_alloc", "<u4"), ("t_free", "<u4"), ("user_id", "<u4")])
RECORD_DTYPE = np.dtype([("addr", "<u8"), ("size", "<u4"), ("meta", "<u4")])
STATS_DTYPE = np.dtype([("n_elems", "<u8"), ("accessed", "<u8"), ("span_lo", "<u8"),
                        ("span_hi", "<u8"), ("largest_unaccessed_run", "<u8"),
                        ("t_first", "<u4"), ("t_last", "<u4"), ("n_access_apis", "<u4"),
                        ("_pad", "<u4")])
REPORT_DTYPE = np.dtype([("flags", "<u4"), ("ea_distance", "<u4"), ("ld_distance", "<u4"),
                         ("ti_ranges", "<u4"), ("ti_max_idle", "<u4"), ("dw_pairs", "<u4"),
                         ("ti_total_idle", "<u8")])
COUNTERS_DTYPE = np.dtype([("records", "<u8"), ("attributed", "<u8"), ("unattributed", "<u8"),
                           ("clipped", "<u8"), ("invalid", "<u8")])
LAYOUT_DTYPE = np.dtype([("bitmap_word", "<u8"), ("hit_word", "<u8"), ("r_lo", "<u4"),
                         ("n_hit_apis", "<u4")])
assert OBJECT_DTYPE.itemsize == 32 and RECORD_DTYPE.itemsize == 16
assert STATS_DTYPE.itemsize == 56 and REPORT_DTYPE.itemsize == 32 and LAYOUT_DTYPE.itemsize == 24

NEVER = 0xFFFFFFFF
FEATURE_STRUCTURED = 1
FEATURE_FREQUENCY = 2
DEP_INTRA, DEP_RAW, DEP_WAW, DEP_WAR = 1, 2, 4, 8
API_ALLOC, API_FREE, API_MEMCPY, API_MEMSET, API_KERNEL = 0, 1, 2, 3, 4
EA, LD, UA, ML, TI, DW, OA, OA_ACTIONABLE = 1, 2, 4, 8, 16, 32, 64, 128
FLAG_NAMES = {EA: "EA", LD: "LD", UA: "UA", ML: "ML", TI: "TI", DW: "DW", OA: "OA",
              OA_ACTIONABLE: "OA_ACTIONABLE"}
STATUS = {0: "DRGPUM_OK", 1: "DRGPUM_EINVAL", 2: "DRGPUM_EOVERLAP", 3: "DRGPUM_ESTATE",
          4: "DRGPUM_ENOMEM", 5: "DRGPUM_ECUDA"}


class Thresholds(ctypes.Structure):
    _fields_ = [("ti_min_idle", ctypes.c_uint32), ("oa_accessed_pct", ctypes.c_uint32),
                ("oa_frag_pct", ctypes.c_uint32)]


class ShadowView(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in ("or_off", "or_words", "bitmap_words", "hit_words",
                                               "first_off", "last_off", "counters_off", "n_obj")]


class Counters(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in COUNTERS_DTYPE.names]


class DrgpumError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


EXPORTS = ["drgpum_create", "drgpum_objects_load", "drgpum_set_features", "drgpum_set_finalize_consume", "drgpum_set_queue_capacity", "drgpum_set_api_group", "drgpum_slice_frequency", "drgpum_set_frequency_capacity", "drgpum_structured",
           "drgpum_frequency", "drgpum_frequency_slots",
           "drgpum_workspace_size",
           "drgpum_workspace_bind", "drgpum_reset", "drgpum_trace_attribute",
           "drgpum_trace_attribute_host", "drgpum_shadow_view", "drgpum_object_layout",
           "drgpum_merge_or", "drgpum_merge_peers", "drgpum_merge_peers_owned", "drgpum_merge_peers_owned_nvls", "drgpum_gather_peers", "drgpum_finalize", "drgpum_object_stats", "drgpum_patterns",
           "drgpum_consistency_errors", "drgpum_path_stats", "drgpum_redundant_pairs",
           "drgpum_redundant_alloc", "drgpum_kahn_levels", "drgpum_dependency_graph",
           "drgpum_patterns_topo", "drgpum_last_error", "drgpum_destroy",
           "drgpum_launch_count"]

_lib = None


def load():
    """Load libdrgpum.so (no CUDA call is made here)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing -- build it with `make lib` (or "
                          "__graft_entry__.build()); there is no CPU fallback")
    L = ctypes.CDLL(LIB_PATH)
    P, U64, U32, I = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
    PP = ctypes.POINTER(ctypes.c_void_p)
    sig = {
        "drgpum_create": ([I, PP], I),
        "drgpum_objects_load": ([P, P, U64, P, U32], I),
        "drgpum_workspace_size": ([P, ctypes.POINTER(U64)], I),
        "drgpum_workspace_bind": ([P, P, U64, P], I),
        "drgpum_reset": ([P, P], I),
        "drgpum_trace_attribute": ([P, P, U64, P], I),
        "drgpum_trace_attribute_host": ([P, P, U64, P], I),
        "drgpum_shadow_view": ([P, ctypes.POINTER(ShadowView)], I),
        "drgpum_object_layout": ([P, P], I),
        "drgpum_merge_or": ([P, P, U32, U64, U64, U64, P], I),
        "drgpum_merge_peers": ([P, P, U32, U32, P], I),
        "drgpum_merge_peers_owned": ([P, P, U32, U32, P], I),
        "drgpum_merge_peers_owned_nvls": ([P, P, U32, U32, P, P], I),
        "drgpum_gather_peers": ([P, P, U32, U32, P], I),
        "drgpum_finalize": ([P, ctypes.POINTER(Thresholds), P], I),
        "drgpum_object_stats": ([P, P, ctypes.POINTER(Counters), P], I),
        "drgpum_patterns": ([P, ctypes.POINTER(Thresholds), P, P], I),
        "drgpum_consistency_errors": ([P, ctypes.POINTER(U64), P], I),
        "drgpum_path_stats": ([P, P, P], I),
        "drgpum_set_features": ([P, U32], I),
        "drgpum_set_finalize_consume": ([P, ctypes.c_int], I),
        "drgpum_set_queue_capacity": ([P, U32, U32], I),
        "drgpum_set_api_group": ([P, P, P], I),
        "drgpum_set_frequency_capacity": ([P, U64], I),
        "drgpum_slice_frequency": ([P, U32, P, P, P], I),
        "drgpum_structured": ([P, P, P, P], I),
        "drgpum_frequency": ([P, U32, P, P, P], I),
        "drgpum_frequency_slots": ([P, P, ctypes.POINTER(U64), P], I),
        "drgpum_redundant_pairs": ([P, P, P, P, U64, U32, P, P, U64, ctypes.POINTER(U64)], I),
        "drgpum_redundant_alloc": ([P, U32, P, P, U64, ctypes.POINTER(U64), P], I),
        "drgpum_kahn_levels": ([U32, P, P, U64, P], I),
        "drgpum_dependency_graph": ([P, P, P, P, P, P, U64, ctypes.POINTER(U64), P], I),
        "drgpum_patterns_topo": ([P, P, P, P, P], I),
        "drgpum_last_error": ([P], ctypes.c_char_p),
        "drgpum_destroy": ([P], None),
        "drgpum_launch_count": ([P], U64),
    }
    for name, (args, res) in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = res
    _lib = L
    return L


def check(ctx, status):
    if status != 0:
        raise DrgpumError(status, load().drgpum_last_error(ctx).decode(errors="replace"))


def redundant_pairs(sizes, first, last, used, pct=10):
    """Host algorithm of NEXT-1 on plain arrays (no GPU needed): list of
    (reuser, donor) object indices."""
    L = load()
    sizes = np.ascontiguousarray(sizes, dtype=np.uint64)
    first = np.ascontiguousarray(first, dtype=np.uint32)
    last = np.ascontiguousarray(last, dtype=np.uint32)
    used = np.ascontiguousarray(used, dtype=np.uint8)
    n = sizes.shape[0]
    cnt = ctypes.c_uint64()
    p = lambda a: ctypes.c_void_p(a.ctypes.data)
    st = L.drgpum_redundant_pairs(p(sizes), p(first), p(last), p(used), n, pct, None, None, 0,
                                  ctypes.byref(cnt))
    if st:
        raise DrgpumError(st, "drgpum_redundant_pairs")
    a = np.zeros(cnt.value, np.uint32)
    b = np.zeros(cnt.value, np.uint32)
    L.drgpum_redundant_pairs(p(sizes), p(first), p(last), p(used), n, pct, p(a), p(b), cnt.value,
                             ctypes.byref(cnt))
    return list(zip(a.tolist(), b.tolist()))


def kahn_levels(n_api, src, dst):
    """NEXT-4 host algorithm on a plain edge list: u32[n_api] Kahn levels."""
    L = load()
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    T = np.zeros(n_api, np.uint32)
    p = lambda a: ctypes.c_void_p(a.ctypes.data)
    st = L.drgpum_kahn_levels(n_api, p(src), p(dst), src.shape[0], p(T))
    if st:
        raise DrgpumError(st, "drgpum_kahn_levels")
    return T
