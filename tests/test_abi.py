"""CPU-side checks of the C-ABI library: it loads, exports every symbol
include/drgpum.h declares, and its host-side validation agrees with the
oracle's (no kernel is launched; without a GPU drgpum_create reports ECUDA but
still returns a context whose host logic works)."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_asplos_linzs23_b200 as pkg
from paper_conf_asplos_linzs23_b200 import _lib
from oracle import validate as oracle_validate
from tracegen import OBJ_DTYPE, NEVER, build_tiny, build_config

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    hdr = open(os.path.join(ROOT, "include", "drgpum.h")).read()
    return sorted(set(re.findall(r"DRGPUM_API[^;(]*?\b(drgpum_\w+)\s*\(", hdr)))


def test_header_declares_the_boundary():
    d = _declared()
    for name in ("drgpum_objects_load", "drgpum_trace_attribute", "drgpum_object_stats",
                 "drgpum_patterns"):
        assert name in d
    assert sorted(_lib.EXPORTS) == d


def test_library_exports_every_declared_symbol():
    L = _lib.load()
    for name in _declared():
        assert hasattr(L, name), name
        assert ctypes.cast(getattr(L, name), ctypes.c_void_p).value


def test_struct_sizes_match_header():
    assert pkg.OBJECT_DTYPE.itemsize == 32 and pkg.RECORD_DTYPE.itemsize == 16
    assert pkg.STATS_DTYPE.itemsize == 56 and pkg.REPORT_DTYPE.itemsize == 32
    assert OBJ_DTYPE == pkg.OBJECT_DTYPE


def _host_ctx():
    L = _lib.load()
    h = ctypes.c_void_p()
    L.drgpum_create(0, ctypes.byref(h))   # ECUDA without a GPU, context still created
    assert h.value
    return L, h


def _load_status(objs, kinds):
    L, h = _host_ctx()
    objs = np.ascontiguousarray(objs)
    kinds = np.ascontiguousarray(kinds, dtype=np.uint8)
    st = L.drgpum_objects_load(h, ctypes.c_void_p(objs.ctypes.data), objs.shape[0],
                               ctypes.c_void_p(kinds.ctypes.data), kinds.shape[0])
    msg = L.drgpum_last_error(h).decode()
    L.drgpum_destroy(h)
    return st, msg


A, F, C, S, K = 0, 1, 2, 3, 4


@pytest.mark.parametrize("rows,kinds", [
    ([(4096, 64, 4, 0, 2, 0)], [A, K, F]),
    ([(4096, 0, 4, 0, 2, 0)], [A, K, F]),
    ([(4096, 64, 3, 0, 2, 0)], [A, K, F]),
    ([(4096, 66, 4, 0, 2, 0)], [A, K, F]),
    ([(2**64 - 32, 64, 4, 0, 2, 0)], [A, K, F]),
    ([(4096, 64, 4, 1, 2, 0)], [A, K, F]),
    ([(4096, 64, 4, 0, 1, 0)], [A, K, F]),
    ([(4096, 64, 4, 0, 5, 0)], [A, K, F]),
    ([(4096, 64, 4, 0, 2, 0)], [A, K, 7]),
    ([(4096, 64, 4, 0, NEVER, 0), (4096 + 32, 64, 4, 1, NEVER, 1)], [A, A, K]),
    ([(4096, 64, 4, 0, 2, 0), (4096 + 32, 64, 4, 3, NEVER, 1)], [A, K, F, A, K]),
    ([(4096, 64, 4, 0, 3, 0), (4096 + 64, 64, 4, 1, NEVER, 1)], [A, A, K, F]),
    ([(4096, 64, 4, 0, 3, 0), (4096 + 63, 64, 4, 1, NEVER, 1)], [A, A, K, F]),
    ([(4096, 64, 4, 0, 3, 0), (0, 2**20, 1, 1, 4, 1)], [A, A, K, F, F]),
    ([(4096, 64, 4, 0, 2, 0), (4000, 256, 4, 3, 5, 1), (4096, 64, 4, 6, 7, 2)],
     [A, K, F, A, K, F, A, F]),
])
def test_validation_matches_oracle(rows, kinds):
    objs = np.zeros(len(rows), dtype=OBJ_DTYPE)
    for i, r in enumerate(rows):
        objs[i] = r
    st, msg = _load_status(objs, kinds)
    assert st == oracle_validate(objs, np.array(kinds, dtype=np.uint8))[0], msg


@pytest.mark.parametrize("seed", range(20))
def test_validation_generated_programs(seed):
    p = build_tiny(seed)
    assert _load_status(p.objects, p.kinds)[0] == 0
    # corrupt: make one object's lifetime overlap a reuser of its address
    objs = p.objects.copy()
    b = objs["base"]
    order = np.argsort(b, kind="stable")
    for i, j in zip(order, order[1:]):
        if b[j] < b[i] + objs["size"][i] and objs["t_free"][i] != NEVER:
            objs["t_free"][i] = NEVER   # i now lives forever over j's range
            want = oracle_validate(objs, p.kinds)[0]
            assert _load_status(objs, p.kinds)[0] == want
            break


def test_c1_loads():
    p = build_config("C1")
    assert _load_status(p.objects, p.kinds)[0] == 0
