"""B200-native DrGPUM per-access object attribution (ASPLOS '23, Lin/Zhou/Su).

The product is libdrgpum.so (C ABI, include/drgpum.h; sm_100a kernels in
csrc/).  This package is its thin Python binding:

    from paper_conf_asplos_linzs23_b200 import Session
    s = Session(objects, api_kinds)       # drgpum_objects_load + workspace_bind
    s.attribute(records_cuda_tensor)      # drgpum_trace_attribute
    stats, counters = s.object_stats()    # drgpum_object_stats
    reports = s.patterns()                # drgpum_patterns

It never imports the CPU oracle (oracle/ is test infrastructure only).
"""
from ._lib import (OBJECT_DTYPE, RECORD_DTYPE, STATS_DTYPE, REPORT_DTYPE, COUNTERS_DTYPE,
                   LAYOUT_DTYPE, NEVER, EA, LD, UA, ML, TI, DW, OA, OA_ACTIONABLE,
                   FLAG_NAMES, DrgpumError, EXPORTS, LIB_PATH, load, redundant_pairs, kahn_levels,
                   DEP_INTRA, DEP_RAW, DEP_WAW, DEP_WAR)
from .session import Session, pinned_array

__all__ = ["Session", "pinned_array", "OBJECT_DTYPE", "RECORD_DTYPE", "STATS_DTYPE", "REPORT_DTYPE",
           "COUNTERS_DTYPE", "LAYOUT_DTYPE", "NEVER", "EA", "LD", "UA", "ML", "TI", "DW",
           "OA", "OA_ACTIONABLE", "FLAG_NAMES", "DrgpumError", "EXPORTS", "LIB_PATH", "load",
           "redundant_pairs", "kahn_levels", "DEP_INTRA", "DEP_RAW", "DEP_WAW", "DEP_WAR"]
