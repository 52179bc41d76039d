"""Seeded synthetic DrGPUM programs and access traces.

This package is the ONE module shared by both sides of the parity check (the
CUDA path in ``paper_conf_asplos_linzs23_b200`` and the CPU oracle in
``oracle/``).  It holds no part of the method's arithmetic: it only *draws*
programs (objects, the GPU-API timeline, access bursts) and expands bursts
into 16-byte access records.  Which object a record belongs to, which bits it
sets, first/last use, and every pattern are decided by the oracle and the CUDA
path independently.

Shapes follow BASELINE.json ``configs`` (C1..C5) and SURVEY.md §8(d); the
recipe of each config is written out in DESIGN.md §"Input recipe".
"""
from .layout import (OBJ_DTYPE, REC_DTYPE, BURST_DTYPE, API_ALLOC, API_FREE,
                     API_MEMCPY, API_MEMSET, API_KERNEL, NEVER,
                     PAT_AFFINE, PAT_RANDOM, PAT_RANGE, PAT_RAW)
from .program import Program, ProgramBuilder, build_config, build_tiny, object_sample, CONFIGS
from .records import gen_records, gen_all_records

__all__ = [
    "OBJ_DTYPE", "REC_DTYPE", "BURST_DTYPE", "API_ALLOC", "API_FREE",
    "API_MEMCPY", "API_MEMSET", "API_KERNEL", "NEVER", "PAT_AFFINE",
    "PAT_RANDOM", "PAT_RANGE", "PAT_RAW", "Program", "ProgramBuilder",
    "build_config", "build_tiny", "object_sample", "CONFIGS", "gen_records", "gen_all_records",
]
