"""Binary layouts of the generator's outputs (plain data, no method logic).

Object (32 B) and record (16 B) layouts are the interchange format of the
boundary: SURVEY.md §8(b).  A record covers bytes [addr, addr+size) and its
``meta`` word packs the issuing GPU API's timestamp (bits 0..30) and the
write flag (bit 31) -- PAPER.md §5.2 l.264 ("accessed memory range (i.e.,
start address and size)") and §5.1 l.238 (timestamps aligned with invocation
order).
"""
import numpy as np

API_ALLOC, API_FREE, API_MEMCPY, API_MEMSET, API_KERNEL = 0, 1, 2, 3, 4
NEVER = 0xFFFFFFFF

OBJ_DTYPE = np.dtype([
    ("base", "<u8"), ("size", "<u8"), ("elem_size", "<u4"),
    ("t_alloc", "<u4"), ("t_free", "<u4"), ("user_id", "<u4"),
])
assert OBJ_DTYPE.itemsize == 32

REC_DTYPE = np.dtype([("addr", "<u8"), ("size", "<u4"), ("meta", "<u4")])
assert REC_DTYPE.itemsize == 16

# Burst patterns.  A burst is a run of consecutive records issued by one API.
#   AFFINE : elem_j = start + (j*stride) mod span      (SEQ sweeps, strided)
#   RANDOM : elem_j = start + hash(seed, burst, j) mod span
#   RANGE  : one record, addr = base + start*E, size = access_size (memcpy/memset)
#   RAW    : one record, addr = base, size = access_size (injected odd records)
PAT_AFFINE, PAT_RANDOM, PAT_RANGE, PAT_RAW = 0, 1, 2, 3

BURST_DTYPE = np.dtype([
    ("base", "<u8"), ("start", "<u8"), ("stride", "<u8"), ("span", "<u8"),
    ("count", "<u8"), ("ts", "<u4"), ("elem", "<u4"), ("access_size", "<u4"),
    ("obj", "<u4"), ("pattern", "u1"), ("is_write", "u1"), ("_pad", "u1", (6,)),
])
assert BURST_DTYPE.itemsize == 64
