"""Device-side record generation (tracegen/gen.cu, built as
tracegen/libtracegen.so): the same pure function ``record(i)`` as
``records.gen_records``, evaluated on the GPU so that traces larger than host
memory (BASELINE configs C3-C5 at full size) can be produced chunk by chunk in
HBM.  Input generation only -- no part of the method's arithmetic.
"""
import ctypes
import os

import numpy as np

_LIB = None
_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libtracegen.so")


def _lib():
    global _LIB
    if _LIB is None:
        if not os.path.exists(_PATH):
            raise RuntimeError(f"{_PATH} missing: run `make tracegen` (or __graft_entry__.build())")
        L = ctypes.CDLL(_PATH)
        L.tg_gen_records.restype = ctypes.c_int
        L.tg_gen_records.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64,
                                     ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p]
        _LIB = L
    return _LIB


class DeviceProgram:
    """A program's burst table resident on a CUDA device."""

    def __init__(self, prog, device="cuda"):
        import torch
        if prog.burst_id is not None:
            raise ValueError("device generation needs a program's own bursts (not an object_sample)")
        self.prog = prog
        self.device = torch.device(device)
        self.bursts = torch.from_numpy(np.ascontiguousarray(prog.bursts).view(np.uint8)).to(self.device)
        self.prefix = torch.from_numpy(np.ascontiguousarray(prog.prefix).view(np.int64)).to(self.device)
        self.nb = len(prog.bursts)

    def gen(self, i0, i1, out=None, stream=None):
        """Records [i0, i1) as a uint8 tensor of 16*(i1-i0) bytes on the device
        (written into ``out`` when given), stream-ordered on ``stream``."""
        import torch
        n = int(i1) - int(i0)
        if out is None:
            out = torch.empty(16 * n, dtype=torch.uint8, device=self.device)
        assert out.numel() >= 16 * n and out.data_ptr() % 16 == 0
        if stream is None:
            stream = torch.cuda.current_stream(self.device)
        rc = _lib().tg_gen_records(self.bursts.data_ptr(), self.prefix.data_ptr(), self.nb,
                                   int(self.prog.seed), int(i0), int(i1), out.data_ptr(),
                                   ctypes.c_void_p(stream.cuda_stream))
        if rc != 0:
            raise RuntimeError(f"tg_gen_records: cudaError {rc}")
        return out[: 16 * n]
