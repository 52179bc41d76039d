"""Session: one DrGPUM attribution context on one CUDA device.

PyTorch supplies device memory (the workspace), streams and -- for multi-GPU
merges (parallel.py) -- process groups.  Everything else is a call into
libdrgpum.so.
"""
import ctypes

import numpy as np
import torch

from . import _lib
from ._lib import (OBJECT_DTYPE, RECORD_DTYPE, STATS_DTYPE, REPORT_DTYPE, COUNTERS_DTYPE,
                   LAYOUT_DTYPE, Thresholds, ShadowView, Counters, check)


def _np_ptr(a):
    return ctypes.c_void_p(a.ctypes.data)


def _stream_handle(stream):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def pinned_array(n, dtype):
    """A numpy array of n ``dtype`` elements in page-locked host memory (a
    torch pinned allocation, kept alive by the array's base): outputs read
    into it (``object_stats(out=...)``, ``patterns(out=...)``) copy at the
    DMA rate instead of through the driver's pageable staging."""
    dtype = np.dtype(dtype)
    t = torch.empty(max(1, n) * dtype.itemsize, dtype=torch.uint8, pin_memory=True)
    a = t.numpy()[:n * dtype.itemsize].view(dtype)
    return a


def _out(out, n, dtype):
    if out is None:
        return np.zeros(n, dtype=dtype)
    if out.dtype != dtype or out.shape != (n,) or not out.flags.c_contiguous:
        raise ValueError(f"out must be a contiguous {dtype} array of {n} elements")
    return out


def _thresholds(th):
    if th is None:
        return Thresholds(2, 80, 80)
    if isinstance(th, Thresholds):
        return th
    return Thresholds(*th)


class Session:
    """Attribute an access trace to the objects of one program.

    objects: array of OBJECT_DTYPE (32-B drgpum_object_t) records.
    kinds:   uint8 array, the GPU-API kind of every timestamp.
    """

    def __init__(self, objects, kinds, device=None, structured=False, frequency=False, workspace_alloc=None,
                 queue_capacity=None, frequency_capacity=None):
        if not torch.cuda.is_available():
            raise RuntimeError("drgpum Session needs a CUDA device (there is no CPU fallback)")
        self.L = _lib.load()
        self.device = torch.device("cuda", torch.cuda.current_device() if device is None
                                   else torch.device(device).index or 0)
        objs = np.asarray(objects)
        self.objects = np.ascontiguousarray(objs if objs.dtype == OBJECT_DTYPE
                                            else objs.view(OBJECT_DTYPE))
        self.kinds = np.ascontiguousarray(kinds, dtype=np.uint8)
        self.n_obj = int(self.objects.shape[0])
        self.n_api = int(self.kinds.shape[0])
        h = ctypes.c_void_p()
        st = self.L.drgpum_create(self.device.index, ctypes.byref(h))
        self._h = h
        check(self._h, st)
        check(self._h, self.L.drgpum_objects_load(self._h, _np_ptr(self.objects), self.n_obj,
                                                  _np_ptr(self.kinds), self.kinds.shape[0]))
        feats = (_lib.FEATURE_STRUCTURED if structured else 0) | (_lib.FEATURE_FREQUENCY if frequency else 0)
        if feats:
            check(self._h, self.L.drgpum_set_features(self._h, feats))
        if frequency_capacity is not None:   # NEXT-2 records per sub-call
            check(self._h, self.L.drgpum_set_frequency_capacity(self._h, int(frequency_capacity)))
        if queue_capacity is not None:   # (range entries, aux entries); tests drive the overflow paths
            check(self._h, self.L.drgpum_set_queue_capacity(self._h, *queue_capacity))
        nbytes = ctypes.c_uint64()
        check(self._h, self.L.drgpum_workspace_size(self._h, ctypes.byref(nbytes)))
        # workspace_alloc(nbytes, device) -> uint8 CUDA tensor (e.g. torch
        # symmetric memory for merge_peers); default torch.empty
        alloc = workspace_alloc or (lambda nb, dev: torch.empty(nb, dtype=torch.uint8, device=dev))
        self.workspace = alloc(max(int(nbytes.value), 256), self.device)
        with torch.cuda.device(self.device):
            check(self._h, self.L.drgpum_workspace_bind(
                self._h, ctypes.c_void_p(self.workspace.data_ptr()), self.workspace.numel(),
                _stream_handle(None)))
        v = ShadowView()
        check(self._h, self.L.drgpum_shadow_view(self._h, ctypes.byref(v)))
        self.view = v

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            self.L.drgpum_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ------------------------------------------------------------ attribution
    def reset(self, stream=None):
        check(self._h, self.L.drgpum_reset(self._h, _stream_handle(stream)))

    def attribute(self, records, stream=None):
        """records: a CUDA tensor holding 16-B records (any dtype, contiguous,
        nbytes % 16 == 0) -> drgpum_trace_attribute; or a host numpy array /
        CPU tensor -> drgpum_trace_attribute_host (pipelined H2D staging)."""
        if isinstance(records, torch.Tensor):
            if not records.is_contiguous():
                raise ValueError("records tensor must be contiguous")
            nbytes = records.numel() * records.element_size()
            if nbytes % 16:
                raise ValueError("records tensor size is not a multiple of 16 bytes")
            n = nbytes // 16
            if records.is_cuda:
                check(self._h, self.L.drgpum_trace_attribute(
                    self._h, ctypes.c_void_p(records.data_ptr()), n, _stream_handle(stream)))
            else:
                check(self._h, self.L.drgpum_trace_attribute_host(
                    self._h, ctypes.c_void_p(records.data_ptr()), n, _stream_handle(stream)))
            return
        a = np.ascontiguousarray(records)
        if a.dtype != RECORD_DTYPE:
            a = a.view(RECORD_DTYPE)
        check(self._h, self.L.drgpum_trace_attribute_host(self._h, _np_ptr(a), a.shape[0],
                                                          _stream_handle(stream)))

    # ------------------------------------------------------------ results
    def set_finalize_consume(self, on=True):
        """drgpum_set_finalize_consume: reduce-and-clear -- finalize zeroes the
        bitmap words it reduces (bitmaps read back as zero afterwards; stats
        and patterns stay valid; attribute / merges need a reset first)."""
        check(self._h, self.L.drgpum_set_finalize_consume(self._h, 1 if on else 0))

    def finalize(self, thresholds=None, stream=None):
        th = _thresholds(thresholds)
        check(self._h, self.L.drgpum_finalize(self._h, ctypes.byref(th), _stream_handle(stream)))

    def object_stats(self, stream=None, out=None):
        out = _out(out, self.n_obj, STATS_DTYPE)
        c = Counters()
        check(self._h, self.L.drgpum_object_stats(self._h, _np_ptr(out), ctypes.byref(c),
                                                  _stream_handle(stream)))
        ctr = np.zeros((), dtype=COUNTERS_DTYPE)
        for k in COUNTERS_DTYPE.names:
            ctr[k] = getattr(c, k)
        return out, ctr

    def patterns(self, thresholds=None, stream=None, out=None):
        out = _out(out, self.n_obj, REPORT_DTYPE)
        th = _thresholds(thresholds)
        check(self._h, self.L.drgpum_patterns(self._h, ctypes.byref(th), _np_ptr(out),
                                              _stream_handle(stream)))
        return out

    def dependency_graph(self, streams, stream=None):
        """NEXT-4: (T u32[n_api], src u32[E], dst u32[E], label u8[E]) of the
        Def 5.1 graph for API stream ids ``streams``."""
        streams = np.ascontiguousarray(streams, dtype=np.uint32)
        if streams.shape[0] != self.n_api:
            raise ValueError("streams must have one entry per API")
        n = ctypes.c_uint64()
        T = np.zeros(self.n_api, np.uint32)
        check(self._h, self.L.drgpum_dependency_graph(self._h, _np_ptr(streams), None, None, None, None,
                                                      0, ctypes.byref(n), _stream_handle(stream)))
        src = np.zeros(n.value, np.uint32)
        dst = np.zeros(n.value, np.uint32)
        lab = np.zeros(n.value, np.uint8)
        check(self._h, self.L.drgpum_dependency_graph(self._h, _np_ptr(streams), _np_ptr(T), _np_ptr(src),
                                                      _np_ptr(dst), _np_ptr(lab), n.value,
                                                      ctypes.byref(n), _stream_handle(stream)))
        return T, src, dst, lab

    def patterns_topo(self, T, thresholds=None, stream=None):
        """NEXT-4: pattern reports on topological timestamps T (u32[n_api])."""
        T = np.ascontiguousarray(T, dtype=np.uint32)
        if T.shape[0] != self.n_api:
            raise ValueError("T must have one entry per API")
        out = np.zeros(self.n_obj, dtype=REPORT_DTYPE)
        th = _thresholds(thresholds)
        check(self._h, self.L.drgpum_patterns_topo(self._h, _np_ptr(T), ctypes.byref(th), _np_ptr(out),
                                                   _stream_handle(stream)))
        return out

    def consistency_errors(self, stream=None):
        e = ctypes.c_uint64()
        check(self._h, self.L.drgpum_consistency_errors(self._h, ctypes.byref(e),
                                                        _stream_handle(stream)))
        return int(e.value)

    def path_stats(self, stream=None):
        """Diagnostics: 32-record tiles per attribution path since the last reset."""
        out = np.zeros(4, dtype=np.uint64)
        check(self._h, self.L.drgpum_path_stats(self._h, _np_ptr(out), _stream_handle(stream)))
        return dict(zip(("affine_union", "affine_words", "tile_fast", "slow"), (int(x) for x in out)))

    def set_api_group(self, in_group=None, stream=None):
        """drgpum_set_api_group: u8[n_api] mask of the APIs the NEXT-2/3
        analyses consider (None = all) [R22b, R23]; set before attributing
        for the structured-access pass."""
        g = None if in_group is None else np.ascontiguousarray(in_group, dtype=np.uint8)
        if g is not None and g.shape[0] != self.n_api:
            raise ValueError("in_group needs one entry per API")
        check(self._h, self.L.drgpum_set_api_group(self._h, None if g is None else _np_ptr(g),
                                                   _stream_handle(stream)))

    def slice_frequency(self, pct=20, stream=None):
        """Slice-level NUAF [R22b]: (match u8[n_obj], moments list of
        (n, S1, S2) Python ints) over the API group; needs frequency=True."""
        m = np.zeros(self.n_obj, np.uint8)
        mo = np.zeros(4 * self.n_obj, np.uint64)
        check(self._h, self.L.drgpum_slice_frequency(self._h, pct, _np_ptr(m), _np_ptr(mo),
                                                     _stream_handle(stream)))
        q = mo.reshape(self.n_obj, 4)
        return m, [(int(a), int(b), int(c) | (int(d) << 64)) for a, b, c, d in q]

    def structured(self, stream=None):
        """NEXT-3: (sa u8[n_obj], overlap u8[n_obj]) over the API group
        (set_api_group); needs structured=True."""
        sa = np.zeros(self.n_obj, np.uint8)
        ov = np.zeros(self.n_obj, np.uint8)
        check(self._h, self.L.drgpum_structured(self._h, _np_ptr(sa), _np_ptr(ov), _stream_handle(stream)))
        return sa, ov

    def frequency(self, pct=20, stream=None):
        """NEXT-2: (count u32[n_obj], first_ts u32[n_obj]) of the APIs at which
        each object matches non-uniform access frequency; needs frequency=True."""
        cnt = np.zeros(self.n_obj, np.uint32)
        first = np.zeros(self.n_obj, np.uint32)
        check(self._h, self.L.drgpum_frequency(self._h, pct, _np_ptr(cnt), _np_ptr(first),
                                               _stream_handle(stream)))
        return cnt, first

    def frequency_slots(self, stream=None):
        """NEXT-2 raw sums: u64[n_slots, 3] = (n, S1, S2) per (object, access API)."""
        n = ctypes.c_uint64()
        check(self._h, self.L.drgpum_frequency_slots(self._h, None, ctypes.byref(n), _stream_handle(stream)))
        out = np.zeros((n.value, 3), np.uint64)
        check(self._h, self.L.drgpum_frequency_slots(self._h, _np_ptr(out), ctypes.byref(n),
                                                     _stream_handle(stream)))
        return out

    def redundant_allocations(self, pct=10, stream=None):
        """NEXT-1: [(reuser, donor), ...] from this session's first/last uses."""
        cnt = ctypes.c_uint64()
        check(self._h, self.L.drgpum_redundant_alloc(self._h, pct, None, None, 0, ctypes.byref(cnt),
                                                     _stream_handle(stream)))
        a = np.zeros(cnt.value, np.uint32)
        b = np.zeros(cnt.value, np.uint32)
        check(self._h, self.L.drgpum_redundant_alloc(self._h, pct, _np_ptr(a), _np_ptr(b), cnt.value,
                                                     ctypes.byref(cnt), _stream_handle(stream)))
        return list(zip(a.tolist(), b.tolist()))

    def layout(self):
        out = np.zeros(self.n_obj, dtype=LAYOUT_DTYPE)
        check(self._h, self.L.drgpum_object_layout(self._h, _np_ptr(out)))
        return out

    def launch_count(self):
        return int(self.L.drgpum_launch_count(self._h))

    # ------------------------------------------------------------ shadow views
    def or_words(self):
        """The OR-mergeable shadow (bitmaps then hit rows) as an int32 CUDA
        tensor aliasing the workspace."""
        v = self.view
        return self.workspace[v.or_off: v.or_off + 4 * v.or_words].view(torch.int32)

    def first_last(self):
        v = self.view
        f = self.workspace[v.first_off: v.first_off + 4 * v.n_obj].view(torch.int32)
        l = self.workspace[v.last_off: v.last_off + 4 * v.n_obj].view(torch.int32)
        return f, l

    def counters_tensor(self):
        v = self.view
        return self.workspace[v.counters_off: v.counters_off + 8 * 5].view(torch.int64)

    def raw_counters(self):
        """All 16 u64 counter slots of the workspace (diagnostics: [5] is the
        range-queue overflow count, [6] the consistency count)."""
        v = self.view
        return self.workspace[v.counters_off: v.counters_off + 8 * 16].view(torch.int64)

    def merge_or(self, src, n_src, src_stride_words, word_lo, word_hi, stream=None):
        check(self._h, self.L.drgpum_merge_or(self._h, ctypes.c_void_p(src.data_ptr()), n_src,
                                              src_stride_words, word_lo, word_hi,
                                              _stream_handle(stream)))

    def merge_peers(self, peer_ptrs, rank, stream=None):
        """drgpum_merge_peers: peer_ptrs = workspace base pointers (ints) of every
        rank, index = rank (this session's own at ``rank``)."""
        arr = (ctypes.c_void_p * len(peer_ptrs))(*[ctypes.c_void_p(int(x)) for x in peer_ptrs])
        check(self._h, self.L.drgpum_merge_peers(self._h, arr, len(peer_ptrs), rank,
                                                 _stream_handle(stream)))

    def merge_peers_owned(self, peer_ptrs, rank, stream=None):
        """drgpum_merge_peers_owned: merge this rank's objects only (then
        finalize + gather_peers)."""
        arr = (ctypes.c_void_p * len(peer_ptrs))(*[ctypes.c_void_p(int(x)) for x in peer_ptrs])
        check(self._h, self.L.drgpum_merge_peers_owned(self._h, arr, len(peer_ptrs), rank,
                                                       _stream_handle(stream)))

    def merge_peers_owned_nvls(self, peer_ptrs, rank, mc_ptr, stream=None):
        """drgpum_merge_peers_owned_nvls: the owned merge, objects touched by
        several ranks read through the NVSwitch multicast mapping mc_ptr."""
        arr = (ctypes.c_void_p * len(peer_ptrs))(*[ctypes.c_void_p(int(x)) for x in peer_ptrs])
        check(self._h, self.L.drgpum_merge_peers_owned_nvls(self._h, arr, len(peer_ptrs), rank,
                                                            ctypes.c_void_p(int(mc_ptr)),
                                                            _stream_handle(stream)))

    def gather_peers(self, peer_ptrs, rank, stream=None):
        """drgpum_gather_peers: share this rank's finalized stats / reports."""
        arr = (ctypes.c_void_p * len(peer_ptrs))(*[ctypes.c_void_p(int(x)) for x in peer_ptrs])
        check(self._h, self.L.drgpum_gather_peers(self._h, arr, len(peer_ptrs), rank,
                                                  _stream_handle(stream)))

    def bitmap(self, o):
        """Object o's bitmap as a bool numpy array (copies from the device)."""
        lay = self.layout()[o]
        ne = int(self.objects["size"][o] // self.objects["elem_size"][o])
        nw = (ne + 31) // 32
        w0 = int(lay["bitmap_word"])
        words = self.or_words()[w0: w0 + nw].cpu().numpy().view(np.uint32)
        return np.unpackbits(words.view(np.uint8), bitorder="little")[:ne].astype(bool)
