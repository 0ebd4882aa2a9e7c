"""Thin ctypes binding of libblastp.so (include/blastp.h), same names as the C-ABI.

Argument marshalling only: every step of the search runs in the library's
CUDA kernels.  There is no CPU fallback -- if libblastp.so is missing the
import fails (build it with ``python -m paper_conf_ipps_zhangwlf14_b200.build``
or ``__graft_entry__.build()``).

PyTorch is used only for what the C-ABI leaves to the caller: device memory
for the device-side output (``search_ungapped_device``) and CUDA streams.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
# BLASTP_LIB: load another build of the same library (A/B timing of kernel
# revisions); it is still this package's C-ABI, never a fallback.
LIB_PATH = os.environ.get("BLASTP_LIB") or os.path.join(_PKG, "libblastp.so")

OK, E_INVALID_ARG, E_BAD_RESIDUE, E_TOO_LONG, E_NOMEM, E_CUDA, E_CAPACITY = 0, -1, -2, -3, -4, -5, -6
FILTER_LEFT, FILTER_EITHER, FILTER_STATEFUL, FILTER_STATEFUL_RB = 0, 1, 2, 3
EXT_DIAGONAL, EXT_HIT, EXT_WINDOW, EXT_HIT_DEDUP = 0, 1, 2, 3

HSP_DTYPE = np.dtype([("query_id", "<i4"), ("subject_id", "<i4"), ("diagonal", "<i4"),
                      ("q_start", "<i4"), ("s_start", "<i4"), ("length", "<i4"),
                      ("score", "<i4")])
HIT_DTYPE = np.dtype([("query_id", "<i4"), ("subject_id", "<i4"), ("q", "<i4"), ("s", "<i4")])
HSP_BYTES = 28
GAPPED_DTYPE = np.dtype([("query_id", "<i4"), ("subject_id", "<i4"), ("q_start", "<i4"),
                         ("q_end", "<i4"), ("s_start", "<i4"), ("s_end", "<i4"),
                         ("score", "<i4"), ("ident", "<i4"), ("gap_opens", "<i4"),
                         ("gap_len", "<i4")])
GAPPED_BYTES = 40


class BlastpError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        super().__init__(f"{where}: {detail} (status {status})")
        self.status = status


class _CParams(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in
                ("word_len", "threshold", "window", "min_gap", "xdrop", "cutoff", "filter_mode",
                 "ext_mode")]


@dataclass
class Params:
    """blastp_params; defaults = BASELINE.json (w=3, T=11, A=40, X=16 raw, cutoff 41)."""
    word_len: int = 3
    threshold: int = 11
    window: int = 40
    min_gap: int = 3
    xdrop: int = 16
    cutoff: int = 41
    filter_mode: int = FILTER_LEFT
    ext_mode: int = EXT_DIAGONAL  # Alg. 3 coverage chain; EXT_HIT = Alg. 4

    def c(self) -> _CParams:
        return _CParams(self.word_len, self.threshold, self.window, self.min_gap, self.xdrop,
                        self.cutoff, self.filter_mode, self.ext_mode)


class _CGappedParams(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in ("gap_open", "gap_extend", "xdrop", "cutoff")]


@dataclass
class GappedParams:
    """blastp_gapped_params (R18-R21): BLASTP defaults, gap cost 11 + 1 per
    residue, gapped X-drop 38 raw (15 bits at lambda 0.267), cutoff 41."""
    gap_open: int = 11
    gap_extend: int = 1
    xdrop: int = 38
    cutoff: int = 41

    def c(self) -> _CGappedParams:
        return _CGappedParams(self.gap_open, self.gap_extend, self.xdrop, self.cutoff)


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build the CUDA library first "
                          "(python -m paper_conf_ipps_zhangwlf14_b200.build)")
    L = ctypes.CDLL(LIB_PATH)
    vp, i32, i64, P = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.POINTER
    L.blastp_params_default.argtypes = [P(_CParams)]
    L.blastp_params_default.restype = None
    L.blastp_strerror.argtypes = [ctypes.c_int]
    L.blastp_strerror.restype = ctypes.c_char_p
    L.blastp_last_error.argtypes = []
    L.blastp_last_error.restype = ctypes.c_char_p
    L.blastp_version.argtypes = []
    L.blastp_version.restype = ctypes.c_char_p
    L.blastp_build_query_table.argtypes = [ctypes.c_char_p, i32, P(_CParams), ctypes.c_int, vp, P(vp)]
    L.blastp_build_query_batch.argtypes = [P(ctypes.c_char_p), P(i32), i32, P(_CParams),
                                           ctypes.c_int, vp, P(vp)]
    L.blastp_pack_db.argtypes = [vp, vp, i64, i32, i32, ctypes.c_int, vp, P(vp)]
    L.blastp_shard_range.argtypes = [vp, i64, i32, i32, P(i64), P(i64)]
    L.blastp_db_info.argtypes = [vp, P(i64), P(i64), P(i64), P(i64), P(i64)]
    if hasattr(L, "blastp_db_long_info"):  # absent in builds older than the long-item plan
        L.blastp_db_long_info.argtypes = [vp, P(i64), P(i64), P(i64)]
    L.blastp_query_table_info.argtypes = [vp, P(i32), P(i64)]
    if hasattr(L, "blastp_query_table_groups"):
        L.blastp_query_table_groups.argtypes = [vp, P(i32), P(i32), P(i32)]
    L.blastp_search_ungapped.argtypes = [vp, vp, P(_CParams), vp, P(vp), P(i64)]
    L.blastp_search_ungapped_device.argtypes = [vp, vp, P(_CParams), vp, vp, i64, vp]
    if hasattr(L, "blastp_search_host_db"):  # absent in older builds (A/B timing)
        L.blastp_search_host_db.argtypes = [vp, vp, vp, i64, i32, i32, P(_CParams), i32, vp, vp,
                                            i64, vp]
    if hasattr(L, "blastp_format_host_db"):  # absent in older builds (A/B timing)
        L.blastp_format_host_db.argtypes = [vp, vp, i64, i32, i32, i32, ctypes.c_int, vp, P(vp)]
        L.blastp_search_formatted_db.argtypes = [vp, vp, P(_CParams), vp, vp, i64, vp]
        L.blastp_host_db_info.argtypes = [vp, P(i64), P(i64), P(i64), P(i32), P(i64)]
        L.blastp_host_db_free.argtypes = [vp]
        L.blastp_host_db_free.restype = None
    L.blastp_sort_hsps_device.argtypes = [vp, i64, vp]
    L.blastp_unique_hsps_device.argtypes = [vp, i64, vp, vp]
    if hasattr(L, "blastp_dedup_covered_device"):  # absent in older builds (A/B timing)
        L.blastp_dedup_covered_device.argtypes = [vp, i64, i32, vp, vp]
    L.blastp_debug_trace.argtypes = [vp, vp, P(_CParams), vp, vp, i64, P(i64), vp, i64, P(i64),
                                     vp, i64, P(i64)]
    L.blastp_debug_hits.argtypes = [vp, vp, P(_CParams), vp, vp, i64, P(i64)]
    L.blastp_debug_passing.argtypes = [vp, vp, P(_CParams), vp, vp, i64, P(i64)]
    L.blastp_debug_stats.argtypes = [vp, vp, P(_CParams), vp, vp, i32]
    if hasattr(L, "blastp_search_ungapped_append"):  # absent in older builds (A/B timing)
        L.blastp_search_ungapped_append.argtypes = [vp, vp, P(_CParams), vp, vp, i64, vp]
        L.blastp_ipc_alloc.argtypes = [ctypes.c_int, i64, P(vp), vp]
        L.blastp_ipc_open.argtypes = [ctypes.c_int, vp, P(vp)]
        L.blastp_ipc_close.argtypes = [vp]
        L.blastp_ipc_free.argtypes = [vp]
    if hasattr(L, "blastp_trim_memory"):
        L.blastp_trim_memory.argtypes = [ctypes.c_int]
    if hasattr(L, "blastp_debug_alu_peak"):  # absent in older builds (A/B timing)
        L.blastp_debug_alu_peak.argtypes = [ctypes.c_int, P(ctypes.c_double)]
    if hasattr(L, "blastp_gapped_extend_device"):  # absent in older builds (A/B timing)
        L.blastp_gapped_params_default.argtypes = [P(_CGappedParams)]
        L.blastp_gapped_params_default.restype = None
        L.blastp_gapped_extend_device.argtypes = [vp, vp, vp, i64, P(_CGappedParams), vp, vp, i64,
                                                  P(i64)]
        L.blastp_search_gapped.argtypes = [vp, vp, P(_CParams), P(_CGappedParams), vp, P(vp),
                                           P(i64), P(vp), P(i64)]
        L.blastp_gapped_free.argtypes = [vp]
        L.blastp_gapped_free.restype = None
    for f in ("blastp_hsp_free", "blastp_query_table_free", "blastp_db_free"):
        getattr(L, f).argtypes = [vp]
        getattr(L, f).restype = None
    return L


lib = _load()

EXPORTED = ["blastp_params_default", "blastp_strerror", "blastp_last_error", "blastp_version",
            "blastp_build_query_table", "blastp_build_query_batch", "blastp_pack_db",
            "blastp_shard_range", "blastp_db_info", "blastp_db_long_info", "blastp_query_table_info",
            "blastp_query_table_groups",
            "blastp_search_ungapped", "blastp_search_ungapped_device", "blastp_search_ungapped_append",
            "blastp_ipc_alloc", "blastp_ipc_open", "blastp_ipc_close", "blastp_ipc_free",
            "blastp_search_host_db",
            "blastp_format_host_db", "blastp_search_formatted_db", "blastp_host_db_info",
            "blastp_host_db_free",
            "blastp_sort_hsps_device", "blastp_unique_hsps_device", "blastp_dedup_covered_device",
            "blastp_debug_trace", "blastp_debug_hits", "blastp_debug_passing", "blastp_debug_stats",
            "blastp_debug_alu_peak", "blastp_trim_memory",
            "blastp_gapped_params_default", "blastp_gapped_extend_device", "blastp_search_gapped",
            "blastp_gapped_free",
            "blastp_hsp_free", "blastp_query_table_free", "blastp_db_free"]


def _check(rc: int, where: str):
    if rc != OK:
        raise BlastpError(rc, where, lib.blastp_last_error().decode(errors="replace") or
                          lib.blastp_strerror(rc).decode())


def _stream_handle(stream) -> int | None:
    if stream is None:
        try:
            import torch
            if torch.cuda.is_available():
                return torch.cuda.current_stream().cuda_stream or None
        except ImportError:
            pass
        return None
    if isinstance(stream, int):
        return stream or None
    return getattr(stream, "cuda_stream", None) or None


def version() -> str:
    return lib.blastp_version().decode()


def params_default() -> Params:
    c = _CParams()
    lib.blastp_params_default(ctypes.byref(c))
    return Params(*(getattr(c, f) for f, _ in _CParams._fields_))


def _as_bytes(q) -> bytes:
    return q.encode() if isinstance(q, str) else bytes(q)


class QueryTable:
    """blastp_query_table handle (one or more queries, query_id = index)."""

    def __init__(self, queries, params: Params | None = None, device: int = 0, stream=None):
        self.params = params or Params()
        qs = [queries] if isinstance(queries, (str, bytes, bytearray)) else list(queries)
        bufs = [_as_bytes(q) for q in qs]
        arr = (ctypes.c_char_p * len(bufs))(*bufs)
        lens = (ctypes.c_int32 * len(bufs))(*[len(b) for b in bufs])
        h = ctypes.c_void_p()
        c = self.params.c()
        _check(lib.blastp_build_query_batch(arr, lens, len(bufs), ctypes.byref(c), device,
                                            _stream_handle(stream), ctypes.byref(h)),
               "blastp_build_query_batch")
        self.handle = h
        self.device = device
        self.lengths = [len(b) for b in bufs]

    @property
    def num_queries(self) -> int:
        n = ctypes.c_int32()
        e = ctypes.c_int64()
        _check(lib.blastp_query_table_info(self.handle, ctypes.byref(n), ctypes.byref(e)),
               "blastp_query_table_info")
        return n.value

    @property
    def groups(self) -> tuple[int, int, int]:
        """(query groups, queries searched alone, sentinel gap) of a batch table."""
        g, a, gap = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
        _check(lib.blastp_query_table_groups(self.handle, ctypes.byref(g), ctypes.byref(a),
                                             ctypes.byref(gap)), "blastp_query_table_groups")
        return g.value, a.value, gap.value

    def launches(self, params: Params | None = None) -> int:
        """Search kernels per shard for a search with `params` (groups when the window fits)."""
        g, a, gap = self.groups
        p = params or self.params
        return g + a if g and p.window + 8 <= gap else self.num_queries

    @property
    def entries(self) -> int:
        n = ctypes.c_int32()
        e = ctypes.c_int64()
        _check(lib.blastp_query_table_info(self.handle, ctypes.byref(n), ctypes.byref(e)),
               "blastp_query_table_info")
        return e.value

    def free(self):
        # lib is None during interpreter shutdown (module globals cleared)
        if getattr(self, "handle", None) and lib is not None:
            lib.blastp_query_table_free(self.handle)
            self.handle = None

    __del__ = free


def build_query_table(query, params: Params | None = None, device: int = 0, stream=None):
    return QueryTable(query, params, device, stream)


def build_query_batch(queries, params: Params | None = None, device: int = 0, stream=None):
    return QueryTable(list(queries), params, device, stream)


def shard_range(offsets: np.ndarray, shard_index: int, num_shards: int) -> tuple[int, int]:
    """Host-only: residue-balanced contiguous subject range of a shard."""
    off = np.ascontiguousarray(offsets, dtype=np.int64)
    lo, hi = ctypes.c_int64(), ctypes.c_int64()
    _check(lib.blastp_shard_range(off.ctypes.data, len(off) - 1, shard_index, num_shards,
                                  ctypes.byref(lo), ctypes.byref(hi)), "blastp_shard_range")
    return lo.value, hi.value


class Database:
    """blastp_db handle: one shard of a database, packed on the GPU."""

    def __init__(self, residues: np.ndarray | bytes, offsets: np.ndarray, shard_index: int = 0,
                 num_shards: int = 1, device: int = 0, stream=None):
        if isinstance(residues, (bytes, bytearray)):
            residues = np.frombuffer(residues, dtype=np.uint8)
        res = residues if residues.flags["C_CONTIGUOUS"] else np.ascontiguousarray(residues)
        off = np.ascontiguousarray(offsets, dtype=np.int64)
        h = ctypes.c_void_p()
        ptr = res.ctypes.data if hasattr(res, "ctypes") else res.data_ptr()
        _check(lib.blastp_pack_db(ptr, off.ctypes.data, len(off) - 1, shard_index, num_shards,
                                  device, _stream_handle(stream), ctypes.byref(h)),
               "blastp_pack_db")
        self.handle = h
        self.device = device
        self._info()

    @classmethod
    def from_pinned(cls, residues_ptr: int, offsets: np.ndarray, shard_index=0, num_shards=1,
                    device=0, stream=None):
        """Pack from a raw host pointer (e.g. a pinned torch tensor's data_ptr())."""
        self = cls.__new__(cls)
        off = np.ascontiguousarray(offsets, dtype=np.int64)
        h = ctypes.c_void_p()
        _check(lib.blastp_pack_db(residues_ptr, off.ctypes.data, len(off) - 1, shard_index,
                                  num_shards, device, _stream_handle(stream), ctypes.byref(h)),
               "blastp_pack_db")
        self.handle = h
        self.device = device
        self._info()
        return self

    def _info(self):
        vals = [ctypes.c_int64() for _ in range(5)]
        _check(lib.blastp_db_info(self.handle, *[ctypes.byref(v) for v in vals]), "blastp_db_info")
        self.nseq, self.residues, self.subject_base, self.stream_bytes, self.num_chunks = \
            (v.value for v in vals)
        self.long_items = self.segments = self.segment_len = None
        if hasattr(lib, "blastp_db_long_info"):
            vals = [ctypes.c_int64() for _ in range(3)]
            _check(lib.blastp_db_long_info(self.handle, *[ctypes.byref(v) for v in vals]),
                   "blastp_db_long_info")
            self.long_items, self.segments, self.segment_len = (v.value for v in vals)

    def free(self):
        if getattr(self, "handle", None) and lib is not None:
            lib.blastp_db_free(self.handle)
            self.handle = None

    __del__ = free


def pack_db(residues, offsets, shard_index=0, num_shards=1, device=0, stream=None) -> Database:
    return Database(residues, offsets, shard_index, num_shards, device, stream)


def search_ungapped(table: QueryTable, db: Database, params: Params | None = None,
                    stream=None) -> np.ndarray:
    """Host variant: canonical-order HSP array (HSP_DTYPE)."""
    c = (params or table.params).c()
    out = ctypes.c_void_p()
    n = ctypes.c_int64()
    _check(lib.blastp_search_ungapped(table.handle, db.handle, ctypes.byref(c),
                                      _stream_handle(stream), ctypes.byref(out), ctypes.byref(n)),
           "blastp_search_ungapped")
    try:
        if n.value == 0:
            return np.zeros(0, dtype=HSP_DTYPE)
        buf = (ctypes.c_char * (n.value * HSP_BYTES)).from_address(out.value)
        return np.frombuffer(bytes(buf), dtype=HSP_DTYPE).copy()
    finally:
        lib.blastp_hsp_free(out)


def search_ungapped_device(table: QueryTable, db: Database, out_ptr: int, capacity: int,
                           count_ptr: int, params: Params | None = None, stream=None):
    """Device variant (async): HSPs appended to device memory at out_ptr
    (capacity records of 28 B), total count written to the int64 at count_ptr."""
    c = (params or table.params).c()
    _check(lib.blastp_search_ungapped_device(table.handle, db.handle, ctypes.byref(c),
                                             _stream_handle(stream), out_ptr, capacity,
                                             count_ptr), "blastp_search_ungapped_device")


def search_ungapped_append(table: QueryTable, db: Database, out_ptr: int, capacity: int,
                           count_ptr: int, params: Params | None = None, stream=None):
    """Append variant (async; blastp_search_ungapped_append): the count at
    count_ptr is not reset, HSPs take the next indices of it; out_ptr /
    count_ptr may be another GPU's buffer mapped with ipc_open (the kernel
    stores its HSPs there over NVLink)."""
    c = (params or table.params).c()
    _check(lib.blastp_search_ungapped_append(table.handle, db.handle, ctypes.byref(c),
                                             _stream_handle(stream), out_ptr, capacity,
                                             count_ptr), "blastp_search_ungapped_append")


def gapped_extend_device(table: QueryTable, db: Database, hsps_ptr: int, n: int, out_ptr: int,
                         capacity: int, gparams: GappedParams | None = None, stream=None) -> int:
    """Gapped extension (blastp_gapped_extend_device, synchronous) of n device
    HSPs of this shard in canonical order at hsps_ptr; alignments written to
    out_ptr (capacity records of 40 B).  Returns their count."""
    g = (gparams or GappedParams()).c()
    cnt = ctypes.c_int64()
    _check(lib.blastp_gapped_extend_device(table.handle, db.handle, hsps_ptr, n, ctypes.byref(g),
                                           _stream_handle(stream), out_ptr, capacity,
                                           ctypes.byref(cnt)), "blastp_gapped_extend_device")
    return int(cnt.value)


def search_gapped(table: QueryTable, db: Database, params: Params | None = None,
                  gparams: GappedParams | None = None, stream=None, want_ungapped: bool = False):
    """Ungapped search + gapped extension on the GPU (blastp_search_gapped):
    GAPPED_DTYPE array in canonical order (and the canonical ungapped list if
    want_ungapped)."""
    c = (params or table.params).c()
    g = (gparams or GappedParams()).c()
    out, n = ctypes.c_void_p(), ctypes.c_int64()
    uout, un = ctypes.c_void_p(), ctypes.c_int64()
    _check(lib.blastp_search_gapped(table.handle, db.handle, ctypes.byref(c), ctypes.byref(g),
                                    _stream_handle(stream), ctypes.byref(out), ctypes.byref(n),
                                    ctypes.byref(uout) if want_ungapped else None,
                                    ctypes.byref(un) if want_ungapped else None),
           "blastp_search_gapped")
    try:
        res = np.zeros(0, dtype=GAPPED_DTYPE)
        if n.value:
            buf = (ctypes.c_char * (n.value * GAPPED_BYTES)).from_address(out.value)
            res = np.frombuffer(bytes(buf), dtype=GAPPED_DTYPE).copy()
        if not want_ungapped:
            return res
        u = np.zeros(0, dtype=HSP_DTYPE)
        if un.value:
            buf = (ctypes.c_char * (un.value * HSP_BYTES)).from_address(uout.value)
            u = np.frombuffer(bytes(buf), dtype=HSP_DTYPE).copy()
        return res, u
    finally:
        lib.blastp_gapped_free(out)
        if want_ungapped:
            lib.blastp_hsp_free(uout)


IPC_HANDLE_BYTES = 64


def ipc_alloc(device: int, nbytes: int) -> tuple[int, bytes]:
    """(device pointer, IPC handle) of a new exported buffer (blastp_ipc_alloc)."""
    ptr = ctypes.c_void_p()
    h = ctypes.create_string_buffer(IPC_HANDLE_BYTES)
    _check(lib.blastp_ipc_alloc(device, nbytes, ctypes.byref(ptr), h), "blastp_ipc_alloc")
    return int(ptr.value), h.raw


def ipc_open(device: int, handle: bytes) -> int:
    """Map another process's exported buffer (blastp_ipc_open); its pointer."""
    ptr = ctypes.c_void_p()
    h = ctypes.create_string_buffer(bytes(handle), IPC_HANDLE_BYTES)
    _check(lib.blastp_ipc_open(device, h, ctypes.byref(ptr)), "blastp_ipc_open")
    return int(ptr.value)


def ipc_close(ptr: int):
    _check(lib.blastp_ipc_close(ptr), "blastp_ipc_close")


def ipc_free(ptr: int):
    _check(lib.blastp_ipc_free(ptr), "blastp_ipc_free")


def search_host_db(table: QueryTable, residues, offsets: np.ndarray, out_ptr: int, capacity: int,
                   count_ptr: int, params: Params | None = None, shard_index: int = 0,
                   num_shards: int = 1, num_parts: int = 0, stream=None):
    """Pipelined search of a host-resident shard (blastp_search_host_db): parts
    are copied host->device while the previous part is searched.  `residues`:
    a numpy uint8 array / bytes, or an int host pointer (e.g. a pinned tensor's
    data_ptr() minus offsets[0]).  HSPs appended at out_ptr (device), total
    count written to the int64 at count_ptr; asynchronous on `stream`."""
    off = np.ascontiguousarray(offsets, dtype=np.int64)
    if isinstance(residues, int):
        ptr, keep = residues, None
    else:
        keep = np.frombuffer(residues, dtype=np.uint8) if isinstance(residues, (bytes, bytearray)) \
            else np.ascontiguousarray(residues)
        ptr = keep.ctypes.data
    c = (params or table.params).c()
    _check(lib.blastp_search_host_db(table.handle, ptr, off.ctypes.data, len(off) - 1, shard_index,
                                     num_shards, ctypes.byref(c), num_parts,
                                     _stream_handle(stream), out_ptr, capacity, count_ptr),
           "blastp_search_host_db")
    return keep


class HostDb:
    """A shard formatted into pinned host memory (blastp_format_host_db)."""

    def __init__(self, handle):
        self.handle = handle
        vals = [ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int32(),
                ctypes.c_int64()]
        _check(lib.blastp_host_db_info(handle, *[ctypes.byref(v) for v in vals]),
               "blastp_host_db_info")
        self.nseq, self.residues, self.subject_base, self.num_parts, self.host_bytes = \
            (v.value for v in vals)

    def free(self):
        if self.handle:
            lib.blastp_host_db_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def format_host_db(residues, offsets: np.ndarray, shard_index: int = 0, num_shards: int = 1,
                   num_parts: int = 0, device: int = 0, stream=None) -> HostDb:
    """Pack a shard once into ready-to-stream parts in pinned host memory."""
    off = np.ascontiguousarray(offsets, dtype=np.int64)
    if isinstance(residues, int):
        ptr = residues
    else:
        keep = np.frombuffer(residues, dtype=np.uint8) if isinstance(residues, (bytes, bytearray)) \
            else np.ascontiguousarray(residues)
        ptr = keep.ctypes.data
    h = ctypes.c_void_p()
    _check(lib.blastp_format_host_db(ptr, off.ctypes.data, len(off) - 1, shard_index, num_shards,
                                     num_parts, device, _stream_handle(stream), ctypes.byref(h)),
           "blastp_format_host_db")
    return HostDb(h.value)


def search_formatted_db(table: QueryTable, hdb: HostDb, out_ptr: int, capacity: int,
                        count_ptr: int, params: Params | None = None, stream=None):
    """Stream a formatted host shard through the search (blastp_search_formatted_db):
    HSPs appended at out_ptr (device), count at count_ptr; asynchronous."""
    c = (params or table.params).c()
    _check(lib.blastp_search_formatted_db(table.handle, hdb.handle, ctypes.byref(c),
                                          _stream_handle(stream), out_ptr, capacity, count_ptr),
           "blastp_search_formatted_db")


def sort_hsps_device(ptr: int, n: int, stream=None):
    _check(lib.blastp_sort_hsps_device(ptr, n, _stream_handle(stream)), "blastp_sort_hsps_device")


def unique_hsps_device(ptr: int, n: int, count_ptr: int, stream=None):
    """Collapse duplicates of a canonically sorted device HSP list in place;
    the new count is written to the device int64 at count_ptr."""
    _check(lib.blastp_unique_hsps_device(ptr, n, count_ptr, _stream_handle(stream)),
           "blastp_unique_hsps_device")


def dedup_covered_device(ptr: int, n: int, cutoff: int, count_ptr: int, stream=None):
    """ext_mode HIT_DEDUP's de-duplication step on device seed records (R17):
    the kept HSPs (canonical order) replace the records; the count is written
    to the device int64 at count_ptr."""
    _check(lib.blastp_dedup_covered_device(ptr, n, cutoff, count_ptr, _stream_handle(stream)),
           "blastp_dedup_covered_device")


STAT_NAMES = ["windows", "rounds", "conflict_rounds", "hits", "passing", "enqueued", "flushes",
              "extended", "accepted", "emitted", "xdrop_residues", "xdrop_lane_slots"]


def debug_stats(table: QueryTable, db: Database, params: Params | None = None,
                stream=None) -> dict:
    """Event counters of a traced search (see blastp_debug_stats)."""
    c = (params or table.params).c()
    buf = (ctypes.c_int64 * len(STAT_NAMES))()
    _check(lib.blastp_debug_stats(table.handle, db.handle, ctypes.byref(c),
                                  _stream_handle(stream), buf, len(STAT_NAMES)),
           "blastp_debug_stats")
    return dict(zip(STAT_NAMES, list(buf)))


def trim_memory(device: int = 0):
    """Return the library pool's unused device memory (blastp_trim_memory)."""
    _check(lib.blastp_trim_memory(device), "blastp_trim_memory")


def debug_alu_peak(device: int = 0) -> float:
    """Measured integer-ALU roof of the device, lane operations per second."""
    v = ctypes.c_double()
    _check(lib.blastp_debug_alu_peak(device, ctypes.byref(v)), "blastp_debug_alu_peak")
    return v.value


@dataclass
class Trace:
    hits: np.ndarray
    passing: np.ndarray
    extensions: np.ndarray


def debug_trace(table: QueryTable, db: Database, params: Params | None = None, stream=None,
                hits_cap: int = 1 << 20, passing_cap: int = 1 << 18,
                exts_cap: int = 1 << 18) -> Trace:
    """Every hit, passing hit and extension of a search (unordered)."""
    c = (params or table.params).c()
    for _ in range(3):
        hb = np.zeros(max(hits_cap, 1), dtype=HIT_DTYPE)
        pb = np.zeros(max(passing_cap, 1), dtype=HIT_DTYPE)
        eb = np.zeros(max(exts_cap, 1), dtype=HSP_DTYPE)
        nh, np_, ne = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        rc = lib.blastp_debug_trace(table.handle, db.handle, ctypes.byref(c),
                                    _stream_handle(stream), hb.ctypes.data, hits_cap,
                                    ctypes.byref(nh), pb.ctypes.data, passing_cap,
                                    ctypes.byref(np_), eb.ctypes.data, exts_cap, ctypes.byref(ne))
        if rc == E_CAPACITY:
            hits_cap = max(hits_cap, nh.value)
            passing_cap = max(passing_cap, np_.value)
            exts_cap = max(exts_cap, ne.value)
            continue
        _check(rc, "blastp_debug_trace")
        return Trace(hb[:nh.value].copy(), pb[:np_.value].copy(), eb[:ne.value].copy())
    raise BlastpError(E_CAPACITY, "blastp_debug_trace", "capacity retries exhausted")
