"""ctypes binding of oracle.c -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Argument marshalling only; every step of the oracle runs in oracle.c.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")

ALPHABET = "ARNDCQEGHILKMFPSTWYVBZX*"
NA = 24

HSP_DTYPE = np.dtype([("query_id", "<i4"), ("subject_id", "<i4"), ("diagonal", "<i4"),
                      ("q_start", "<i4"), ("s_start", "<i4"), ("length", "<i4"),
                      ("score", "<i4")])


_SRC_GAPPED = os.path.join(_HERE, "gapped.c")


def build(force: bool = False) -> str:
    """Compile oracle.c + gapped.c into liboracle.so (plain gcc, no CUDA)."""
    deps = [_SRC, _SRC_GAPPED, os.path.join(_HERE, "oracle.h")]
    if (not force and os.path.exists(_LIB_PATH)
            and os.path.getmtime(_LIB_PATH) >= max(os.path.getmtime(d) for d in deps)):
        return _LIB_PATH
    tmp = _LIB_PATH + f".tmp{os.getpid()}"
    subprocess.check_call(["gcc", "-O2", "-std=c99", "-Wall", "-Wextra", "-shared", "-fPIC",
                           "-pthread", _SRC, _SRC_GAPPED, "-o", tmp])
    os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


class _Params(ctypes.Structure):
    _fields_ = [("word_len", ctypes.c_int32), ("threshold", ctypes.c_int32),
                ("window", ctypes.c_int32), ("min_gap", ctypes.c_int32),
                ("xdrop", ctypes.c_int32), ("cutoff", ctypes.c_int32),
                ("filter_mode", ctypes.c_int32), ("ext_mode", ctypes.c_int32)]


class _HitList(ctypes.Structure):
    _fields_ = [("cap", ctypes.c_int64), ("count", ctypes.c_int64),
                ("subject", ctypes.c_void_p), ("q", ctypes.c_void_p), ("s", ctypes.c_void_p)]


@dataclass
class Params:
    """R3/R6/R8-R10 parameters (defaults = BASELINE.json configs)."""
    word_len: int = 3
    threshold: int = 11
    window: int = 40
    min_gap: int = 3
    xdrop: int = 16
    cutoff: int = 41
    filter_mode: int = 0  # 0 LEFT, 1 EITHER, 2 STATEFUL (Alg. 1 lasthit walk, R15),
    #                       3 STATEFUL + Alg. 1 L13's reach-back (R16)
    ext_mode: int = 0  # 0 DIAGONAL (Alg. 3 coverage chain), 1 HIT (Alg. 4)

    def _c(self) -> _Params:
        return _Params(self.word_len, self.threshold, self.window, self.min_gap, self.xdrop,
                       self.cutoff, self.filter_mode, self.ext_mode)


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        L = _lib
        L.oracle_encode.restype = ctypes.c_int64
        L.oracle_encode.argtypes = [ctypes.c_char_p, ctypes.c_int64, ctypes.c_void_p]
        L.oracle_neighbourhood.restype = ctypes.c_int64
        L.oracle_neighbourhood.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p,
                                           ctypes.c_int32, ctypes.c_int32, ctypes.c_int32,
                                           ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64]
        L.oracle_xdrop_pairs.restype = None
        L.oracle_xdrop_pairs.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32,
                                         ctypes.c_int32, ctypes.c_void_p, ctypes.c_int32,
                                         ctypes.c_int32, ctypes.POINTER(ctypes.c_int32),
                                         ctypes.POINTER(ctypes.c_int32),
                                         ctypes.POINTER(ctypes.c_int32)]
        L.oracle_two_hit.restype = None
        L.oracle_two_hit.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32,
                                     ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p]
        L.oracle_two_hit_stateful_rb.restype = None
        L.oracle_two_hit_stateful_rb.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p,
                                                 ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32,
                                                 ctypes.c_void_p]
        L.oracle_two_hit_stateful.restype = None
        L.oracle_two_hit_stateful.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p,
                                              ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p]
        L.oracle_gapped_dir.restype = ctypes.c_int32
        L.oracle_gapped_dir.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p,
                                        ctypes.c_int32, ctypes.c_void_p, ctypes.c_int32,
                                        ctypes.c_int32, ctypes.c_int32, ctypes.c_int32] + \
            [ctypes.POINTER(ctypes.c_int32)] * 5
        L.oracle_gapped_hsps.restype = ctypes.c_int64
        L.oracle_gapped_hsps.argtypes = [
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32,  # queries, qlens, nq
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64,  # db, off, nseq, base
            ctypes.c_void_p, ctypes.c_int64,  # hsps, n
            ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32,
            ctypes.c_int32,  # matrix, na, gap_open, gap_extend, xdrop, cutoff
            ctypes.c_void_p, ctypes.c_int64]
        L.oracle_search.restype = ctypes.c_int64
        L.oracle_search.argtypes = [
            ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32,  # query, lq, qid
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64,  # db, off, nseq, base
            ctypes.c_void_p, ctypes.c_int32, ctypes.POINTER(_Params),  # matrix, na, params
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32,  # table off/pos, nthreads
            ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64,  # out, cap, ext, cap
            ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(_HitList), ctypes.POINTER(_HitList)]
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def blosum62() -> np.ndarray:
    """The oracle's BLOSUM62 (24x24 int32), read from the compiled library."""
    arr = (ctypes.c_int32 * (NA * NA)).in_dll(lib(), "ORACLE_BLOSUM62")
    return np.array(arr, dtype=np.int32).reshape(NA, NA)


def alphabet() -> str:
    return bytes((ctypes.c_char * (NA + 1)).in_dll(lib(), "ORACLE_ALPHABET"))[:NA].decode()


def encode(seq: str | bytes) -> np.ndarray:
    """R1 encoding; raises ValueError on an invalid residue."""
    b = seq.encode() if isinstance(seq, str) else bytes(seq)
    out = np.zeros(len(b), dtype=np.uint8)
    r = lib().oracle_encode(b, len(b), _ptr(out))
    if r < 0:
        raise ValueError(f"invalid residue at index {-r - 1}: {b[-r - 1:-r]!r}")
    return out


def neighbourhood(query: np.ndarray, matrix: np.ndarray, T: int, word_len: int = 3):
    """R3 brute-force neighbourhood table (CSR: off[na^w+1], pos[])."""
    q = np.ascontiguousarray(query, dtype=np.uint8)
    m = np.ascontiguousarray(matrix, dtype=np.int32)
    na = m.shape[0]
    off = np.zeros(na ** word_len + 1, dtype=np.int64)
    total = lib().oracle_neighbourhood(_ptr(q), len(q), _ptr(m), na, word_len, T, _ptr(off),
                                       None, 0)
    pos = np.zeros(max(total, 1), dtype=np.int32)
    lib().oracle_neighbourhood(_ptr(q), len(q), _ptr(m), na, word_len, T, _ptr(off), _ptr(pos),
                               total)
    return off, pos[:total]


def xdrop_pairs(a: np.ndarray, b: np.ndarray, matrix: np.ndarray, X: int, step: int = 1,
                start: int = 0, n: int | None = None):
    """R8 X-drop over pairs (a[start+k*step], b[start+k*step]); returns (best, len, steps)."""
    a = np.ascontiguousarray(a, dtype=np.uint8)
    b = np.ascontiguousarray(b, dtype=np.uint8)
    m = np.ascontiguousarray(matrix, dtype=np.int32)
    if n is None:
        n = (len(a) - start) if step > 0 else start + 1
    best, ln, steps = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
    pa = ctypes.c_void_p(a.ctypes.data + start)
    pb = ctypes.c_void_p(b.ctypes.data + start)
    lib().oracle_xdrop_pairs(pa, pb, n, step, _ptr(m), m.shape[0], X, ctypes.byref(best),
                             ctypes.byref(ln), ctypes.byref(steps))
    return best.value, ln.value, steps.value


def two_hit(s, min_gap: int = 3, window: int = 40, mode: int = 0) -> np.ndarray:
    s = np.ascontiguousarray(s, dtype=np.int32)
    out = np.zeros(len(s), dtype=np.uint8)
    lib().oracle_two_hit(_ptr(s), len(s), min_gap, window, mode, _ptr(out))
    return out.astype(bool)


def two_hit_stateful(s, ext_end, min_gap: int = 3, window: int = 40) -> np.ndarray:
    """Alg. 1 L8-19 walk (R15): which hits of one diagonal are extended, given the
    subject end of the extension from each hit."""
    s = np.ascontiguousarray(s, dtype=np.int32)
    e = np.ascontiguousarray(ext_end, dtype=np.int32)
    assert len(e) == len(s)
    out = np.zeros(len(s), dtype=np.uint8)
    lib().oracle_two_hit_stateful(_ptr(s), len(s), _ptr(e), min_gap, window, _ptr(out))
    return out.astype(bool)


def two_hit_stateful_rb(s, ext_start, ext_end, min_gap: int = 3, window: int = 40) -> np.ndarray:
    """Alg. 1 L8-19 walk with L13's reach-back (R16): an extension is kept only
    if its subject start is at or before the lasthit it was triggered by."""
    s = np.ascontiguousarray(s, dtype=np.int32)
    a = np.ascontiguousarray(ext_start, dtype=np.int32)
    e = np.ascontiguousarray(ext_end, dtype=np.int32)
    assert len(a) == len(e) == len(s)
    out = np.zeros(len(s), dtype=np.uint8)
    lib().oracle_two_hit_stateful_rb(_ptr(s), len(s), _ptr(a), _ptr(e), min_gap, window,
                                     _ptr(out))
    return out.astype(bool)


@dataclass
class SearchResult:
    hsps: np.ndarray            # HSP_DTYPE, canonical order, score >= cutoff
    extensions: np.ndarray      # every extension performed (HSP_DTYPE)
    hits: np.ndarray | None     # (subject, q, s) int32 [n,3] if requested
    passing: np.ndarray | None  # (subject, q, s) passing hits if requested


def search(query: np.ndarray, db: np.ndarray, offsets: np.ndarray, params: Params | None = None,
           *, query_id: int = 0, subject_base: int = 0, matrix: np.ndarray | None = None,
           table=None, nthreads: int = 1, want_hits: bool = False,
           want_extensions: bool = True, cap_hint: int = 0) -> SearchResult:
    """Oracle search of one query (codes) against db codes with offsets[nseq+1]."""
    p = params or Params()
    q = np.ascontiguousarray(query, dtype=np.uint8)
    d = np.ascontiguousarray(db, dtype=np.uint8)
    off = np.ascontiguousarray(offsets, dtype=np.int64)
    m = np.ascontiguousarray(blosum62() if matrix is None else matrix, dtype=np.int32)
    nseq = len(off) - 1
    cp = p._c()
    t_off = t_pos = None
    if table is not None:
        t_off = np.ascontiguousarray(table[0], dtype=np.int64)
        t_pos = np.ascontiguousarray(table[1], dtype=np.int32)
    hl = ps = None
    hbufs = []
    cap_h = 0
    if want_hits:
        cap_h = 1 << 16
    for attempt in range(8):
        if want_hits:
            hbufs = [np.zeros(cap_h, dtype=np.int32) for _ in range(6)]
            hl = _HitList(cap_h, 0, hbufs[0].ctypes.data, hbufs[1].ctypes.data, hbufs[2].ctypes.data)
            ps = _HitList(cap_h, 0, hbufs[3].ctypes.data, hbufs[4].ctypes.data, hbufs[5].ctypes.data)
        cap = max(1 << 12, int(cap_hint))  # output buffer size only (a rerun if too small)
        for _ in range(8):
            out = np.zeros(cap, dtype=HSP_DTYPE)
            ext = np.zeros(cap * 8 if want_extensions else 1, dtype=HSP_DTYPE)
            ext_n = ctypes.c_int64(0)
            n = lib().oracle_search(_ptr(q), len(q), query_id, _ptr(d), _ptr(off), nseq,
                                    subject_base, _ptr(m), m.shape[0], ctypes.byref(cp),
                                    None if t_off is None else _ptr(t_off),
                                    None if t_pos is None else _ptr(t_pos), nthreads,
                                    _ptr(out), cap, _ptr(ext) if want_extensions else None,
                                    len(ext) if want_extensions else 0, ctypes.byref(ext_n),
                                    ctypes.byref(hl) if hl is not None else None,
                                    ctypes.byref(ps) if ps is not None else None)
            if n < 0:
                raise RuntimeError(f"oracle_search failed ({n})")
            if n <= cap and (not want_extensions or ext_n.value <= len(ext)):
                break
            cap = max(int(n), int(ext_n.value) // 8 + 1, cap) * 2
        if want_hits and (hl.count > cap_h or ps.count > cap_h):
            cap_h = int(max(hl.count, ps.count)) + 1
            continue
        break
    hits = passing = None
    if want_hits:
        hits = np.stack([hbufs[0][:hl.count], hbufs[1][:hl.count], hbufs[2][:hl.count]], axis=1)
        passing = np.stack([hbufs[3][:ps.count], hbufs[4][:ps.count], hbufs[5][:ps.count]], axis=1)
    exts = ext[:ext_n.value].copy() if want_extensions else np.zeros(0, dtype=HSP_DTYPE)
    return SearchResult(out[:n].copy(), exts, hits, passing)


# ---- gapped extension of the HSP hand-off (gapped.c; R18-R22) ----

GAPPED_DTYPE = np.dtype([("query_id", "<i4"), ("subject_id", "<i4"), ("q_start", "<i4"),
                         ("q_end", "<i4"), ("s_start", "<i4"), ("s_end", "<i4"),
                         ("score", "<i4"), ("ident", "<i4"), ("gap_opens", "<i4"),
                         ("gap_len", "<i4")])


@dataclass
class GappedParams:
    """R18/R19/R21 (BLASTP defaults: gap cost 11 + 1 per residue, gapped X-drop
    15 bits = 38 raw at the gapped lambda 0.267, report cutoff 41)."""
    gap_open: int = 11
    gap_extend: int = 1
    xdrop: int = 38
    cutoff: int = 41


def gapped_dir(a: np.ndarray, b: np.ndarray, matrix: np.ndarray, gp: GappedParams | None = None):
    """One direction (R19/R22): (score, bi, bj, ident, gap_opens, gap_len)."""
    gp = gp or GappedParams()
    a = np.ascontiguousarray(a, dtype=np.uint8)
    b = np.ascontiguousarray(b, dtype=np.uint8)
    m = np.ascontiguousarray(matrix, dtype=np.int32)
    outs = [ctypes.c_int32() for _ in range(5)]
    sc = lib().oracle_gapped_dir(_ptr(a), len(a), _ptr(b), len(b), _ptr(m), m.shape[0],
                                 gp.gap_open, gp.gap_extend, gp.xdrop,
                                 *[ctypes.byref(o) for o in outs])
    if sc < 0:
        raise MemoryError("oracle_gapped_dir")
    return (int(sc), *[int(o.value) for o in outs])


def gapped_hsps(queries, db: np.ndarray, offsets: np.ndarray, hsps: np.ndarray,
                gp: GappedParams | None = None, subject_base: int = 0,
                matrix: np.ndarray | None = None) -> np.ndarray:
    """R20/R21 over a canonical HSP list; queries = list of code arrays
    (index = query_id).  Returns GAPPED_DTYPE records in canonical order."""
    gp = gp or GappedParams()
    qs = [np.ascontiguousarray(q, dtype=np.uint8) for q in queries]
    qptr = (ctypes.c_void_p * max(1, len(qs)))(*[q.ctypes.data for q in qs])
    qlen = np.array([len(q) for q in qs] or [0], dtype=np.int32)
    d = np.ascontiguousarray(db, dtype=np.uint8)
    off = np.ascontiguousarray(offsets, dtype=np.int64)
    h = np.ascontiguousarray(hsps).view(HSP_DTYPE) if len(hsps) else np.zeros(0, HSP_DTYPE)
    m = np.ascontiguousarray(blosum62() if matrix is None else matrix, dtype=np.int32)
    cap = max(1, len(h))
    out = np.zeros(cap, dtype=GAPPED_DTYPE)
    n = lib().oracle_gapped_hsps(ctypes.cast(qptr, ctypes.c_void_p), _ptr(qlen), len(qs),
                                 _ptr(d), _ptr(off), len(off) - 1, subject_base, _ptr(h), len(h),
                                 _ptr(m), m.shape[0], gp.gap_open, gp.gap_extend, gp.xdrop,
                                 gp.cutoff, _ptr(out), cap)
    if n < 0:
        raise ValueError("oracle_gapped_hsps: bad HSP (query / subject id) or allocation failure")
    return out[:n].copy()
