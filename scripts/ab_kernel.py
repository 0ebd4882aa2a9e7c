"""Interleaved A/B device timing of libblastp builds in ONE process on one box
(the workload generated once): python scripts/ab_kernel.py <rounds> lib1.so lib2.so ...

Each library gets its own table + packed DB through its own C-ABI handles; every
round times `steps` searches per library with CUDA events on one stream and
prints ms/search; the HSP counts of all libraries must agree.  Env: AB_CONFIG (3),
AB_SCALE (1.0), AB_STEPS (5), AB_QLEN (a config-3 query length override)."""
import ctypes
import os
import statistics
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from synth import config_workload  # noqa: E402


class CParams(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in ("word_len", "threshold", "window", "min_gap",
                                              "xdrop", "cutoff", "filter_mode", "ext_mode")]


def load(path):
    L = ctypes.CDLL(os.path.abspath(path))
    vp, i32, i64, P = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.POINTER
    L.blastp_build_query_table.argtypes = [ctypes.c_char_p, i32, P(CParams), ctypes.c_int, vp,
                                           P(vp)]
    L.blastp_pack_db.argtypes = [vp, vp, i64, i32, i32, ctypes.c_int, vp, P(vp)]
    L.blastp_search_ungapped_device.argtypes = [vp, vp, P(CParams), vp, vp, i64, vp]
    L.blastp_last_error.restype = ctypes.c_char_p
    return L


def main():
    rounds = int(sys.argv[1])
    libs = sys.argv[2:]
    cfg = int(os.environ.get("AB_CONFIG", "3"))
    scale = float(os.environ.get("AB_SCALE", "1.0"))
    steps = int(os.environ.get("AB_STEPS", "5"))
    (q,), db = config_workload(cfg, scale=scale)
    torch.cuda.set_device(0)
    s = torch.cuda.current_stream()
    sp = ctypes.c_void_p(s.cuda_stream)
    p = CParams(3, 11, 40, 3, 16, 41, int(os.environ.get("AB_FILTER", "0")),
                int(os.environ.get("AB_EXT", "0")))
    cap = db.residues // 500 + (1 << 20)
    out = torch.empty((cap, 7), dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    off = np.ascontiguousarray(db.offsets, dtype=np.int64)
    inst = []
    for path in libs:
        L = load(path)
        t = ctypes.c_void_p()
        rc = L.blastp_build_query_table(q, len(q), ctypes.byref(p), 0, sp, ctypes.byref(t))
        assert rc == 0, L.blastp_last_error()
        d = ctypes.c_void_p()
        rc = L.blastp_pack_db(db.ascii.ctypes.data, off.ctypes.data, len(off) - 1, 0, 1, 0, sp,
                              ctypes.byref(d))
        assert rc == 0, L.blastp_last_error()
        inst.append((os.path.basename(path), L, t, d))
    counts = {}
    times = {n: [] for n, *_ in inst}
    for r in range(rounds + 1):
        for name, L, t, d in inst:
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
            torch.cuda.synchronize()
            ev[0].record(s)
            for _ in range(steps):
                rc = L.blastp_search_ungapped_device(t, d, ctypes.byref(p), sp, out.data_ptr(),
                                                     cap, cnt.data_ptr())
                assert rc == 0, L.blastp_last_error()
            ev[1].record(s)
            torch.cuda.synchronize()
            ms = ev[0].elapsed_time(ev[1]) / steps
            counts.setdefault(name, int(cnt.item()))
            assert counts[name] == int(cnt.item())
            if r > 0:  # round 0 warms up
                times[name].append(ms)
                print(f"round {r} {name:28s} {ms:8.3f} ms/search", flush=True)
    print("--- median ms/search (HSPs)")
    base = None
    for name in times:
        m = statistics.median(times[name])
        base = base or m
        print(f"{name:28s} {m:8.3f}  ({100 * (m / base - 1):+5.1f}%)  hsps {counts[name]}")
    if os.environ.get("AB_NO_CHECK") != "1":
        assert len(set(counts.values())) == 1, counts


if __name__ == "__main__":
    main()
