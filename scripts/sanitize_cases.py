"""Small searches for compute-sanitizer (memcheck / racecheck / synccheck /
initcheck): config 1 on every kernel variant and filter mode, the poly-W
low-complexity case (hit-dense rounds, long same-diagonal groups), long
subjects through the segment plan (warp kernel lists + walker, list overflow
BLASTP_SEGCAP=4; diagonal-range segments of the block kernel and STATEFUL),
a query batch (groups), HIT_DEDUP, the PSSM switch.  Each search is checked
against the oracle so a sanitizer run is also a parity run.
usage: python scripts/sanitize_cases.py [quick]"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
from oracle import oracle as orc  # noqa: E402
from paper_conf_ipps_zhangwlf14_b200 import blastp as bp  # noqa: E402
from synth import config_workload, gen_db, gen_query  # noqa: E402
from test_gpu_parity import _long_subject_db  # noqa: E402


def check(q, ascii, off, p, label):
    t = bp.build_query_table(q, p)
    d = bp.pack_db(ascii, off)
    g = [tuple(x) for x in bp.search_ungapped(t, d, p).tolist()]
    t.free()
    d.free()
    P = orc.Params(word_len=p.word_len, threshold=p.threshold, window=p.window,
                   min_gap=p.min_gap, xdrop=p.xdrop, cutoff=p.cutoff, filter_mode=p.filter_mode,
                   ext_mode=1 if p.ext_mode == 1 else 0)
    r = orc.search(orc.encode(q), orc.encode(ascii.tobytes()), np.asarray(off, np.int64), P)
    exp = [tuple(x) for x in r.hsps.tolist()]
    assert g == exp, (label, len(g), len(exp))
    print(f"ok {label}: {len(g)} HSPs", flush=True)


def main():
    quick = len(sys.argv) > 1 and sys.argv[1] == "quick"
    (q1,), db1 = config_workload(1, scale=0.3 if quick else 1.0)
    polyq = "W" * 200 + "AAAAQQQQ" * 6 + "W" * 40
    subs = ["W" * 600, "A" * 150 + "W" * 40, "WA" * 200, "Q" * 300, "W" * 3]
    pa = np.frombuffer("".join(subs).encode(), np.uint8).copy()
    po = np.concatenate([[0], np.cumsum([len(s) for s in subs])]).astype(np.int64)
    qL = gen_query(21, 300).decode()
    la, lo = _long_subject_db(qL)
    for kernel in ("block", "warp", "cta"):
        os.environ["BLASTP_KERNEL"] = kernel
        modes = [(0, 0), (1, 0), (0, 1), (2, 0), (3, 0)] if kernel != "block" else [(0, 0), (0, 1), (0, 3)]
        for fm, em in modes:
            check(q1, db1.ascii, db1.offsets, bp.Params(filter_mode=fm, ext_mode=em),
                  f"{kernel} config1 filter{fm} ext{em}")
        check(polyq, pa, po, bp.Params(), f"{kernel} poly-W")
        check(qL, la, lo, bp.Params(), f"{kernel} long subjects")
    os.environ["BLASTP_KERNEL"] = "warp"
    for cap in ("4", "150"):
        os.environ["BLASTP_SEGCAP"] = cap
        check(qL, la, lo, bp.Params(), f"warp long subjects SEGCAP={cap}")
    os.environ.pop("BLASTP_SEGCAP")
    check(qL, la, lo, bp.Params(filter_mode=2), "warp long subjects STATEFUL")
    os.environ.pop("BLASTP_KERNEL")
    os.environ["BLASTP_SCORE"] = "pssm"
    check(q1, db1.ascii, db1.offsets, bp.Params(), "block PSSM")
    os.environ.pop("BLASTP_SCORE")
    qs = [gen_query(300 + i, L) for i, L in enumerate([60, 120, 200, 350])]
    dbq = gen_db(301, 302, n_subjects=150, mean_len=300.0, queries=qs, plant_frac=0.5)
    t = bp.build_query_batch(qs, bp.Params())
    d = bp.pack_db(dbq.ascii, dbq.offsets)
    g = bp.search_ungapped(t, d, bp.Params())
    assert len(g) > 10
    print(f"ok query groups: {len(g)} HSPs", flush=True)
    t.free()
    d.free()
    # the append entry (peer-buffer protocol, here into a local buffer; the
    # system-scope fence per HSP) and the formatted DB streamed through one
    # reused part slot
    import torch
    t = bp.build_query_table(q1, bp.Params())
    d = bp.pack_db(db1.ascii, db1.offsets)
    cap = 1 << 16
    out = torch.empty((cap, 7), dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    for _ in range(2):  # appends accumulate
        bp.search_ungapped_append(t, d, out.data_ptr(), cap, cnt.data_ptr())
    n = int(cnt.item())
    exp = len(bp.search_ungapped(t, d))
    assert n == 2 * exp, (n, exp)
    print(f"ok append: {n} HSPs (2 x {exp})", flush=True)
    os.environ["BLASTP_PIPE_SLOTS"] = "1"
    h = bp.format_host_db(db1.ascii, db1.offsets, num_parts=5)
    cnt.zero_()
    bp.search_formatted_db(t, h, out.data_ptr(), cap, cnt.data_ptr())
    assert int(cnt.item()) == exp
    print(f"ok formatted, 1 slot x 5 parts: {exp} HSPs", flush=True)
    os.environ.pop("BLASTP_PIPE_SLOTS")
    h.free()
    t.free()
    d.free()
    del out, cnt
    torch.cuda.empty_cache()
    torch._C._host_emptyCache()  # the pinned staging buffer of .item()
    bp.trim_memory(0)  # pool memory back to the device: memcheck's leak check sees only leaks


if __name__ == "__main__":
    main()
