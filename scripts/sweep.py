"""Strategy sweep on B200 (the paper's E1-E3 comparisons, re-run
on this implementation): kernel variant (warp rings / CTA bins, BLASTP_KERNEL)
x extension strategy (diagonal-based Alg. 3 / hit-based Alg. 4 / window-based
Alg. 5, warp variant; the CTA variant runs Alg. 3 for WINDOW) x two-hit
reading (LEFT / EITHER / STATEFUL = Alg. 1's lasthit walk / STATEFUL_RB, DIAGONAL and
warp only; the block kernel: LEFT with DIAGONAL / HIT) on configs 1-3.  Device time per search (CUDA events
on the launch stream, median of `reps` after 2 warm-ups), residues/s and the
HSP/extension counts of each cell.

usage: python scripts/sweep.py [out.json] [reps]
"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangwlf14_b200 import blastp as bp  # noqa: E402
from synth import config_workload  # noqa: E402

out_path = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/sweep.json"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
torch.cuda.set_device(0)
stream = torch.cuda.current_stream()
rows = []
for cfg in (1, 2, 3):
    (q,), db = config_workload(cfg)
    d = bp.pack_db(db.ascii, db.offsets, stream=stream)
    cap = max(1 << 20, db.residues // 50)
    out = torch.empty((cap, 7), dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    for kernel in ("block", "warp", "cta"):
        os.environ["BLASTP_KERNEL"] = kernel
        for ext_mode in (0, 1, 2, 3):
            for filt in (0, 1, 2, 3):
                if filt >= 2 and (ext_mode != 0 or kernel != "warp"):
                    continue
                if kernel == "block" and (filt != 0 or ext_mode == 2):
                    continue  # the block kernel runs LEFT with DIAGONAL / HIT (/ HIT_DEDUP)
                if kernel == "cta" and ext_mode == 3:
                    continue
                p = bp.Params(filter_mode=filt, ext_mode=ext_mode)
                t = bp.build_query_table(q, p, stream=stream)
                ms = []
                for i in range(reps + 2):
                    a = torch.cuda.Event(enable_timing=True)
                    b = torch.cuda.Event(enable_timing=True)
                    a.record(stream)
                    bp.search_ungapped_device(t, d, out.data_ptr(), cap, cnt.data_ptr(), p, stream)
                    b.record(stream)
                    torch.cuda.synchronize()
                    if i >= 2:
                        ms.append(a.elapsed_time(b))
                n = int(cnt.item())
                med = statistics.median(ms)
                row = {"config": cfg, "query_len": len(q), "residues": db.residues,
                       "kernel": kernel,
                       "ext_mode": ["DIAGONAL", "HIT", "WINDOW", "HIT_DEDUP(search)"][ext_mode],
                       "filter": ["LEFT", "EITHER", "STATEFUL", "STATEFUL_RB"][filt], "ms": med,
                       "residues_per_s": db.residues / (med / 1e3), "hsps": n}
                rows.append(row)
                print(f"config {cfg} {kernel:4s} {row['ext_mode']:8s} {row['filter']:6s} "
                      f"{med:9.3f} ms  {row['residues_per_s']:.3e} res/s  {n} HSPs", flush=True)
    del d
json.dump(rows, open(out_path, "w"), indent=1)
