"""Time the gapped stage on config 3's ungapped list (device-resident input),
CUDA events on the launch stream; a sweep of the pass-1 ring width and
blocks per SM (BLASTP_GAPPED_RING / _BPS), then search + gapped together."""
import os
import sys
import time

import numpy as np
import torch

from paper_conf_ipps_zhangwlf14_b200 import blastp as bp
from synth import config_workload

(q,), db = config_workload(3)
s = torch.cuda.current_stream()
t = bp.build_query_table(q, stream=s)
d = bp.pack_db(db.ascii, db.offsets, stream=s)
u = bp.search_ungapped(t, d, stream=s)
dev = torch.from_numpy(u.view(np.int32).reshape(-1, 7).copy()).cuda()
out = torch.zeros((len(u), 10), dtype=torch.int32, device="cuda")


def run(reps=3):
    ms = []
    for rep in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(s)
        n = bp.gapped_extend_device(t, d, dev.data_ptr(), len(u), out.data_ptr(), len(u), stream=s)
        e1.record(s)
        torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
    return n, sorted(ms)[len(ms) // 2]


# --sweep: ring width x blocks per SM; --env 'K=V,K=V;K=V': explicit settings
sweep = "--sweep" in sys.argv
combos = [{"BLASTP_GAPPED_RING": r, "BLASTP_GAPPED_BPS": b} for r in ("128", "256", "512")
          for b in ("4", "8", "16")] if sweep else [{}]
if "--env" in sys.argv:
    spec = sys.argv[sys.argv.index("--env") + 1]
    combos = [dict(kv.split("=") for kv in c.split(",") if kv) for c in spec.split(";")]
KNOBS = ("BLASTP_GAPPED_RING", "BLASTP_GAPPED_BPS", "BLASTP_GAPPED_TBBUF", "BLASTP_GAPPED_STORE")
for combo in combos:
    for k in KNOBS:
        os.environ.pop(k, None)
    os.environ.update(combo)
    ring, bps = combo, ""
    run(1)
    os.environ["BLASTP_GAPPED_VERBOSE"] = "1"
    run(1)
    sys.stderr.flush()
    os.environ.pop("BLASTP_GAPPED_VERBOSE")
    n, ms = run()
    print(f"{combo}: {len(u)} HSPs -> {n} alignments, {ms:.2f} ms device (median of 3)",
          flush=True)
for k in KNOBS:
    os.environ.pop(k, None)
g = out[:n].cpu().numpy().view(bp.GAPPED_DTYPE).ravel()
print("gap_opens>0:", int((g["gap_opens"] > 0).sum()), "mean len", float((g["q_end"] - g["q_start"]).mean()))
for rep in range(3):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    r, uu = bp.search_gapped(t, d, stream=s, want_ungapped=True)
    e1.record(s)
    torch.cuda.synchronize()
    print(f"search_gapped: {len(uu)} HSPs, {len(r)} alignments, {e0.elapsed_time(e1):.2f} ms")
