"""Time the gapped stage on config 3's ungapped list (device-resident input),
CUDA events on the launch stream, plus the search alone for context."""
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
for rep in range(4):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    w0 = time.perf_counter()
    e0.record(s)
    n = bp.gapped_extend_device(t, d, dev.data_ptr(), len(u), out.data_ptr(), len(u), stream=s)
    e1.record(s)
    torch.cuda.synchronize()
    print(f"gapped: {len(u)} HSPs -> {n} alignments, {e0.elapsed_time(e1):.2f} ms device "
          f"({(time.perf_counter() - w0) * 1e3:.2f} ms wall)")
g = out[:n].cpu().numpy().view(bp.GAPPED_DTYPE).ravel()
print("gap_opens>0:", int((g["gap_opens"] > 0).sum()), "mean len", float((g["q_end"] - g["q_start"]).mean()))
for rep in range(3):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    r, uu = bp.search_gapped(t, d, stream=s, want_ungapped=True)
    e1.record(s)
    torch.cuda.synchronize()
    print(f"search_gapped: {len(uu)} HSPs, {len(r)} alignments, {e0.elapsed_time(e1):.2f} ms")
