"""Part-size sweep of the formatted-host-DB stream (blastp_search_formatted_db) on config 3:
for each (first part residues, growth %) the image is formatted, then searched 4 times
end to end (host clock, synchronised; D2H of the HSP count only).  Device time of the
resident search printed for reference.

usage: python scripts/fmt_sweep.py [scale]
"""
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangwlf14_b200 import blastp as bp  # noqa: E402
from synth import config_workload  # noqa: E402

scale = float(sys.argv[1]) if len(sys.argv) > 1 and sys.argv[1][0].isdigit() else 1.0
(q,), db = config_workload(3, scale=scale)
pinned = torch.empty(db.residues, dtype=torch.uint8, pin_memory=True)
pinned.copy_(torch.from_numpy(db.ascii))
off = torch.from_numpy(db.offsets.astype("int64")).pin_memory().numpy()
t = bp.build_query_table(q)
cap = 1 << 22
out = torch.empty(cap * 7, dtype=torch.int32, device="cuda")
cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
d = bp.Database.from_pinned(pinned.data_ptr(), off, 0, 1)
for _ in range(3):
    bp.search_ungapped_device(t, d, out.data_ptr(), cap, cnt.data_ptr())
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(5):
    bp.search_ungapped_device(t, d, out.data_ptr(), cap, cnt.data_ptr())
torch.cuda.synchronize()
print(f"resident search: {1e3 * (time.perf_counter() - t0) / 5:.2f} ms", flush=True)
d.free()
grid = [(1 << 24, 150, 0), (1 << 24, 140, 0), (1 << 24, 130, 0), (1 << 24, 120, 0),
        (1 << 23, 130, 0), (1 << 25, 130, 0), (1 << 23, 140, 0), (0, 0, 32), (0, 0, 48)]
if "--wide" in sys.argv:
    grid += [(1 << 24, 200, 0), (1 << 24, 300, 0), (0, 0, 4), (0, 0, 16)]
for first, growth, parts in grid:
    if parts == 0:
        os.environ["BLASTP_PIPE_FIRST"] = str(first)
        os.environ["BLASTP_PIPE_GROWTH"] = str(growth)
    h = bp.format_host_db(pinned.data_ptr(), off, num_parts=parts)
    ms = []
    for it in range(5):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        bp.search_formatted_db(t, h, out.data_ptr(), cap, cnt.data_ptr())
        n = int(cnt.item())
        torch.cuda.synchronize()
        if it:
            ms.append(1e3 * (time.perf_counter() - t0))
    print(f"first {first:>9d} growth {growth:3d} parts {h.num_parts:2d}: "
          f"{statistics.median(ms):.2f} ms (min {min(ms):.2f}), {n} HSPs", flush=True)
    h.free()
