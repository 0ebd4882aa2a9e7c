"""Timeline of blastp_search_host_db on config 3 (BLASTP_DEBUG_PIPE=1)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["BLASTP_DEBUG_PIPE"] = "1"
import torch
from paper_conf_ipps_zhangwlf14_b200 import blastp as bp
from synth import config_workload
(q,), db = config_workload(3, scale=float(sys.argv[1]) if len(sys.argv) > 1 else 1.0)
pinned = torch.empty(db.residues, dtype=torch.uint8, pin_memory=True)
pinned.copy_(torch.from_numpy(db.ascii))
t = bp.build_query_table(q)
off = torch.from_numpy(db.offsets.astype("int64")).pin_memory().numpy() if "--pageable" not in sys.argv else db.offsets
cap = 1 << 22
out = torch.empty(cap * 7, dtype=torch.int32, device="cuda")
cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
for it in range(3):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    bp.search_host_db(t, pinned.data_ptr(), off, out.data_ptr(), cap, cnt.data_ptr(),
                      num_parts=int(sys.argv[2]) if len(sys.argv) > 2 and sys.argv[2].isdigit() else 0)
    n = int(cnt.item()); torch.cuda.synchronize()
    print(f"iteration {it}: {1e3 * (time.perf_counter() - t0):.2f} ms, {n} HSPs", flush=True)
