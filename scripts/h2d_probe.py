"""H2D bandwidth from pinned memory vs blastp_pack_db time (config 3 DB)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_zhangwlf14_b200 import blastp as bp
from synth import config_workload
(q,), db = config_workload(3, scale=1.0)
pinned = torch.empty(db.residues, dtype=torch.uint8, pin_memory=True)
pinned.copy_(torch.from_numpy(db.ascii))
dev = torch.empty(db.residues, dtype=torch.uint8, device="cuda")
s = torch.cuda.Stream()
for size in (1 << 24, 1 << 26, 1 << 28, db.residues):
    for it in range(3):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        with torch.cuda.stream(s):
            dev[:size].copy_(pinned[:size], non_blocking=True)
        s.synchronize()
        dt = time.perf_counter() - t0
    print(f"H2D {size/1e6:8.1f} MB: {dt*1e3:7.2f} ms  {size/dt/1e9:6.1f} GB/s", flush=True)
for it in range(3):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    d = bp.Database.from_pinned(pinned.data_ptr(), db.offsets, 0, 1)
    torch.cuda.synchronize(); dt = time.perf_counter() - t0
    d.free()
    print(f"pack_db whole: {dt*1e3:.2f} ms ({db.residues/dt/1e9:.1f} GB/s)", flush=True)
print(os.popen("nvidia-smi -q | grep -i -A3 'PCIe Generation\\|Link Width' | head -20").read())
print(os.popen("numactl --hardware 2>/dev/null | head -5; nproc").read())
