"""Summarise one ncu --set full capture of the search kernel into
profiles/ncu_search_kernel.json (what bench.py's roofline keys read), tagged
with the csrc hash of the source tree it was built from -- run it on the tree
the capture was taken with.  usage: python scripts/capture_json.py <rep> [out]"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from bench import csrc_hash  # noqa: E402

rep = sys.argv[1]
out = sys.argv[2] if len(sys.argv) > 2 else os.path.join(ROOT, "profiles", "ncu_search_kernel.json")
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__thread_inst_executed_per_inst_executed.ratio",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "smsp__inst_executed.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active"]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units, vals = rows[0], rows[1], rows[2]
d = {}
for m in want:
    if m in hdr:
        v = vals[hdr.index(m)].replace(",", "")
        try:
            d[m] = float(v)
        except ValueError:
            d[m] = v
d["units"] = {m: units[hdr.index(m)] for m in want if m in hdr}
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
rd = float(d["dram__bytes_read.sum"]) * scale[d["units"]["dram__bytes_read.sum"]]
wr = float(d["dram__bytes_write.sum"]) * scale[d["units"]["dram__bytes_write.sum"]]
d["dram_bytes_per_launch"] = rd + wr
d["kernel"] = vals[hdr.index("Kernel Name")] if "Kernel Name" in hdr else "?"
d["source"] = f"ncu --set full capture {os.path.basename(rep)} (one config-3 launch)"
d["csrc_sha"] = csrc_hash()
with open(out, "w") as f:
    json.dump(d, f, indent=1)
print(json.dumps({k: d[k] for k in ("kernel", "dram_bytes_per_launch", "smsp__inst_executed.sum",
                                    "gpu__time_duration.sum", "csrc_sha")}))
