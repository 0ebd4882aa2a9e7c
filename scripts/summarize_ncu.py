"""Summarise an ncu full capture + launch list into profiles/<round>/ (text + JSON).

usage: python scripts/summarize_ncu.py <prof.ncu-rep> <launches.csv> <outdir> [label]
Writes ncu_<label>_details.txt, ncu_<label>_hotspots.txt, launches_<label>.txt and
profiles/ncu_search_kernel.json (read by bench.py for roofline.traffic).
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

rep, launches, outdir = sys.argv[1:4]
label = sys.argv[4] if len(sys.argv) > 4 else "search"
os.makedirs(outdir, exist_ok=True)


def ncu(*args):
    return subprocess.run(["ncu", "-i", rep, *args], capture_output=True, text=True).stdout


# details page
det = list(csv.reader(io.StringIO(ncu("--page", "details", "--csv"))))
hdr = det[0]
rows = [dict(zip(hdr, r)) for r in det[1:]]
kernel = rows[0]["Kernel Name"] if rows else "?"
with open(os.path.join(outdir, f"ncu_{label}_details.txt"), "w") as f:
    f.write(f"kernel: {kernel}\n")
    for d in rows:
        if d.get("Metric Name"):
            f.write(f"{d['Section Name'][:34]:34s} {d['Metric Name'][:52]:52s} "
                    f"{d['Metric Unit'][:12]:12s} {d['Metric Value']}\n")
# raw metrics we cite
raw = list(csv.reader(io.StringIO(ncu("--page", "raw", "--csv"))))
rh, units, vals = raw[0], raw[1], raw[2]
R = dict(zip(rh, vals))
U = dict(zip(rh, units))


def num(k):
    v = R.get(k, "")
    try:
        return float(v.replace(",", ""))
    except ValueError:
        return None


def to_bytes(k):
    v, u = num(k), U.get(k, "byte")
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}
    return None if v is None else v * scale.get(u, 1)


keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "lts__t_bytes.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__thread_inst_executed_per_inst_executed.ratio",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "smsp__inst_executed.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"]
summary = {k: R.get(k) for k in keys if k in R}
summary["units"] = {k: U.get(k) for k in keys if k in R}
rd, wr = to_bytes("dram__bytes_read.sum"), to_bytes("dram__bytes_write.sum")
summary["dram_bytes_per_launch"] = (rd or 0) + (wr or 0) if rd is not None else None
summary["kernel"] = kernel
summary["source"] = f"ncu --set full capture {os.path.basename(rep)} (one launch)"
with open(os.path.join(outdir, f"ncu_{label}_raw.json"), "w") as f:
    json.dump(summary, f, indent=1)
with open(os.path.join(os.path.dirname(outdir.rstrip("/")), "ncu_search_kernel.json"), "w") as f:
    json.dump(summary, f, indent=1)
# launch list summary
rows = list(csv.reader(open(launches)))
start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
h = rows[start]
agg = collections.defaultdict(list)
for r in rows[start + 1:]:
    d = dict(zip(h, r))
    if d.get("Metric Name") == "gpu__time_duration.sum":
        agg[d["Kernel Name"][:70]].append(float(d["Metric Value"].replace(",", "")))
tot = sum(sum(v) for v in agg.values())
with open(os.path.join(outdir, f"launches_{label}.txt"), "w") as f:
    f.write("ncu --metrics gpu__time_duration.sum --clock-control none "
            "(bench.py --steps 3 --warmup 3; cold-cache, serialised: compare shares)\n")
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        f.write(f"{k:70s} n={len(v):3d} total {sum(v)/1e6:9.3f} ms share {100*sum(v)/tot:5.1f}% "
                f"mean {sum(v)/len(v)/1e6:8.3f} ms\n")
print(open(os.path.join(outdir, f"launches_{label}.txt")).read())
print(json.dumps(summary, indent=1))
