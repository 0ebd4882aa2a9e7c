"""Per-kernel HBM roofline of every kernel libblastp.so launches (config 3).

Phase 1 (under ncu): `python scripts/kernel_roofline.py run` exercises every
kernel once on config 3 (q1054 vs 1.2G residues): blastp_pack_db (layout,
chunk, pack kernels), the warp and CTA search kernels (ext_mode DIAGONAL and
HIT), the host variant's GPU canonical sort (key/radix/gather kernels) and
the pipelined host-DB search.
Phase 2: `python scripts/kernel_roofline.py summarize <ncu.csv> <out.json> [peak_gbs]`
turns the ncu CSV (metrics below) into per-kernel time, DRAM bytes and the
achieved fraction of the HBM peak.

ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,\
sm__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none --csv \
--log-file gpurun_out/kernels.csv python scripts/kernel_roofline.py run
"""
import collections
import csv
import io
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def run():
    import torch

    from paper_conf_ipps_zhangwlf14_b200 import blastp as bp
    from synth import config_workload
    torch.cuda.set_device(0)
    s = torch.cuda.current_stream()
    (q,), db = config_workload(3)
    d = bp.pack_db(db.ascii, db.offsets, stream=s)
    cap = db.residues // 500
    out = torch.empty((cap, 7), dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    for kernel in ("warp", "cta"):
        os.environ["BLASTP_KERNEL"] = kernel
        for ext_mode in (0, 1):
            p = bp.Params(ext_mode=ext_mode)
            t = bp.build_query_table(q, p, stream=s)
            bp.search_ungapped_device(t, d, out.data_ptr(), cap, cnt.data_ptr(), p, s)
    os.environ["BLASTP_KERNEL"] = "warp"
    t = bp.build_query_table(q, stream=s)
    bp.search_ungapped(t, d, stream=s)  # + GPU canonical sort
    bp.search_host_db(t, db.ascii, db.offsets, out.data_ptr(), cap, cnt.data_ptr(), stream=s)
    torch.cuda.synchronize()


def summarize(path, out_path, peak=6650.0):
    text = open(path).read()
    text = text[text.index('"ID"'):]
    per = collections.defaultdict(lambda: collections.defaultdict(list))
    for r in csv.DictReader(io.StringIO(text)):
        name = r["Kernel Name"].split("(")[0].replace("void ", "")
        v = float(r["Metric Value"].replace(",", ""))
        u = r["Metric Unit"]
        m = r["Metric Name"]
        if m == "gpu__time_duration.sum":
            v = v * {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "nsecond": 1e-6, "ms": 1.0,
                     "msecond": 1.0}.get(u, 1.0)
        elif m.startswith("dram__bytes"):
            v = v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6,
                     "GB": 1e9}.get(u, 1)
        per[(name, r["ID"])][m].append(v)
    kern = collections.defaultdict(lambda: {"launches": 0, "ms": 0.0, "dram_bytes": 0.0,
                                            "sm_pct": []})
    for (name, _), ms in per.items():
        k = kern[name]
        k["launches"] += 1
        k["ms"] += ms["gpu__time_duration.sum"][0]
        k["dram_bytes"] += ms["dram__bytes_read.sum"][0] + ms["dram__bytes_write.sum"][0]
        k["sm_pct"].append(ms["sm__throughput.avg.pct_of_peak_sustained_elapsed"][0])
    rows = []
    for name, k in sorted(kern.items(), key=lambda x: -x[1]["ms"]):
        gbs = k["dram_bytes"] / (k["ms"] / 1e3) / 1e9 if k["ms"] else 0.0
        rows.append({"kernel": name, "launches": k["launches"], "ms_total": k["ms"],
                     "ms_per_launch": k["ms"] / k["launches"],
                     "dram_bytes_per_launch": k["dram_bytes"] / k["launches"],
                     "dram_gbs": gbs, "hbm_frac": gbs / peak,
                     "sm_throughput_pct": sum(k["sm_pct"]) / len(k["sm_pct"])})
    json.dump({"peak_gbs": peak, "source": os.path.basename(path),
               "note": "ncu --clock-control none, serialised cold-cache launches; dram_gbs = "
                       "measured DRAM bytes / kernel duration",
               "kernels": rows}, open(out_path, "w"), indent=1)
    for r in rows:
        print(f"{r['kernel'][:60]:60s} n={r['launches']:3d} {r['ms_per_launch']:9.3f} ms "
              f"{r['dram_bytes_per_launch'] / 1e6:10.1f} MB {r['dram_gbs']:8.1f} GB/s "
              f"({100 * r['hbm_frac']:5.1f}% HBM)  SM {r['sm_throughput_pct']:5.1f}%")


if __name__ == "__main__":
    if sys.argv[1] == "run":
        run()
    else:
        summarize(sys.argv[2], sys.argv[3], float(sys.argv[4]) if len(sys.argv) > 4 else 6650.0)
