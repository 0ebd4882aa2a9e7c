#!/usr/bin/env python
"""bench.py -- database residues/s of the B200 BLASTP hot path (hit detection +
two-hit filter + X-drop ungapped extension), BASELINE.json's metric.

  python bench.py [--gpus N --steps K --warmup W] [--impl ours|reference]
  torchrun --nproc-per-node N bench.py --gpus N ...      (N > 1, NCCL)

Workload: BASELINE config 3 -- query length 1054
against the env_nr-shaped synthetic database (6.0M subjects, ~1.2G residues,
RR frequencies, 0.5% planted homologs).  At N > 1 the same database is
sharded by subject range over the ranks (config 4, strong scaling) and the
HSPs are gathered to rank 0 over NCCL inside every step.

One step = one full search of every query against the (local shard of the)
database: the fused search kernel(s) plus, at N > 1, the HSP gather.  The
database (1.2 GB) is larger than L2 (126 MB), so no flush is needed between
steps.  Device time: CUDA events on the launching stream, barrier +
synchronize around the timed region, max over ranks.

e2e: the same metric through the C-ABI with HOST buffers: each step packs the
shard from pinned host memory (H2D inside blastp_pack_db), searches, gathers
(N > 1) and reads the HSP list back to the host.

--impl reference: the CPU oracle (oracle/, test infrastructure) timed on the
host cores on a bounded sample of the same workload, rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "database residues/sec (hit detect + ungapped ext) at 1/2/4/8 B200; % HBM roofline"
UNIT = "residues/s"
ORACLE_SAMPLE_RQ = 48_000_000  # oracle sample per step: residue-queries at q1054-equivalent


def parse_args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", type=int, default=3, choices=[1, 2, 3, 5],
                    help="BASELINE config; 5 = 64 queries vs the nr-shaped DB cut into 8 "
                         "shards, rank r searching shard r (weak scaling)")
    ap.add_argument("--query-lens", default="1054",
                    help="comma list of query lengths searched as one batch (config 4: 127,517,1054)")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-gapped", action="store_true",
                    help="skip the gapped-stage measurement (SURVEY 8(f) rank 4)")
    ap.add_argument("--gather", choices=["p2p", "nccl"], default="p2p",
                    help="N > 1: HSPs appended by the search kernels into rank 0's buffer over "
                         "NVLink (CUDA IPC), or per-rank lists gathered with NCCL")
    ap.add_argument("--scale", type=float, default=1.0, help="DB scale (tests only)")
    return ap.parse_args()


def env_rank():
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("LOCAL_RANK", "0")),
            int(os.environ.get("WORLD_SIZE", "1")))


# --------------------------------------------------------------- workload

def shard_plan(args, world):
    """(shard count, whole-job residues are those of shards [0, world)).
    Configs 1-3: the DB is cut into `world` shards (strong scaling, config 4).
    Config 5: the DB is cut into max(8, world) shards and rank r owns shard r
    (weak scaling: per-GPU work is fixed; at N = 8 the job is all of config 5)."""
    return max(8, world) if args.config == 5 else world


def workload(args, rank, world):
    from paper_conf_ipps_zhangwlf14_b200.dist import shard_subjects
    from synth import CONFIGS, config_offsets, gen_db, gen_queries, gen_query
    c = CONFIGS[args.config]
    if args.config == 5:
        queries = gen_queries(c["query_seed"], 64, 100, 2000)
        lens = [len(q) for q in queries]
    else:
        lens = [int(x) for x in args.query_lens.split(",")] if args.config == 3 else [c["query_len"]]
        queries = [gen_query(c["query_seed"] if L == c["query_len"] else L, L) for L in lens]
    full_off = config_offsets(args.config, args.scale)
    nshards = shard_plan(args, world)
    lo, hi = shard_subjects(full_off, rank, nshards)
    ns, tr = c["n_subjects"], c["total_residues"]
    if args.scale != 1.0:
        ns = None if ns is None else max(1, int(ns * args.scale))
        tr = None if tr is None else max(1000, int(tr * args.scale))
    db = gen_db(c["db_seed"], c["plant_seed"], n_subjects=ns, total_residues=tr,
                mean_len=c["mean_len"], queries=queries, plant_frac=c["plant_frac"],
                subject_range=(lo, hi))
    if args.config == 5:
        _, job_hi = shard_subjects(full_off, world - 1, nshards)
        desc = (f"config5: 64 queries (len U[100,2000], {sum(lens)} residues) vs "
                f"{c['name'].split('_vs_')[-1]} synthetic DB ({len(full_off) - 1} subjects, "
                f"{int(full_off[-1])} residues) cut into {nshards} shards; shards 0..{world - 1} "
                f"searched, one per GPU ({int(full_off[job_hi] - full_off[0])} residues)")
    else:
        desc = (f"config{args.config}{'/4' if world > 1 else ''}: q{'+'.join(map(str, lens))} vs "
                f"{c['name'].split('_vs_')[-1]} synthetic DB ({len(full_off) - 1} subjects, "
                f"{int(full_off[-1])} residues)" +
                (f", sharded over {world} GPUs" if world > 1 else ""))
    return queries, db, full_off, (lo, hi), desc


# --------------------------------------------------------------- clocks

class ClockSampler:
    """nvidia-smi sampled every 100 ms while the timed region runs."""
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.tmp = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"], stdout=self.tmp,
                stderr=subprocess.DEVNULL)
        except OSError:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        self.proc.wait()
        self.tmp.flush()
        rows = []
        with open(self.tmp.name) as f:
            for line in f:
                parts = [p.strip() for p in line.split(",")]
                if len(parts) >= 8 and parts[0].replace(".", "").isdigit():
                    rows.append(parts)
        os.unlink(self.tmp.name)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm = [float(r[0]) for r in rows]
        mx = max(float(r[1]) for r in rows)
        loaded = [v for v in sm if v > 0.5 * mx] or sm
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({n for r in rows for n, v in zip(names, r[4:8]) if v == "Active"})
        return {"sm_mhz": statistics.median(loaded), "sm_max_mhz": mx, "reasons": reasons,
                "samples": len(rows), "power_w_max": max(float(r[2]) for r in rows
                                                         if r[2].replace(".", "").isdigit())}


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


def ncu_capture():
    """The committed ncu --set full summary of the search kernel (config 3)."""
    p = os.path.join(ROOT, "profiles", "ncu_search_kernel.json")
    if not os.path.exists(p):
        return {}
    with open(p) as f:
        return json.load(f)


# --------------------------------------------------------------- oracle (CPU) legs

def oracle_sample(queries, db):
    """The one oracle sample definition (the --impl reference arm and the
    cpu_baseline key): the first subjects of the workload's database holding
    ORACLE_SAMPLE_RQ residue-queries (all queries), re-searched every step."""
    # the oracle's work scales with residues x query length: the sample holds
    # ORACLE_SAMPLE_RQ residue-queries of a 1054-residue query's worth
    want = ORACLE_SAMPLE_RQ * 1054 // max(1, sum(len(q) for q in queries))
    nsub = max(1, min(int(np.searchsorted(db.offsets, want)), db.nseq))
    return nsub, db.offsets[: nsub + 1]


def oracle_rate(queries, db, steps, warmup):
    """Times the oracle (oracle/, as it stands) on the host's cores over the
    sample: residue-queries per second, mean step time."""
    from oracle import oracle as o
    Qs = [o.encode(q) for q in queries]
    tables = [o.neighbourhood(Q, o.blosum62(), 11) for Q in Qs]
    nsub, sub_off = oracle_sample(queries, db)
    codes = o.encode(db.ascii[: sub_off[-1]].tobytes())
    cores = os.cpu_count() or 1
    times = []
    for i in range(warmup + steps):
        t0 = time.perf_counter()
        for Q, tab in zip(Qs, tables):
            o.search(Q, codes, sub_off, table=tab, nthreads=cores, want_extensions=False)
        if i >= warmup:
            times.append(time.perf_counter() - t0)
    res = int(sub_off[-1]) * len(Qs)
    return {"value": res * len(times) / sum(times), "unit": UNIT, "cores": cores,
            "kind": "oracle", "ms_per_step": 1e3 * sum(times) / len(times),
            "sample": f"first {nsub} subjects ({int(sub_off[-1])} residues) of the workload's "
                      f"database x {len(Qs)} quer{'y' if len(Qs) == 1 else 'ies'} per step "
                      f"(scan + two-hit filter + extension; table prebuilt), {cores} pthreads, "
                      f"{steps} steps after {warmup} warm-up"}


def run_reference(args):
    rank, _, world = env_rank()
    if rank != 0:
        return  # rank 0 alone runs the CPU arm
    queries, db, full_off, (lo, hi), desc = workload(args, 0, 1)
    r = oracle_rate(queries, db, args.steps, args.warmup)
    value = r["value"]
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": r["ms_per_step"],
            "higher_is_better": True, "scaling": "weak" if args.config == 5 else "strong",
            "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": desc, "sample": r["sample"]},
            "cpu_baseline": r,
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# --------------------------------------------------------------- roofline inputs

def csrc_hash():
    """sha256 of the CUDA sources + header: ties a committed ncu capture to the
    build it was taken on."""
    import glob
    import hashlib
    h = hashlib.sha256()
    pkg = os.path.join(ROOT, "paper_conf_ipps_zhangwlf14_b200", "csrc")
    for f in sorted(glob.glob(os.path.join(pkg, "*.cu")) + glob.glob(os.path.join(pkg, "*.cuh"))
                    + [os.path.join(ROOT, "include", "blastp.h")]):
        with open(f, "rb") as fh:
            h.update(os.path.basename(f).encode() + b"\0" + fh.read())
    return h.hexdigest()[:16]


# SURVEY.md 8(d)'s operation budget of the method itself (not of any kernel):
# per DB residue scanned (word code + table probe), per hit (position load,
# diagonal, key, bin append, sort share, two-hit test) and per X-drop step.
OPS_PER_RESIDUE, OPS_PER_HIT, OPS_PER_XDROP_STEP = 10, 30, 5


def main():
    args = parse_args()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhangwlf14_b200 import blastp as bp
    from paper_conf_ipps_zhangwlf14_b200.dist import gather_hsps

    rank, local_rank, world = env_rank()
    # one GPU per rank; BLASTP_DIST_BACKEND=gloo lets several ranks share a
    # device (a functional check of the sharded path on a 1-GPU box)
    backend = os.environ.get("BLASTP_DIST_BACKEND", "nccl")
    local_rank = local_rank % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    stream = torch.cuda.current_stream()

    def all_reduce_max(t):
        if world > 1:
            if backend == "nccl":
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
            else:
                c = t.cpu()
                dist.all_reduce(c, op=dist.ReduceOp.MAX)
                t.copy_(c)
        return t

    queries, db, full_off, (lo, hi), desc = workload(args, rank, world)
    params = bp.Params()
    # setup outside the timed region, reported separately: the
    # query table build (a1) and the shard pack from pinned host memory (a2)
    bp.build_query_batch(queries[:1], params, device=local_rank, stream=stream).free()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    table = bp.build_query_batch(queries, params, device=local_rank, stream=stream)
    torch.cuda.synchronize()
    table_ms = 1e3 * (time.perf_counter() - t0)
    nq = len(queries)
    # pinned copy of this rank's residues: the e2e input and the pack source
    pinned = torch.empty(max(1, db.residues), dtype=torch.uint8, pin_memory=True)
    pinned[: db.residues].copy_(torch.from_numpy(db.ascii))
    base_ptr = pinned.data_ptr() - int(full_off[lo])
    # the offsets are step input too: pinned, so their copy is asynchronous
    off_pinned = torch.from_numpy(np.ascontiguousarray(full_off, dtype=np.int64)).pin_memory()
    full_off = off_pinned.numpy()
    nshards = shard_plan(args, world)
    bp.Database.from_pinned(base_ptr, full_off, rank, nshards, device=local_rank,
                            stream=stream).free()  # warm the allocator pool
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    gdb = bp.Database.from_pinned(base_ptr, full_off, rank, nshards, device=local_rank,
                                  stream=stream)
    torch.cuda.synchronize()
    pack_ms = 1e3 * (time.perf_counter() - t0)
    assert gdb.subject_base == lo and gdb.residues == db.residues
    cap = max(1 << 20, gdb.residues // 500 * nq)
    out = torch.empty((cap, 7), dtype=torch.int32, device=dev)
    cnt = torch.zeros(1, dtype=torch.int64, device=dev)

    # N > 1: the search kernels append into rank 0's buffer over NVLink
    # (dist.PeerHspBuffer, CUDA IPC) -- the gather fused into the search;
    # --gather nccl: per-rank buffers + the NCCL count/point-to-point gather
    peer = None
    if world > 1 and args.gather == "p2p":
        from paper_conf_ipps_zhangwlf14_b200.dist import PeerHspBuffer
        peer = PeerHspBuffer(cap * world)

    def search():
        bp.search_ungapped_device(table, gdb, out.data_ptr(), cap, cnt.data_ptr(), params, stream)

    def step(events=None):
        if peer is not None:
            peer.search(table, gdb, params, canonical=False, events=events)
            return
        if events:
            events[0].record(stream)
        search()
        if events:
            events[1].record(stream)
        if world > 1:
            n = int(cnt.item())
            gather_hsps(out[: min(n, cap)])

    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize()
    n_hsp = int(cnt.item())
    assert n_hsp <= cap, "HSP buffer too small"
    if peer is not None:
        search()  # this rank's own count (n_hsp) for the roofline's HSP bytes
        torch.cuda.synchronize()
        n_hsp = int(cnt.item())

    # ---- timed region -------------------------------------------------------
    clocks = ClockSampler(local_rank)
    clocks.start()
    time.sleep(0.3)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    t_start.record(stream)
    for k in range(args.steps):
        step(ev[k])
    t_end.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    elapsed_ms = t_start.elapsed_time(t_end)
    kern_ms = [a.elapsed_time(b) for a, b in ev]
    t = torch.tensor([elapsed_ms, statistics.mean(kern_ms)], dtype=torch.float64, device=dev)
    all_reduce_max(t)
    elapsed_ms, kern_avg_ms = float(t[0]), float(t[1])
    # whole-job residues: every shard a rank searched (configs 1-3: the DB)
    from paper_conf_ipps_zhangwlf14_b200.dist import shard_subjects
    total_residues = int(full_off[shard_subjects(full_off, world - 1, nshards)[1]] - full_off[0])
    value = total_residues * nq * args.steps / (elapsed_ms / 1e3)

    # ---- rooflines of the dominant kernel (the search kernel) --------------
    # (1) HBM, the metric's roofline: algorithmic bytes = 1 B
    # per residue per query pass + 28 B per HSP written, over the kernel's
    # CUDA-event time; DRAM traffic from the committed ncu capture when it was
    # taken on this very source tree (csrc hash), else null.
    peak, peak_src = peaks()
    alg_bytes = gdb.residues * nq + n_hsp * 28
    kern_s = kern_avg_ms / 1e3  # the mean search-kernel time, max over ranks
    achieved = alg_bytes / kern_s / 1e9
    capt = ncu_capture()
    src_sha = csrc_hash()
    fresh = bool(capt) and capt.get("csrc_sha") == src_sha and args.config == 3 and nq == 1
    frac_shard = gdb.residues / max(1, total_residues)
    traffic = capt["dram_bytes_per_launch"] * frac_shard if fresh else None
    capt_note = (f"{capt.get('source')} ({capt.get('kernel')}), csrc {capt.get('csrc_sha')}"
                 + (f", x {frac_shard:.4f} (this rank's residue share)" if fresh and world > 1
                    else "")) if fresh else \
        (f"no capture of this build (csrc {src_sha}; committed capture is csrc "
         f"{capt.get('csrc_sha')}, config 3 single query only)")
    hbm_roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": traffic, "kernel": "search kernel",
                "kernel_ms": 1e3 * kern_s, "alg_bytes_per_launch": alg_bytes // nq,
                "alg_bytes_per_unit": "1 B per residue per query pass + 28 B per HSP",
                "peak_source": peak_src, "traffic_source": capt_note}
    # (2) on chip: the METHOD's integer work (SURVEY 8(d) op budget x this
    # search's event counts, blastp_debug_stats, one traced launch outside the
    # timed region) per kernel second vs the measured integer-ALU roof of this
    # device (blastp_debug_alu_peak); the kernel's own warp instructions per
    # residue from the capture of this build beside it.
    onchip = None
    try:
        st = bp.debug_stats(table, gdb, params, stream)
        torch.cuda.synchronize()
        alu_peak = bp.debug_alu_peak(local_rank)
        ops = (OPS_PER_RESIDUE * gdb.residues * nq + OPS_PER_HIT * st["hits"]
               + OPS_PER_XDROP_STEP * st["xdrop_residues"])
        winst = (float(capt["smsp__inst_executed.sum"]) * frac_shard / max(1, gdb.residues * nq)
                 if fresh else None)
        onchip = {"bound": "alu", "achieved": ops / kern_s, "peak": alu_peak,
                  "unit": "int lane-ops/s", "frac": ops / kern_s / alu_peak,
                  "method_ops_per_residue": ops / max(1, gdb.residues * nq),
                  "ops_model": f"SURVEY 8(d): {OPS_PER_RESIDUE}/residue scanned + "
                               f"{OPS_PER_HIT}/hit + {OPS_PER_XDROP_STEP}/X-drop residue",
                  "events_per_residue": {k: st[k] / max(1, gdb.residues * nq)
                                         for k in ("hits", "passing", "extended", "accepted",
                                                   "xdrop_residues")},
                  "peak_source": "blastp_debug_alu_peak: measured integer add/xor lane-"
                                 "instructions/s, 32 warps per SM, this device",
                  "kernel_warp_inst_per_residue": winst,
                  "warp_inst_source": capt_note}
    except Exception as ex:  # noqa: BLE001 -- the roofline is a report, not the step
        onchip = {"error": str(ex)}

    # the step's result lands in pinned host memory (an asynchronous copy)
    hsp_host = torch.empty(cap * 7, dtype=torch.int32, pin_memory=True)

    def d2h_pinned(res):
        if res is None:
            return None
        flat = res.reshape(-1)
        dst = hsp_host[: flat.numel()] if flat.numel() <= hsp_host.numel() else \
            torch.empty(flat.numel(), dtype=torch.int32, pin_memory=True)
        dst.copy_(flat, non_blocking=True)
        return dst

    # ---- e2e through the C-ABI with host buffers ---------------------------
    e2e = None
    if not args.no_e2e and args.e2e_steps > 0:
        times, h2d, d2h = [], 0, 0
        for k in range(args.e2e_steps + 1):
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            # the public end-to-end entry point for a host-resident shard:
            # parts are copied H2D while the previous part is searched
            bp.search_host_db(table, base_ptr, full_off, out.data_ptr(), cap, cnt.data_ptr(),
                              params, shard_index=rank, num_shards=nshards, stream=stream)
            n = int(cnt.item())
            res = out[: min(n, cap)]
            if world > 1:
                res = gather_hsps(res)
            host = d2h_pinned(res)
            torch.cuda.synchronize()
            dt = time.perf_counter() - t0
            tt = torch.tensor([dt], dtype=torch.float64, device=dev)
            all_reduce_max(tt)
            if k > 0:  # first e2e step is a warm-up
                times.append(float(tt[0]))
            h2d = db.residues + 8 * (hi - lo + 1)
            d2h = 8 + (host.numel() * 4 if host is not None else 0)
        e2e = {"value": total_residues * nq / statistics.mean(times), "unit": UNIT,
               "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "ms_per_step": 1e3 * statistics.mean(times),
               "path": "blastp_search_host_db(pinned host; H2D of part k+1 overlaps the search "
                       "of part k) + "
                       + ("NCCL gather + " if world > 1 else "") + "D2H of the HSP list"}

    # ---- e2e from a formatted host database (the makeblastdb layout: the
    # shard packed once into pinned host memory, outside the timed region):
    # every step copies each part H2D on a copy stream and searches it as soon
    # as it lands (no per-part kernel or host synchronisation) + D2H of the HSPs
    e2e_fmt = None
    if not args.no_e2e and args.e2e_steps > 0 and hasattr(bp.lib, "blastp_format_host_db"):
        t0 = time.perf_counter()
        hdb = bp.format_host_db(base_ptr, full_off, shard_index=rank, num_shards=nshards,
                                stream=stream)
        fmt_ms = 1e3 * (time.perf_counter() - t0)
        times = []
        for k in range(args.e2e_steps + 1):
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            bp.search_formatted_db(table, hdb, out.data_ptr(), cap, cnt.data_ptr(), params,
                                   stream=stream)
            n = int(cnt.item())
            res = out[: min(n, cap)]
            if world > 1:
                res = gather_hsps(res)
            host = d2h_pinned(res)
            torch.cuda.synchronize()
            dt = time.perf_counter() - t0
            tt = torch.tensor([dt], dtype=torch.float64, device=dev)
            all_reduce_max(tt)
            if k > 0:
                times.append(float(tt[0]))
        h2d = hdb.host_bytes
        d2h = 8 + (host.numel() * 4 if host is not None else 0)
        e2e_fmt = {"value": total_residues * nq / statistics.mean(times), "unit": UNIT,
                   "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
                   "ms_per_step": 1e3 * statistics.mean(times),
                   "format_ms": fmt_ms, "parts": hdb.num_parts,
                   "path": "blastp_format_host_db once (pinned host image of the packed parts, "
                           "outside the timed region), then per step blastp_search_formatted_db "
                           "(H2D of part k+1 on a copy stream while part k is searched) + "
                           + ("NCCL gather + " if world > 1 else "") + "D2H of the HSP list"}
        hdb.free()

    # ---- e2e with the shard resident in HBM (a search service: the database
    # is loaded once; each step's inputs are the query strings, its result the
    # HSP list): query table build from host strings (H2D + GPU build) +
    # search + D2H of the HSPs through the C-ABI
    e2e_res = None
    if not args.no_e2e and args.e2e_steps > 0:
        times = []
        for k in range(args.e2e_steps + 1):
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            tq = bp.build_query_batch(queries, params, device=local_rank, stream=stream)
            bp.search_ungapped_device(tq, gdb, out.data_ptr(), cap, cnt.data_ptr(), params, stream)
            n = int(cnt.item())
            res = out[: min(n, cap)]
            if world > 1:
                res = gather_hsps(res)
            host = d2h_pinned(res)
            torch.cuda.synchronize()
            dt = time.perf_counter() - t0
            tq.free()
            tt = torch.tensor([dt], dtype=torch.float64, device=dev)
            all_reduce_max(tt)
            if k > 0:
                times.append(float(tt[0]))
        e2e_res = {"value": total_residues * nq / statistics.mean(times), "unit": UNIT,
                   "h2d_bytes_per_step": int(sum(len(q) for q in queries)),
                   "d2h_bytes_per_step": int(8 + (host.numel() * 4 if host is not None else 0)),
                   "ms_per_step": 1e3 * statistics.mean(times),
                   "path": "blastp_build_query_batch (host strings -> GPU table) + "
                           "blastp_search_ungapped_device on the HBM-resident shard + "
                           + ("NCCL gather + " if world > 1 else "") + "D2H of the HSP list"}

    # ---- the gapped consumer of this step's HSP list,
    # outside the headline: the rank's own list sorted (R11), then
    # blastp_gapped_extend_device timed with CUDA events on the stream
    gapped = None
    if not args.no_gapped and hasattr(bp.lib, "blastp_gapped_extend_device") and peer is None:
        try:
            search()
            torch.cuda.synchronize()
            ng = int(cnt.item())
            hs = out[:ng].clone()
            bp.sort_hsps_device(hs.data_ptr(), ng, stream)
            gout = torch.empty((max(ng, 1), 10), dtype=torch.int32, device=dev)
            gms = []
            for k in range(4):
                g0 = torch.cuda.Event(enable_timing=True)
                g1 = torch.cuda.Event(enable_timing=True)
                g0.record(stream)
                m = bp.gapped_extend_device(table, gdb, hs.data_ptr(), ng, gout.data_ptr(), ng,
                                            stream=stream)
                g1.record(stream)
                torch.cuda.synchronize()
                if k > 0:
                    gms.append(g0.elapsed_time(g1))
            gmean = statistics.mean(gms)
            # the two stages through the public host-result call (search +
            # canonical order + gapped stage + D2H of the alignments)
            ems = []
            for k in range(3):
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                al = bp.search_gapped(table, gdb, params, stream=stream)
                ems.append(1e3 * (time.perf_counter() - t0))
            gapped = {"hsps_in": ng, "alignments_out": int(m), "ms": gmean,
                      "hsps_per_s": ng / (gmean / 1e3),
                      "path": "blastp_gapped_extend_device on the rank's canonical device HSP "
                              "list (affine Gotoh X-drop, R18-R22; 3 timed calls after 1 warm-up)",
                      "search_plus_gapped_host_ms": statistics.median(ems[1:]),
                      "search_plus_gapped_path": "blastp_search_gapped (search, canonical sort, "
                                                 "gapped stage, alignments copied to the host; "
                                                 f"{len(al)} alignments), wall clock, median of 2 "
                                                 "after 1 warm-up"}
            del hs, gout
        except Exception as ex:  # noqa: BLE001 -- a report beside the headline
            gapped = {"error": str(ex)}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = oracle_rate(queries, db, steps=3, warmup=1)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": max(args.warmup, 3),
            "ms_per_step": elapsed_ms / args.steps, "higher_is_better": True,
            "scaling": "weak" if args.config == 5 else "strong", "vs_baseline": None,
            "dtype": "int32", "data": "synthetic",
            "config": {"workload": desc, "query_lens": [len(q) for q in queries],
                       "db_subjects": int(len(full_off) - 1), "db_residues": total_residues,
                       "shard_residues_rank0": int(gdb.residues),
                       "params": {"word_len": 3, "T": 11, "A": 40, "X": 16, "cutoff": 41,
                                  "filter": "LEFT"},
                       "l2": "inputs larger than L2 (DB shard >> 126 MB), no flush",
                       "hsps_per_step": n_hsp,
                       "parallelism": f"db-shard{world}" + (f" (of {nshards})" if nshards != world
                                                             else ""),
                       "gather": None if world == 1 else (
                           "p2p: every rank's search kernel appends its HSPs into rank 0's "
                           "buffer over NVLink (CUDA IPC, blastp_search_ungapped_append)"
                           if peer is not None else "NCCL count all_gather + point-to-point")},
            # the metric's roofline (HBM) and the on-chip one
            "roofline": hbm_roof,
            "onchip_roofline": onchip,
            "setup": {"query_table_ms": table_ms, "pack_db_ms": pack_ms,
                      "note": "outside the timed region: host table build (+ H2D) of all "
                              "queries; blastp_pack_db of the rank's shard from pinned host "
                              "memory (H2D + encode kernels)"},
            "clocks": clk,
            # e2e: the formatted host database streamed every step (the
            # production layout); the ASCII-streaming and HBM-resident paths
            # beside it
            "e2e": e2e_fmt or e2e,
            "e2e_ascii_db": e2e if e2e_fmt else None,
            "e2e_resident_db": e2e_res,
            "gpu_launches": args.steps * (table.launches(params)
                                          if hasattr(table, "launches") else nq),
            "cpu_baseline": cpu,
            "gapped_stage": gapped,
        }
        print(json.dumps(line), flush=True)
    if peer is not None:
        peer.free()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
