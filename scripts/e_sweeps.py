"""The paper's kernel-design experiments re-run on B200 (one process, one box,
interleaved rounds, median device ms per search; HSP lists must agree):

  E2 (Fig. 15): X-drop scores from BLOSUM62 + query codes vs a
     PSSM in shared memory vs a PSSM in global memory, queries 127 / 517 / 1054
     (BLASTP_SCORE=blosum|pssm|pssm_global; block kernel).
  E1 (Fig. 14): bins per warp in the CTA variant
     (the paper's binning kernel): producer warps np -> a window of 32 np
     positions binned into 32 np + Lq diagonal bins, (32 np + Lq) / np per warp
     (BLASTP_CTA_NP / BLASTP_CTA_NC; query 517).

usage: python scripts/e_sweeps.py <out.json> [rounds] [db_scale]"""
import json
import os
import statistics
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_zhangwlf14_b200 import blastp as bp  # noqa: E402
from synth import CONFIGS, config_workload, gen_query  # noqa: E402


def time_search(t, d, p, steps=3):
    s = torch.cuda.current_stream()
    cap = d.residues // 200 + (1 << 20)
    out = torch.empty((cap, 7), dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    bp.search_ungapped_device(t, d, out.data_ptr(), cap, cnt.data_ptr(), p, s)  # warm
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(s)
    for _ in range(steps):
        bp.search_ungapped_device(t, d, out.data_ptr(), cap, cnt.data_ptr(), p, s)
    e1.record(s)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / steps, int(cnt.item())


def sweep(name, arms, t, d, p, rounds, env_key):
    times = {a: [] for a in arms}
    counts = {}
    for _ in range(rounds):
        for arm, envs in arms.items():
            saved = {k: os.environ.get(k) for k in envs}
            os.environ.update(envs)
            try:
                ms, n = time_search(t, d, p)
            finally:
                for k, v in saved.items():
                    if v is None:
                        os.environ.pop(k, None)
                    else:
                        os.environ[k] = v
            times[arm].append(ms)
            counts.setdefault(arm, n)
            assert counts[arm] == n
    assert len(set(counts.values())) == 1, counts
    res = {a: {"ms": statistics.median(v), "runs": v} for a, v in times.items()}
    print(f"== {name}: " + "  ".join(f"{a} {r['ms']:.3f} ms" for a, r in res.items()), flush=True)
    return res


def main():
    out_path = sys.argv[1]
    rounds = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    scale = float(sys.argv[3]) if len(sys.argv) > 3 else 1.0
    torch.cuda.set_device(0)
    (_,), db = config_workload(3, scale=scale)
    d = bp.pack_db(db.ascii, db.offsets)
    report = {"db": f"config-3 DB x {scale} ({db.residues} residues, {db.nseq} subjects)",
              "E2": {}, "E1": {}}
    seeds = {127: CONFIGS[1]["query_seed"], 517: CONFIGS[2]["query_seed"],
             1054: CONFIGS[3]["query_seed"]}
    p = bp.Params()
    for L in (127, 517, 1054):
        t = bp.build_query_table(gen_query(seeds[L], L), p)
        arms = {"blosum62": {"BLASTP_SCORE": "blosum"}, "pssm_smem": {"BLASTP_SCORE": "pssm"},
                "pssm_global": {"BLASTP_SCORE": "pssm_global"}}
        report["E2"][f"q{L}"] = sweep(f"E2 q{L}", arms, t, d, p, rounds, "BLASTP_SCORE")
    t = bp.build_query_table(gen_query(seeds[517], 517), p)
    arms = {}
    for np_, nc in ((4, 8), (8, 8), (12, 8), (16, 8), (20, 8), (24, 8), (28, 4)):
        bins = (32 * np_ + 517) / np_
        arms[f"np{np_}_nc{nc}_bins{bins:.0f}"] = {"BLASTP_KERNEL": "cta", "BLASTP_CTA_NP": str(np_),
                                                  "BLASTP_CTA_NC": str(nc)}
    report["E1"]["q517"] = sweep("E1 q517 (cta)", arms, t, d, p, rounds, "BLASTP_CTA_NP")
    with open(out_path, "w") as f:
        json.dump(report, f, indent=1)


if __name__ == "__main__":
    main()
