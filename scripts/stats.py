"""Per-residue event rates of the GPU search (blastp_debug_stats) on the
BASELINE configs -- compares with SURVEY.md section 8's hit statistics."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_zhangwlf14_b200 import blastp as bp  # noqa: E402
from synth import config_workload  # noqa: E402

out = {}
for cfg, scale in [(1, 1.0), (2, 1.0), (3, 0.1)]:
    (q,), db = config_workload(cfg, scale=scale)
    t = bp.build_query_table(q)
    d = bp.pack_db(db.ascii, db.offsets)
    s = bp.debug_stats(t, d)
    R = db.residues
    rates = {k: v / R for k, v in s.items()}
    rates["passing_frac"] = s["passing"] / max(1, s["hits"])
    rates["hits_per_round"] = s["hits"] / max(1, s["rounds"])
    rates["conflict_round_frac"] = s["conflict_rounds"] / max(1, s["rounds"])
    rates["xdrop_residues_per_ext"] = s["xdrop_residues"] / max(1, s["extended"])
    rates["xdrop_lane_util"] = s["xdrop_residues"] / max(1, s["xdrop_lane_slots"])
    rates["speculative_waste"] = 1 - s["accepted"] / max(1, s["extended"])
    out[f"config{cfg}@{scale}"] = {"residues": R, "counts": s, "rates": rates}
    print(f"config {cfg} (scale {scale}, {R} residues, q{len(q)}):")
    for k, v in rates.items():
        print(f"   {k:24s} {v:.5g}")
json.dump(out, open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/stats.json", "w"), indent=1)
