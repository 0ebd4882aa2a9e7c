"""Query-group budget sweep on config 5 (64 queries vs a scaled shard 0 of 8):
device time of the batch search per BLASTP_GROUP_LEN (read at table build),
CUDA events, median of 3 after 1 warm-up.

usage: python scripts/group_sweep.py [scale]
"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangwlf14_b200 import blastp as bp  # noqa: E402
from paper_conf_ipps_zhangwlf14_b200.dist import shard_subjects  # noqa: E402
from synth import CONFIGS, config_offsets, gen_db, gen_queries  # noqa: E402

scale = float(sys.argv[1]) if len(sys.argv) > 1 else 0.25
c = CONFIGS[5]
queries = gen_queries(c["query_seed"], 64, 100, 2000)
full_off = config_offsets(5, scale)
lo, hi = shard_subjects(full_off, 0, 8)
db = gen_db(c["db_seed"], c["plant_seed"], n_subjects=max(1, int(c["n_subjects"] * scale))
            if c["n_subjects"] else None,
            total_residues=max(1000, int(c["total_residues"] * scale)) if c["total_residues"]
            else None, mean_len=c["mean_len"], queries=queries, plant_frac=c["plant_frac"],
            subject_range=(lo, hi))
d = bp.pack_db(db.ascii, db.offsets - db.offsets[0])
stream = torch.cuda.current_stream()
cap = 1 << 23
out = torch.empty((cap, 7), dtype=torch.int32, device="cuda")
cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
print(f"shard: {d.nseq} subjects, {d.residues} residues", flush=True)
for budget in ("0", "768", "1024", "1280", "1536", "2048", "3072"):
    if budget == "0":
        os.environ["BLASTP_GROUP"] = "0"
    else:
        os.environ.pop("BLASTP_GROUP", None)
        os.environ["BLASTP_GROUP_LEN"] = budget
    t = bp.build_query_batch(queries, bp.Params(), stream=stream)
    ms = []
    for i in range(4):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        bp.search_ungapped_device(t, d, out.data_ptr(), cap, cnt.data_ptr(), stream=stream)
        b.record(stream)
        torch.cuda.synchronize()
        if i:
            ms.append(a.elapsed_time(b))
    g, alone, _ = t.groups
    print(f"budget {budget:>5}: {statistics.median(ms):9.2f} ms, launches {t.launches()}, "
          f"groups {g}, alone {alone}, {int(cnt.item())} HSPs", flush=True)
    t.free()
