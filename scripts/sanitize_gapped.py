"""Small gapped-stage runs for compute-sanitizer: config 1 (scaled) through
blastp_search_gapped with every code path of gapped.cu -- default, pairs
redone with big rings (BLASTP_GAPPED_RING=16), every traceback re-run in pass
2 over several store windows (TBBUF=0, STORE=4096), small logs (TBBUF=256),
and the pipelined batch with unit-buffer overflow -- each checked against the
gapped oracle, so a sanitizer run is also a parity run."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from oracle import oracle as orc  # noqa: E402
from paper_conf_ipps_zhangwlf14_b200 import blastp as bp  # noqa: E402
from synth import config_workload, gen_db, gen_queries  # noqa: E402

KNOBS = ("BLASTP_GAPPED_RING", "BLASTP_GAPPED_TBBUF", "BLASTP_GAPPED_STORE", "BLASTP_GAPPED_PIPE",
         "BLASTP_PIPE_CAP")


def expected(queries, ascii, off):
    codes = orc.encode(ascii.tobytes())
    off = np.asarray(off, np.int64)
    lists = [orc.search(orc.encode(q), codes, off, orc.Params(), query_id=k).hsps
             for k, q in enumerate(queries)]
    u = np.concatenate(lists)
    u = np.sort(u, order=list(u.dtype.names))
    return orc.gapped_hsps([orc.encode(q) for q in queries], codes, off, u)


def run(queries, ascii, off, knobs, label):
    for k in KNOBS:
        os.environ.pop(k, None)
    os.environ.update(knobs)
    t = bp.build_query_batch(queries) if len(queries) > 1 else bp.build_query_table(queries[0])
    d = bp.pack_db(ascii, off)
    g = bp.search_gapped(t, d)
    t.free()
    d.free()
    e = expected(queries, ascii, off)
    assert len(g) == len(e) and (g.view(np.int32) == e.view(np.int32)).all(), (label, len(g), len(e))
    print(f"ok {label}: {len(g)} alignments", flush=True)


def main():
    (q1,), db1 = config_workload(1, scale=0.3)
    for knobs in ({}, {"BLASTP_GAPPED_RING": "16"},
                  {"BLASTP_GAPPED_TBBUF": "0", "BLASTP_GAPPED_STORE": "4096"},
                  {"BLASTP_GAPPED_TBBUF": "256"}):
        run([q1], db1.ascii, db1.offsets, knobs, f"config1 {knobs}")
    qs = gen_queries(77, 6, 100, 600)
    db = gen_db(78, 79, n_subjects=400, mean_len=300.0, queries=qs, plant_frac=0.2)
    run(qs, db.ascii, db.offsets, {"BLASTP_GAPPED_PIPE": "1", "BLASTP_PIPE_CAP": "7"},
        "batch pipelined, unit overflow")
    bp.trim_memory(0) if hasattr(bp, "trim_memory") else None
    try:
        import torch
        torch.cuda.empty_cache()
    except Exception:  # noqa: BLE001
        pass


if __name__ == "__main__":
    main()
