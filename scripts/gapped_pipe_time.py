"""Fig. 12 overlap on one GPU: search_gapped over a query batch, pipelined
(unit u+1 searched while unit u is gapped on a second stream) vs the two
stages one after the other (BLASTP_GAPPED_PIPE=0), and the search alone.
Config 4's three queries and config 5's 64 queries against config 3's
database (device-resident), CUDA events on the launch stream."""
import os
import sys

import torch

from paper_conf_ipps_zhangwlf14_b200 import blastp as bp
from synth import CONFIGS, config_workload, gen_queries, gen_query

(_,), db = config_workload(3)
s = torch.cuda.current_stream()
d = bp.pack_db(db.ascii, db.offsets, stream=s)
sets = {"config4 (127/517/1054)": [gen_query(CONFIGS[1]["query_seed"], 127),
                                   gen_query(CONFIGS[2]["query_seed"], 517),
                                   gen_query(CONFIGS[3]["query_seed"], 1054)],
        "config5 queries (64 x 100-2000)": gen_queries(CONFIGS[5]["query_seed"], 64, 100, 2000)}


def timed(fn, reps=3):
    ms = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(s)
        r = fn()
        e1.record(s)
        torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
    return r, sorted(ms)[len(ms) // 2]


for name, qs in sets.items():
    t = bp.build_query_batch(qs, stream=s)
    g, a, _ = t.groups
    u, ms_u = timed(lambda: bp.search_ungapped(t, d, stream=s))
    os.environ["BLASTP_GAPPED_PIPE"] = "0"
    r0, ms_seq = timed(lambda: bp.search_gapped(t, d, stream=s))
    os.environ["BLASTP_GAPPED_PIPE"] = "1"
    r1, ms_pipe = timed(lambda: bp.search_gapped(t, d, stream=s))
    same = len(r0) == len(r1) and bool((r0 == r1).all())
    print(f"{name}: {g} groups + {a} alone; search {ms_u:.1f} ms ({len(u)} HSPs); search+gapped "
          f"sequential {ms_seq:.1f} ms, pipelined {ms_pipe:.1f} ms ({len(r1)} alignments, "
          f"identical={same})", flush=True)
