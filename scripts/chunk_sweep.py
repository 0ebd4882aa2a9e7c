"""Chunk-size sweep (BLASTP_CHUNK, read at pack time) on configs 1 and 2: device time
per search (CUDA events, median of 20 after 3 warm-ups).

usage: python scripts/chunk_sweep.py [configs e.g. 1,2] [chunk sizes e.g. 128,256]
"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_zhangwlf14_b200 import blastp as bp  # noqa: E402
from synth import config_workload  # noqa: E402

stream = torch.cuda.current_stream()
cfgs = [int(x) for x in sys.argv[1].split(",")] if len(sys.argv) > 1 else [1, 2]
sizes = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else \
    [128, 256, 384, 512, 768, 1024]
for cfg in cfgs:
    (q,), db = config_workload(cfg)
    t = bp.build_query_table(q, stream=stream)
    cap = 1 << 20
    out = torch.empty((cap, 7), dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    for chunk in [None] + sizes:
        if chunk is None:
            os.environ.pop("BLASTP_CHUNK", None)
        else:
            os.environ["BLASTP_CHUNK"] = str(chunk)
        d = bp.pack_db(db.ascii, db.offsets, stream=stream)
        torch.cuda.synchronize()
        ms = []
        for i in range(23 if cfg < 3 else 8):
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record(stream)
            bp.search_ungapped_device(t, d, out.data_ptr(), cap, cnt.data_ptr(), stream=stream)
            b.record(stream)
            torch.cuda.synchronize()
            if i >= 3:
                ms.append(a.elapsed_time(b))
        print(f"config {cfg} chunk {chunk or 'default':>7}: {statistics.median(ms):.4f} ms "
              f"({int(cnt.item())} HSPs)", flush=True)
        d.free()
