"""The gapped stage on config 5's shard 0 of 8 (64 queries x 1.9G residues,
~21.5M HSPs): both pass-1a forms, CUDA events on the stream, verbose stats."""
import os
import sys
from types import SimpleNamespace

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from bench import workload  # noqa: E402  (the bench's own shard generation)
from paper_conf_ipps_zhangwlf14_b200 import blastp as bp  # noqa: E402

args = SimpleNamespace(config=5, scale=1.0, query_lens="1054", gpus=1)
queries, db, full_off, (lo, hi), desc = workload(args, 0, 1)
s = torch.cuda.current_stream()
t = bp.build_query_batch(queries, stream=s)
d = bp.pack_db(db.ascii, full_off[lo:hi + 1] - full_off[lo], stream=s)
u = bp.search_ungapped(t, d, stream=s)
dev = torch.from_numpy(u.view(np.int32).reshape(-1, 7).copy()).cuda()
out = torch.zeros((len(u), 10), dtype=torch.int32, device="cuda")
for form in ("warp", "thread", "warp", "thread"):
    os.environ["BLASTP_GAPPED_KERNEL"] = form
    os.environ["BLASTP_GAPPED_VERBOSE"] = "1"
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(s)
    n = bp.gapped_extend_device(t, d, dev.data_ptr(), len(u), out.data_ptr(), len(u), stream=s)
    e1.record(s)
    torch.cuda.synchronize()
    sys.stderr.flush()
    print(f"{form}: {len(u)} HSPs -> {n} alignments, {e0.elapsed_time(e1):.1f} ms", flush=True)
