"""Multi-process (world_size 2 and 3, gloo, CPU) coverage of the sharded path:
shard planning, global subject ids, and the count + padded all_gather that
brings every rank's HSPs to rank 0.  The per-shard search is the oracle here
(the GPU search is covered by tests/test_gpu_parity.py)."""
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q, ascii, offsets, result_path, empty_rank):
    sys.path.insert(0, ROOT)
    from oracle import oracle as o
    from paper_conf_ipps_zhangwlf14_b200.dist import search_sharded, shard_subjects

    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    try:
        def search_fn(lo, hi):
            if rank == empty_rank:
                return torch.zeros((0, 7), dtype=torch.int32)
            sub = offsets[lo:hi + 1]
            codes = o.encode(ascii[sub[0]:sub[-1]].tobytes())
            r = o.search(o.encode(q), codes, sub - sub[0], subject_base=lo)
            return torch.from_numpy(r.hsps.view(np.int32).reshape(-1, 7).copy())

        out = search_sharded(search_fn, offsets)
        lo, hi = shard_subjects(offsets, rank, world)
        assert 0 <= lo <= hi <= len(offsets) - 1
        if rank == 0:
            np.save(result_path, out.numpy())
        else:
            assert out is None
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,empty_rank", [(2, -1), (3, -1), (2, 1)])
def test_sharded_gather_equals_single_process(orc, tmp_path, world, empty_rank):
    from synth import config_workload
    (q,), db = config_workload(1)
    whole = orc.search(orc.encode(q), orc.encode(db.ascii.tobytes()), db.offsets).hsps
    path = str(tmp_path / "out.npy")
    mp.spawn(_worker, args=(world, _free_port(), q, db.ascii, db.offsets, path, empty_rank),
             nprocs=world, join=True)
    got = np.load(path)
    exp = whole.view(np.int32).reshape(-1, 7)
    if empty_rank < 0:
        assert (got == exp).all() and len(got) == len(exp) > 10
    else:
        from paper_conf_ipps_zhangwlf14_b200.dist import shard_subjects
        lo, hi = shard_subjects(db.offsets, empty_rank, world)
        keep = (exp[:, 1] < lo) | (exp[:, 1] >= hi)
        assert (got == exp[keep]).all()


def test_shard_subjects_matches_c_abi():
    from paper_conf_ipps_zhangwlf14_b200 import build
    build.build()
    from paper_conf_ipps_zhangwlf14_b200 import blastp as bp
    from paper_conf_ipps_zhangwlf14_b200.dist import shard_subjects
    rng = np.random.default_rng(5)
    off = np.concatenate([[7], 7 + np.cumsum(rng.integers(0, 900, size=5000))]).astype(np.int64)
    for world in (1, 2, 4, 8, 16):
        for k in range(world):
            assert shard_subjects(off, k, world) == bp.shard_range(off, k, world)


def _gapped_worker(rank, world, port, q, ascii, offsets, result_path):
    sys.path.insert(0, ROOT)
    from oracle import oracle as o
    from paper_conf_ipps_zhangwlf14_b200.dist import gapped_sharded

    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    try:
        def gapped_fn(lo, hi):
            sub = offsets[lo:hi + 1]
            codes = o.encode(ascii[sub[0]:sub[-1]].tobytes())
            r = o.search(o.encode(q), codes, sub - sub[0], subject_base=lo)
            g = o.gapped_hsps([o.encode(q)], codes, sub - sub[0], r.hsps, subject_base=lo)
            return torch.from_numpy(g.view(np.int32).reshape(-1, 10).copy())

        out = gapped_sharded(gapped_fn, offsets)
        if rank == 0:
            np.save(result_path, out.numpy())
        else:
            assert out is None
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_gapped_gather_equals_whole_db(orc, tmp_path, world):
    """The gapped consumer per shard (the oracle standing in for each rank's
    GPU stage) gathered to rank 0 equals the gapped stage over the whole
    database: (query, subject) pairs never span shards."""
    from synth import config_workload
    (q,), db = config_workload(1)
    codes = orc.encode(db.ascii.tobytes())
    u = orc.search(orc.encode(q), codes, db.offsets).hsps
    whole = orc.gapped_hsps([orc.encode(q)], codes, db.offsets, u)
    path = str(tmp_path / "gapped.npy")
    mp.spawn(_gapped_worker, args=(world, _free_port(), q, db.ascii, db.offsets, path),
             nprocs=world, join=True)
    got = np.load(path)
    exp = whole.view(np.int32).reshape(-1, 10)
    assert len(got) == len(exp) > 10 and (got == exp).all()
