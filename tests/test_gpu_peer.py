"""The fused search + gather (dist.PeerHspBuffer, blastp_search_ungapped_append):
2 and 3 processes share the one GPU of the box (gloo for the host-side
collectives, the exported buffer mapped through CUDA IPC on that device);
every rank's search kernel appends into rank 0's buffer and rank 0's list must
equal the oracle's search of the whole database."""
import os
import socket
import sys

import numpy as np
import pytest
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, queries, ascii, offsets, result_path, cap, ext_mode, repeats,
            filter_mode=0):
    sys.path.insert(0, ROOT)
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhangwlf14_b200 import blastp as bp
    from paper_conf_ipps_zhangwlf14_b200.dist import PeerHspBuffer

    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    try:
        p = bp.Params(ext_mode=ext_mode, filter_mode=filter_mode)
        table = bp.build_query_batch(queries, p)
        db = bp.pack_db(ascii, offsets, rank, world)
        buf = PeerHspBuffer(cap)
        outs = []
        for _ in range(repeats):  # the buffer is reused (count reset each search)
            res = buf.search(table, db, p)
            outs.append(None if res is None else res.cpu().numpy().copy())
        grown = buf.capacity
        buf.free()
        db.free()
        table.free()
        if rank == 0:
            for o in outs[1:]:
                assert (o == outs[0]).all()
            np.save(result_path, outs[0])
            np.save(result_path + ".cap.npy", np.array([grown]))
        else:
            assert all(o is None for o in outs)
    finally:
        dist.destroy_process_group()


def _oracle_hsps(orc, queries, db, filter_mode=0):
    parts = []
    for qi, q in enumerate(queries):
        r = orc.search(orc.encode(q), orc.encode(db.ascii.tobytes()), db.offsets,
                       orc.Params(filter_mode=filter_mode))
        h = r.hsps.view(np.int32).reshape(-1, 7).copy()
        h[:, 0] = qi
        parts.append(h)
    allh = np.concatenate(parts)
    return allh[np.lexsort(allh.T[::-1])]


@pytest.mark.parametrize("world,cap,ext,filt", [(2, 1 << 16, "diagonal", 0),
                                                 (3, 7, "diagonal", 0),
                                                 (2, 1 << 16, "hit_dedup", 0),
                                                 (3, 1 << 16, "diagonal", 2),
                                                 (2, 100, "diagonal", 3)])
def test_peer_append_equals_oracle(orc, tmp_path, world, cap, ext, filt):
    """filt: 0 LEFT (block kernel), 2 STATEFUL / 3 STATEFUL_RB (warp kernel)."""
    from paper_conf_ipps_zhangwlf14_b200 import blastp as bp
    from synth import config_workload
    (q,), db = config_workload(1)
    queries = [q, q[:60]]
    exp = _oracle_hsps(orc, queries, db, filt)
    path = str(tmp_path / "out.npy")
    ext_mode = {"diagonal": bp.EXT_DIAGONAL, "hit_dedup": bp.EXT_HIT_DEDUP}[ext]
    mp.spawn(_worker, args=(world, _free_port(), queries, db.ascii, db.offsets, path, cap,
                            ext_mode, 2, filt), nprocs=world, join=True)
    got = np.load(path)
    assert len(exp) > 10
    assert got.shape == exp.shape and (got == exp).all()
    if cap < len(exp):  # the overflow path grew the buffer
        assert int(np.load(path + ".cap.npy")[0]) >= len(exp)


def test_peer_append_empty_rank(orc, tmp_path):
    """More ranks than subjects: some ranks search an empty shard and append
    nothing; rank 0's list is still the oracle's."""
    from synth import config_workload
    (q,), db = config_workload(1)
    keep = 2
    off = db.offsets[: keep + 1].copy()
    ascii = db.ascii[: int(off[-1])].copy()

    class _Db:
        pass
    small = _Db()
    small.ascii, small.offsets = ascii, off
    exp = _oracle_hsps(orc, [q], small)
    path = str(tmp_path / "out.npy")
    mp.spawn(_worker, args=(4, _free_port(), [q], ascii, off, path, 1 << 12, 0, 1),
             nprocs=4, join=True)
    got = np.load(path)
    assert got.shape == exp.shape and (got == exp).all()
