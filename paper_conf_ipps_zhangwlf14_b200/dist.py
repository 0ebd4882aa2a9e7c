"""Multi-GPU: one process per GPU, subject-range shards, HSP gather over NCCL.

The database shards by contiguous subject ranges balanced by residues
(blastp_shard_range); subjects are independent, so each rank
searches its shard with no data-path communication.  The one exchange is the
result: every rank's HSP list (int32 x 7 per HSP, device memory) is gathered
to rank 0 -- one all_gather of the counts, then exact-size point-to-point
transfers into rank 0's output (gather_hsps) -- in rank order.  Because shards are contiguous in subject id and each rank's list
is canonical (R11), the concatenation is already canonical for one query;
for query batches rank 0 re-sorts (query_id major) on the GPU.

The collective code is backend-agnostic (NCCL on GPUs, gloo in the CPU tests).

PeerHspBuffer fuses the gather into the search instead: rank dst exports one
HSP buffer (CUDA IPC), every rank maps it, and every rank's search kernel
appends its HSPs straight into it over NVLink / NVSwitch
(blastp_search_ungapped_append) -- no gather step, the transfer overlaps the
search record by record; two tiny collectives order the count reset before
and every rank's kernel completion after.
"""
from __future__ import annotations

from typing import Callable

import numpy as np

HSP_FIELDS = 7
GAPPED_FIELDS = 10  # blastp_gapped records (the gapped consumer)


def shard_subjects(offsets: np.ndarray, rank: int, world: int) -> tuple[int, int]:
    """[lo, hi) of this rank's shard (same rule as blastp_shard_range)."""
    off = np.asarray(offsets, dtype=np.int64)
    total = int(off[-1] - off[0])

    def first_at(k: int) -> int:
        if k <= 0:
            return 0
        if k >= world:
            return len(off) - 1
        target = total * k // world
        return int(np.searchsorted(off - off[0], target, side="left"))

    lo, hi = first_at(rank), first_at(rank + 1)
    return lo, max(lo, hi)


def gather_hsps(local, group=None, dst: int = 0, fields: int = HSP_FIELDS):
    """Gather [n_r, fields] int32 record tensors of every rank onto rank `dst`
    (HSPs: 7 fields; gapped alignments: 10, gather_gapped).

    Returns the concatenation in rank order on rank dst (None elsewhere).
    One collective for the counts (all_gather_into_tensor of one int64 per
    rank, read back once), then exact-size point-to-point transfers batched
    in one group (NCCL: one ncclGroupStart/End): rank dst receives each
    rank's list straight into its slice of the output -- no padding, no
    concatenation copy, and no rank receives lists it does not keep.  Works
    for any torch.distributed backend; tensors stay on their device.
    """
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    if world == 1:
        return local
    if local.is_cuda and dist.get_backend(group) != "nccl":
        # gloo (functional multi-rank checks on one device): collectives on host
        out = gather_hsps(local.cpu(), group, dst, fields)
        return None if out is None else out.to(local.device)
    dev = local.device
    n = torch.tensor([local.shape[0]], dtype=torch.int64, device=dev)
    counts_t = torch.empty(world, dtype=torch.int64, device=dev)
    dist.all_gather_into_tensor(counts_t, n, group=group)
    counts = counts_t.tolist()  # the one host synchronisation of the gather
    glob = (lambda r: r) if group is None else (lambda r: dist.get_global_rank(group, r))
    ops = []
    out = None
    if rank == dst:
        out = local.new_empty((sum(counts), fields))
        offs = np.concatenate([[0], np.cumsum(counts)]).astype(np.int64)
        for r in range(world):
            if counts[r] == 0:
                continue
            view = out[int(offs[r]): int(offs[r + 1])]
            if r == rank:
                view.copy_(local)
            else:
                ops.append(dist.P2POp(dist.irecv, view, glob(r), group))
    elif counts[rank] > 0:
        ops.append(dist.P2POp(dist.isend, local.contiguous(), glob(dst), group))
    if ops:
        for req in dist.batch_isend_irecv(ops):
            req.wait()
    return out


def gather_gapped(local, group=None, dst: int = 0):
    """gather_hsps for [n_r, 10] int32 gapped alignments.  Shards partition
    the subjects and a (query, subject) pair's alignments are made on the
    shard holding the subject, so the rank-order concatenation is the whole
    database's gapped list (canonical for one query; batches re-sort by
    query id)."""
    return gather_hsps(local, group, dst, GAPPED_FIELDS)


def gapped_sharded(gapped_fn: Callable[[int, int], "object"], offsets: np.ndarray, group=None,
                   dst: int = 0):
    """Run `gapped_fn(lo, hi)` (search + gapped stage of this rank's shard,
    a [n, 10] int32 tensor with GLOBAL subject ids) and gather to rank dst."""
    import torch.distributed as dist
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    lo, hi = shard_subjects(offsets, rank, world)
    return gather_gapped(gapped_fn(lo, hi), group=group, dst=dst)


def search_sharded(search_fn: Callable[[int, int], "object"], offsets: np.ndarray, group=None,
                   dst: int = 0):
    """Run `search_fn(lo, hi)` on this rank's shard and gather the results.

    search_fn returns a [n, 7] int32 tensor of HSPs with GLOBAL subject ids.
    """
    import torch.distributed as dist
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    lo, hi = shard_subjects(offsets, rank, world)
    local = search_fn(lo, hi)
    return gather_hsps(local, group=group, dst=dst)


def gpu_shard_search(table, residues_local: np.ndarray, offsets_full: np.ndarray, rank: int,
                     world: int, params=None, capacity: int | None = None, stream=None):
    """Pack this rank's shard -- only its bytes need to be resident on the
    host -- and search it on the current CUDA device, all on `stream` (torch's
    current stream by default; the output buffers are allocated on it and the
    count is read after the search on it).  Returns a device [n, 7] int32
    tensor (global subject ids, canonical order)."""
    import torch

    from . import blastp as bp

    off = np.ascontiguousarray(offsets_full, dtype=np.int64)
    lo, hi = shard_subjects(off, rank, world)
    s = stream if stream is not None else torch.cuda.current_stream()
    with torch.cuda.stream(s):
        # libblastp reads residues at base + offsets[i] for the shard's subjects
        # only; hand it a base such that base + offsets[lo] is the local buffer.
        base = residues_local.ctypes.data - int(off[lo])
        db = bp.Database.from_pinned(base, off, rank, world, device=torch.cuda.current_device(),
                                     stream=s)
        assert db.subject_base == lo
        try:
            cap = capacity or max(4096, db.residues // 1000 * max(1, table.num_queries))
            while True:
                out = torch.empty((cap, 7), dtype=torch.int32, device="cuda")
                cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
                bp.search_ungapped_device(table, db, out.data_ptr(), cap, cnt.data_ptr(), params,
                                          s)
                n = int(cnt.item())  # a copy on s, after the search
                if n <= cap:
                    break
                cap = n + n // 4 + 1024
            res = out[:n]
            bp.sort_hsps_device(res.data_ptr(), n, s)
            return res
        finally:
            db.free()


class _DevMem:
    """A raw device range as a torch tensor (zero-copy, __cuda_array_interface__)."""

    def __init__(self, ptr: int, shape: tuple, typestr: str):
        self.__cuda_array_interface__ = {"shape": shape, "typestr": typestr, "data": (ptr, False),
                                         "strides": None, "version": 2}


class PeerHspBuffer:
    """One HSP buffer in rank `dst`'s device memory that the search kernels of
    every rank write into directly (blastp_search_ungapped_append over a CUDA
    IPC mapping: NVLink / NVSwitch stores between GPUs; ranks sharing one
    device, as in the 1-GPU tests, map it on that device).

    Layout: the int64 count at offset 0, `capacity` blastp_hsp records from
    offset HEADER.  search() returns the canonical [n, 7] int32 list on rank
    dst (a view of the buffer, valid until the next search) and None on the
    other ranks; a count above capacity re-runs the search with a buffer
    grown to fit (every rank reads the shared count, so all agree).
    """

    HEADER = 256

    def __init__(self, capacity: int, group=None, dst: int = 0):
        import torch
        import torch.distributed as dist

        from . import blastp as bp
        self._bp = bp
        self.group = group
        self.dst = dst
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.nccl = dist.get_backend(group) == "nccl"
        self.device = torch.cuda.current_device()
        self.ptr = 0
        self.capacity = 0
        self._alloc(max(1, int(capacity)))

    def _glob(self, r: int) -> int:
        import torch.distributed as dist
        return r if self.group is None else dist.get_global_rank(self.group, r)

    def _alloc(self, capacity: int):
        import torch
        import torch.distributed as dist
        bp = self._bp
        nbytes = self.HEADER + capacity * bp.HSP_BYTES
        h = bytes(bp.IPC_HANDLE_BYTES)
        if self.rank == self.dst:
            self.ptr, h = bp.ipc_alloc(self.device, nbytes)
        ht = torch.frombuffer(bytearray(h), dtype=torch.uint8)
        if self.nccl:
            ht = ht.cuda()
        dist.broadcast(ht, src=self._glob(self.dst), group=self.group)
        if self.rank != self.dst:
            self.ptr = bp.ipc_open(self.device, bytes(ht.cpu().numpy()))
        self.capacity = capacity
        self.count = torch.as_tensor(_DevMem(self.ptr, (1,), "<i8"), device="cuda")
        self.out = torch.as_tensor(_DevMem(self.ptr + self.HEADER, (capacity, HSP_FIELDS), "<i4"),
                                   device="cuda")

    def _sync(self):
        """Every rank's preceding work on its current stream is complete
        before any rank's following work: a stream-ordered all_reduce under
        NCCL; a host synchronisation + barrier under gloo."""
        import torch
        import torch.distributed as dist
        if self.nccl:
            dist.all_reduce(torch.ones(1, device="cuda"), group=self.group)
        else:
            torch.cuda.synchronize()
            dist.barrier(group=self.group)

    def free(self):
        import torch.distributed as dist
        if not self.ptr:
            return
        self.count = self.out = None
        self._sync()  # nobody still writes or reads
        if self.rank != self.dst:
            self._bp.ipc_close(self.ptr)
        dist.barrier(group=self.group)  # every mapping closed before the free
        if self.rank == self.dst:
            self._bp.ipc_free(self.ptr)
        self.ptr = 0

    def search(self, table, db, params=None, canonical: bool = True, events=None):
        """This rank's shard `db` searched into the shared buffer.  canonical:
        rank dst sorts the list (R11; HIT_DEDUP: de-duplicates it), else it is
        returned in append order.  events: optional (start, end) CUDA events
        recorded around this rank's search launch (kernel timing)."""
        bp = self._bp
        while True:
            if self.rank == self.dst:
                self.count.zero_()
            self._sync()  # the reset precedes every append
            if events:
                events[0].record()
            bp.search_ungapped_append(table, db, self.out.data_ptr(), self.capacity,
                                      self.count.data_ptr(), params)
            if events:
                events[1].record()
            self._sync()  # every rank's kernel (and its NVLink stores) completed
            n = int(self.count.item())
            if n <= self.capacity:
                break
            self._sync()  # every rank read the count before the buffer goes
            old = self.ptr
            self.count = self.out = None
            if self.rank != self.dst:
                bp.ipc_close(old)
            self._sync()
            if self.rank == self.dst:
                bp.ipc_free(old)
            self._alloc(n + n // 4 + 1024)
        if self.rank != self.dst:
            return None
        res = self.out[:n]
        if not canonical:
            return res
        p = params or table.params
        if p.ext_mode == bp.EXT_HIT_DEDUP:
            import torch
            kept = torch.zeros(1, dtype=torch.int64, device="cuda")
            bp.dedup_covered_device(res.data_ptr(), n, p.cutoff, kept.data_ptr())
            return res[: int(kept.item())]
        bp.sort_hsps_device(res.data_ptr(), n)
        return res
