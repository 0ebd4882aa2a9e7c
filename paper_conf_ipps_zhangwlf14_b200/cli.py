"""Command line: ungapped BLASTP search of FASTA queries against a FASTA database.

    python -m paper_conf_ipps_zhangwlf14_b200.cli QUERIES.fa DB.fa [options] > hits.tsv

Reads both files, packs the database onto the GPU (or streams it from a
formatted host image with --stream), searches every query (a batch: short
queries share one scan as query groups) and prints one tab-separated line per
HSP in canonical order (R11):

    query  subject  q_start  s_start  length  score  diagonal

with FASTA identifiers (first word of the header) and 0-based starts; with
--gapped, the gapped consumer of those HSPs (R18-R22) instead, one
line per gapped alignment:

    query  subject  q_start  q_end  s_start  s_end  score  identities  gap_opens  gap_residues

(ends exclusive).  All of
the search runs in libblastp.so (include/blastp.h); this module only parses
FASTA and formats the result.  Options map to blastp_params (P:L143-144 T,
P:L1344-1351 A, Fig. 8 X; R3-R15).
"""
from __future__ import annotations

import argparse
import sys

import numpy as np


def read_fasta(path: str) -> tuple[list[str], bytes, np.ndarray]:
    """(ids, concatenated residues, offsets[n+1]) of a FASTA file; residue
    letters are kept as written (the library validates and encodes them)."""
    ids: list[str] = []
    seqs: list[bytes] = []
    cur: list[bytes] = []
    with open(path, "rb") as f:
        for raw in f:
            line = raw.strip()
            if not line:
                continue
            if line.startswith(b">"):
                if ids:
                    seqs.append(b"".join(cur))
                cur = []
                head = line[1:].split()
                ids.append(head[0].decode(errors="replace") if head else f"seq{len(ids)}")
            else:
                if not ids:
                    raise ValueError(f"{path}: sequence data before the first '>' header")
                cur.append(line)
    if ids:
        seqs.append(b"".join(cur))
    lens = np.array([len(s) for s in seqs], dtype=np.int64)
    off = np.zeros(len(seqs) + 1, dtype=np.int64)
    np.cumsum(lens, out=off[1:])
    return ids, b"".join(seqs), off


def main(argv: list[str] | None = None) -> int:
    ap = argparse.ArgumentParser(description=__doc__.split("\n\n")[0])
    ap.add_argument("queries", help="query FASTA")
    ap.add_argument("db", help="database FASTA")
    ap.add_argument("--threshold", "-T", type=int, default=11)
    ap.add_argument("--window", "-A", type=int, default=40)
    ap.add_argument("--xdrop", "-X", type=int, default=16)
    ap.add_argument("--cutoff", type=int, default=41)
    ap.add_argument("--filter", choices=["left", "either", "stateful", "stateful_rb"], default="left")
    ap.add_argument("--ext", choices=["diagonal", "hit", "window"], default="diagonal")
    ap.add_argument("--stream", action="store_true",
                    help="keep the database in pinned host memory (formatted image) and stream it "
                         "(each part's copy overlaps the previous part's search; the shard's "
                         "device image must fit in HBM)")
    ap.add_argument("--gapped", action="store_true",
                    help="run the gapped stage on the HSPs (blastp_search_gapped) and print the "
                         "gapped alignments (resident database, one GPU)")
    ap.add_argument("--gap-open", type=int, default=11)
    ap.add_argument("--gap-extend", type=int, default=1)
    ap.add_argument("--gapped-xdrop", type=int, default=38)
    ap.add_argument("--gapped-cutoff", type=int, default=41)
    ap.add_argument("--device", type=int, default=0)
    ap.add_argument("--distributed", action="store_true",
                    help="one process per GPU under torchrun: each rank searches a residue-"
                         "balanced subject range, HSPs gathered to rank 0 (dist.py), which prints")
    ap.add_argument("--gather", choices=["p2p", "nccl"], default="p2p",
                    help="--distributed: the search kernels append into rank 0's buffer over "
                         "NVLink (CUDA IPC), or per-rank lists gathered with NCCL")
    args = ap.parse_args(argv)
    if args.gapped and (args.stream or args.distributed):
        ap.error("--gapped runs on a resident database on one GPU (no --stream / --distributed)")

    import os

    import torch

    from . import blastp as bp
    rank, world = 0, 1
    if args.distributed:
        import torch.distributed as dist
        rank = int(os.environ.get("RANK", "0"))
        world = int(os.environ.get("WORLD_SIZE", "1"))
        args.device = int(os.environ.get("LOCAL_RANK", "0")) % max(1, torch.cuda.device_count())
        torch.cuda.set_device(args.device)
        dist.init_process_group(os.environ.get("BLASTP_DIST_BACKEND", "nccl"))

    qids, qres, qoff = read_fasta(args.queries)
    sids, sres, soff = read_fasta(args.db)
    if not qids:
        print("no queries", file=sys.stderr)
        return 1
    queries = [qres[qoff[i]:qoff[i + 1]] for i in range(len(qids))]
    # a query shorter than one word (3 residues) has no hits: skipped with a
    # warning, the others keep their ids
    keep = [i for i, q in enumerate(queries) if len(q) >= 3]
    for i in range(len(queries)):
        if i not in keep:
            print(f"warning: query {qids[i]} shorter than 3 residues: skipped", file=sys.stderr)
    if not keep:
        print("no searchable queries", file=sys.stderr)
        return 1
    qids = [qids[i] for i in keep]
    queries = [queries[i] for i in keep]
    p = bp.Params(threshold=args.threshold, window=args.window, xdrop=args.xdrop,
                  cutoff=args.cutoff,
                  filter_mode={"left": bp.FILTER_LEFT, "either": bp.FILTER_EITHER,
                               "stateful": bp.FILTER_STATEFUL,
                               "stateful_rb": bp.FILTER_STATEFUL_RB}[args.filter],
                  ext_mode={"diagonal": bp.EXT_DIAGONAL, "hit": bp.EXT_HIT,
                            "window": bp.EXT_WINDOW}[args.ext])
    torch.cuda.set_device(args.device)
    table = bp.build_query_batch(queries, p, device=args.device)
    residues = np.frombuffer(sres, dtype=np.uint8)
    if world > 1:
        # this rank's shard (blastp_shard_range), HSPs with global subject ids,
        # gathered in rank order (canonical per query; re-sorted on rank 0)
        import torch.distributed as dist

        from .dist import gather_hsps
        # an error on one rank (e.g. a bad residue in its shard only) is agreed
        # on by all ranks before the gather, so none waits forever in it
        err = None
        d = None
        local = torch.zeros((0, 7), dtype=torch.int32, device="cuda")
        try:
            d = bp.pack_db(residues, soff, rank, world, device=args.device)
            if args.gather == "nccl":
                local = torch.from_numpy(bp.search_ungapped(table, d, p).view(np.int32)
                                         .reshape(-1, 7).copy()).cuda()
                d.free()
                d = None
        except bp.BlastpError as ex:
            err = ex
        flag = torch.tensor([1 if err else 0], dtype=torch.int32,
                            device="cuda" if dist.get_backend() == "nccl" else "cpu")
        dist.all_reduce(flag, op=dist.ReduceOp.MAX)
        if int(flag.item()):
            dist.destroy_process_group()
            if err:
                print(f"rank {rank}: {err}", file=sys.stderr)
            return 1
        if args.gather == "p2p":
            # every rank's search kernel stores its HSPs into rank 0's buffer
            from .dist import PeerHspBuffer
            buf = PeerHspBuffer(max(1 << 16, len(residues) // 1000 * len(queries)))
            res = buf.search(table, d, p)  # canonical on rank 0
            hsps = None if res is None else res.cpu().numpy()
            buf.free()
            d.free()
            dist.destroy_process_group()
            if rank != 0:
                return 0
        else:
            allh = gather_hsps(local)
            dist.destroy_process_group()
            if rank != 0:
                return 0
            n = allh.shape[0]
            flat = allh.contiguous().view(-1)
            bp.sort_hsps_device(flat.data_ptr(), n)
            hsps = flat.view(n, 7).cpu().numpy()
    elif args.stream:
        h = bp.format_host_db(residues, soff, device=args.device)
        cap = max(1 << 16, len(residues) // 1000 * len(queries))  # grown below if short
        while True:
            out = torch.empty(cap * 7, dtype=torch.int32, device="cuda")
            cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
            bp.search_formatted_db(table, h, out.data_ptr(), cap, cnt.data_ptr(), p)
            n = int(cnt.item())
            if n <= cap:
                break
            cap = n + 1024
        bp.sort_hsps_device(out.data_ptr(), n)
        hsps = out[: n * 7].view(n, 7).cpu().numpy()
        h.free()
    elif args.gapped:
        db = bp.pack_db(residues, soff, device=args.device)
        gp = bp.GappedParams(args.gap_open, args.gap_extend, args.gapped_xdrop, args.gapped_cutoff)
        al = bp.search_gapped(table, db, p, gp)
        db.free()
        w = sys.stdout.write
        for qi, si, q0, q1, s0, s1, sc, idn, gop, gl in al.view(np.int32).reshape(-1, 10).tolist():
            w(f"{qids[qi]}\t{sids[si]}\t{q0}\t{q1}\t{s0}\t{s1}\t{sc}\t{idn}\t{gop}\t{gl}\n")
        return 0
    else:
        db = bp.pack_db(residues, soff, device=args.device)
        hsps = bp.search_ungapped(table, db, p).view(np.int32).reshape(-1, 7)
        db.free()
    w = sys.stdout.write
    for qi, si, diag, qs, ss, ln, sc in hsps.tolist():
        w(f"{qids[qi]}\t{sids[si]}\t{qs}\t{ss}\t{ln}\t{sc}\t{diag}\n")
    return 0


if __name__ == "__main__":
    sys.exit(main())
