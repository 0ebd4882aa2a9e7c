"""The FASTA command line (paper_conf_ipps_zhangwlf14_b200/cli.py): FASTA parsing
on CPU; on the GPU its TSV equals the oracle's HSPs (resident and streamed DB)."""
import os

import numpy as np
import pytest

from synth import gen_db, gen_query


def _write_fasta(path, ids, seqs, width=60):
    with open(path, "w") as f:
        for i, s in zip(ids, seqs):
            f.write(f">{i} description text\n")
            for k in range(0, len(s), width):
                f.write(s[k:k + width] + "\n")
            f.write("\n")


def test_read_fasta(tmp_path):
    from paper_conf_ipps_zhangwlf14_b200.cli import read_fasta
    p = tmp_path / "a.fa"
    p.write_text(">q1 first\nMKVL\nAGG\n\n>q2\n>q3 x y\nWW\n")
    ids, res, off = read_fasta(str(p))
    assert ids == ["q1", "q2", "q3"]
    assert res == b"MKVLAGGWW"
    assert off.tolist() == [0, 7, 7, 9]
    bad = tmp_path / "b.fa"
    bad.write_text("MKV\n>q\nAA\n")
    with pytest.raises(ValueError):
        read_fasta(str(bad))


@pytest.mark.gpu
def test_cli_matches_oracle(tmp_path, capsys, orc):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_ipps_zhangwlf14_b200 import cli
    qs = [gen_query(900 + i, L).decode() for i, L in enumerate([127, 300, 60])]
    db = gen_db(901, 902, n_subjects=200, mean_len=250.0, queries=[q.encode() for q in qs],
                plant_frac=0.4)
    subs = [db.ascii[db.offsets[i]:db.offsets[i + 1]].tobytes().decode()
            for i in range(len(db.offsets) - 1)]
    qids = [f"query{i}" for i in range(len(qs))]
    sids = [f"subj{i}" for i in range(len(subs))]
    _write_fasta(tmp_path / "q.fa", qids, qs)
    _write_fasta(tmp_path / "d.fa", sids, subs)
    codes = orc.encode(db.ascii.tobytes())
    tuples = sorted(tuple(h) for i, q in enumerate(qs)
                    for h in orc.search(orc.encode(q), codes, db.offsets, query_id=i).hsps.tolist())
    exp_lines = [f"{qids[qi]}\t{sids[si]}\t{q0}\t{s0}\t{ln}\t{sc}\t{diag}"
                 for qi, si, diag, q0, s0, ln, sc in tuples]
    assert len(exp_lines) > 20
    for extra in ([], ["--stream"]):
        assert cli.main([str(tmp_path / "q.fa"), str(tmp_path / "d.fa"), *extra]) == 0
        out = capsys.readouterr().out.strip().split("\n")
        assert out == exp_lines, extra
    assert cli.main([str(tmp_path / "q.fa"), str(tmp_path / "d.fa"), "--filter", "stateful"]) == 0
    assert len(capsys.readouterr().out.strip().split("\n")) > 20
    # --gapped: the gapped stage over the same HSPs vs the oracle's gapped stage
    u = np.array(tuples, dtype=np.int32).view(orc.HSP_DTYPE).ravel()
    g = orc.gapped_hsps([orc.encode(q) for q in qs], codes, db.offsets, u)
    exp_g = [f"{qids[r[0]]}\t{sids[r[1]]}\t" + "\t".join(str(int(x)) for x in list(r)[2:])
             for r in g.tolist()]
    assert cli.main([str(tmp_path / "q.fa"), str(tmp_path / "d.fa"), "--gapped"]) == 0
    assert capsys.readouterr().out.strip().split("\n") == exp_g and len(exp_g) > 20


@pytest.mark.gpu
@pytest.mark.parametrize("gather,port", [("p2p", 29561), ("nccl", 29562)])
def test_cli_distributed_two_ranks(tmp_path, gather, port):
    """--distributed under torchrun (2 ranks sharing the one GPU through the
    gloo backend): rank 0 prints exactly the single-process table."""
    import subprocess
    import sys

    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    qs = [gen_query(910 + i, L).decode() for i, L in enumerate([200, 90])]
    db = gen_db(911, 912, n_subjects=300, mean_len=250.0, queries=[q.encode() for q in qs],
                plant_frac=0.4)
    subs = [db.ascii[db.offsets[i]:db.offsets[i + 1]].tobytes().decode()
            for i in range(len(db.offsets) - 1)]
    _write_fasta(tmp_path / "q.fa", [f"q{i}" for i in range(len(qs))], qs)
    _write_fasta(tmp_path / "d.fa", [f"s{i}" for i in range(len(subs))], subs)
    args = [str(tmp_path / "q.fa"), str(tmp_path / "d.fa")]
    env = dict(os.environ, PYTHONPATH=root, BLASTP_DIST_BACKEND="gloo")
    one = subprocess.run([sys.executable, "-m", "paper_conf_ipps_zhangwlf14_b200.cli", *args],
                         capture_output=True, text=True, env=env, cwd=root, timeout=300)
    assert one.returncode == 0, one.stderr
    two = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
                          "--nproc-per-node", "2", "--master-addr", "127.0.0.1",
                          "--master-port", str(port), "-m", "paper_conf_ipps_zhangwlf14_b200.cli",
                          *args, "--distributed", "--gather", gather],
                         capture_output=True, text=True, env=env, cwd=root, timeout=300)
    assert two.returncode == 0, two.stderr[-2000:]
    assert one.stdout.count("\n") > 20
    assert two.stdout == one.stdout
