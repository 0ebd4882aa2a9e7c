"""GPU parity of the gapped-extension consumer (DESIGN.md
R18-R22): blastp_search_gapped / blastp_gapped_extend_device through the
C-ABI vs the oracle's gapped stage (oracle/gapped.c) run on the oracle's own
ungapped list, record by record (bit-exact: integer arithmetic)."""
import os

import numpy as np
import pytest

from synth import config_workload, gen_db, gen_query

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def bp():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_ipps_zhangwlf14_b200 import build
    build.build()
    from paper_conf_ipps_zhangwlf14_b200 import blastp
    return blastp


@pytest.fixture(params=["thread", "warp"], autouse=True)
def gapped_kernel(request, monkeypatch):
    """Every gapped test runs on both pass-1a forms (BLASTP_GAPPED_KERNEL):
    a thread per direction, and a warp per direction with its rows computed
    32 columns at a time."""
    monkeypatch.setenv("BLASTP_GAPPED_KERNEL", request.param)
    return request.param


def assert_same(got, exp, what):
    got, exp = np.asarray(got), np.asarray(exp)
    if len(got) == len(exp) and (got.view(np.int32).reshape(-1, 10) ==
                                 exp.view(np.int32).reshape(-1, 10)).all():
        return
    n = min(len(got), len(exp))
    g = got.view(np.int32).reshape(-1, 10)[:n]
    e = exp.view(np.int32).reshape(-1, 10)[:n]
    bad = np.nonzero((g != e).any(axis=1))[0]
    i = int(bad[0]) if len(bad) else n
    raise AssertionError(f"{what}: {len(got)} GPU vs {len(exp)} oracle alignments; first "
                         f"divergence at {i}: gpu {tuple(got[i]) if i < len(got) else None} "
                         f"oracle {tuple(exp[i]) if i < len(exp) else None}")


def oracle_gapped(orc, queries, ascii, offsets, gp, p=None, nthreads=None):
    """The oracle's ungapped list of every query (its own search), then its
    gapped stage over that list."""
    codes = orc.encode(ascii.tobytes())
    off = np.asarray(offsets, dtype=np.int64)
    off = off - off[0]
    P = orc.Params() if p is None else p
    lists = []
    for k, q in enumerate(queries):
        r = orc.search(orc.encode(q), codes, off, P, nthreads=nthreads or os.cpu_count() or 8,
                       want_extensions=False, query_id=k,
                       cap_hint=max(1 << 16, int(off[-1]) // 2000))
        lists.append(r.hsps)
    u = np.concatenate(lists) if lists else np.zeros(0, orc.HSP_DTYPE)
    u = np.sort(u, order=list(u.dtype.names))
    OG = orc.GappedParams(gap_open=gp.gap_open, gap_extend=gp.gap_extend, xdrop=gp.xdrop,
                          cutoff=gp.cutoff)
    return u, orc.gapped_hsps([orc.encode(q) for q in queries], codes, off, u, OG)


def check(bp, orc, queries, ascii, offsets, gp=None, what="", min_count=1):
    gp = gp or bp.GappedParams()
    t = bp.build_query_batch(queries) if len(queries) > 1 else bp.build_query_table(queries[0])
    d = bp.pack_db(ascii, offsets)
    got, ung = bp.search_gapped(t, d, gparams=gp, want_ungapped=True)
    u, exp = oracle_gapped(orc, queries, ascii, offsets, gp)
    assert (ung.view(np.int32).reshape(-1, 7) == u.view(np.int32).reshape(-1, 7)).all()
    assert_same(got, exp, what)
    assert len(exp) >= min_count
    return got


def test_config1_gapped(bp, orc):
    """Config 1 (q127 vs 1,000 subjects, 5% planted homologs)."""
    (q,), db = config_workload(1)
    g = check(bp, orc, [q], db.ascii, db.offsets, what="config 1", min_count=20)
    assert (g["gap_opens"] > 0).any() or len(g) < 50


def test_config2_gapped(bp, orc):
    """Config 2 (q517 vs 20M residues): every alignment identical."""
    (q,), db = config_workload(2)
    g = check(bp, orc, [q], db.ascii, db.offsets, what="config 2", min_count=1000)
    assert (g["gap_opens"] > 0).sum() > 100


def test_config3_gapped_full(bp, orc):
    """Config 3 at full size (q1054 vs 1.2G residues): the gapped stage over
    the complete ungapped list (~286K HSPs), every alignment identical."""
    (q,), db = config_workload(3)
    check(bp, orc, [q], db.ascii, db.offsets, what="config 3", min_count=10000)


@pytest.mark.parametrize("knobs", [{"BLASTP_GAPPED_RING": "16"}, {"BLASTP_GAPPED_RING": "64"},
                                   {"BLASTP_GAPPED_TBBUF": "0", "BLASTP_GAPPED_STORE": "4096"},
                                   {"BLASTP_GAPPED_TBBUF": "256"},
                                   {"BLASTP_GAPPED_TBBUF": "1024", "BLASTP_GAPPED_RING": "32"}],
                         ids=["ring16", "ring64", "pass2-store4k", "tbuf256", "tbuf1k-ring32"])
def test_ring_overflow_and_store_windows(bp, orc, monkeypatch, knobs):
    """Pairs whose DP rows outgrow the per-thread ring are redone with
    subject-sized rings; directions whose codes outgrow the per-thread store
    are traced by pass 2, whose stores split into several windows: same
    results."""
    for k, v in knobs.items():
        monkeypatch.setenv(k, v)
    (q,), db = config_workload(1)
    check(bp, orc, [q], db.ascii, db.offsets, what=str(knobs), min_count=20)


def test_batch_and_shard_device_entry(bp, orc):
    """A three-query batch against the shards of a database with long subjects:
    blastp_gapped_extend_device over each shard's sorted device list
    (global subject ids) equals the oracle's shard-by-shard result."""
    import torch
    queries = [gen_query(11, 160), gen_query(12, 700), gen_query(13, 1500)]
    db = gen_db(31, 32, n_subjects=3000, mean_len=300.0, queries=queries, plant_frac=0.1)
    # one long subject holding copies of every query (long alignments, big rows)
    t = bp.build_query_batch(queries)
    for k in range(3):
        lo, hi = bp.shard_range(db.offsets, k, 3)
        sub_off = db.offsets[lo:hi + 1]
        d = bp.pack_db(db.ascii, db.offsets, k, 3)
        u = bp.search_ungapped(t, d)
        assert len(u) > 0
        dev = torch.from_numpy(u.view(np.int32).reshape(-1, 7).copy()).cuda()
        out = torch.zeros((len(u), 10), dtype=torch.int32, device="cuda")
        n = bp.gapped_extend_device(t, d, dev.data_ptr(), len(u), out.data_ptr(), len(u))
        got = out[:n].cpu().numpy().view(bp.GAPPED_DTYPE).ravel()
        codes = orc.encode(db.ascii[sub_off[0]:sub_off[-1]].tobytes())
        OG = orc.GappedParams()
        exp = orc.gapped_hsps([orc.encode(q) for q in queries], codes, sub_off - sub_off[0],
                              u.view(orc.HSP_DTYPE), OG, subject_base=lo)
        assert_same(got, exp, f"shard {k}")


def test_long_subjects_and_copies(bp, orc):
    """Subjects of 8K-36,805 residues with planted query copies and indels:
    long gapped alignments (rows far from the seed, big traceback stores)."""
    rng = np.random.default_rng(77)
    q = gen_query(4040, 1200)
    alpha = np.frombuffer(b"ARNDCQEGHILKMFPSTWYV", dtype=np.uint8)
    subs = []
    for k in range(12):
        L = int(rng.integers(8192, 36806))
        s = alpha[rng.integers(0, 20, size=L)].copy()
        for _ in range(4):  # copies of query segments with a few indels
            a = int(rng.integers(0, 1000))
            ln = int(rng.integers(60, 200))
            seg = np.frombuffer(q[a:a + ln], dtype=np.uint8).copy()
            for _ in range(int(rng.integers(0, 4))):
                c = int(rng.integers(1, len(seg) - 1))
                seg = np.delete(seg, c) if rng.random() < 0.5 else np.insert(seg, c, alpha[rng.integers(0, 20)])
            pos = int(rng.integers(0, L - len(seg)))
            s[pos:pos + len(seg)] = seg
        subs.append(s)
    ascii = np.concatenate(subs)
    off = np.concatenate([[0], np.cumsum([len(s) for s in subs])]).astype(np.int64)
    g = check(bp, orc, [q], ascii, off, what="long subjects", min_count=20)
    assert (g["gap_opens"] > 0).any()
    assert (g["q_end"] - g["q_start"]).max() >= 60


@pytest.mark.parametrize("go,ge,x,cut", [(11, 1, 38, 41), (5, 2, 20, 30), (0, 1, 10, 20),
                                         (11, 1, 0, 41), (11, 1, 200, 60)])
def test_gapped_params(bp, orc, go, ge, x, cut):
    """Gap costs, X-drop and cutoff variations (X = 0: only cells at the best
    survive) on random planted databases."""
    q = gen_query(99, 300)
    db = gen_db(101, 102, n_subjects=800, mean_len=250.0, queries=[q], plant_frac=0.2)
    check(bp, orc, [q], db.ascii, db.offsets, bp.GappedParams(go, ge, x, cut),
          what=f"params {go}/{ge}/{x}/{cut}")


def test_hit_dedup_list_gaps_like_diagonal(bp, orc):
    """ext_mode HIT_DEDUP hands off DIAGONAL's list (R17): same gapped result."""
    (q,), db = config_workload(1)
    t = bp.build_query_table(q)
    d = bp.pack_db(db.ascii, db.offsets)
    a = bp.search_gapped(t, d, bp.Params(ext_mode=bp.EXT_HIT_DEDUP))
    b = bp.search_gapped(t, d, bp.Params())
    assert_same(a, b, "HIT_DEDUP vs DIAGONAL")


def test_errors_and_capacity(bp, orc):
    import torch
    (q,), db = config_workload(1)
    t = bp.build_query_table(q)
    d = bp.pack_db(db.ascii, db.offsets)
    u = bp.search_ungapped(t, d)
    assert len(u) > 10
    dev = torch.from_numpy(u.view(np.int32).reshape(-1, 7).copy()).cuda()
    out = torch.zeros((len(u), 10), dtype=torch.int32, device="cuda")
    n = bp.gapped_extend_device(t, d, dev.data_ptr(), len(u), out.data_ptr(), len(u))
    assert n > 2
    # capacity too small: CAPACITY, the first records written, the count reported
    with pytest.raises(bp.BlastpError) as ei:
        bp.gapped_extend_device(t, d, dev.data_ptr(), len(u), out.data_ptr(), 2)
    assert ei.value.status == bp.E_CAPACITY
    # pairs out of order, a query id outside the table, a seed outside the query
    rev = torch.flip(dev, dims=[0]).contiguous()
    with pytest.raises(bp.BlastpError) as ei:
        bp.gapped_extend_device(t, d, rev.data_ptr(), len(u), out.data_ptr(), len(u))
    assert ei.value.status == bp.E_INVALID_ARG
    bad = dev.clone()
    bad[0, 0] = 5
    with pytest.raises(bp.BlastpError) as ei:
        bp.gapped_extend_device(t, d, bad.data_ptr(), len(u), out.data_ptr(), len(u))
    assert ei.value.status == bp.E_INVALID_ARG
    bad = dev.clone()
    bad[0, 3] = 10 ** 6
    with pytest.raises(bp.BlastpError) as ei:
        bp.gapped_extend_device(t, d, bad.data_ptr(), len(u), out.data_ptr(), len(u))
    assert ei.value.status == bp.E_INVALID_ARG
    with pytest.raises(bp.BlastpError):
        bp.gapped_extend_device(t, d, dev.data_ptr(), len(u), out.data_ptr(), len(u),
                                bp.GappedParams(gap_extend=0))
    assert bp.gapped_extend_device(t, d, dev.data_ptr(), 0, out.data_ptr(), len(u)) == 0


@pytest.mark.parametrize("knobs", [{}, {"BLASTP_PIPE_CAP": "7"}], ids=["pipe", "pipe-overflow"])
def test_batch_pipeline_equals_sequential_and_oracle(bp, orc, monkeypatch, knobs):
    """Fig. 12's overlap: a batch whose launch units (query groups, lone
    queries) are searched on one stream while the previous unit is gapped on
    another gives the oracle's result, as the sequential two-stage run does;
    unit buffers that overflow are regrown and the unit re-run."""
    from synth import gen_queries
    queries = gen_queries(77, 12, 100, 900)
    db = gen_db(78, 79, n_subjects=2500, mean_len=300.0, queries=queries, plant_frac=0.2)
    t = bp.build_query_batch(queries)
    assert t.groups[0] >= 1
    d = bp.pack_db(db.ascii, db.offsets)
    for k, v in knobs.items():
        monkeypatch.setenv(k, v)
    monkeypatch.setenv("BLASTP_GAPPED_PIPE", "1")
    got, ung = bp.search_gapped(t, d, want_ungapped=True)
    monkeypatch.setenv("BLASTP_GAPPED_PIPE", "0")
    seq, sung = bp.search_gapped(t, d, want_ungapped=True)
    assert_same(got, seq, "pipelined vs sequential")
    assert (ung == sung).all()
    u, exp = oracle_gapped(orc, queries, db.ascii, db.offsets, bp.GappedParams())
    assert_same(got, exp, "pipelined vs oracle")
    assert len(exp) > 100


def test_config4_gapped_sharded_full(bp, orc, gapped_kernel):
    """Config 4 at full size: queries 127/517/1054 (one batch) against config
    3's database cut into 4 shards; each shard's gapped stage on the GPU
    (blastp_search_gapped), concatenated and sorted, equals the oracle's gapped
    stage over the oracle's whole-database list (pairs never span shards)."""
    if gapped_kernel != "warp":
        pytest.skip("the thread form is covered by config 3; one form at this size")
    from synth import CONFIGS
    (_,), db = config_workload(3)
    queries = [gen_query(CONFIGS[1]["query_seed"], 127), gen_query(CONFIGS[2]["query_seed"], 517),
               gen_query(CONFIGS[3]["query_seed"], 1054)]
    t = bp.build_query_batch(queries)
    parts = []
    for k in range(4):
        d = bp.pack_db(db.ascii, db.offsets, k, 4)
        parts.append(bp.search_gapped(t, d))
        d.free()
    got = np.concatenate(parts)
    got = np.sort(got, order=list(got.dtype.names))
    _, exp = oracle_gapped(orc, queries, db.ascii, db.offsets, bp.GappedParams())
    assert_same(got, exp, "config 4, 4 shards")
    assert len(exp) > 100000


def test_constructed_hsp_lists_edges(bp, orc, gapped_kernel):
    """HSP lists built by hand rather than by the search: seeds at both ends
    of the query and the subject (empty directions), length-0 and length-1
    HSPs, exact duplicates, 150 HSPs on one (query, subject) pair (R21's box
    test over a long chain, equal scores keeping canonical order), poly-W
    rows wide enough for the big-ring pass, the last subject of the shard --
    all against the oracle, on both pass-1a forms."""
    import torch
    rng = np.random.default_rng(2024)
    q = gen_query(606, 400)
    qc = orc.encode(q)
    alpha = np.frombuffer(b"ARNDCQEGHILKMFPSTWYV", dtype=np.uint8)
    subs = [alpha[rng.integers(0, 20, size=int(rng.integers(50, 900)))].copy() for _ in range(40)]
    subs[3][100:300] = np.frombuffer(q[50:250], dtype=np.uint8)      # a long copy
    subs[7] = np.frombuffer(b"W" * 700, dtype=np.uint8).copy()        # poly-W: wide rows
    subs[-1][:120] = np.frombuffer(q[-120:], dtype=np.uint8)          # last subject, query end
    ascii = np.concatenate(subs)
    off = np.concatenate([[0], np.cumsum([len(s) for s in subs])]).astype(np.int64)
    lens = [len(s) for s in subs]
    recs = []

    def add(sid, qs, ss, ln, score):
        recs.append((0, sid, ss - qs, qs, ss, ln, score))
    add(0, 0, 0, 0, 50)                      # seed at both starts: left directions empty
    add(1, 399, lens[1] - 1, 1, 45)          # seed at both ends (middle pair = the last pair)
    add(2, 399, 0, 0, 44)                    # qm = lq: right direction has no rows
    add(5, 10, 20, 6, 60)
    add(5, 10, 20, 6, 60)                    # an exact duplicate: inside the first box
    for k in range(150):                     # one long chain on the pair (0, 3)
        qs = int(rng.integers(0, 390))
        ss = int(rng.integers(0, lens[3] - 10))
        add(3, qs, ss, int(rng.integers(0, 10)), int(rng.integers(41, 90)) if k % 7 else 55)
    add(7, 0, 0, 3, 41)                      # poly-W subject vs the query's W's
    add(7, 200, 600, 3, 41)
    add(39, 280, 0, 120, 300)                # the last subject: the copy of the query's end
    h = np.array(sorted(recs), dtype=np.int32)
    d = bp.pack_db(ascii, off)
    t = bp.build_query_table(q)
    dev = torch.from_numpy(h.copy()).cuda()
    out = torch.zeros((len(h), 10), dtype=torch.int32, device="cuda")
    for knobs in ({}, {"BLASTP_GAPPED_RING": "16"}):
        for k_, v in knobs.items():
            os.environ[k_] = v
        try:
            n = bp.gapped_extend_device(t, d, dev.data_ptr(), len(h), out.data_ptr(), len(h))
        finally:
            for k_ in knobs:
                os.environ.pop(k_, None)
        got = out[:n].cpu().numpy().view(bp.GAPPED_DTYPE).ravel()
        exp = orc.gapped_hsps([qc], orc.encode(ascii.tobytes()), off,
                              h.view(orc.HSP_DTYPE).ravel(), orc.GappedParams())
        assert_same(got, exp, f"constructed list {knobs}")
        assert len(exp) >= 4  # the copies, poly-W; most chain seeds fall inside the copy's box


_C5 = {}


def _c5_gapped_chunk(bounds):
    a, b = bounds
    o = _C5["orc"]
    return o.gapped_hsps(_C5["qcodes"], _C5["codes"], _C5["off"], _C5["u"][a:b])


@pytest.mark.skipif(os.environ.get("BLASTP_FULL_CONFIG5") != "1",
                    reason="~12 min of oracle time on 16 cores: run once per round with "
                           "BLASTP_FULL_CONFIG5=1 (log in profiles/)")
def test_config5_shard_gapped_full(bp, orc, gapped_kernel):
    """Config 5, one full shard: the 64 queries against shard 0 of 8 (~1.9G
    residues); the GPU's gapped alignments equal the oracle's gapped stage run
    over the oracle's own complete ungapped list (split at pair boundaries
    over the host's cores; ~21.5M HSPs)."""
    if gapped_kernel != "warp":
        pytest.skip("the default form at this size")
    import multiprocessing as mp
    import time
    from paper_conf_ipps_zhangwlf14_b200.dist import shard_subjects
    from synth import config_offsets
    off = config_offsets(5)
    lo, hi = shard_subjects(off, 0, 8)
    queries, db = config_workload(5, subject_range=(lo, hi))
    loc = (db.offsets - db.offsets[0]).astype(np.int64)
    t0 = time.perf_counter()
    got = bp.search_gapped(bp.build_query_batch(queries), bp.pack_db(db.ascii, loc))
    t_gpu = time.perf_counter() - t0
    t0 = time.perf_counter()
    codes = orc.encode(db.ascii.tobytes())
    lists = [orc.search(orc.encode(q), codes, loc, orc.Params(), nthreads=os.cpu_count() or 8,
                        want_extensions=False, query_id=k, cap_hint=int(loc[-1]) // 500).hsps
             for k, q in enumerate(queries)]
    u = np.concatenate(lists)
    u = np.sort(u, order=list(u.dtype.names))
    t_search = time.perf_counter() - t0
    t0 = time.perf_counter()
    # chunks of the canonical list split at (query, subject) boundaries
    nproc = os.cpu_count() or 8
    cuts = [0]
    for c in range(1, nproc):
        i = len(u) * c // nproc
        while 0 < i < len(u) and (u["query_id"][i], u["subject_id"][i]) == \
                (u["query_id"][i - 1], u["subject_id"][i - 1]):
            i += 1
        cuts.append(max(i, cuts[-1]))
    cuts.append(len(u))
    _C5.update(orc=orc, qcodes=[orc.encode(q) for q in queries], codes=codes, off=loc, u=u)
    with mp.get_context("fork").Pool(nproc) as pool:
        parts = pool.map(_c5_gapped_chunk, list(zip(cuts[:-1], cuts[1:])))
    exp = np.concatenate(parts)
    t_gapped = time.perf_counter() - t0
    _C5.clear()
    assert_same(got, exp, "config 5 shard 0 of 8, gapped")
    print(f"config5 shard 0/8 gapped parity: {len(u)} HSPs -> {len(exp)} alignments; GPU search + "
          f"gapped {t_gpu:.1f} s (incl. table build + pack); oracle search {t_search:.0f} s, "
          f"oracle gapped {t_gapped:.0f} s on {nproc} processes")


@pytest.mark.parametrize("mode,ext_mode", [(0, 1), (1, 0), (2, 0), (3, 0)],
                         ids=["HIT", "EITHER", "STATEFUL", "STATEFUL_RB"])
def test_gapped_over_other_readings(bp, orc, mode, ext_mode):
    """The gapped stage consumes whatever list a search reading hands off --
    ext_mode HIT's one record per seed (duplicates inside each other's boxes,
    R21), EITHER, STATEFUL, STATEFUL_RB -- identically to the oracle's gapped
    stage over the oracle's list of the same reading (config 1)."""
    (q,), db = config_workload(1)
    p = bp.Params(filter_mode=mode, ext_mode=ext_mode)
    t = bp.build_query_table(q, p)
    d = bp.pack_db(db.ascii, db.offsets)
    got = bp.search_gapped(t, d, p)
    P = orc.Params(filter_mode=mode, ext_mode=ext_mode)
    _, exp = oracle_gapped(orc, [q], db.ascii, db.offsets, bp.GappedParams(), p=P)
    assert_same(got, exp, f"config 1 {p}")
    assert len(exp) > 5
