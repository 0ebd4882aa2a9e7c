"""GPU parity: the CUDA path through the C-ABI vs the CPU oracle, element by
element (bit-exact: all arithmetic is integer).  Run with -m gpu on a B200."""
import os

import numpy as np
import pytest

from synth import config_workload, gen_db, gen_query

pytestmark = pytest.mark.gpu

ALPHA = "ARNDCQEGHILKMFPSTWYVBZX*"


@pytest.fixture(scope="module")
def bp():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_ipps_zhangwlf14_b200 import build
    build.build()
    from paper_conf_ipps_zhangwlf14_b200 import blastp
    return blastp


@pytest.fixture(params=["cta", "warp", "block"], autouse=True)
def kernel_variant(request, monkeypatch):
    """Every parity test runs on every kernel variant (BLASTP_KERNEL): the
    block kernel (default where eligible: LEFT, window >= 31 + min_gap; the
    warp kernel otherwise), the warp kernel and the CTA kernel."""
    monkeypatch.setenv("BLASTP_KERNEL", request.param)
    return request.param


def tuples(a):
    return [tuple(int(v) for v in x) for x in a.tolist()]


def hit_set(a):
    return sorted((int(h[0]), int(h[1]), int(h[2]), int(h[3])) for h in a)


def oracle_run(orc, q_ascii, ascii, offsets, p, want_hits=False, nthreads=1, query_id=0):
    # ext_mode WINDOW (Alg. 5) computes Alg. 3's extensions: the oracle's DIAGONAL mode
    P = orc.Params(word_len=p.word_len, threshold=p.threshold, window=p.window,
                   min_gap=p.min_gap, xdrop=p.xdrop, cutoff=p.cutoff, filter_mode=p.filter_mode,
                   ext_mode=1 if p.ext_mode == 1 else 0)
    codes = orc.encode(ascii.tobytes() if hasattr(ascii, "tobytes") else ascii)
    return orc.search(orc.encode(q_ascii), codes, np.asarray(offsets, dtype=np.int64), P,
                      want_hits=want_hits, nthreads=nthreads, query_id=query_id)


def gpu_run(bp, q_ascii, ascii, offsets, p, trace=False):
    t = bp.build_query_table(q_ascii, p)
    d = bp.pack_db(ascii, offsets)
    hsps = bp.search_ungapped(t, d, p)
    tr = bp.debug_trace(t, d, p) if trace else None
    return hsps, tr


def assert_same(bp, orc, q, ascii, offsets, p, trace=True, nthreads=1):
    g, tr = gpu_run(bp, q, ascii, offsets, p, trace)
    r = oracle_run(orc, q, ascii, offsets, p, want_hits=trace, nthreads=nthreads)
    assert tuples(g) == tuples(r.hsps), (len(g), len(r.hsps))
    if trace:
        oh = sorted((0, int(a), int(b), int(c)) for a, b, c in r.hits)
        op = sorted((0, int(a), int(b), int(c)) for a, b, c in r.passing)
        assert hit_set(tr.hits) == oh
        assert hit_set(tr.passing) == op
        ext = np.sort(tr.extensions, order=list(tr.extensions.dtype.names))
        assert tuples(ext) == tuples(r.extensions)
    return g, r


# ------------------------------------------------------------------ configs

@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("ext_mode", [0, 1, 2])
def test_config1_full_trace(bp, orc, mode, ext_mode):
    """Config 1 (q127 vs 1,000 subjects): hits, passing hits, every extension
    and the HSP list identical to the oracle, both filter readings, all three
    extension strategies (Alg. 3 diagonal-based, Alg. 4 hit-based, Alg. 5
    window-based = Alg. 3's results)."""
    (q,), db = config_workload(1)
    p = bp.Params(filter_mode=mode, ext_mode=ext_mode)
    g, r = assert_same(bp, orc, q, db.ascii, db.offsets, p)
    assert len(g) > 10


# Complete oracle lists at full size, computed once per session on all host
# cores and shared by the kernel-variant parametrisation: key -> canonical
# HSP array of one query (query_id 0).
_ORACLE_FULL = {}


def oracle_full(orc, key, q_ascii, ascii, offsets, p):
    """The oracle's complete HSP list of one query against a whole (shard of
    a) database, all host cores, no sampling."""
    k = (key, bytes(q_ascii if isinstance(q_ascii, bytes) else q_ascii.encode()), p.filter_mode,
         1 if p.ext_mode == 1 else 0, p.window, p.min_gap)
    if k not in _ORACLE_FULL:
        codes = _ORACLE_FULL.get(("codes", key))
        if codes is None:
            codes = orc.encode(ascii.tobytes())
            _ORACLE_FULL[("codes", key)] = codes
        P = orc.Params(word_len=p.word_len, threshold=p.threshold, window=p.window,
                       min_gap=p.min_gap, xdrop=p.xdrop, cutoff=p.cutoff,
                       filter_mode=p.filter_mode, ext_mode=1 if p.ext_mode == 1 else 0)
        off = np.asarray(offsets, dtype=np.int64)
        r = orc.search(orc.encode(q_ascii), codes, off - off[0], P, nthreads=os.cpu_count() or 8,
                       want_extensions=False, cap_hint=max(1 << 16, int(off[-1] - off[0]) // 2000))
        _ORACLE_FULL[k] = r.hsps
    return _ORACLE_FULL[k]


def assert_lists_equal(got, exp, what):
    """Element-by-element equality of two canonical HSP arrays; on a mismatch
    report the first divergence."""
    got = np.asarray(got)
    exp = np.asarray(exp)
    if len(got) == len(exp) and (got == exp).all():
        return
    n = min(len(got), len(exp))
    bad = np.nonzero(got[:n] != exp[:n])[0]
    i = int(bad[0]) if len(bad) else n
    raise AssertionError(f"{what}: {len(got)} GPU vs {len(exp)} oracle HSPs; first divergence at "
                         f"{i}: gpu {tuple(got[i]) if i < len(got) else None} oracle "
                         f"{tuple(exp[i]) if i < len(exp) else None}")


def _with_qid(a, qid):
    a = a.copy()
    a["query_id"] = qid
    return a


_CONFIG2 = {}


def _config2():
    if not _CONFIG2:
        _CONFIG2["w"] = config_workload(2)
    return _CONFIG2["w"]


@pytest.mark.parametrize("mode,ext_mode", [(0, 0), (1, 0), (2, 0), (3, 0), (0, 1), (0, 2)],
                         ids=["LEFT", "EITHER", "STATEFUL", "STATEFUL_RB", "HIT", "WINDOW"])
def test_config2_full(bp, orc, mode, ext_mode):
    """Config 2 (q517 vs 20M residues): the complete HSP list identical to the
    oracle's, every filter reading (R6 LEFT / EITHER, R15 STATEFUL) and every
    extension strategy (Alg. 3 diagonal, Alg. 4 hit, Alg. 5 window)."""
    (q,), db = _config2()
    p = bp.Params(filter_mode=mode, ext_mode=ext_mode)
    g = bp.search_ungapped(bp.build_query_table(q, p), bp.pack_db(db.ascii, db.offsets), p)
    exp = oracle_full(orc, "config2", q, db.ascii, db.offsets, p)
    assert_lists_equal(g, exp, f"config 2 {p}")
    assert len(g) > 1000


_CONFIG3 = {}


def _config3():
    """Config 3's workload, generated once per test session (~1.2 GB)."""
    if not _CONFIG3:
        _CONFIG3["w"] = config_workload(3)
    return _CONFIG3["w"]


def _config3_db(bp):
    if "db" not in _CONFIG3:
        (_,), db = _config3()
        _CONFIG3["db"] = bp.pack_db(db.ascii, db.offsets)
    return _CONFIG3["db"]


def rescore(orc, queries, ascii, offsets, g, subject_base=0, n=2000):
    """P5 on a deterministic sample of HSPs: score = the BLOSUM62 sum over the
    segment, read from the sequences."""
    B = orc.blosum62()
    Qs = [orc.encode(q) for q in queries]
    rng = np.random.default_rng(0)
    for h in g[rng.choice(len(g), size=min(n, len(g)), replace=False)]:
        a = offsets[h["subject_id"]] + h["s_start"] - offsets[subject_base]
        S = orc.encode(ascii[a:a + h["length"]].tobytes())
        Q = Qs[h["query_id"]]
        assert B[Q[h["q_start"]:h["q_start"] + h["length"]], S].sum() == h["score"]


@pytest.mark.parametrize("mode", [0, 1, 2, 3], ids=["LEFT", "EITHER", "STATEFUL", "STATEFUL_RB"])
def test_config3_full(bp, orc, kernel_variant, mode):
    """Config 3 at full size (q1054 vs 6.0M subjects / ~1.2G residues, the
    bench launch): the complete HSP list identical to the oracle's complete
    list (no sampling), both R6 readings and the STATEFUL walk."""
    if kernel_variant == "cta" and mode >= 2:
        pytest.skip("STATEFUL runs on the warp variant only")
    if kernel_variant == "block" and mode != 0:
        pytest.skip("EITHER and STATEFUL run on the warp kernel (the block kernel is LEFT only)")
    (q,), db = _config3()
    p = bp.Params(filter_mode=mode)
    g = bp.search_ungapped(bp.build_query_table(q, p), _config3_db(bp), p)
    exp = oracle_full(orc, "config3", q, db.ascii, db.offsets, p)
    assert len(exp) > 10000
    assert_lists_equal(g, exp, f"config 3 {p}")
    rescore(orc, [q], db.ascii, db.offsets, g)


def test_config4_sharded_full(bp, orc, kernel_variant):
    """Config 4: queries 127/517/1054 (one batch) against config 3's database
    cut into 1, 2, 4 and 8 residue-balanced subject-range shards (one per GPU
    in production; here shard by shard on one device).  The concatenation of
    the shards' lists (dist.gather_hsps) is, for every shard count, exactly the
    oracle's complete list of the three queries against the whole database."""
    if kernel_variant == "cta":
        pytest.skip("shard arithmetic is kernel-independent; the cta variant is covered "
                    "by config 3")
    from synth import CONFIGS, gen_query
    (_,), db = _config3()
    queries = [gen_query(CONFIGS[1]["query_seed"], 127), gen_query(CONFIGS[2]["query_seed"], 517),
               gen_query(CONFIGS[3]["query_seed"], 1054)]
    p = bp.Params()
    exp = np.concatenate([_with_qid(oracle_full(orc, "config3", q, db.ascii, db.offsets, p), i)
                          for i, q in enumerate(queries)])
    exp = np.sort(exp, order=list(exp.dtype.names))
    t = bp.build_query_batch(queries, p)
    for n in (1, 2, 4, 8):
        parts = []
        for k in range(n):
            d = _config3_db(bp) if n == 1 else bp.pack_db(db.ascii, db.offsets, k, n)
            parts.append(bp.search_ungapped(t, d, p))
            if n > 1:
                d.free()
        cat = np.concatenate(parts)
        # per-shard canonical order; the gathered list sorted by query first
        got = np.sort(cat, order=list(cat.dtype.names))
        assert_lists_equal(got, exp, f"config 4, {n} shards")
    assert len(exp) > 10000


def assert_sampled_parity(bp, orc, queries, ascii, offsets, g, p, blocks, subject_base=0,
                          rescore_n=2000):
    """Full-size parity where the oracle cannot redo the whole search in the
    default suite (config 5: 64 queries x 1.9G residues per shard): every GPU
    HSP of a deterministic sample is re-scored from the sequences (P5), and
    for each subject block [lo, hi) (global ids) the oracle re-searches the
    block for every query and the GPU's HSPs on those subjects must be
    identical.  test_config5_shard_full runs the complete comparison."""
    rescore(orc, queries, ascii, offsets, g, subject_base, rescore_n)
    B = orc.blosum62()
    Qs = [orc.encode(q) for q in queries]
    P = orc.Params(word_len=p.word_len, threshold=p.threshold, window=p.window,
                   min_gap=p.min_gap, xdrop=p.xdrop, cutoff=p.cutoff, filter_mode=p.filter_mode,
                   ext_mode=1 if p.ext_mode == 1 else 0)
    tables = [orc.neighbourhood(Q, B, p.threshold) for Q in Qs]
    for lo, hi in blocks:
        sub_off = offsets[lo:hi + 1]
        blk = orc.encode(ascii[sub_off[0] - offsets[subject_base]:
                               sub_off[-1] - offsets[subject_base]].tobytes())
        exp = []
        for qi, (Q, tab) in enumerate(zip(Qs, tables)):
            r = orc.search(Q, blk, sub_off - sub_off[0], P, query_id=qi, table=tab,
                           nthreads=os.cpu_count() or 8)
            e = r.hsps.copy()
            e["subject_id"] += lo
            exp += tuples(e)
        sel = g[(g["subject_id"] >= lo) & (g["subject_id"] < hi)]
        assert tuples(sel) == sorted(exp), (lo, hi)


def test_config5_shard_sampled(bp, orc, kernel_variant):
    """Config 5: the batch of 64 queries (len U[100, 2000]) against one
    eighth of the nr-shaped 40M-subject database (~1.9G residues: the shard
    one of the 8 GPUs owns; first and last shard), full size, in one batched
    search.  Sampled oracle parity on subject blocks for all 64 queries."""
    if kernel_variant != "block":
        pytest.skip("the 64-query full-size shard runs on the default (block) kernel")
    from paper_conf_ipps_zhangwlf14_b200.dist import shard_subjects
    from synth import config_offsets
    off = config_offsets(5)
    for k in (0, 7):
        lo, hi = shard_subjects(off, k, 8)
        queries, db = config_workload(5, subject_range=(lo, hi))
        assert len(queries) == 64
        p = bp.Params()
        t = bp.build_query_batch(queries, p)
        # the shard alone is resident (as on its GPU): pack it as shard 0 of 1
        # of its own subjects, then map the subject ids back to global ones
        d = bp.pack_db(db.ascii, db.offsets - db.offsets[0])
        g = bp.search_ungapped(t, d, p)
        del d
        if k == 7:
            # the same shard streamed from its formatted host image (the e2e
            # path) gives the identical list
            import torch
            h = bp.format_host_db(db.ascii, db.offsets - db.offsets[0])
            cap = len(g) + 1024
            out = torch.zeros(cap * 7, dtype=torch.int32, device="cuda")
            cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
            bp.search_formatted_db(t, h, out.data_ptr(), cap, cnt.data_ptr(), p)
            nf = int(cnt.item())
            assert nf == len(g)
            bp.sort_hsps_device(out.data_ptr(), nf)
            fm = out[: nf * 7].view(nf, 7).cpu().numpy()
            h.free()
            del out
            assert np.array_equal(fm, g.view(np.int32).reshape(-1, 7))
        g["subject_id"] += lo
        assert len(g) > 100000
        assert set(np.unique(g["query_id"])) == set(range(64))
        n = hi - lo
        blocks = [(lo + j, lo + min(j + 600, n)) for j in range(0, n, n // 6)][:6]
        assert_sampled_parity(bp, orc, queries, db.ascii, off, g, p, blocks, subject_base=lo)




@pytest.mark.skipif(os.environ.get("BLASTP_FULL_CONFIG5") != "1",
                    reason="~10 min of oracle time on 16 cores: run once per round with "
                           "BLASTP_FULL_CONFIG5=1 (log in profiles/)")
def test_config5_shard_full(bp, orc, kernel_variant):
    """Config 5, one full shard with no sampling: the 64 queries (len
    U[100, 2000]) against shard 0 of 8 of the nr-shaped database (~1.9G
    residues, ~5M subjects); the GPU list equals the oracle's complete list of
    all 64 queries."""
    if kernel_variant != "block":
        pytest.skip("the 64-query full-size shard runs on the default (block) kernel")
    import time
    from paper_conf_ipps_zhangwlf14_b200.dist import shard_subjects
    from synth import config_offsets
    off = config_offsets(5)
    lo, hi = shard_subjects(off, 0, 8)
    queries, db = config_workload(5, subject_range=(lo, hi))
    p = bp.Params()
    t0 = time.perf_counter()
    g = bp.search_ungapped(bp.build_query_batch(queries, p),
                           bp.pack_db(db.ascii, db.offsets - db.offsets[0]), p)
    t_gpu = time.perf_counter() - t0
    t0 = time.perf_counter()
    exp = np.concatenate([_with_qid(oracle_full(orc, "config5s0", q, db.ascii, db.offsets, p), i)
                          for i, q in enumerate(queries)])
    t_orc = time.perf_counter() - t0
    exp = np.sort(exp, order=list(exp.dtype.names))
    assert_lists_equal(g, exp, "config 5 shard 0 of 8")
    print(f"config5 shard 0/8 full parity: {len(g)} HSPs, {hi - lo} subjects, "
          f"{int(db.offsets[-1] - db.offsets[0])} residues, 64 queries; GPU search "
          f"{t_gpu:.1f} s (incl. table build + pack), oracle {t_orc:.1f} s on "
          f"{os.cpu_count()} threads")


@pytest.mark.parametrize("T", [8, 11, 13])
def test_query_table_builders_agree(bp, orc, monkeypatch, T):
    """The GPU table builder (default) and the host enumeration
    (BLASTP_TABLE_BUILD=host) give the same table: same entry count and the
    same hit trace as the oracle's brute-force neighbourhood (R3)."""
    q = gen_query(41, 600).decode() + "WWWCCCBZX*"
    db = gen_db(42, 43, n_subjects=120, mean_len=300.0, queries=[q.encode()], plant_frac=0.3)
    p = bp.Params(threshold=T)
    entries = []
    for how in ("gpu", "host"):
        monkeypatch.setenv("BLASTP_TABLE_BUILD", how)
        entries.append(bp.build_query_table(q, p).entries)
        assert_same(bp, orc, q, db.ascii, db.offsets, p, trace=True)
    off, pos = orc.neighbourhood(orc.encode(q), orc.blosum62(), T)
    assert entries[0] == entries[1] == len(pos)


# ------------------------------------------------------------------ fuzz

def _rand_db(rng, n, lo, hi, q=None, plant=0.3):
    subs = []
    for _ in range(n):
        L = int(rng.integers(lo, hi + 1))
        s = rng.choice(list(ALPHA[:20]), size=L)
        if q is not None and L > 10 and len(q) >= 5 and rng.random() < plant:
            k = int(rng.integers(5, min(L, len(q)) + 1))
            a = int(rng.integers(0, len(q) - k + 1))
            b = int(rng.integers(0, L - k + 1))
            seg = np.array(list(q[a:a + k]))
            mut = rng.random(k) < 0.25
            seg[mut] = rng.choice(list(ALPHA[:20]), size=int(mut.sum()))
            s[b:b + k] = seg
        subs.append("".join(s))
    off = np.concatenate([[0], np.cumsum([len(s) for s in subs])]).astype(np.int64)
    return np.frombuffer("".join(subs).encode(), dtype=np.uint8).copy(), off


def test_fuzz_small_random(bp, orc):
    rng = np.random.default_rng(99)
    for case in range(120):
        lq = int(rng.choice([3, 5, 17, 64, 127, 300, 517]))
        q = "".join(rng.choice(list(ALPHA[:20] if case % 4 else ALPHA), size=lq))
        ascii, off = _rand_db(rng, int(rng.integers(1, 60)), 0, 400, q)
        p = bp.Params(threshold=int(rng.choice([11, 11, 9, 13])),
                      window=int(rng.choice([40, 40, 10, 80, 3])),
                      min_gap=int(rng.choice([3, 3, 1, 2, 5])),
                      xdrop=int(rng.choice([16, 16, 5, 30])),
                      cutoff=int(rng.choice([41, 20, 0])),
                      filter_mode=int(case % 2), ext_mode=int((case // 2) % 3))
        assert_same(bp, orc, q, ascii, off, p, trace=True)


@pytest.mark.parametrize("W,A", [(1, 32), (3, 34), (3, 35), (8, 39), (8, 40), (3, 255),
                                 (8, 256), (2, 100)])
def test_block_state_window_limits(bp, orc, kernel_variant, W, A):
    """The block kernel's validity edge (A >= 31 + W, A <= 256): every window
    / min_gap pair at and next to it, on hit-dense planted data with long runs
    of hits per diagonal, compared at trace level (hits, passing hits,
    extensions) with the oracle; every kernel variant takes the same pairs."""
    rng = np.random.default_rng(1000 + 7 * W + A)
    q = gen_query(31 + W, 400).decode()
    ascii, off = _rand_db(rng, 40, 50, 900, q, plant=0.8)
    for ext in (0, 1):
        assert_same(bp, orc, q, ascii, off,
                    bp.Params(window=A, min_gap=W, threshold=9, ext_mode=ext), trace=True)


def test_adversarial_low_complexity(bp, orc):
    """Poly-W query vs poly-W subjects: every (q, s) is a hit (the hit-dense
    slow path), plus runs of mixed low-complexity residues."""
    q = "W" * 300 + "AAAAQQQQ" * 10 + "W" * 50
    subs = ["W" * 1000, "A" * 200 + "W" * 40, "WA" * 300, "Q" * 500, "W" * 3]
    ascii = np.frombuffer("".join(subs).encode(), dtype=np.uint8).copy()
    off = np.concatenate([[0], np.cumsum([len(s) for s in subs])]).astype(np.int64)
    for mode in (0, 1):
        assert_same(bp, orc, q, ascii, off, bp.Params(filter_mode=mode), trace=True)
    assert_same(bp, orc, q, ascii, off, bp.Params(ext_mode=1), trace=True)
    assert_same(bp, orc, q, ascii, off, bp.Params(ext_mode=2), trace=True)


def test_edge_cases(bp, orc):
    q = gen_query(3, 200).decode()
    # empty subjects, subjects shorter than a word, query itself, long subject
    long_s = gen_query(4, 36805).decode()
    long_s = long_s[:20000] + q + long_s[20000 + len(q):]
    subs = ["", "A", "MK", q, "", q[::-1], long_s, q[:3], q[-5:], ""]
    ascii = np.frombuffer("".join(subs).encode(), dtype=np.uint8).copy()
    off = np.concatenate([[0], np.cumsum([len(s) for s in subs])]).astype(np.int64)
    g, r = assert_same(bp, orc, q, ascii, off, bp.Params(), trace=True)
    assert any(h[1] == 3 and h[2] == 0 for h in tuples(g))  # the self hit
    # query of exactly one word
    assert_same(bp, orc, "WCW", ascii, off, bp.Params(threshold=5), trace=True)
    # a database with no subjects at all
    empty = np.zeros(0, dtype=np.uint8)
    g, _ = gpu_run(bp, q, empty, np.zeros(1, dtype=np.int64), bp.Params())
    assert len(g) == 0


def test_pack_tiny_and_mixed_subjects(bp, orc):
    """Runs of empty and 1-5 residue subjects (more than 32 subject starts in
    one 512-byte pack tile: the pack kernel's general path), lowercase and
    U/O/J residues, and ordinary subjects between them: every hit, passing
    hit, extension and HSP identical to the oracle (a word spanning two
    subjects, a wrong sentinel or a shifted residue would show up as a hit)."""
    rng = np.random.default_rng(31)
    q = gen_query(32, 400).decode()
    subs = []
    for blk in range(60):
        if blk % 3 == 0:
            subs += ["".join(rng.choice(list(ALPHA[:20]), size=int(L)))
                     for L in rng.integers(0, 6, size=int(rng.integers(40, 300)))]
        else:
            L = int(rng.integers(50, 900))
            s = list(rng.choice(list(ALPHA[:20] + "uojbzx"), size=L))
            a, n = int(rng.integers(0, 300)), int(rng.integers(20, 100))
            b = int(rng.integers(0, max(1, L - n)))
            s[b:b + n] = list(q[a:a + n])[:max(0, L - b)]
            subs.append("".join(s[:L]))
    ascii = np.frombuffer("".join(subs).encode(), dtype=np.uint8).copy()
    off = np.concatenate([[0], np.cumsum([len(s) for s in subs])]).astype(np.int64)
    g, r = assert_same(bp, orc, q, ascii, off, bp.Params(), trace=True)
    assert len(g) > 20
    for k in range(3):  # shards start at arbitrary subjects
        shard = tuples(bp.search_ungapped(bp.build_query_table(q), bp.pack_db(ascii, off, k, 3)))
        assert shard == [h for h in tuples(g) if h[1] in range(*_shard_ids(bp, off, k, 3))]


def _shard_ids(bp, off, k, n):
    d = bp.pack_db(np.zeros(int(off[-1]), np.uint8) + ord("A"), off, k, n)
    return d.subject_base, d.subject_base + d.nseq


def _long_subject_db(q):
    """Long subjects (> 2C residues: split into segments) with copies of the
    query planted across segment boundaries (exact ones, so an extension and
    its ext_reach run from one segment into the next), one subject longer
    than the 16-bit frame (65536), and short subjects around them."""
    rng = np.random.default_rng(5)
    L = len(q)

    def subject(n, plants):
        s = list(gen_query(int(rng.integers(1, 1 << 30)), n).decode())
        for pos, exact in plants:
            seg = list(q)
            if not exact:
                for i in np.nonzero(rng.random(L) < 0.3)[0]:
                    seg[i] = ALPHA[int(rng.integers(0, 20))]
            s[pos:pos + L] = seg
        return "".join(s[:n])

    subs = [gen_query(11, 120).decode(), "",
            subject(40000, [(2048 - 100, True), (4096 - 7, False), (9000, True),
                            (20480 - L // 2, True), (39000, False)]),
            gen_query(12, 300).decode(),
            subject(9000, [(100, True), (4000, True), (4100 + L, False)]),
            subject(5000, [(2000, True)]),
            subject(70000, [(1000, True), (32768 - 50, True), (65536 - 80, True), (69000, False)]),
            q, gen_query(13, 700).decode(), "MK"]
    ascii = np.frombuffer("".join(subs).encode(), dtype=np.uint8).copy()
    off = np.concatenate([[0], np.cumsum([len(s) for s in subs])]).astype(np.int64)
    return ascii, off


@pytest.mark.parametrize("knobs", [{}, {"BLASTP_SEGLEN": "256"}, {"BLASTP_SEGCAP": "4"},
                                   {"BLASTP_SEGCAP": "150"}, {"BLASTP_SEGMENTS": "0"}],
                         ids=["default", "seglen256", "overflow_all", "overflow_some", "off"])
def test_long_subjects_segmented(bp, orc, monkeypatch, kernel_variant, knobs):
    """The long-subject plan (segments filtered in parallel, one walker per
    long chunk, list-overflow fallback) gives the oracle's results exactly:
    hits, passing hits, extensions and HSPs, both filter readings."""
    q = gen_query(21, 300).decode()
    ascii, off = _long_subject_db(q)
    for k, v in knobs.items():
        monkeypatch.setenv(k, v)
    d = bp.pack_db(ascii, off)
    assert d.long_items >= 4
    if knobs.get("BLASTP_SEGMENTS") == "0":
        assert d.segments == 0
    else:
        assert d.segments >= (40000 + 9000 + 5000 + 70000) // d.segment_len
    for mode, window, ext in ((0, 40, 0), (1, 40, 0), (0, 80, 0), (0, 256, 0), (0, 40, 1),
                              (0, 40, 2)):
        p = bp.Params(filter_mode=mode, window=window, ext_mode=ext)
        g, r = assert_same(bp, orc, q, ascii, off, p, trace=True)
        assert len(g) > 10
    # repeated searches on one db (segment publication epochs)
    t = bp.build_query_table(q, bp.Params())
    first = tuples(bp.search_ungapped(t, d, bp.Params()))
    for _ in range(3):
        assert tuples(bp.search_ungapped(t, d, bp.Params())) == first


def test_long_query_2000(bp, orc):
    q = gen_query(2000, 2000)
    db = gen_db(7, 8, n_subjects=400, mean_len=375.0, queries=[q], plant_frac=0.2)
    assert_same(bp, orc, q, db.ascii, db.offsets, bp.Params(), trace=True)


def test_longest_query(bp, orc, kernel_variant):
    """BLASTP_MAX_QUERY_LEN (16,000): the diagonal ring is ~96 KB per warp,
    so a CTA holds two warps and the lookup table stays in global memory;
    results identical to the oracle.  One residue more is rejected.  The
    CTA variant's per-CTA diagonal state does not fit shared memory at this
    length: forcing it (BLASTP_KERNEL=cta) fails loudly."""
    q = gen_query(16000, 16000)
    db = gen_db(9, 10, n_subjects=150, mean_len=375.0, queries=[q], plant_frac=0.3)
    if kernel_variant == "cta":
        with pytest.raises(bp.BlastpError, match="invalid configuration"):
            gpu_run(bp, q, db.ascii, db.offsets, bp.Params())
        return
    g, _ = assert_same(bp, orc, q, db.ascii, db.offsets, bp.Params(), trace=False,
                       nthreads=os.cpu_count() or 8)
    assert len(g) > 20
    with pytest.raises(bp.BlastpError) as e:
        bp.build_query_table(gen_query(16001, 16001))
    assert e.value.status == -3  # BLASTP_E_TOO_LONG


# ------------------------------------------------------------------ API

def test_device_variant_and_sort_match_host_variant(bp, orc):
    import torch
    (q,), db = config_workload(1)
    p = bp.Params()
    t = bp.build_query_table(q, p)
    d = bp.pack_db(db.ascii, db.offsets)
    host = bp.search_ungapped(t, d, p)
    cap = len(host) + 5
    out = torch.zeros(cap * 7, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    bp.search_ungapped_device(t, d, out.data_ptr(), cap, cnt.data_ptr(), p)
    n = int(cnt.item())
    assert n == len(host)
    bp.sort_hsps_device(out.data_ptr(), n)
    dev = out[: n * 7].view(n, 7).cpu().numpy()
    assert [tuple(x) for x in dev.tolist()] == tuples(host)
    # a too-small buffer still reports the full count
    small = torch.zeros(7 * 3, dtype=torch.int32, device="cuda")
    bp.search_ungapped_device(t, d, small.data_ptr(), 3, cnt.data_ptr(), p)
    assert int(cnt.item()) == len(host)


def test_hit_mode_dedup_device(bp, orc):
    """Alg. 4 (ext_mode HIT) returns one extension per passing hit; the
    de-duplication step the paper leaves before gapped extension
    (blastp_unique_hsps_device after the canonical sort) gives exactly the
    distinct HSPs of the oracle's HIT list; on a DIAGONAL list it is a no-op."""
    import torch
    (q,), db = config_workload(1)
    d = bp.pack_db(db.ascii, db.offsets)
    for ext_mode in (1, 0):
        p = bp.Params(ext_mode=ext_mode)
        t = bp.build_query_table(q, p)
        cap = 1 << 16
        out = torch.zeros(cap * 7, dtype=torch.int32, device="cuda")
        cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
        bp.search_ungapped_device(t, d, out.data_ptr(), cap, cnt.data_ptr(), p)
        n = int(cnt.item())
        bp.sort_hsps_device(out.data_ptr(), n)
        bp.unique_hsps_device(out.data_ptr(), n, cnt.data_ptr())
        m = int(cnt.item())
        got = [tuple(x) for x in out[: m * 7].view(m, 7).cpu().numpy().tolist()]
        ref = tuples(oracle_run(orc, q, db.ascii, db.offsets, p).hsps)
        assert got == sorted(set(ref))
        if ext_mode == 1:
            assert m < n  # there were duplicates
        else:
            assert m == n


def test_hit_dedup_equals_diagonal(bp, orc):
    """ext_mode HIT_DEDUP (R17): Alg. 4 extends every passing hit, then the
    de-duplication step walks each diagonal's extensions in seed
    order with Alg. 3's coverage rule -- the result is exactly the oracle's
    DIAGONAL list (config 1, a long-subject DB, random small cases); the
    device variant's seed records reduce to the same list through
    blastp_dedup_covered_device."""
    import torch
    cases = []
    (q,), db = config_workload(1)
    cases.append((q, db.ascii, db.offsets, bp.Params()))
    q2 = gen_query(21, 300).decode()
    a2, o2 = _long_subject_db(q2)
    cases.append((q2, a2, o2, bp.Params(window=80)))
    rng = np.random.default_rng(4)
    for _ in range(20):
        lq = int(rng.choice([17, 64, 300]))
        qq = "".join(rng.choice(list(ALPHA[:20]), size=lq))
        a3, o3 = _rand_db(rng, int(rng.integers(1, 40)), 0, 400, qq, plant=0.6)
        cases.append((qq, a3, o3, bp.Params(window=int(rng.choice([40, 10])),
                                            cutoff=int(rng.choice([41, 20])))))
    n_hit_extra = 0
    for qq, aa, oo, p in cases:
        pd = bp.Params(**{**p.__dict__, "ext_mode": bp.EXT_HIT_DEDUP})
        t = bp.build_query_table(qq, pd)
        d = bp.pack_db(aa, oo)
        got = tuples(bp.search_ungapped(t, d, pd))
        exp = tuples(oracle_run(orc, qq, aa, oo, p).hsps)
        assert got == exp
        hit = tuples(bp.search_ungapped(t, d, bp.Params(**{**p.__dict__, "ext_mode": 1})))
        n_hit_extra += len(hit) - len(exp)
        cap = 1 << 16
        out = torch.zeros(cap * 7, dtype=torch.int32, device="cuda")
        cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
        bp.search_ungapped_device(t, d, out.data_ptr(), cap, cnt.data_ptr(), pd)
        n = int(cnt.item())
        assert n <= cap
        bp.dedup_covered_device(out.data_ptr(), n, pd.cutoff, cnt.data_ptr())
        m = int(cnt.item())
        assert [tuple(x) for x in out[: m * 7].view(m, 7).cpu().numpy().tolist()] == exp
    assert n_hit_extra > 0  # Alg. 4 alone returns more (duplicates / covered seeds)


@pytest.mark.parametrize("score", ["pssm", "pssm_global"])
def test_pssm_scores_identical(bp, orc, monkeypatch, kernel_variant, score):
    """The PSSM switch (paper E2; BLASTP_SCORE) is perf-only: the
    X-drop reads PSSM[q][a] = BLOSUM62[query[q]][a] instead of the matrix and
    the query code -- every hit, passing hit, extension and HSP identical to
    the oracle (config 1 traced, config 2 complete, long subjects)."""
    if kernel_variant != "block":
        pytest.skip("the PSSM switch is the block kernel's")
    monkeypatch.setenv("BLASTP_SCORE", score)
    (q,), db = config_workload(1)
    assert_same(bp, orc, q, db.ascii, db.offsets, bp.Params())
    q2 = gen_query(21, 300).decode()
    a2, o2 = _long_subject_db(q2)
    assert_same(bp, orc, q2, a2, o2, bp.Params(ext_mode=1))
    (q3,), db3 = _config2()
    p = bp.Params()
    g = bp.search_ungapped(bp.build_query_table(q3, p), bp.pack_db(db3.ascii, db3.offsets), p)
    assert_lists_equal(g, oracle_full(orc, "config2", q3, db3.ascii, db3.offsets, p), "config 2")


@pytest.mark.parametrize("np_nc", [(8, 8), (16, 16), (28, 4)])
def test_cta_bins_per_warp_knobs(bp, orc, monkeypatch, kernel_variant, np_nc):
    """The E1 knobs of the CTA variant (producer / consumer warps: bins per
    warp) leave results unchanged (config 1 traced, long subjects)."""
    if kernel_variant != "cta":
        pytest.skip("CTA-variant knobs")
    monkeypatch.setenv("BLASTP_CTA_NP", str(np_nc[0]))
    monkeypatch.setenv("BLASTP_CTA_NC", str(np_nc[1]))
    (q,), db = config_workload(1)
    assert_same(bp, orc, q, db.ascii, db.offsets, bp.Params())
    q2 = gen_query(21, 300).decode()
    a2, o2 = _long_subject_db(q2)
    assert_same(bp, orc, q2, a2, o2, bp.Params(filter_mode=1))


def _host_db_search(bp, t, ascii, off, p, **kw):
    import torch
    cap = 1 << 16
    out = torch.zeros(cap * 7, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    bp.search_host_db(t, ascii, off, out.data_ptr(), cap, cnt.data_ptr(), p, **kw)
    n = int(cnt.item())
    assert n <= cap
    bp.sort_hsps_device(out.data_ptr(), n)
    return [tuple(x) for x in out[: n * 7].view(n, 7).cpu().numpy().tolist()]


def test_search_host_db_pipelined_parts(bp, orc):
    """blastp_search_host_db (parts copied while the previous part is
    searched) equals pack + search of the whole shard, for automatic and
    explicit part counts, shards, a query batch and long subjects."""
    q = gen_query(21, 300).decode()
    ascii, off = _long_subject_db(q)
    rng = np.random.default_rng(8)
    a2, o2 = _rand_db(rng, 3000, 0, 600, q)
    ascii = np.concatenate([a2, ascii])
    off = np.concatenate([o2, o2[-1] + off[1:]]).astype(np.int64)
    p = bp.Params()
    t = bp.build_query_table(q, p)
    whole = tuples(bp.search_ungapped(t, bp.pack_db(ascii, off), p))
    r = oracle_run(orc, q, ascii, off, p, nthreads=4)
    assert whole == tuples(r.hsps)
    for parts in (0, 1, 2, 7, 50):
        assert _host_db_search(bp, t, ascii, off, p, num_parts=parts) == whole, parts
    for k in range(3):  # a shard's parts: global subject ids
        shard = tuples(bp.search_ungapped(t, bp.pack_db(ascii, off, k, 3), p))
        assert _host_db_search(bp, t, ascii, off, p, shard_index=k, num_shards=3,
                               num_parts=4) == shard
    qs = [q, gen_query(22, 127).decode()]
    tb = bp.build_query_batch(qs, p)
    assert _host_db_search(bp, tb, ascii, off, p, num_parts=3) == \
        tuples(bp.search_ungapped(tb, bp.pack_db(ascii, off), p))
    # no subjects at all
    assert _host_db_search(bp, t, np.zeros(0, np.uint8), np.zeros(1, np.int64), p) == []


def _formatted_search(bp, t, hdb, p):
    import torch
    cap = 1 << 16
    out = torch.zeros(cap * 7, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    bp.search_formatted_db(t, hdb, out.data_ptr(), cap, cnt.data_ptr(), p)
    n = int(cnt.item())
    assert n <= cap
    bp.sort_hsps_device(out.data_ptr(), n)
    return [tuple(x) for x in out[: n * 7].view(n, 7).cpu().numpy().tolist()]


def test_formatted_host_db(bp, orc):
    """blastp_format_host_db + blastp_search_formatted_db (parts packed once
    into pinned host memory, streamed by copies only) equals pack + search of
    the whole shard: automatic and explicit part counts, shards, repeated
    searches of one image, a query batch, every filter mode and long subjects
    (segment plans travel with the image)."""
    q = gen_query(21, 300).decode()
    ascii, off = _long_subject_db(q)
    rng = np.random.default_rng(9)
    a2, o2 = _rand_db(rng, 3000, 0, 600, q)
    ascii = np.concatenate([a2, ascii])
    off = np.concatenate([o2, o2[-1] + off[1:]]).astype(np.int64)
    t = bp.build_query_table(q, bp.Params())
    d = bp.pack_db(ascii, off)
    for p in (bp.Params(), bp.Params(filter_mode=1), bp.Params(filter_mode=2),
              bp.Params(ext_mode=1)):
        whole = tuples(bp.search_ungapped(t, d, p))
        for parts in (0, 1, 3, 7):
            hdb = bp.format_host_db(ascii, off, num_parts=parts)
            assert hdb.nseq == len(off) - 1 and hdb.residues == int(off[-1])
            assert parts == 0 or hdb.num_parts == parts
            assert _formatted_search(bp, t, hdb, p) == whole, (p, parts)
            assert _formatted_search(bp, t, hdb, p) == whole  # the image is reusable
            hdb.free()
    p = bp.Params()
    assert tuples(bp.search_ungapped(t, d, p)) == tuples(oracle_run(orc, q, ascii, off, p,
                                                                    nthreads=4).hsps)
    for k in range(3):
        shard = tuples(bp.search_ungapped(t, bp.pack_db(ascii, off, k, 3), p))
        hdb = bp.format_host_db(ascii, off, shard_index=k, num_shards=3, num_parts=2)
        assert _formatted_search(bp, t, hdb, p) == shard
    qs = [q, gen_query(22, 127).decode()]
    tb = bp.build_query_batch(qs, p)
    hdb = bp.format_host_db(ascii, off, num_parts=4)
    assert _formatted_search(bp, tb, hdb, p) == tuples(bp.search_ungapped(tb, d, p))
    empty = bp.format_host_db(np.zeros(0, np.uint8), np.zeros(1, np.int64))
    assert _formatted_search(bp, t, empty, p) == []


@pytest.mark.parametrize("slots", ["1", "2"])
def test_formatted_host_db_slot_ring(bp, monkeypatch, slots):
    """The formatted search's bounded device memory: with 1 or 2 part slots
    for 9 parts every slot is reused (each copy waits for the search of the
    slot's previous part) and the result still equals the resident search."""
    monkeypatch.setenv("BLASTP_PIPE_SLOTS", slots)
    q = gen_query(23, 400).decode()
    rng = np.random.default_rng(11)
    ascii, off = _rand_db(rng, 4000, 0, 700, q)
    t = bp.build_query_table(q, bp.Params())
    d = bp.pack_db(ascii, off)
    for p in (bp.Params(), bp.Params(filter_mode=2)):
        whole = tuples(bp.search_ungapped(t, d, p))
        assert len(whole) > 10
        hdb = bp.format_host_db(ascii, off, num_parts=9)
        assert _formatted_search(bp, t, hdb, p) == whole
        hdb.free()


def test_formatted_host_db_config3_full_size(bp):
    """Config 3 at full size (the bench's e2e path): the formatted image
    streamed in parts gives exactly the resident shard's HSP list (the
    resident list is itself pinned to the oracle by
    test_config3_full)."""
    import torch
    (q,), db = _config3()
    p = bp.Params()
    t = bp.build_query_table(q, p)
    cap = 1 << 20
    outs = []
    for mode in ("resident", "formatted"):
        out = torch.zeros(cap * 7, dtype=torch.int32, device="cuda")
        cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
        if mode == "resident":
            d = bp.pack_db(db.ascii, db.offsets)
            bp.search_ungapped_device(t, d, out.data_ptr(), cap, cnt.data_ptr(), p)
            n = int(cnt.item())
            d.free()
        else:
            h = bp.format_host_db(db.ascii, db.offsets)
            assert h.num_parts > 4
            bp.search_formatted_db(t, h, out.data_ptr(), cap, cnt.data_ptr(), p)
            n = int(cnt.item())
            h.free()
        assert 10000 < n <= cap
        bp.sort_hsps_device(out.data_ptr(), n)
        outs.append(out[: n * 7].cpu())
    assert torch.equal(outs[0], outs[1])


def _same_start_db(orc):
    """A seeded DB whose oracle HSP list holds two HSPs of one diagonal with
    the same start and different ends (a later seed beyond the first HSP's
    end whose left extension reaches back to the same start): the canonical
    order then depends on the length field (R11)."""
    rng = np.random.default_rng(7)
    q = gen_query(77, 300).decode()
    for _ in range(40):
        subs = []
        for _ in range(50):
            s = list(rng.choice(list(ALPHA[:20]), size=400))
            a, b, n = int(rng.integers(0, 200)), int(rng.integers(0, 300)), int(rng.integers(30, 90))
            seg = list(q[a:a + n])
            for i in np.nonzero(rng.random(len(seg)) < 0.35)[0]:
                seg[i] = ALPHA[int(rng.integers(0, 20))]
            s[b:b + len(seg)] = seg
            subs.append("".join(s[:400]))
        ascii = np.frombuffer("".join(subs).encode(), dtype=np.uint8).copy()
        off = np.arange(0, 50 * 400 + 1, 400, dtype=np.int64)
        h = tuples(orc.search(orc.encode(q), orc.encode(ascii.tobytes()), off).hsps)
        if len({x[:4] for x in h}) < len(h):
            return q, ascii, off
    raise AssertionError("no same-start HSP pair generated")


def test_same_start_hsps_canonical_order(bp, orc):
    """HSPs equal in (query, subject, diagonal, q_start) are ordered by
    length as R11 requires, on the host (GPU-sorted) and device variants."""
    q, ascii, off = _same_start_db(orc)
    for ext_mode in (0, 1, 2):
        p = bp.Params(ext_mode=ext_mode)
        g, r = assert_same(bp, orc, q, ascii, off, p, trace=True)
        assert len({x[:4] for x in tuples(g)}) < len(g)


def test_query_batch_equals_single_queries(bp, orc):
    qs = [gen_query(11 + i, L) for i, L in enumerate([100, 350, 900])]
    db = gen_db(12, 13, n_subjects=500, mean_len=300.0, queries=qs, plant_frac=0.3)
    p = bp.Params()
    d = bp.pack_db(db.ascii, db.offsets)
    batch = bp.search_ungapped(bp.build_query_batch(qs, p), d, p)
    exp = []
    for i, q in enumerate(qs):
        exp += tuples(oracle_run(orc, q, db.ascii, db.offsets, p, query_id=i).hsps)
    assert tuples(batch) == sorted(exp)


def test_query_groups_equal_single_queries(bp, orc):
    """A batch of short queries is searched as query groups (members
    concatenated with sentinel gaps >= A + 8, one scan per group; SURVEY 8(f)
    rank 1): HSPs identical to the oracle's per-query searches for every
    filter and extension mode, for a window that fits the gap (groups) and one
    that does not (query by query), with planted homologs of every member,
    long subjects (segments) and the formatted host database path."""
    import torch
    rng = np.random.default_rng(77)
    lens = [60, 90, 120, 150, 200, 240, 310, 400, 3, 17, 520, 700, 45]
    qs = [gen_query(300 + i, L) for i, L in enumerate(lens)]
    db = gen_db(301, 302, n_subjects=400, mean_len=300.0, queries=qs, plant_frac=0.5)
    lq, lo = _long_subject_db(qs[7].decode())
    ascii = np.concatenate([db.ascii, lq])
    off = np.concatenate([db.offsets, db.offsets[-1] + lo[1:]]).astype(np.int64)
    d = bp.pack_db(ascii, off)
    for build_window in (40, 256):
        tb = bp.build_query_batch(qs, bp.Params(window=build_window))
        g, alone, gap = tb.groups
        assert g >= 2 and gap == build_window + 8
        for p in (bp.Params(), bp.Params(filter_mode=1), bp.Params(filter_mode=2),
                  bp.Params(ext_mode=1), bp.Params(ext_mode=2), bp.Params(window=80),
                  bp.Params(window=256)):
            assert tb.launches(p) == (g + alone if p.window + 8 <= gap else len(qs))
            got = tuples(bp.search_ungapped(tb, d, p))
            exp = []
            for i, q in enumerate(qs):
                exp += tuples(oracle_run(orc, q, ascii, off, p, query_id=i, nthreads=4).hsps)
            assert got == sorted(exp), (build_window, p)
            assert len(got) > 100
    # the formatted host database streams the groups too
    tb = bp.build_query_batch(qs, bp.Params())
    h = bp.format_host_db(ascii, off, num_parts=3)
    cap = 1 << 18
    out = torch.zeros(cap * 7, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    bp.search_formatted_db(tb, h, out.data_ptr(), cap, cnt.data_ptr())
    n = int(cnt.item())
    bp.sort_hsps_device(out.data_ptr(), n)
    assert [tuple(x) for x in out[: n * 7].view(n, 7).cpu().numpy().tolist()] == \
        tuples(bp.search_ungapped(tb, d, bp.Params()))
    # grouping off: same results
    import os as _os
    _os.environ["BLASTP_GROUP"] = "0"
    try:
        t0 = bp.build_query_batch(qs, bp.Params())
        assert t0.groups[0] == 0
        assert tuples(bp.search_ungapped(t0, d, bp.Params())) == \
            tuples(bp.search_ungapped(tb, d, bp.Params()))
    finally:
        del _os.environ["BLASTP_GROUP"]


def test_sharded_union_equals_whole(bp, orc):
    (q,), db = config_workload(1)
    p = bp.Params()
    t = bp.build_query_table(q, p)
    whole = tuples(bp.search_ungapped(t, bp.pack_db(db.ascii, db.offsets), p))
    for n in (2, 3, 8):
        parts = []
        for k in range(n):
            parts += tuples(bp.search_ungapped(t, bp.pack_db(db.ascii, db.offsets, k, n), p))
        assert parts == whole  # contiguous ranges, canonical order per shard


def test_bad_residue_reported(bp):
    ascii = np.frombuffer(b"MKVLA-GG", dtype=np.uint8).copy()
    with pytest.raises(bp.BlastpError) as e:
        bp.pack_db(ascii, np.array([0, 8], dtype=np.int64))
    assert e.value.status == bp.E_BAD_RESIDUE
    with pytest.raises(bp.BlastpError) as e:
        bp.build_query_table("MKV1", bp.Params())
    assert e.value.status == bp.E_BAD_RESIDUE


def test_formatted_db_and_groups_errors(bp):
    """Error paths of the formatted host database and of query batches: a bad
    residue or a decreasing offset fails the format with the pack's status,
    a bad query in a batch fails the whole batch, NULL handles are rejected."""
    import ctypes
    bad = np.frombuffer(b"MKVLAGGQ-RST", dtype=np.uint8).copy()
    with pytest.raises(bp.BlastpError) as e:
        bp.format_host_db(bad, np.array([0, 6, 12], dtype=np.int64), num_parts=2)
    assert e.value.status == bp.E_BAD_RESIDUE
    ok = np.frombuffer(b"MKVLAGGQWRST", dtype=np.uint8).copy()
    with pytest.raises(bp.BlastpError) as e:
        bp.format_host_db(ok, np.array([0, 8, 6, 12], dtype=np.int64))
    assert e.value.status == bp.E_INVALID_ARG
    with pytest.raises(bp.BlastpError) as e:
        bp.build_query_batch(["MKVLAGG", "MKV1LL", "WWWAAA"], bp.Params())
    assert e.value.status == bp.E_BAD_RESIDUE
    t = bp.build_query_table("MKVLAGGQ", bp.Params())
    rc = bp.lib.blastp_search_formatted_db(t.handle, None, ctypes.byref(bp.Params().c()), None,
                                           None, 0, None)
    assert rc == bp.E_INVALID_ARG
    assert bp.lib.blastp_query_table_groups(None, None, None, None) == bp.E_INVALID_ARG
    assert bp.lib.blastp_host_db_info(None, None, None, None, None, None) == bp.E_INVALID_ARG
    bp.lib.blastp_host_db_free(None)  # no-op


def test_debug_stats_match_oracle_counts(bp, orc):
    """Event counters of the kernel agree with the oracle's lists (config 1)."""
    (q,), db = config_workload(1)
    p = bp.Params()
    t = bp.build_query_table(q, p)
    d = bp.pack_db(db.ascii, db.offsets)
    s = bp.debug_stats(t, d, p)
    r = oracle_run(orc, q, db.ascii, db.offsets, p, want_hits=True)
    assert s["hits"] == len(r.hits)
    assert s["passing"] == len(r.passing)
    assert s["accepted"] == len(r.extensions)
    assert s["emitted"] == len(r.hsps)
    assert s["extended"] >= s["accepted"] and s["enqueued"] >= s["extended"] - 0


def test_pack_rejects_bad_offsets(bp):
    ascii = np.frombuffer(b"MKVLAGGAAA", dtype=np.uint8).copy()
    with pytest.raises(bp.BlastpError) as e:
        bp.pack_db(ascii, np.array([0, 6, 4, 10], dtype=np.int64))
    assert e.value.status == bp.E_INVALID_ARG


def test_graft_smoke_entry(bp):
    import __graft_entry__ as g
    g.smoke()
