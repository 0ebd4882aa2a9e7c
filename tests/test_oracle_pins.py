"""Pins of the oracle against things other than itself:
exhaustive brute force on tiny inputs, closed forms, invariants, planted
exact copies and the independent oracle-B formulation."""
import os
from collections import defaultdict

import numpy as np
import pytest

from oracle.oracle_b import search_b
from synth import RR_FREQ, gen_db, gen_query

STD = "ARNDCQEGHILKMFPSTWYV"


def rr_codes(rng, n, alphabet):
    p = np.array([RR_FREQ[c] for c in STD])
    p /= p.sum()
    letters = rng.choice(len(STD), size=n, p=p)
    return np.array([alphabet.index(STD[i]) for i in letters], dtype=np.uint8)


def direct_hits(Q, S, M, T=11, w=3):
    """All (q, s) with word score >= T by direct O(Lq*Ls) scoring (numpy)."""
    lq, ls = len(Q), len(S)
    if lq < w or ls < w:
        return set()
    P = M[np.ix_(Q, S)].astype(np.int64)  # pair scores [lq, ls]
    W = P[: lq - w + 1, : ls - w + 1].copy()
    for k in range(1, w):
        W += P[k: lq - w + 1 + k, k: ls - w + 1 + k]
    qs, ss = np.nonzero(W >= T)
    return set(zip(qs.tolist(), ss.tolist()))


# ------------------------------------------------------------------ P2 (R3)

def test_exhaustive_word_pairs_tiny(orc, B62):
    """Table-based hits == direct scoring of every word pair (P2)."""
    al = orc.alphabet()
    rng = np.random.default_rng(7)
    for case in range(300):
        lq, ls = rng.integers(1, 41, size=2)
        if case % 3 == 0:  # include B/Z/X/* letters too
            Q = rng.integers(0, 24, size=lq).astype(np.uint8)
            S = rng.integers(0, 24, size=ls).astype(np.uint8)
        else:
            Q, S = rr_codes(rng, lq, al), rr_codes(rng, ls, al)
        T = int(rng.choice([11, 11, 8, 13]))
        r = orc.search(Q, S, np.array([0, ls]), orc.Params(threshold=T), want_hits=True)
        got = {(int(h[1]), int(h[2])) for h in r.hits}
        assert len(got) == len(r.hits)
        assert got == direct_hits(Q, S, B62, T), case


def test_neighbourhood_sizes(orc, B62):
    """Neighbourhood-size statistics: AAA 1, LLL 1, CCC 58,
    IYP 29, WWW 118; mean over the 8000 standard words 34.37, RR-weighted
    18.96, max 163."""
    al = orc.alphabet()
    idx = [al.index(c) for c in STD]
    # neighbour words over the 20 standard letters (the statistics' domain)
    std_words = np.array([(a * 24 + b) * 24 + c for a in idx for b in idx for c in idx])
    size = {}
    for w in ["AAA", "LLL", "CCC", "IYP", "WWW"]:
        off, pos = orc.neighbourhood(orc.encode(w), B62, 11)
        assert list(np.unique(pos)) == [0]
        size[w] = int((off[std_words + 1] - off[std_words]).sum())
    assert size == {"AAA": 1, "LLL": 1, "CCC": 58, "IYP": 29, "WWW": 118}
    # all 8000 standard words at once: a query that enumerates them would be
    # 24k long; use per-position counts from one long table instead.
    words = np.array([[a, b, c] for a in idx for b in idx for c in idx], dtype=np.uint8)
    q = words.reshape(-1)  # word k sits at position 3k (other positions ignored)
    off, pos = orc.neighbourhood(q, B62, 11)
    std_pos = np.concatenate([pos[off[v]:off[v + 1]] for v in std_words])
    counts = np.bincount(std_pos, minlength=len(q))[::3][:8000]
    p = np.array([RR_FREQ[c] for c in STD])
    p /= p.sum()
    pw = np.einsum("i,j,k->ijk", p, p, p).reshape(-1)
    assert abs(counts.mean() - 34.37) < 0.01
    assert abs((counts * pw).sum() - 18.96) < 0.01
    assert counts.min() == 1 and counts.max() == 163


# ------------------------------------------------------------------ P3 (R4)

def _p_hit(B62, al, T=11):
    """P[S(w,w') >= T] for w, w' ~ RR^3, by exact convolution."""
    idx = [al.index(c) for c in STD]
    p = np.array([RR_FREQ[c] for c in STD])
    p /= p.sum()
    S = B62[np.ix_(idx, idx)]
    lo = S.min()
    dist = np.zeros(S.max() - lo + 1)
    for i in range(20):
        for j in range(20):
            dist[S[i, j] - lo] += p[i] * p[j]
    tot = np.convolve(np.convolve(dist, dist), dist)
    scores = np.arange(len(tot)) + 3 * lo
    return tot[scores >= T].sum()


def test_expected_hit_count_closed_form(orc, B62):
    al = orc.alphabet()
    ph = _p_hit(B62, al)
    assert abs(ph - 0.0021009693) < 1e-9
    rng = np.random.default_rng(11)
    lq = 300
    Q = rr_codes(rng, lq, al)
    lens = rng.integers(50, 400, size=800)
    offs = np.concatenate([[0], np.cumsum(lens)])
    db = rr_codes(rng, int(offs[-1]), al)
    r = orc.search(Q, db, offs, want_hits=True)
    n_words_s = int((lens - 2).sum())
    # E[hits | query] = n_words_s * sum_q P_RR[S(Q[q:q+3], v) >= T], v ~ RR^3,
    # by direct enumeration of the 8000 standard words (no table).
    idx = np.array([al.index(c) for c in STD])
    p = np.array([RR_FREQ[c] for c in STD])
    p /= p.sum()
    pw = np.einsum("i,j,k->ijk", p, p, p)
    per_q = []
    for q in range(lq - 2):
        sc = (B62[Q[q], idx][:, None, None] + B62[Q[q + 1], idx][None, :, None]
              + B62[Q[q + 2], idx][None, None, :])
        per_q.append(pw[sc >= 11].sum())
    expect = n_words_s * float(np.sum(per_q))
    assert abs(len(r.hits) - expect) < 6 * np.sqrt(expect), (len(r.hits), expect)


# ------------------------------------------------------------------ P4 (R8)

def test_xdrop_infinite_x_is_max_prefix(orc):
    rng = np.random.default_rng(3)
    M = np.diag(np.arange(-8, 9)).astype(np.int32)  # letter k scores k-8 vs itself
    for _ in range(300):
        n = int(rng.integers(0, 80))
        sc = rng.integers(-8, 9, size=n)
        seq = (sc + 8).astype(np.uint8)
        best, ln, steps = orc.xdrop_pairs(seq, seq, M, 10 ** 9, n=n)
        cs = np.concatenate([[0], np.cumsum(sc)])
        assert best == max(0, cs.max()) and steps == n
        assert ln == (int(np.argmax(cs)) if cs.max() > 0 else 0)


def test_xdrop_stop_rule_random(orc):
    """R8 stop rule written from Fig. 8: stop at the first k with
    best_k - run_k >= X; best over the consumed prefix, shortest argmax."""
    rng = np.random.default_rng(5)
    M = np.diag(np.arange(-8, 9)).astype(np.int32)
    for _ in range(500):
        n = int(rng.integers(0, 60))
        X = int(rng.integers(1, 30))
        sc = rng.integers(-8, 9, size=n)
        seq = (sc + 8).astype(np.uint8)
        best, ln, steps = orc.xdrop_pairs(seq, seq, M, X, n=n)
        run = np.cumsum(sc)
        bst = np.maximum.accumulate(np.maximum(run, 0))
        stop = np.nonzero(bst - run >= X)[0]
        k = int(stop[0]) + 1 if len(stop) else n
        cs = np.concatenate([[0], run[:k]])
        assert steps == k
        assert best == cs.max() and ln == int(np.argmax(cs))


# ------------------------------------------------------------- P5-P8 (R6-R10)

def _check_invariants(orc, B62, Q, db, offs, r, p):
    by_diag = defaultdict(list)
    for subj, q, s in r.hits:
        by_diag[(int(subj), int(s - q))].append(int(s))
    passing = {(int(a), int(b), int(c)) for a, b, c in r.passing}
    # P7: brute-force pairwise filter
    for (subj, d), ss in by_diag.items():
        ss.sort()
        for h in ss:
            ok = any(p.min_gap <= (h - x if p.filter_mode == 0 else abs(h - x)) < p.window
                     for x in ss)
            assert ((subj, h - d, h) in passing) == ok
    exts = defaultdict(list)
    for e in r.extensions:
        exts[(int(e["subject_id"]), int(e["diagonal"]))].append(e)
    for (subj, d), es in exts.items():
        S = db[offs[subj]:offs[subj + 1]]
        es.sort(key=lambda e: e["s_start"])
        prev_end = -1
        for e in es:
            qs, ss, L, sc = (int(e[k]) for k in ("q_start", "s_start", "length", "score"))
            assert ss - qs == d and L >= p.word_len
            pair = B62[Q[qs:qs + L], S[ss:ss + L]].astype(int)
            assert pair.sum() == sc  # P5
            end = ss + L - 1
            assert end > prev_end  # P8: strictly increasing reach
            prev_end = end
    # P8 / north_star: every passing hit is extended or covered
    for (subj, d), ss in by_diag.items():
        es = sorted(exts.get((subj, d), []), key=lambda e: e["s_start"])
        reach, ei = -1, 0
        for h in sorted(ss):
            if (subj, h - d, h) not in passing:
                continue
            if h <= reach:
                continue
            e = es[ei]
            ei += 1
            assert e["s_start"] <= h and h + p.word_len - 1 <= e["s_start"] + e["length"] - 1
            reach = int(e["s_start"] + e["length"] - 1)
        assert ei == len(es)
    # P6: maximality of each side (shortest argmax; stop point honest)
    for e in r.extensions:
        subj = int(e["subject_id"])
        S = db[offs[subj]:offs[subj + 1]]
        qs, ss, L = int(e["q_start"]), int(e["s_start"]), int(e["length"])
        d = ss - qs
        # right end: scores beyond the end until X-drop never exceed
        tail = []
        k = 0
        while qs + L + k < len(Q) and ss + L + k < len(S):
            tail.append(B62[Q[qs + L + k], S[ss + L + k]])
            k += 1
        run = np.cumsum(tail) if tail else np.zeros(0)
        for v in run:
            assert v <= 0
            if v <= -p.xdrop:
                break
    hsp = r.hsps
    assert (hsp["score"] >= p.cutoff).all()
    emitted = {tuple(x) for x in r.extensions[r.extensions["score"] >= p.cutoff].tolist()}
    assert emitted == {tuple(x) for x in hsp.tolist()}


@pytest.mark.parametrize("mode", [0, 1])
def test_invariants_random_related(orc, B62, mode):
    al = orc.alphabet()
    rng = np.random.default_rng(100 + mode)
    Q = rr_codes(rng, 150, al)
    subs = []
    for i in range(120):
        S = rr_codes(rng, int(rng.integers(5, 300)), al)
        if i % 3 == 0 and len(S) > 40:  # mutated query segment
            L = int(rng.integers(20, min(120, len(S))))
            a = int(rng.integers(0, len(Q) - L))
            b = int(rng.integers(0, len(S) - L + 1))
            seg = Q[a:a + L].copy()
            mut = rng.random(L) < 0.35
            seg[mut] = rr_codes(rng, int(mut.sum()), al)
            S[b:b + L] = seg
        subs.append(S)
    offs = np.concatenate([[0], np.cumsum([len(s) for s in subs])])
    db = np.concatenate(subs)
    p = orc.Params(filter_mode=mode)
    r = orc.search(Q, db, offs, p, want_hits=True)
    assert len(r.extensions) > 20 and len(r.hsps) > 5
    _check_invariants(orc, B62, Q, db, offs, r, p)


# ------------------------------------------------------------------ P9

def test_planted_exact_copies_are_spanned(orc):
    q = gen_query(9, 400)
    db = gen_db(77, 78, n_subjects=3000, mean_len=250, queries=[q], plant_frac=0.2)
    Q = orc.encode(q)
    codes = orc.encode(db.ascii.tobytes())
    r = orc.search(Q, codes, db.offsets)
    exts = defaultdict(list)
    for e in r.extensions:
        exts[(int(e["subject_id"]), int(e["diagonal"]))].append(e)
    n = 0
    for pl in db.plants:
        if not pl["exact"] or pl["length"] < 6:
            continue
        d = int(pl["s_start"] - pl["q_start"])
        a, b = int(pl["s_start"]), int(pl["s_start"] + pl["length"] - 1)
        es = exts[(int(pl["subject"]), d)]
        assert any(e["s_start"] <= a and e["s_start"] + e["length"] - 1 >= b for e in es)
        n += 1
    assert n >= 20


# ------------------------------------------------------------------ P10

def _oracle_b_cases(rng, al, n):
    for case in range(n):
        kind = case % 6
        lq = int(rng.integers(1, 61))
        ls = int(rng.integers(0, 61))
        Q = rr_codes(rng, lq, al)
        if kind == 0:
            subs = [rr_codes(rng, ls, al)]
        elif kind == 1:  # subject = mutated query
            S = Q.copy()
            mut = rng.random(lq) < 0.3
            S[mut] = rr_codes(rng, int(mut.sum()), al)
            subs = [S, rr_codes(rng, ls, al)]
        elif kind == 2:  # several subjects, some shorter than a word
            subs = [rr_codes(rng, int(rng.integers(0, 8)), al) for _ in range(3)] + \
                   [np.concatenate([Q[: lq // 2], rr_codes(rng, 5, al), Q[lq // 2:]])]
        elif kind == 3:  # any letters incl. B/Z/X/*
            Q = rng.integers(0, 24, size=lq).astype(np.uint8)
            subs = [rng.integers(0, 24, size=ls).astype(np.uint8), Q[::-1].copy()]
        elif kind == 4:  # hits at both ends of the subject
            subs = [np.concatenate([Q[:5], rr_codes(rng, ls, al), Q[-5:]])]
        else:  # low complexity
            c = al.index(str(rng.choice(list("WAQC"))))
            Q = np.full(lq, c, dtype=np.uint8)
            subs = [np.full(ls, c, dtype=np.uint8), rr_codes(rng, ls, al)]
        yield Q, subs


def test_oracle_b_agrees_on_random_tiny_cases(orc, B62):
    al = orc.alphabet()
    rng = np.random.default_rng(2024)
    n = int(os.environ.get("ORACLE_B_CASES", "600"))
    M = B62.tolist()
    checked_ext = 0
    for i, (Q, subs) in enumerate(_oracle_b_cases(rng, al, n)):
        mode = i % 2
        ext_mode = (i // 2) % 2  # DIAGONAL (Alg. 3) / HIT (Alg. 4)
        T = 11 if i % 5 else 9
        X = int(rng.choice([16, 16, 5, 30]))
        cutoff = int(rng.choice([41, 20]))
        offs = np.concatenate([[0], np.cumsum([len(s) for s in subs])]).astype(np.int64)
        db = np.concatenate(subs).astype(np.uint8) if offs[-1] else np.zeros(0, np.uint8)
        p = orc.Params(threshold=T, xdrop=X, cutoff=cutoff, filter_mode=mode, ext_mode=ext_mode)
        r = orc.search(Q, db, offs, p, query_id=3, subject_base=10)
        hb, eb = search_b(Q, subs, M, T=T, X=X, cutoff=cutoff, mode=mode, query_id=3,
                          subject_base=10, ext_mode=ext_mode)
        assert [tuple(x) for x in r.hsps.tolist()] == hb, i
        assert [tuple(x) for x in r.extensions.tolist()] == eb, i
        checked_ext += len(eb)
    assert checked_ext > 200


def test_multithreaded_equals_single(orc):
    q = gen_query(5, 300)
    db = gen_db(55, 56, n_subjects=2000, mean_len=200, queries=[q], plant_frac=0.1)
    Q = orc.encode(q)
    codes = orc.encode(db.ascii.tobytes())
    r1 = orc.search(Q, codes, db.offsets, nthreads=1)
    r4 = orc.search(Q, codes, db.offsets, nthreads=4)
    assert (r1.hsps == r4.hsps).all() and (r1.extensions == r4.extensions).all()
    assert len(r1.hsps) > 50


@pytest.mark.parametrize("mode", [0, 1])
def test_hit_mode_extends_every_passing_hit(orc, mode):
    """Alg. 4: one extension per passing hit, duplicates kept;
    the diagonal-based (Alg. 3) extensions are a sub-multiset of them (a
    covered hit is skipped, an uncovered one is extended identically)."""
    from collections import Counter
    q = gen_query(31, 400)
    db = gen_db(32, 33, n_subjects=600, mean_len=250, queries=[q], plant_frac=0.3)
    Q = orc.encode(q)
    codes = orc.encode(db.ascii.tobytes())
    hit = orc.search(Q, codes, db.offsets, orc.Params(filter_mode=mode, ext_mode=1),
                     want_hits=True)
    diag = orc.search(Q, codes, db.offsets, orc.Params(filter_mode=mode, ext_mode=0),
                      want_hits=True)
    assert len(hit.extensions) == len(hit.passing) == len(diag.passing)
    ch = Counter(tuple(x) for x in hit.extensions.tolist())
    cd = Counter(tuple(x) for x in diag.extensions.tolist())
    assert not (cd - ch)
    assert len(hit.extensions) > len(diag.extensions) > 50
    # duplicates: several seeds inside one planted copy give the same HSP
    assert any(v > 1 for v in ch.values())
    assert sorted(tuple(x) for x in hit.hsps.tolist()) == \
        sorted(x for x in (tuple(y) for y in hit.extensions.tolist()) if x[6] >= 41)
