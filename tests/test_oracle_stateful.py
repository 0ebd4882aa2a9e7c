"""Pins of the STATEFUL filter mode (filter_mode 2: Alg. 1 L8-19, P:L664-689,
reading R15 in DESIGN.md) against things other than the oracle itself:
hand-walked examples (tests/golden/alg1_stateful.json), the reduction to the
LEFT test (R6) on diagonals of at most two hits, the covering-extension
special case, the trigger-spacing invariant, and the independent oracle-B
formulation (direct word scoring, oracle/oracle_b.py) on random tiny cases."""
import json
import os
from collections import defaultdict

import numpy as np
import pytest

from oracle.oracle_b import search_b
from synth import gen_db, gen_query

from test_oracle_pins import _oracle_b_cases, rr_codes

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_hand_walked_examples(orc):
    with open(os.path.join(GOLD, "alg1_stateful.json")) as f:
        g = json.load(f)
    for c in g["cases"]:
        got = orc.two_hit_stateful(c["s"], c["ext_end"], c["W"], c["A"])
        assert list(got) == c["trigger"], c["name"]
        # the LEFT test (R6) on the same hits, for contrast: these cases are
        # chosen so that the two rules differ
        left = orc.two_hit(c["s"], c["W"], c["A"], 0)
        assert list(left) == c["left_pass"], c["name"]


def _random_diagonal(rng, n, span=120):
    s = np.sort(rng.choice(span, size=n, replace=False)).astype(np.int32)
    ext = s + 2 + rng.integers(0, 25, size=n).astype(np.int32)
    return s, ext


def test_two_hits_reduce_to_left():
    """With at most two hits on a diagonal Alg. 1 triggers exactly when the
    second hit lies W <= h - p < A after the first: the LEFT test (R6)."""
    from oracle import oracle as orc
    rng = np.random.default_rng(15)
    for _ in range(3000):
        n = int(rng.integers(1, 3))
        s, ext = _random_diagonal(rng, n, span=int(rng.integers(3, 90)))
        W, A = int(rng.integers(1, 5)), int(rng.integers(2, 60))
        assert list(orc.two_hit_stateful(s, ext, W, A)) == list(orc.two_hit(s, W, A, 0))


def test_covering_extension_single_trigger(orc):
    """An extension that reaches past every later hit leaves lasthit beyond
    them: at most one trigger, at the first hit whose distance to the last
    non-overlapping hit before it lies in [W, A)."""
    rng = np.random.default_rng(16)
    for _ in range(2000):
        s, _ = _random_diagonal(rng, int(rng.integers(1, 12)))
        ext = np.full(len(s), s[-1] + 5, dtype=np.int32)
        trig = orc.two_hit_stateful(s, ext, 3, 40)
        assert trig.sum() <= 1
        # expected: walk with hit-only updates until the first trigger
        last, want = None, None
        for k, h in enumerate(s.tolist()):
            if last is None or h - last >= 40:
                last = h
            elif h - last >= 3:
                want = k
                break
        assert list(np.nonzero(trig)[0]) == ([] if want is None else [want])


def test_trigger_spacing_invariant(orc):
    """Between consecutive triggers k1 < k2: s[k2] - ext_end[k1] >= W (the
    second seed lies beyond the first extension, no overlap), and a trigger
    always has a lasthit (a hit or an extension end) less than A before it."""
    rng = np.random.default_rng(17)
    for _ in range(2000):
        s, ext = _random_diagonal(rng, int(rng.integers(1, 20)))
        trig = np.nonzero(orc.two_hit_stateful(s, ext, 3, 40))[0]
        for a, b in zip(trig[:-1], trig[1:]):
            assert s[b] - ext[a] >= 3
        for k in trig:
            before = [int(x) for x in s[:k]] + [int(ext[j]) for j in trig if j < k]
            assert any(3 <= s[k] - v < 40 for v in before)


def test_oracle_b_agrees_stateful(orc, B62):
    """oracle.c's STATEFUL search == oracle-B's (direct word scoring, Alg. 1 as a
    position scan) on random tiny cases, HSPs and every extension."""
    al = orc.alphabet()
    rng = np.random.default_rng(2025)
    M = B62.tolist()
    n_ext = 0
    for i, (Q, subs) in enumerate(_oracle_b_cases(rng, al, 300)):
        T = 11 if i % 5 else 9
        X = int(rng.choice([16, 16, 5, 30]))
        cutoff = int(rng.choice([41, 20]))
        offs = np.concatenate([[0], np.cumsum([len(s) for s in subs])]).astype(np.int64)
        db = np.concatenate(subs).astype(np.uint8) if offs[-1] else np.zeros(0, np.uint8)
        p = orc.Params(threshold=T, xdrop=X, cutoff=cutoff, filter_mode=2)
        r = orc.search(Q, db, offs, p, query_id=3, subject_base=10)
        hb, eb = search_b(Q, subs, M, T=T, X=X, cutoff=cutoff, mode=2, query_id=3,
                          subject_base=10)
        assert [tuple(x) for x in r.hsps.tolist()] == hb, i
        assert [tuple(x) for x in r.extensions.tolist()] == eb, i
        n_ext += len(eb)
    assert n_ext > 100


def test_stateful_search_invariants(orc, B62):
    """On a planted DB: every extension is seeded at a hit, its score is the
    BLOSUM62 sum over its segment (P5), seeds on a diagonal lie beyond the
    previous extension (no overlap, R15), and the extended hits are exactly the
    walk's triggers over the hits of each diagonal."""
    q = gen_query(41, 300)
    db = gen_db(42, 43, n_subjects=400, mean_len=250, queries=[q], plant_frac=0.3)
    Q = orc.encode(q)
    codes = orc.encode(db.ascii.tobytes())
    offs = db.offsets
    r = orc.search(Q, codes, offs, orc.Params(filter_mode=2), want_hits=True)
    assert len(r.extensions) > 50 and len(r.hsps) > 20
    hits = defaultdict(list)
    for subj, qq, ss in r.hits.tolist():
        hits[(subj, ss - qq)].append(ss)
    trig = {(int(a), int(c) - int(b), int(c)) for a, b, c in r.passing.tolist()}
    assert len(trig) == len(r.extensions)
    by_diag = defaultdict(list)
    for e in r.extensions:
        S = codes[offs[e["subject_id"]]:offs[e["subject_id"] + 1]]
        qs, ss, L = int(e["q_start"]), int(e["s_start"]), int(e["length"])
        assert int(e["score"]) == int(sum(B62[Q[qs + k], S[ss + k]] for k in range(L)))
        by_diag[(int(e["subject_id"]), int(e["diagonal"]))].append((ss, ss + L - 1))
    for key, segs in by_diag.items():
        segs.sort()
        for (a0, b0), (a1, b1) in zip(segs, segs[1:]):
            assert b0 < b1
    # the walk over each diagonal's hits, with each hit's extension end from
    # the pinned X-drop (R8) directly, reproduces the search's triggers
    n_checked = 0
    for (subj, d), ss in hits.items():
        ss = sorted(ss)
        if len(ss) < 2:
            assert (subj, d, ss[0]) not in trig
            continue
        S = codes[offs[subj]:offs[subj + 1]]
        ends = []
        for h in ss:
            qq = h - d
            n = min(len(Q) - (qq + 3), len(S) - (h + 3))
            _, rlen, _ = orc.xdrop_pairs(Q[qq + 3:], S[h + 3:], B62, 16, n=n)
            ends.append(h + 2 + rlen)
        want = orc.two_hit_stateful(ss, ends, 3, 40)
        assert [bool(x) for x in want] == [(subj, d, s_) in trig for s_ in ss]
        n_checked += 1
    assert n_checked > 200


# ---------------------------------------------------------------------------
# filter_mode 3: STATEFUL with Alg. 1 L13's reach-back (reading R16)
# ---------------------------------------------------------------------------

def test_reachback_hand_walked_examples(orc):
    with open(os.path.join(GOLD, "alg1_reachback.json")) as f:
        g = json.load(f)
    for c in g["cases"]:
        got = orc.two_hit_stateful_rb(c["s"], c["ext_start"], c["ext_end"], c["W"], c["A"])
        assert list(got) == c["trigger"], c["name"]
        assert list(orc.two_hit_stateful(c["s"], c["ext_end"], c["W"], c["A"])) == \
            c["stateful"], c["name"]


def test_reachback_limits(orc):
    """Extensions that always reach back (start before every hit) give the
    STATEFUL walk (R15) exactly; extensions that never do (start after every
    hit) give no extension at all, whatever the hits."""
    rng = np.random.default_rng(18)
    for _ in range(2000):
        s, ext = _random_diagonal(rng, int(rng.integers(1, 16)), span=int(rng.integers(16, 150)))
        W, A = int(rng.integers(1, 5)), int(rng.integers(2, 60))
        always = np.full(len(s), -1, dtype=np.int32)
        never = np.full(len(s), 10 ** 6, dtype=np.int32)
        assert list(orc.two_hit_stateful_rb(s, always, ext, W, A)) == \
            list(orc.two_hit_stateful(s, ext, W, A))
        assert not orc.two_hit_stateful_rb(s, never, ext, W, A).any()


def test_reachback_kept_extensions_reach_back(orc):
    """Every kept extension starts at or before the last hit (or extension
    end) the walk pairs it with, and a dropped one makes its hit the
    lasthit: replaying the walk by hand reproduces the triggers."""
    rng = np.random.default_rng(19)
    for _ in range(2000):
        n = int(rng.integers(1, 14))
        s, ext = _random_diagonal(rng, n)
        start = (s - rng.integers(0, 20, size=n)).astype(np.int32)
        trig = orc.two_hit_stateful_rb(s, start, ext, 3, 40)
        last = None
        for k in range(n):
            h = int(s[k])
            if last is None or h - last >= 40:
                assert not trig[k]
                last = h
            elif h - last < 3:
                assert not trig[k]
            elif start[k] <= last:
                assert trig[k]
                last = int(ext[k])
            else:
                assert not trig[k]
                last = h


def test_oracle_b_agrees_reachback(orc, B62):
    """oracle.c's STATEFUL_RB search == oracle-B's (Alg. 1 as a position scan with
    direct word scoring and the reach-back test) on random tiny cases."""
    al = orc.alphabet()
    rng = np.random.default_rng(2026)
    M = B62.tolist()
    n_ext = n_diff = 0
    for i, (Q, subs) in enumerate(_oracle_b_cases(rng, al, 300)):
        T = 11 if i % 5 else 9
        X = int(rng.choice([16, 16, 5, 30]))
        cutoff = int(rng.choice([41, 20]))
        offs = np.concatenate([[0], np.cumsum([len(s) for s in subs])]).astype(np.int64)
        db = np.concatenate(subs).astype(np.uint8) if offs[-1] else np.zeros(0, np.uint8)
        p = orc.Params(threshold=T, xdrop=X, cutoff=cutoff, filter_mode=3)
        r = orc.search(Q, db, offs, p, query_id=3, subject_base=10)
        hb, eb = search_b(Q, subs, M, T=T, X=X, cutoff=cutoff, mode=3, query_id=3,
                          subject_base=10)
        assert [tuple(x) for x in r.hsps.tolist()] == hb, i
        assert [tuple(x) for x in r.extensions.tolist()] == eb, i
        _, e2 = search_b(Q, subs, M, T=T, X=X, cutoff=cutoff, mode=2, query_id=3,
                         subject_base=10)
        n_ext += len(eb)
        n_diff += eb != e2
    assert n_ext > 50 and n_diff > 10  # the reach-back changes real searches
