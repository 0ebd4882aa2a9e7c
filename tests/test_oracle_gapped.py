"""Pins of the gapped-extension oracle (oracle/gapped.c; R18-R22):
independent formulations (every alignment path enumerated on tiny inputs; a
textbook full-matrix Gotoh in Python), closed forms (identical sequences, one
deletion), a hand-worked X-drop cut, and the HSP-list rules (seed, order,
containment, cutoff, ids)."""
import numpy as np
import pytest

GO, GE = 11, 1


@pytest.fixture(scope="module")
def M(orc):
    return orc.blosum62()


def brute_best(a, b, m, go=GO, ge=GE):
    """Best anchored score per end cell by enumerating every path of moves
    D (a and b), I (a only), J (b only) from the corner; each maximal run of I
    (or J) moves of length k costs go + ge * k."""
    la, lb = len(a), len(b)
    H = {}

    def walk(i, j, score, prev):
        key = (i, j)
        if key not in H or score > H[key]:
            H[key] = score
        if i < la and j < lb:
            walk(i + 1, j + 1, score + int(m[a[i], b[j]]), "D")
        if i < la:
            walk(i + 1, j, score - (ge if prev == "I" else go + ge), "I")
        if j < lb:
            walk(i, j + 1, score - (ge if prev == "J" else go + ge), "J")

    walk(0, 0, 0, "")
    best, bi, bj = 0, 0, 0
    for i in range(la + 1):
        for j in range(lb + 1):
            if H[(i, j)] > best:
                best, bi, bj = H[(i, j)], i, j
    return best, bi, bj


def path_stats(a, b, m, target, ti, tj, go=GO, ge=GE):
    """Every (ident, gap_opens, gap_len) of the paths from the corner to
    (ti, tj) that score `target`."""
    out = set()

    def walk(i, j, score, prev, idn, gop, gl):
        if (i, j) == (ti, tj) and score == target:
            out.add((idn, gop, gl))
        if i < ti and j < tj:
            walk(i + 1, j + 1, score + int(m[a[i], b[j]]), "D", idn + int(a[i] == b[j]), gop, gl)
        if i < ti:
            walk(i + 1, j, score - (ge if prev == "I" else go + ge), "I", idn,
                 gop + (prev != "I"), gl + 1)
        if j < tj:
            walk(i, j + 1, score - (ge if prev == "J" else go + ge), "J", idn,
                 gop + (prev != "J"), gl + 1)

    walk(0, 0, 0, "", 0, 0, 0)
    return out


def textbook_gotoh(a, b, m, go=GO, ge=GE):
    """Full-matrix Gotoh (no X-drop), written from the textbook recurrences
    in Python: (best, bi, bj) with the first maximum in row-major order."""
    NEG = -10 ** 9
    la, lb = len(a), len(b)
    H = [[NEG] * (lb + 1) for _ in range(la + 1)]
    E = [[NEG] * (lb + 1) for _ in range(la + 1)]
    F = [[NEG] * (lb + 1) for _ in range(la + 1)]
    H[0][0] = 0
    for j in range(1, lb + 1):
        E[0][j] = -(go + ge * j)
        H[0][j] = E[0][j]
    for i in range(1, la + 1):
        F[i][0] = -(go + ge * i)
        H[i][0] = F[i][0]
        for j in range(1, lb + 1):
            E[i][j] = max(E[i][j - 1] - ge, H[i][j - 1] - go - ge)
            F[i][j] = max(F[i - 1][j] - ge, H[i - 1][j] - go - ge)
            H[i][j] = max(H[i - 1][j - 1] + int(m[a[i - 1], b[j - 1]]), E[i][j], F[i][j])
    best, bi, bj = 0, 0, 0
    for i in range(la + 1):
        for j in range(lb + 1):
            if H[i][j] > best:
                best, bi, bj = H[i][j], i, j
    return best, bi, bj


def test_brute_force_paths_tiny(orc, M):
    rng = np.random.default_rng(5)
    gp = orc.GappedParams(xdrop=10 ** 6)
    for _ in range(120):
        la, lb = int(rng.integers(0, 6)), int(rng.integers(0, 6))
        a = rng.integers(0, 20, size=la).astype(np.uint8)
        b = rng.integers(0, 20, size=lb).astype(np.uint8)
        if rng.random() < 0.4 and la and lb:  # similar pairs: gaps compete
            b = a.copy() if rng.random() < 0.5 else np.delete(a, int(rng.integers(0, la)))
        sc, bi, bj, idn, gop, gl = orc.gapped_dir(a, b, M, gp)
        best, ti, tj = brute_best(list(a), list(b), M)
        assert (sc, bi, bj) == (best, ti, tj)
        if sc > 0:
            assert (idn, gop, gl) in path_stats(list(a), list(b), M, sc, bi, bj)


def test_textbook_gotoh_random(orc, M):
    rng = np.random.default_rng(6)
    gp = orc.GappedParams(xdrop=10 ** 6)
    for _ in range(60):
        la, lb = int(rng.integers(1, 30)), int(rng.integers(1, 30))
        a = rng.integers(0, 24, size=la).astype(np.uint8)
        b = a[: lb].copy() if rng.random() < 0.5 else rng.integers(0, 24, size=lb).astype(np.uint8)
        if len(b) > 4 and rng.random() < 0.5:  # indels inside a similar pair
            b = np.concatenate([b[:3], rng.integers(0, 20, size=2).astype(np.uint8), b[3:]])
        sc, bi, bj = orc.gapped_dir(a, b, M, gp)[:3]
        assert (sc, bi, bj) == textbook_gotoh(list(a), list(b), M)


def test_closed_forms(orc, M):
    a = orc.encode("MKVLAAGIVG")
    self_score = int(sum(M[c, c] for c in a))
    assert orc.gapped_dir(a, a, M) == (self_score, 10, 10, 10, 0, 0) and self_score == 46
    # one A deleted: 9 identities, one gap of one residue (46 - 4 - 12)
    b = orc.encode("MKVLAGIVG")
    assert orc.gapped_dir(a, b, M) == (30, 10, 9, 9, 1, 1)
    # nothing positive: the empty extension
    assert orc.gapped_dir(orc.encode("WWW"), orc.encode("PPP"), M)[:3] == (0, 0, 0)
    assert orc.gapped_dir(np.zeros(0, np.uint8), a, M)[:3] == (0, 0, 0)


def test_xdrop_cut_hand_worked(orc, M):
    """a = WW P^5 W^10, b = WW W^15.  After the first WW (best 22) the cheapest
    way on is the 5-residue gap over a's P's: 22 - (11 + 5) = 6, then ten W/W
    pairs: 116 at (17, 12).  The gap's last cell sits exactly 16 below the
    best: X = 16 keeps it (R19: dead only if H < best - X), X = 15 kills every
    path and the extension ends at the WW."""
    a = orc.encode("WW" + "P" * 5 + "W" * 10)
    b = orc.encode("WW" + "W" * 15)
    assert M[orc.encode("W")[0], orc.encode("W")[0]] == 11
    assert M[orc.encode("P")[0], orc.encode("W")[0]] == -4
    assert orc.gapped_dir(a, b, M, orc.GappedParams(xdrop=16))[:3] == (116, 17, 12)
    assert orc.gapped_dir(a, b, M, orc.GappedParams(xdrop=15))[:3] == (22, 2, 2)
    assert textbook_gotoh(list(a), list(b), M) == (116, 17, 12)


def _hsp(qid, sid, qs, ss, ln, sc):
    return (qid, sid, ss - qs, qs, ss, ln, sc)


def test_hsp_list_rules(orc, M):
    """R20 seed, R21 order / containment / cutoff, ids and subject_base."""
    rng = np.random.default_rng(7)
    q = rng.integers(0, 20, size=200).astype(np.uint8)
    s0 = rng.integers(0, 20, size=400).astype(np.uint8)
    s0[100:160] = q[20:80]                   # planted copy: query 20..80 at subject 100..160
    s1 = rng.integers(0, 20, size=300).astype(np.uint8)
    s1[50:90] = q[150:190]                   # subject 1: query 150..190 at 50..90
    db = np.concatenate([s0, s1])
    off = np.array([0, 400, 700], np.int64)
    ungapped = lambda qs, ss, ln: int(sum(M[q[qs + k], db[ss + k]] for k in range(ln)))  # noqa
    hs = [_hsp(0, 7, 20, 100, 60, ungapped(20, 100, 60)),     # the copy
          _hsp(0, 7, 30, 110, 20, ungapped(30, 110, 20)),     # seed inside the copy's box
          _hsp(0, 8, 150, 50, 40, ungapped(150, 450, 40))]    # subject 8 = local 1
    h = np.array(sorted(hs), dtype=np.int32).view(orc.HSP_DTYPE).ravel()
    out = orc.gapped_hsps([q], db, off, h, subject_base=7)
    assert len(out) == 2  # the second HSP of subject 7 is contained
    g0, g1 = out[0], out[1]
    assert (g0["query_id"], g0["subject_id"], g1["subject_id"]) == (0, 7, 8)
    # the copy is at least spanned: the seed (50, 130) extends to both copy ends
    assert g0["q_start"] <= 20 and g0["q_end"] >= 80 and g0["s_start"] <= 100
    assert g0["s_end"] >= 160 and g0["s_end"] - g0["s_start"] >= 60
    assert g0["score"] >= int(sum(M[c, c] for c in q[20:80]))
    # every field recomputed from the oracle's own pieces
    qm, sm = 20 + 30, 100 + 30
    R = orc.gapped_dir(q[qm:], s0[sm:], M)
    L = orc.gapped_dir(q[:qm][::-1], s0[:sm][::-1], M)
    assert g0["score"] == R[0] + L[0] and g0["q_end"] == qm + R[1] and g0["s_start"] == sm - L[2]
    # cutoff above every score: nothing reported; a query id out of range: error
    assert len(orc.gapped_hsps([q], db, off, h, orc.GappedParams(cutoff=10 ** 6), 7)) == 0
    bad = h.copy()
    bad["query_id"][0] = 3
    with pytest.raises(ValueError):
        orc.gapped_hsps([q], db, off, bad, subject_base=7)


def test_order_decides_containment(orc, M):
    """Two overlapping HSPs of one pair: the higher-scoring one is extended
    first, whatever the canonical order; the other is skipped when its seed
    falls inside the first alignment's box."""
    rng = np.random.default_rng(8)
    q = rng.integers(0, 20, size=120).astype(np.uint8)
    s = rng.integers(0, 20, size=200).astype(np.uint8)
    s[40:100] = q[10:70]
    off = np.array([0, 200], np.int64)
    lo = _hsp(0, 0, 10, 40, 10, 5)      # canonical first, low score
    hi = _hsp(0, 0, 12, 42, 50, 999)    # its seed (37, 67) lies inside the copy
    h = np.array(sorted([lo, hi]), dtype=np.int32).view(orc.HSP_DTYPE).ravel()
    out = orc.gapped_hsps([q], s, off, h)
    assert len(out) == 1
    qm, sm = 12 + 25, 42 + 25
    R = orc.gapped_dir(q[qm:], s[sm:], M)
    L = orc.gapped_dir(q[:qm][::-1], s[:sm][::-1], M)
    assert out[0]["score"] == R[0] + L[0]


def test_all_letters_and_both_directions_agree(orc, M):
    """Reversing both sequences mirrors a full-length alignment: the score of
    aligning a against b from the start equals that of their reverses when
    the best cell is the far corner (exact copies with an indel)."""
    for seed in range(10):
        rng = np.random.default_rng(100 + seed)
        a = rng.integers(0, 24, size=40).astype(np.uint8)
        k = int(rng.integers(5, 35))
        b = np.concatenate([a[:k], a[k + 1:]])
        f = orc.gapped_dir(a, b, M)
        r = orc.gapped_dir(a[::-1].copy(), b[::-1].copy(), M)
        if (f[1], f[2]) == (40, 39) and (r[1], r[2]) == (40, 39):
            assert f[0] == r[0]
