"""oracle-B: a second, independent formulation of the hot path.

TEST INFRASTRUCTURE ONLY.  Pure Python, tiny inputs only.  It shares nothing
with oracle.c except the definition of the method in PAPER.md:

* no lookup table: every (query, subject) word pair on a diagonal is scored
  directly (the definition of a hit, R3/R4);
* the two-hit test is an O(n^2) pair loop over the hits of a diagonal
  (R6);
* X-drop is a direct loop over the diagonal, written from the ChangeSinceBest
  / DropFlag description of Fig. 8 (R8);
* coverage follows Alg. 3 L19-23 (R10); ext_mode=1 is Alg. 4
  (P:L1465-1486): every passing hit is extended, no coverage test;
* mode=2 (STATEFUL, R15) is Alg. 1 L8-19 written as a scan of
  the diagonal position by position with the lasthit register; mode=3 adds
  L13's reach-back (R16): an extension whose subject start lies after the
  lasthit is dropped and the hit becomes the lasthit.

Results are returned as a sorted list of 7-tuples (R11).
"""
from __future__ import annotations


def _extend_one_side(Q, S, q0, s0, step, M, X):
    """Walk from (q0, s0) in direction `step`; return (gain, length)."""
    total = 0
    best, best_len = 0, 0
    k = 0
    while 0 <= q0 + k * step < len(Q) and 0 <= s0 + k * step < len(S):
        total += M[Q[q0 + k * step]][S[s0 + k * step]]
        k += 1
        change_since_best = total - best
        if change_since_best > 0:  # new highest score (strictly higher)
            best, best_len = total, k
            continue
        if -change_since_best >= X:  # DropFlag
            break
    return best, best_len


def search_b(Q, subjects, M, *, T=11, w=3, A=40, W=3, X=16, cutoff=41, mode=0,
             query_id=0, subject_base=0, ext_mode=0):
    """Return (hsps, extensions) as sorted lists of 7-tuples
    (query_id, subject_id, diagonal, q_start, s_start, length, score)."""
    Q = [int(c) for c in Q]
    lq = len(Q)
    hsps, exts = [], []
    for i, S in enumerate(subjects):
        S = [int(c) for c in S]
        ls = len(S)
        sid = subject_base + i
        for d in range(-(lq - w), ls - w + 1):
            # hits on this diagonal, s ascending (direct word scoring)
            H = []
            for s in range(max(0, d), ls - w + 1):
                q = s - d
                if q + w > lq:
                    break
                if sum(M[Q[q + j]][S[s + j]] for j in range(w)) >= T:
                    H.append(s)
            if not H:
                continue
            if mode in (2, 3):
                # Alg. 1: one register per diagonal, updated at every hit
                lasthit = None
                for h in H:
                    dist = None if lasthit is None else h - lasthit
                    if dist is None or dist >= A:
                        lasthit = h          # L17-19
                    elif dist >= W:          # L11-16
                        q = h - d
                        seed = sum(M[Q[q + j]][S[h + j]] for j in range(w))
                        gr, rl = _extend_one_side(Q, S, q + w, h + w, +1, M, X)
                        gl, ll = _extend_one_side(Q, S, q - 1, h - 1, -1, M, X)
                        rec = (query_id, sid, d, q - ll, h - ll, ll + w + rl, seed + gl + gr)
                        if mode == 3 and h - ll > lasthit:  # does not reach back
                            lasthit = h
                            continue
                        exts.append(rec)
                        if rec[6] >= cutoff:
                            hsps.append(rec)
                        lasthit = h + w - 1 + rl
                continue
            reach = -1
            for h in H:
                if mode == 0:
                    ok = any(W <= h - p < A for p in H)
                else:
                    ok = any(W <= abs(h - p) < A for p in H)
                if not ok or (ext_mode == 0 and h <= reach):
                    continue
                q = h - d
                seed = sum(M[Q[q + j]][S[h + j]] for j in range(w))
                gr, rl = _extend_one_side(Q, S, q + w, h + w, +1, M, X)
                gl, ll = _extend_one_side(Q, S, q - 1, h - 1, -1, M, X)
                rec = (query_id, sid, d, q - ll, h - ll, ll + w + rl, seed + gl + gr)
                reach = h + w - 1 + rl
                exts.append(rec)
                if rec[6] >= cutoff:
                    hsps.append(rec)
    return sorted(hsps), sorted(exts)
