"""The paper's worked examples, run through the oracle (fixtures in tests/golden/,
each citing its PAPER.md passage)."""
import json
import os

import numpy as np
import pytest

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def _codes(s, alphabet):
    return np.array([alphabet.index(c) for c in s], dtype=np.uint8)


def test_fig2a_dfa_example(orc):
    g = _load("fig2a_dfa.json")
    al = g["alphabet"]
    M = np.full((3, 3), g["mismatch"], dtype=np.int32)
    np.fill_diagonal(M, g["match"])
    q = _codes(g["query"], al)
    s = _codes(g["subject"], al)
    P = orc.Params(threshold=g["threshold"], word_len=g["word_len"])
    r = orc.search(q, s, np.array([0, len(s)]), P, matrix=M, want_hits=True)
    got = sorted((int(h[1]), int(h[2])) for h in r.hits)
    assert got == [tuple(x) for x in g["expected_hits_q_s"]]
    assert [sq - qq for qq, sq in got] == g["expected_diagonals"]
    # the neighbourhood of BABBC under T=3 is exactly its own words
    off, pos = orc.neighbourhood(q, M, g["threshold"])
    nz = {int(v): list(pos[off[v]:off[v + 1]]) for v in range(27) if off[v + 1] > off[v]}
    word = lambda w: sum(al.index(c) * 3 ** (2 - i) for i, c in enumerate(w))
    assert nz == {word("BAB"): [0], word("ABB"): [1], word("BBC"): [2]}


def test_fig3_fig5_hits_diagonals_bins(orc):
    g = _load("fig3_fig5_binning.json")
    al = g["alphabet"]
    na = len(al)
    off = np.zeros(na ** 3 + 1, dtype=np.int64)
    lists = {}
    for w, qs in g["table"].items():
        lists[sum(al.index(c) * na ** (2 - i) for i, c in enumerate(w))] = qs
    pos = []
    for v in range(na ** 3):
        pos += lists.get(v, [])
        off[v + 1] = len(pos)
    s = _codes(g["subject"], al)
    q = _codes("D" * g["query_len"], al)
    M = np.full((na, na), -1, dtype=np.int32)
    np.fill_diagonal(M, 1)
    r = orc.search(q, s, np.array([0, len(s)]), orc.Params(), matrix=M,
                   table=(off, np.array(pos)), want_hits=True)
    got = [(int(h[1]), int(h[2])) for h in r.hits]
    assert sorted(got) == sorted(tuple(x) for x in g["expected_hits_q_s"])
    # thread 3's diagonals, in query-position order
    assert [s_ - q_ for q_, s_ in got if s_ == 3] == g["expected_diagonals_for_s3"]
    bins = {str(b): set() for b in range(g["num_bins"])}
    for q_, s_ in got:
        bins[str((s_ - q_) % g["num_bins"])].add((q_, s_))
    assert bins == {k: {tuple(x) for x in v} for k, v in g["expected_bins"].items()}


@pytest.mark.parametrize("mode,key", [(0, "expected_left"), (1, "expected_either")])
def test_fig7_two_hit_filter(orc, mode, key):
    g = _load("fig7_sort_filter.json")
    for d, ss in g["diagonals"].items():
        got = orc.two_hit(ss, g["min_gap"], g["window"], mode)
        assert list(got) == g[key][d], (d, mode)
    if mode == 1:  # the figure's own output
        kept = [(s - int(d), s) for d, ss in g["diagonals"].items()
                for s, k in zip(ss, orc.two_hit(ss, 3, 40, 1)) if k]
        assert sorted(kept) == sorted(tuple(x) for x in g["figure_kept_after_filtering"])


def test_fig7_filter_through_full_search(orc):
    """Same example end-to-end: injected Fig. 3 table, passing hits per mode."""
    g3 = _load("fig3_fig5_binning.json")
    al = g3["alphabet"]
    na = len(al)
    off = np.zeros(na ** 3 + 1, dtype=np.int64)
    lists = {sum(al.index(c) * na ** (2 - i) for i, c in enumerate(w)): qs
             for w, qs in g3["table"].items()}
    pos = []
    for v in range(na ** 3):
        pos += lists.get(v, [])
        off[v + 1] = len(pos)
    s = _codes(g3["subject"], al)
    q = _codes("D" * g3["query_len"], al)
    M = np.full((na, na), -1, dtype=np.int32)
    np.fill_diagonal(M, 1)
    for mode, exp in [(0, {(6, 8), (11, 13), (7, 13)}),
                      (1, {(1, 3), (6, 8), (11, 13), (2, 8), (7, 13)})]:
        r = orc.search(q, s, np.array([0, len(s)]), orc.Params(filter_mode=mode), matrix=M,
                       table=(off, np.array(pos)), want_hits=True)
        assert {(int(p[1]), int(p[2])) for p in r.passing} == exp


def test_fig8_window_xdrop(orc):
    g = _load("fig8_window_xdrop.json")
    sc = g["scores"]
    pos = g["positions"]
    # PrefixSum row: leftward from 0, rightward from 1
    i0 = pos.index(0)
    left = np.cumsum(sc[i0::-1])
    right = np.cumsum(sc[i0 + 1:])
    row = list(left[::-1]) + list(right)
    assert row == g["prefix_sum_row"]
    # run both windows through the oracle's X-drop via a diagonal matrix
    vals = sorted(set(sc))
    M = np.zeros((len(vals), len(vals)), dtype=np.int32)
    for i, v in enumerate(vals):
        M[i, i] = v
    X = g["dropoff"]
    R = g["right"]
    seq = np.array([vals.index(v) for v in R["scores_from_pos_1"]], dtype=np.uint8)
    best, ln, steps = orc.xdrop_pairs(seq, seq, M, X)
    assert (best, ln) == (R["best"], R["best_len"])
    assert ln == R["best_pos"]  # window starts at position 1
    assert steps == R["stop_pos"]  # the stop fires at +7 (EndPos 7)
    run = np.cumsum(R["scores_from_pos_1"])
    csb = list((run - np.maximum.accumulate(run))[R["best_len"]:])
    assert csb == R["change_since_best_after_best"]
    flags = [p for p, c in zip(range(1, 9), run - np.maximum.accumulate(run)) if c <= -X]
    assert flags == R["drop_flag_positions"]
    L = g["left"]
    seq = np.array([vals.index(v) for v in L["scores_from_pos_0_leftward"]], dtype=np.uint8)
    best, ln, steps = orc.xdrop_pairs(seq, seq, M, X)
    assert (best, ln) == (L["best"], L["best_len"])
    assert -(ln - 1) == L["best_pos"]
    assert steps == len(seq) and not L["stops"]
    # a step backwards (step=-1) over the reversed array gives the same answer
    rev = seq[::-1].copy()
    assert orc.xdrop_pairs(rev, rev, M, X, step=-1, start=len(rev) - 1)[:2] == (17, 7)
