"""Pins of the oracle's constants and encoding.

Not retyping: lambda_u is a closed-form property of BLOSUM62 + the RR
background that NCBI publishes (0.3176); a wrong entry moves it.
"""
import numpy as np
import pytest
from scipy.optimize import brentq

from synth import RR_FREQ



def _rr_vec(alphabet):
    p = np.zeros(len(alphabet))
    for i, c in enumerate(alphabet):
        p[i] = RR_FREQ.get(c, 0.0)
    return p / p.sum()


def test_alphabet_order(orc):
    assert orc.alphabet() == "ARNDCQEGHILKMFPSTWYVBZX*"


def test_blosum62_symmetric_and_known_entries(orc, B62):
    assert B62.shape == (24, 24)
    assert (B62 == B62.T).all()
    a = orc.alphabet()
    S = lambda x, y: B62[a.index(x), a.index(y)]
    assert S("W", "W") == 11 and S("C", "C") == 9 and S("A", "A") == 4
    assert S("*", "*") == 1 and S("A", "*") == -4
    # every self score of the 20 standard letters is positive (used by P9)
    std = [a.index(c) for c in RR_FREQ]
    assert all(B62[i, i] >= 4 for i in std)


def test_blosum62_lambda_matches_ncbi(orc, B62):
    """Karlin-Altschul lambda_u solves sum p_a p_b exp(lambda s_ab) = 1."""
    a = orc.alphabet()
    p = _rr_vec(a)
    P = np.outer(p, p)
    expected = float((P * B62).sum())
    assert expected < 0  # local-alignment statistics need a negative mean
    assert abs(expected - (-0.952)) < 0.01
    lam = brentq(lambda x: (P * np.exp(x * B62)).sum() - 1.0, 1e-3, 2.0)
    assert abs(lam - 0.3176) < 1e-3, lam
    # derived params: X = ceil(7 ln2 / lambda), cutoff 41
    assert int(np.ceil(7 * np.log(2) / 0.3176)) == 16
    assert int((22 * np.log(2) + np.log(0.134)) / 0.3176) == 41


def test_encode_roundtrip_and_errors(orc):
    a = orc.alphabet()
    codes = orc.encode(a)
    assert list(codes) == list(range(24))
    assert list(orc.encode("arndc")) == [0, 1, 2, 3, 4]
    x = a.index("X")
    assert list(orc.encode("UOJuoj")) == [x] * 6
    for bad in ["AC-D", "A1", "A C", "A\x00"]:
        with pytest.raises(ValueError):
            orc.encode(bad)
