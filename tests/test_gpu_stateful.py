"""GPU parity of filter_mode STATEFUL (Alg. 1 L8-19; reading R15):
the warp kernel's lasthit walk (decided at enqueue, finished at the flush in
queue order) vs the CPU oracle, element by element -- every hit, every
extended hit, every extension and the HSP list.  Run with -m gpu on a B200."""
import os

import numpy as np
import pytest

from synth import config_workload, gen_db, gen_query
from test_gpu_parity import _long_subject_db, _rand_db, assert_same, ALPHA

pytestmark = pytest.mark.gpu


@pytest.fixture(params=[2, 3], ids=["STATEFUL", "STATEFUL_RB"])
def st(request):
    """BLASTP_FILTER_STATEFUL (R15) and _STATEFUL_RB (R15 + R16 reach-back)."""
    return request.param


@pytest.fixture(scope="module")
def bp():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_ipps_zhangwlf14_b200 import build
    build.build()
    from paper_conf_ipps_zhangwlf14_b200 import blastp
    assert blastp.FILTER_STATEFUL == 2 and blastp.FILTER_STATEFUL_RB == 3
    return blastp


@pytest.fixture(params=["warp", "cta"], autouse=True)
def kernel_variant(request, monkeypatch):
    """BLASTP_KERNEL=cta must route STATEFUL to the warp kernel, same results."""
    monkeypatch.setenv("BLASTP_KERNEL", request.param)
    return request.param


def test_config1_full_trace(bp, orc, st):
    (q,), db = config_workload(1)
    g, r = assert_same(bp, orc, q, db.ascii, db.offsets, bp.Params(filter_mode=st))
    assert len(g) > 10 and len(r.passing) > 100


# Configs 2 and 3 in STATEFUL mode (complete lists vs the oracle, no
# sampling): test_gpu_parity.py::test_config2_full[STATEFUL] and
# ::test_config3_full[STATEFUL].


def test_fuzz_small_random(bp, orc, st):
    rng = np.random.default_rng(1515)
    for case in range(80):
        lq = int(rng.choice([3, 5, 17, 64, 127, 300, 517]))
        q = "".join(rng.choice(list(ALPHA[:20] if case % 4 else ALPHA), size=lq))
        ascii, off = _rand_db(rng, int(rng.integers(1, 60)), 0, 400, q)
        p = bp.Params(threshold=int(rng.choice([11, 11, 9, 13])),
                      window=int(rng.choice([40, 40, 10, 80, 3])),
                      min_gap=int(rng.choice([3, 3, 1, 2, 5])),
                      xdrop=int(rng.choice([16, 16, 5, 30])),
                      cutoff=int(rng.choice([41, 20, 0])), filter_mode=st)
        assert_same(bp, orc, q, ascii, off, p, trace=True)


def test_adversarial_low_complexity(bp, orc, st):
    """Every (q, s) a hit: long runs of hits per diagonal inside one round and
    across flushes (many conditional entries per diagonal, chains split over
    two flushes), fresh-subject entries on a still-pending diagonal."""
    q = "W" * 300 + "AAAAQQQQ" * 10 + "W" * 50
    subs = ["W" * 1000, "A" * 200 + "W" * 40, "WA" * 300, "Q" * 500, "W" * 3, "W" * 45,
            "W" * 44, "CW" * 30]
    ascii = np.frombuffer("".join(subs).encode(), dtype=np.uint8).copy()
    off = np.concatenate([[0], np.cumsum([len(s) for s in subs])]).astype(np.int64)
    for window, W in ((40, 3), (10, 3), (80, 1), (3, 2)):
        assert_same(bp, orc, q, ascii, off, bp.Params(filter_mode=st, window=window, min_gap=W),
                    trace=True)


@pytest.mark.parametrize("knobs", [{}, {"BLASTP_SEGLEN": "256"}, {"BLASTP_SEGMENTS": "0"}],
                         ids=["default", "seglen256", "whole"])
def test_long_subjects_diagonal_segments(bp, orc, st, monkeypatch, knobs):
    """Long subjects are split by diagonal range in STATEFUL mode: segment j
    owns the diagonals [d_j, d_j + seg_len) (segment 0 also those below the
    chunk start), walks [d_j, d_j + seg_len + Lq) and holds each of its
    diagonals' whole lasthit walk; with segments off they are walked whole.
    Exact copies of the query are planted across segment boundaries, and
    one subject is longer than the 16-bit frame (rebases with pending
    entries flushed first)."""
    for k, v in knobs.items():
        monkeypatch.setenv(k, v)
    q = gen_query(21, 300).decode()
    ascii, off = _long_subject_db(q)
    d = bp.pack_db(ascii, off)
    assert (d.segments == 0) == ("BLASTP_SEGMENTS" in knobs)
    for window in (40, 256):
        g, _ = assert_same(bp, orc, q, ascii, off, bp.Params(filter_mode=st, window=window),
                           trace=True)
        assert len(g) > 10


def test_long_query_2000(bp, orc, st):
    q = gen_query(2000, 2000)
    db = gen_db(7, 8, n_subjects=400, mean_len=375.0, queries=[q], plant_frac=0.2)
    assert_same(bp, orc, q, db.ascii, db.offsets, bp.Params(filter_mode=st), trace=True)


def test_stateful_requires_diagonal_ext_mode(bp, st):
    q = gen_query(3, 100).decode()
    for ext in (1, 2):
        with pytest.raises(bp.BlastpError) as e:
            t = bp.build_query_table(q, bp.Params())
            d = bp.pack_db(np.frombuffer(q.encode(), np.uint8).copy(), np.array([0, len(q)]))
            bp.search_ungapped(t, d, bp.Params(filter_mode=st, ext_mode=ext))
        assert e.value.status == -1  # BLASTP_E_INVALID_ARG
