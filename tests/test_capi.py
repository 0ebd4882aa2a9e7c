"""C-ABI checks that need no GPU: the library loads, exports every symbol
declared in include/blastp.h, and its host-only logic (defaults, sharding,
argument validation) behaves as documented."""
import ctypes
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def bp():
    from paper_conf_ipps_zhangwlf14_b200 import build
    build.build()
    from paper_conf_ipps_zhangwlf14_b200 import blastp
    return blastp


def declared_functions():
    src = open(os.path.join(ROOT, "include", "blastp.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(blastp_[a-z_0-9]+)\s*\(", src)))


def test_library_exports_every_declared_symbol(bp):
    names = declared_functions()
    assert len(names) >= 19
    lib = ctypes.CDLL(bp.LIB_PATH)
    for n in names:
        assert hasattr(lib, n), n
    assert sorted(bp.EXPORTED) == names


def test_built_for_sm100a(bp):
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", bp.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


def test_params_default_matches_baseline(bp):
    p = bp.params_default()
    assert (p.word_len, p.threshold, p.window, p.min_gap, p.xdrop, p.cutoff, p.filter_mode,
            p.ext_mode) == (3, 11, 40, 3, 16, 41, 0, 0)
    assert bp.Params() == p


def test_strerror_and_version(bp):
    assert bp.lib.blastp_strerror(0) == b"ok"
    assert bp.lib.blastp_strerror(-2) == b"invalid residue character"
    assert "sm_100a" in bp.version()


def test_shard_range_balances_residues(bp):
    rng = np.random.default_rng(1)
    lens = rng.integers(10, 800, size=10000)
    off = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
    total = off[-1]
    for n in (1, 2, 3, 4, 8):
        ranges = [bp.shard_range(off, k, n) for k in range(n)]
        assert ranges[0][0] == 0 and ranges[-1][1] == 10000
        for (a, b), (c, d) in zip(ranges, ranges[1:]):
            assert b == c
        for k, (a, b) in enumerate(ranges):
            # first subject of shard k: first i with off[i] >= total*k/n
            assert a == int(np.searchsorted(off, total * k // n, side="left"))
            share = (off[b] - off[a]) / total
            assert abs(share - 1 / n) < 800 / total + 1e-9
    # offsets not starting at zero
    assert bp.shard_range(off + 1234, 1, 4) == bp.shard_range(off, 1, 4)
    # empty database and more shards than subjects
    assert bp.shard_range(np.zeros(1, dtype=np.int64), 0, 8) == (0, 0)
    small = np.array([0, 5, 10], dtype=np.int64)
    rs = [bp.shard_range(small, k, 8) for k in range(8)]
    assert sum(b - a for a, b in rs) == 2


def test_shard_range_rejects_bad_arguments(bp):
    off = np.array([0, 5], dtype=np.int64)
    for k, n in [(-1, 2), (2, 2), (0, 0)]:
        with pytest.raises(bp.BlastpError) as e:
            bp.shard_range(off, k, n)
        assert e.value.status == bp.E_INVALID_ARG


def test_invalid_params_rejected_before_any_gpu_work(bp):
    for bad in [dict(word_len=4), dict(min_gap=0), dict(window=0), dict(xdrop=0),
                dict(xdrop=200), dict(filter_mode=7), dict(ext_mode=4), dict(threshold=500)]:
        with pytest.raises(bp.BlastpError) as e:
            bp.build_query_table("MKVLAAGIVALLA", bp.Params(**bad))
        assert e.value.status == bp.E_INVALID_ARG, bad


def test_gapped_defaults_and_validation_without_gpu(bp, orc):
    """The gapped stage's defaults equal the oracle's (R18-R21: 11 + 1 per
    residue, X-drop 38, cutoff 41), the record is 40 bytes with the oracle's
    field order, and bad arguments fail before any device work."""
    g = bp._CGappedParams()
    bp.lib.blastp_gapped_params_default(ctypes.byref(g))
    o = orc.GappedParams()
    assert (g.gap_open, g.gap_extend, g.xdrop, g.cutoff) == (o.gap_open, o.gap_extend, o.xdrop,
                                                             o.cutoff)
    assert bp.GAPPED_DTYPE.itemsize == 40 and bp.GAPPED_DTYPE.names == orc.GAPPED_DTYPE.names
    cnt = ctypes.c_int64()
    rc = bp.lib.blastp_gapped_extend_device(None, None, None, 0, ctypes.byref(g), None, None, 0,
                                            ctypes.byref(cnt))
    assert rc == bp.E_INVALID_ARG
