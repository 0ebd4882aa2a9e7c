"""Seeded synthetic queries and databases (recipe: DESIGN.md "Input recipe").

* Residues: iid from the Robinson-Robinson background frequencies (NCBI
  ``Robinson_prob``), drawn by inverse CDF over a
  65536-entry table (probabilities quantised to 1/65536).
* Subject lengths: lognormal, sigma = 0.7, mean-matched mu = ln(mean) -
  sigma^2/2, rounded and clipped to [10, 36805] (NR's longest sequence,
  P:L1219-1222).  Deterministically, subject i with i % 100000 == 50000 is
  redrawn U[8192, 36805], and a DB of >= 1e5 subjects has subject n//2 of
  length exactly 36805.
* Planted homologs: a fraction of subjects receives a copy of a query
  segment (length U[20,150]); each copied residue is kept with probability
  0.6, else redrawn from the background; 10% of plants are exact copies.
  The plant overwrites the subject at a uniform start (length preserved).
  Plants are recorded (subject, s_start, query_id, q_start, length, exact).

Everything is generated per block of 65536 subjects from
``SeedSequence([seed, block])``, so any subject range (a shard) can be
regenerated alone.  Output is ASCII (uint8) concatenated + int64 offsets.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

# NCBI Robinson & Robinson background, per 1000.
RR_FREQ = {
    "A": 78.05, "C": 19.25, "D": 53.64, "E": 62.95, "F": 38.56, "G": 73.77, "H": 21.99,
    "I": 51.42, "K": 57.44, "L": 90.19, "M": 22.43, "N": 44.87, "P": 52.03, "Q": 42.64,
    "R": 51.29, "S": 71.20, "T": 58.41, "V": 64.41, "W": 13.30, "Y": 32.16,
}

MAX_LEN = 36805
BLOCK = 65536


def _rr_lut() -> np.ndarray:
    letters = sorted(RR_FREQ)
    p = np.array([RR_FREQ[c] for c in letters], dtype=np.float64)
    p /= p.sum()
    edges = np.rint(np.cumsum(p) * 65536).astype(np.int64)
    edges[-1] = 65536
    lut = np.zeros(65536, dtype=np.uint8)
    start = 0
    for c, e in zip(letters, edges):
        lut[start:e] = ord(c)
        start = e
    return lut


_LUT = _rr_lut()


def _draw_residues(rng: np.random.Generator, n: int) -> np.ndarray:
    return _LUT[rng.integers(0, 65536, size=n, dtype=np.uint16)]


def gen_query(seed: int, length: int) -> bytes:
    """RR-distributed query of the given length (ASCII)."""
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0x51])))
    return _draw_residues(rng, length).tobytes()


def gen_queries(seed: int, n: int, lo: int, hi: int) -> list[bytes]:
    """n queries with lengths U[lo, hi] (config 5)."""
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0x52])))
    lens = rng.integers(lo, hi + 1, size=n)
    return [gen_query(seed * 1000 + i, int(L)) for i, L in enumerate(lens)]


@dataclass
class SyntheticDB:
    ascii: np.ndarray          # uint8, all subjects concatenated
    offsets: np.ndarray        # int64 [nseq+1]
    plants: np.ndarray         # structured array, see PLANT_DTYPE
    first_subject: int = 0     # global index of subject 0 of this (sub)range
    meta: dict = field(default_factory=dict)

    @property
    def nseq(self) -> int:
        return len(self.offsets) - 1

    @property
    def residues(self) -> int:
        return int(self.offsets[-1] - self.offsets[0])

    def subject(self, i: int) -> bytes:
        return self.ascii[self.offsets[i]:self.offsets[i + 1]].tobytes()


PLANT_DTYPE = np.dtype([("subject", "<i8"), ("s_start", "<i4"), ("query_id", "<i4"),
                        ("q_start", "<i4"), ("length", "<i4"), ("exact", "?")])


def _lengths(seed: int, n_subjects: int | None, total_residues: int | None, mean_len: float):
    """All subject lengths (cheap; needed to locate any block)."""
    sigma = 0.7
    mu = np.log(mean_len) - sigma * sigma / 2
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0x1E])))
    chunks, tot, n = [], 0, 0
    while True:
        k = BLOCK if n_subjects is None else min(BLOCK * 16, n_subjects - n)
        if k <= 0:
            break
        L = np.rint(rng.lognormal(mu, sigma, size=k))
        L = np.clip(L, 10, MAX_LEN).astype(np.int64)
        chunks.append(L)
        n += k
        tot += int(L.sum())
        if n_subjects is None and total_residues is not None and tot >= total_residues:
            break
    lens = np.concatenate(chunks) if chunks else np.zeros(0, dtype=np.int64)
    if n_subjects is None and total_residues is not None:
        cut = int(np.searchsorted(np.cumsum(lens), total_residues)) + 1
        lens = lens[:cut]
    n = len(lens)
    long_idx = np.arange(50000, n, 100000)
    if len(long_idx):
        lrng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0x10])))
        lens[long_idx] = lrng.integers(8192, MAX_LEN + 1, size=len(long_idx))
    if n >= 100000:
        lens[n // 2] = MAX_LEN
    return lens


def gen_db(seed: int, plant_seed: int, *, n_subjects: int | None = None,
           total_residues: int | None = None, mean_len: float = 200.0,
           queries: list[bytes] | None = None, plant_frac: float = 0.0,
           subject_range: tuple[int, int] | None = None) -> SyntheticDB:
    """Generate a database (or only subjects [lo, hi) of it, for one shard)."""
    lens = _lengths(seed, n_subjects, total_residues, mean_len)
    n = len(lens)
    lo, hi = (0, n) if subject_range is None else subject_range
    hi = min(hi, n)
    sub = lens[lo:hi]
    offsets = np.zeros(hi - lo + 1, dtype=np.int64)
    np.cumsum(sub, out=offsets[1:])
    ascii = np.empty(int(offsets[-1]), dtype=np.uint8)
    b0, b1 = lo // BLOCK, (hi - 1) // BLOCK if hi > lo else lo // BLOCK - 1
    plants = []
    qarr = [np.frombuffer(q, dtype=np.uint8) for q in (queries or [])]
    for b in range(b0, b1 + 1):
        s_lo, s_hi = b * BLOCK, min((b + 1) * BLOCK, n)
        rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, 0xB, b])))
        blk_lens = lens[s_lo:s_hi]
        blk = _draw_residues(rng, int(blk_lens.sum()))
        blk_off = np.zeros(len(blk_lens) + 1, dtype=np.int64)
        np.cumsum(blk_lens, out=blk_off[1:])
        if plant_frac > 0 and qarr:
            prng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([plant_seed, 0xC, b])))
            chosen = np.nonzero(prng.random(len(blk_lens)) < plant_frac)[0]
            for j in chosen:
                qi = int(prng.integers(0, len(qarr)))
                Q = qarr[qi]
                L = int(prng.integers(20, 151))
                L = min(L, int(blk_lens[j]), len(Q))
                qs = int(prng.integers(0, len(Q) - L + 1))
                ss = int(prng.integers(0, int(blk_lens[j]) - L + 1))
                exact = bool(prng.random() < 0.1)
                seg = Q[qs:qs + L].copy()
                if not exact:
                    keep = prng.random(L) < 0.6
                    seg[~keep] = _draw_residues(prng, int((~keep).sum()))
                a = blk_off[j] + ss
                blk[a:a + L] = seg
                plants.append((s_lo + j, ss, qi, qs, L, exact))
        # copy the requested part of this block
        c_lo, c_hi = max(s_lo, lo), min(s_hi, hi)
        src = blk[blk_off[c_lo - s_lo]:blk_off[c_hi - s_lo]]
        ascii[offsets[c_lo - lo]:offsets[c_hi - lo]] = src
    pl = np.array([p for p in plants if lo <= p[0] < hi], dtype=PLANT_DTYPE)
    if len(pl):
        pl["subject"] -= lo
    return SyntheticDB(ascii, offsets, pl, first_subject=lo,
                       meta=dict(seed=seed, plant_seed=plant_seed, n_total=n,
                                 residues_total=int(lens.sum()), mean_len=mean_len,
                                 plant_frac=plant_frac))


# BASELINE.json configs (SURVEY.md 8(d) seeds).
CONFIGS = {
    1: dict(name="q127_vs_1k_subjects", query_len=127, query_seed=127, db_seed=1001,
            plant_seed=2001, n_subjects=1000, total_residues=None, mean_len=250.0,
            plant_frac=0.05),
    2: dict(name="q517_vs_20M_residues", query_len=517, query_seed=517, db_seed=1002,
            plant_seed=2002, n_subjects=None, total_residues=20_000_000, mean_len=200.0,
            plant_frac=0.05),
    3: dict(name="q1054_vs_env_nr_shaped_6M_subjects", query_len=1054, query_seed=1054,
            db_seed=1003, plant_seed=2003, n_subjects=6_000_000, total_residues=None,
            mean_len=200.0, plant_frac=0.005),
    5: dict(name="64_queries_vs_nr_shaped_40M_subjects", query_len=None, query_seed=4242,
            db_seed=1005, plant_seed=2005, n_subjects=40_000_000, total_residues=None,
            mean_len=375.0, plant_frac=0.005),
}


def config_offsets(cfg: int, scale: float = 1.0) -> np.ndarray:
    """Full int64 offsets of a config's database (lengths only, no residues),
    enough to plan shards before generating just one range."""
    c = CONFIGS[cfg]
    ns, tr = c["n_subjects"], c["total_residues"]
    if scale != 1.0:
        ns = None if ns is None else max(1, int(ns * scale))
        tr = None if tr is None else max(1000, int(tr * scale))
    lens = _lengths(c["db_seed"], ns, tr, c["mean_len"])
    off = np.zeros(len(lens) + 1, dtype=np.int64)
    np.cumsum(lens, out=off[1:])
    return off


def config_workload(cfg: int, *, subject_range=None, scale: float = 1.0):
    """(queries, db) for a BASELINE.json config.  scale < 1 shrinks the DB
    (same generator, fewer subjects) for quick tests."""
    c = CONFIGS[cfg]
    if c["query_len"] is None:
        queries = gen_queries(c["query_seed"], 64, 100, 2000)
    else:
        queries = [gen_query(c["query_seed"], c["query_len"])]
    ns = c["n_subjects"]
    tr = c["total_residues"]
    if scale != 1.0:
        ns = None if ns is None else max(1, int(ns * scale))
        tr = None if tr is None else max(1000, int(tr * scale))
    db = gen_db(c["db_seed"], c["plant_seed"], n_subjects=ns, total_residues=tr,
                mean_len=c["mean_len"], queries=queries, plant_frac=c["plant_frac"],
                subject_range=subject_range)
    return queries, db
