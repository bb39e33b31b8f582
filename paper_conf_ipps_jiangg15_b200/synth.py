"""Seeded synthetic inputs shaped like the paper's workloads (shared by tests, bench and smoke).

This module holds NO arithmetic of the method (no quantisation, no DP, no
statistics of scores): it only draws float log-odds profiles and digitised
sequence databases.  It is the one module both the CUDA path and the CPU oracle
are fed from.

* Profiles: Pfam-like HMMs, M from 48 to 2405.  Match emissions
  e_k ~ Dirichlet(20 f) mixed 0.98/0.02 with the background f; transitions
  M->(M,I,D) ~ Dir(18,1,1), I->(M,I) ~ Dir(5,5), D->(M,D) ~ Dir(7,3);
  occupancy-weighted local entry (HMMER 3.0 local configuration, reading R8);
  degenerate codes B J Z O U X get the background-weighted expected score and
  the gap codes - * ~ get -inf (reading R22).
* Databases: Swiss-Prot / UniProt-shaped: lognormal lengths,
  background residues, 0.05% X, 0.01% long (titin-like) sequences, optional
  planted homologs (segments emitted from the profile's match states).
  Residues come from a counter-based generator (splitmix64 of the global
  residue index) so any shard of a 10 M-sequence DB can be materialised alone.
"""
from __future__ import annotations

import numpy as np

# Residue order of the digital alphabet (Fig 6; Easel order, reading R23/D3).
ALPHABET = "ACDEFGHIKLMNPQRSTVWY-BJZOUX*~"
NCANON = 20
NALPHA = 29
CODE_X = ALPHABET.index("X")

# HMMER3 amino-acid background (reading R34), canonical order A..Y.
BACKGROUND = np.array([
    0.0787945, 0.0151600, 0.0535222, 0.0668298, 0.0397062, 0.0695071, 0.0229198, 0.0590092,
    0.0594422, 0.0963728, 0.0237718, 0.0414386, 0.0482904, 0.0395639, 0.0540978, 0.0683364,
    0.0540687, 0.0673417, 0.0114135, 0.0304133], dtype=np.float64)
BACKGROUND = BACKGROUND / BACKGROUND.sum()

_DEGEN = {"B": "DN", "J": "IL", "Z": "EQ", "O": "K", "U": "C", "X": ALPHABET[:NCANON]}
_GAPS = "-*~"

# BASELINE.json configs.
CONFIGS = {
    1: dict(M=64, pseed=1064, N=1000, mu_ln=5.42, sigma=0.75, dseed=11, planted=0.0),
    2: dict(M=200, pseed=1200, N=550_000, mu_ln=5.60, sigma=0.75, dseed=12, planted=0.0),
    3: dict(M=400, pseed=1400, N=550_000, mu_ln=5.60, sigma=0.75, dseed=12, planted=0.001),
    4: dict(M=2048, pseed=3048, N=550_000, mu_ln=5.60, sigma=0.75, dseed=12, planted=0.0),
    5: dict(M=(100, 500, 1000), pseed=(1100, 1500, 2000), N=10_000_000, mu_ln=5.55, sigma=0.80,
            dseed=15, planted=0.0),
}


class Profile:
    """Float32 log-odds profile: msc [M][29] (nats), tsc [M][8] (nats), plus the
    match emission probabilities ``emit`` [M][20] used to plant homologs."""

    def __init__(self, msc, tsc, emit):
        self.msc = np.ascontiguousarray(msc, dtype=np.float32)
        self.tsc = np.ascontiguousarray(tsc, dtype=np.float32)
        self.emit = emit
        self.M = self.msc.shape[0]


def make_profile(M: int, seed: int, stress: bool = False, dd=(7.0, 3.0), uniform_entry: bool = False) -> Profile:
    """Dirichlet profile of length M.  ``stress`` skips the background mix (log-odds
    down to ~ -45 nats, exercising the -inf clamps); ``dd`` sets D->(M,D) (use
    (1, 9) for the adversarial long-D-chain profile)."""
    rng = np.random.default_rng(seed)
    f = BACKGROUND
    e = rng.dirichlet(20.0 * f, size=M)
    if not stress:
        e = 0.98 * e + 0.02 * f
    e = np.maximum(e, 1e-300)
    with np.errstate(divide="ignore"):
        lo = np.log(e / f)                              # [M][20]
    msc = np.full((M, NALPHA), -np.inf, dtype=np.float64)
    msc[:, :NCANON] = lo
    for sym, members in _DEGEN.items():
        idx = [ALPHABET.index(c) for c in members]
        w = f[idx]
        msc[:, ALPHABET.index(sym)] = (lo[:, idx] * w).sum(axis=1) / w.sum()
    for g in _GAPS:
        msc[:, ALPHABET.index(g)] = -np.inf

    # node 0 (begin) and nodes 1..M transitions, probabilities
    tm = rng.dirichlet([18.0, 1.0, 1.0], size=M + 1)   # M->M, M->I, M->D
    ti = rng.dirichlet([5.0, 5.0], size=M + 1)         # I->M, I->I
    td = rng.dirichlet(list(dd), size=M + 1)           # D->M, D->D
    # occupancy-weighted local entry (HMMER 3.0 p7_hmm_CalculateOccupancy + local config)
    occ = np.zeros(M + 1)
    occ[1] = tm[0, 0] + tm[0, 1]
    for k in range(2, M + 1):
        occ[k] = occ[k - 1] * (tm[k - 1, 0] + tm[k - 1, 1]) + (1.0 - occ[k - 1]) * td[k - 1, 0]
    Z = sum(occ[k] * (M - k + 1) for k in range(1, M + 1))
    if uniform_entry:
        tbm = np.full(M, np.log(2.0 / (M * (M + 1.0))))
    else:
        tbm = np.log(occ[1:] / Z)

    with np.errstate(divide="ignore"):
        tsc = np.full((M, 8), -np.inf, dtype=np.float64)
        tsc[:, 0] = tbm                                 # B->M_k
        tsc[1:, 1] = np.log(tm[1:M, 0])                 # M_{k-1}->M_k
        tsc[1:, 2] = np.log(ti[1:M, 0])                 # I_{k-1}->M_k
        tsc[1:, 3] = np.log(td[1:M, 0])                 # D_{k-1}->M_k
        tsc[:M - 1, 4] = np.log(tm[1:M, 2])             # M_k->D_{k+1}
        tsc[:M - 1, 5] = np.log(tm[1:M, 1])             # M_k->I_k
        tsc[:M - 1, 6] = np.log(ti[1:M, 1])             # I_k->I_k
        tsc[:M - 1, 7] = np.log(td[1:M, 1])             # D_k->D_{k+1}
    return Profile(msc.astype(np.float32), tsc.astype(np.float32), e)


# ---------------------------------------------------------------- databases
def _splitmix64(x: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


# residue sampler: 0.05% X, canonical residues by the background (DESIGN.md input recipe)
_PX = 0.0005
_CDF = np.concatenate([np.cumsum(BACKGROUND * (1.0 - _PX)), [1.0]])
_SYMS = np.concatenate([np.arange(NCANON), [CODE_X]]).astype(np.uint8)


# 16-bit inverse-CDF table: a residue is _TABLE[top 16 bits of splitmix64(position ^ key)]
_TABLE = _SYMS[np.searchsorted(_CDF, (np.arange(65536) + 0.5) / 65536.0, side="right").clip(0, NCANON)]


def _residues_at(key: int, pos: np.ndarray) -> np.ndarray:
    """Residues at global positions ``pos`` (uint64) of DB stream ``key``."""
    k = np.uint64((int(key) * 0xD1B54A32D192ED03) & 0xFFFFFFFFFFFFFFFF)
    return _TABLE[(_splitmix64(pos ^ k) >> np.uint64(48)).astype(np.intp)]


class Database:
    """A digitised DB in caller order: ``lengths`` [N] int32 and, once materialised,
    ``dsq`` (uint8 codes 0..28, concatenated) with ``off`` [N+1] int64."""

    def __init__(self, lengths, seed, planted_ids=(), profile=None):
        self.lengths = np.ascontiguousarray(lengths, dtype=np.int32)
        self.N = len(self.lengths)
        self.seed = seed
        self.gstart = np.zeros(self.N + 1, dtype=np.int64)
        np.cumsum(self.lengths, out=self.gstart[1:])
        self.planted_ids = np.asarray(planted_ids, dtype=np.int64)
        self.profile = profile

    @property
    def residues(self) -> int:
        return int(self.gstart[-1])

    def materialize(self, ids=None):
        """Return (dsq, off) for sequences ``ids`` (default: all, caller order)."""
        ids = np.arange(self.N, dtype=np.int64) if ids is None else np.asarray(ids, dtype=np.int64)
        L = self.lengths[ids].astype(np.int64)
        off = np.zeros(len(ids) + 1, dtype=np.int64)
        np.cumsum(L, out=off[1:])
        total = int(off[-1])
        dsq = np.empty(total, dtype=np.uint8)
        step = 1 << 22
        shift = self.gstart[ids] - off[:-1]           # global position = local position + shift

        def fill(a):
            b = min(total, a + step)
            j0 = int(np.searchsorted(off, a, side="right")) - 1
            j1 = int(np.searchsorted(off, b - 1, side="right"))
            lo = np.maximum(off[j0:j1], a)
            hi = np.minimum(off[j0 + 1:j1 + 1], b)
            pos = np.repeat(shift[j0:j1], hi - lo) + np.arange(a, b, dtype=np.int64)
            dsq[a:b] = _residues_at(self.seed, pos.astype(np.uint64))

        chunks = range(0, total, step)
        if len(chunks) > 1:                           # disjoint slices; numpy releases the GIL
            import concurrent.futures as cf
            import os
            with cf.ThreadPoolExecutor(max_workers=min(len(chunks), os.cpu_count() or 1)) as ex:
                list(ex.map(fill, chunks))
        else:
            for a in chunks:
                fill(a)
        if len(self.planted_ids) and self.profile is not None:
            where = {int(s): j for j, s in enumerate(ids)}
            for s in self.planted_ids:
                j = where.get(int(s))
                if j is None:
                    continue
                seg = _homolog(self.profile, int(s), self.seed, int(L[j]))
                a = int(off[j]) + (int(L[j]) - len(seg)) // 2
                dsq[a:a + len(seg)] = seg
        return dsq, off


def _homolog(profile: Profile, sid: int, seed: int, L: int) -> np.ndarray:
    """A 50-300 residue segment emitted from consecutive match states (planted homolog)."""
    rng = np.random.default_rng([seed, 7, sid])
    n = int(min(L, rng.integers(50, 301), profile.M))
    k0 = int(rng.integers(0, profile.M - n + 1))
    seg = np.empty(n, dtype=np.uint8)
    for j in range(n):
        seg[j] = rng.choice(NCANON, p=profile.emit[k0 + j] / profile.emit[k0 + j].sum())
    return seg


def make_lengths(N: int, mu_ln: float, sigma: float, seed: int, lmin: int = 10, lmax: int = 35213,
                 long_frac: float = 1e-4) -> np.ndarray:
    rng = np.random.default_rng(seed)
    L = np.rint(rng.lognormal(mu_ln, sigma, size=N)).clip(lmin, lmax).astype(np.int32)
    nlong = int(round(N * long_frac))
    if nlong:
        idx = rng.choice(N, size=nlong, replace=False)
        L[idx] = rng.integers(5000, lmax + 1, size=nlong)
    return L


def make_db(N: int, mu_ln: float, sigma: float, seed: int, planted: float = 0.0,
            profile: Profile | None = None, **kw) -> Database:
    L = make_lengths(N, mu_ln, sigma, seed, **kw)
    planted_ids = ()
    if planted > 0 and profile is not None:
        rng = np.random.default_rng([seed, 3])
        planted_ids = np.sort(rng.choice(N, size=max(1, int(round(N * planted))), replace=False))
    return Database(L, seed, planted_ids, profile)


def config(cfg: int, which: int = 0, N: int | None = None):
    """(Profile, Database) of BASELINE config ``cfg`` (``which`` picks M for config 5)."""
    c = CONFIGS[cfg]
    M, ps = c["M"], c["pseed"]
    if isinstance(M, tuple):
        M, ps = M[which], ps[which]
    prof = make_profile(M, ps)
    db = make_db(N or c["N"], c["mu_ln"], c["sigma"], c["dseed"], planted=c["planted"], profile=prof)
    return prof, db


def random_dsq(rng: np.random.Generator, L: int, alphabet: int = NALPHA) -> np.ndarray:
    """Uniform codes 0..alphabet-1 (edge-case tests: degenerate and gap residues)."""
    return rng.integers(0, alphabet, size=L).astype(np.uint8)
