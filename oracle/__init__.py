"""CPU oracle for the hmmsearch hot path (MSV + Viterbi filter) -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_ipps_jiangg15_b200``) never imports it, and this package never
imports the product path: the two share no code.  The arithmetic lives in
``hmg_oracle.c`` (plain C, scalar, explicit saturation after every operation,
full D->D closure on every row); this module only builds it with gcc and
marshals numpy arrays through ctypes.

Every function cites the paper passage it follows (P:NNN = PAPER.md line).
Parity status per function:
  quantisation constants ........ pinned (closed forms, tests/test_oracle.py)
  MSV DP ......................... pinned (brute-force path enumeration incl. segments
                                   chained through J above base 190, wide-int recompute,
                                   invariants, closed forms at L=1 and for two segments)
  Viterbi DP ..................... pinned (brute-force Plan-7 paths, wide-int
                                   recompute, ungapped special case)
  nats / null1 / Gumbel / pass ... pinned (closed forms, golden VF-nats table written by
                                   tests/golden/make_vit_nats.py, textbook Gumbel, direct
                                   MSV / Viterbi pass decisions over a (raw, L, mu, F) grid,
                                   statistical pass fractions at F1 and F2)
  Forward score (f2) ............. pinned (brute-force sum over all Plan-7 paths with
                                   N/J/C loops, closed form for a one-node model)
  agreement with HMMER 3.0 itself  parity unpinned (no HMMER source or scores
                                   on this box; R1-R34)
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "hmg_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

NALPHA = 29  # 20 standard + 6 degenerate + 3 gap codes


def build(force: bool = False) -> str:
    """Compile hmg_oracle.c into liboracle.so (gcc -O2, pthreads)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp.%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-pthread",
                               "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        c_int, c_float, c_double, c_i64, c_p = (ctypes.c_int, ctypes.c_float, ctypes.c_double,
                                                ctypes.c_int64, ctypes.c_void_p)
        sig = {
            "or_ub": (c_int, [c_float]), "or_bb": (c_int, [c_float, c_int]), "or_w": (c_int, [c_float]),
            "or_tjb_b": (c_int, [c_int]), "or_move_w": (c_int, [c_int]), "or_tbm_b": (c_int, [c_int]),
            "or_tec_b": (c_int, []), "or_xw_e": (c_int, []),
            "or_quant_msv": (c_int, [c_int, c_p, c_p, c_p, c_p, c_p]),
            "or_quant_vit": (c_int, [c_int, c_p, c_p, c_p, c_p, c_p]),
            "or_msv_seq": (c_int, [c_int, c_p, c_int, c_int, c_int, c_p, c_int, c_int]),
            "or_vit_seq": (c_int, [c_int, c_p, c_p, c_p, c_int, c_int]),
            "or_msv_db": (None, [c_int, c_p, c_int, c_int, c_int, c_p, c_p, c_p, c_i64, c_int, c_p]),
            "or_vit_db": (None, [c_int, c_p, c_p, c_p, c_p, c_p, c_i64, c_int, c_p]),
            "or_msv_nats": (c_float, [c_int, c_int]), "or_vit_nats": (c_float, [c_int, c_int]),
            "or_null1": (c_float, [c_int]), "or_gumbel_surv": (c_double, [c_double, c_double, c_double]),
            "or_pvalue": (c_double, [c_float, c_int, c_double, c_double]),
            "or_msv_pass": (c_int, [c_int, c_int, c_double, c_double, c_double]),
            "or_vit_pass": (c_int, [c_int, c_int, c_double, c_double, c_double]),
            "or_bits": (c_double, [c_float, c_int]),
            "or_fwd_seq": (c_double, [c_int, c_p, c_p, c_p, c_int, c_p]),
            "or_fwd_db": (None, [c_int, c_p, c_p, c_p, c_p, c_p, c_i64, c_int, c_p]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


# ---------------------------------------------------------------- quantisation
class MSVProfile:
    """Byte profile (Alg 1 l.15; HMMER 3.0 byte system, R1/R3/R4/R7)."""

    def __init__(self, msc: np.ndarray):
        msc = np.ascontiguousarray(msc, dtype=np.float32)
        self.M = msc.shape[0]
        self.cost = np.zeros((NALPHA, self.M), dtype=np.uint8)
        b, t, e = ctypes.c_int(), ctypes.c_int(), ctypes.c_int()
        lib().or_quant_msv(self.M, _ptr(msc), _ptr(self.cost), ctypes.byref(b), ctypes.byref(t), ctypes.byref(e))
        self.bias, self.tbm, self.tec = b.value, t.value, e.value


class VitProfile:
    """Word profile (Alg 2 l.9/15-17; HMMER 3.0 word system, R2/R5/R6)."""

    def __init__(self, msc: np.ndarray, tsc: np.ndarray):
        msc = np.ascontiguousarray(msc, dtype=np.float32)
        tsc = np.ascontiguousarray(tsc, dtype=np.float32)
        self.M = msc.shape[0]
        self.rsc = np.zeros((NALPHA, self.M), dtype=np.int16)
        self.tr = np.zeros((8, self.M), dtype=np.int16)
        d = ctypes.c_int()
        lib().or_quant_vit(self.M, _ptr(msc), _ptr(tsc), _ptr(self.rsc), _ptr(self.tr), ctypes.byref(d))
        self.ddbound = d.value


def ub(s: float) -> int: return lib().or_ub(s)
def bb(s: float, bias: int) -> int: return lib().or_bb(s, bias)
def w(s: float) -> int: return lib().or_w(s)
def tjb_b(L: int) -> int: return lib().or_tjb_b(L)
def move_w(L: int) -> int: return lib().or_move_w(L)
def tbm_b(M: int) -> int: return lib().or_tbm_b(M)
def tec_b() -> int: return lib().or_tec_b()
def xw_e() -> int: return lib().or_xw_e()


# ---------------------------------------------------------------- filters
def msv_seq(p: MSVProfile, dsq: np.ndarray, tjb: int = -1) -> int:
    """Raw MSV score (xJ; 255 = overflow) of one digitised sequence, Alg 1.
    ``tjb`` >= 0 fixes the length parameter instead of tjb_b(len(dsq))."""
    d = np.ascontiguousarray(dsq, dtype=np.uint8)
    return lib().or_msv_seq(p.M, _ptr(p.cost), p.bias, p.tbm, p.tec, _ptr(d), len(d), tjb)


def vit_seq(p: VitProfile, dsq: np.ndarray, move: int = 1) -> int:
    """Raw Viterbi-filter score (xC; 32767 overflow, -32768 no path), Alg 2.
    ``move`` <= 0 fixes the N/J/C move score instead of move_w(len(dsq))."""
    d = np.ascontiguousarray(dsq, dtype=np.uint8)
    return lib().or_vit_seq(p.M, _ptr(p.rsc), _ptr(p.tr), _ptr(d), len(d), move)


def msv_db(p: MSVProfile, dsq: np.ndarray, off: np.ndarray, ids=None, nthreads: int | None = None) -> np.ndarray:
    """Raw MSV of sequences ``ids`` (default all) of a concatenated DB, threaded over sequences."""
    dsq = np.ascontiguousarray(dsq, dtype=np.uint8)
    off = np.ascontiguousarray(off, dtype=np.int64)
    n = len(off) - 1 if ids is None else len(ids)
    idp = None
    if ids is not None:
        ids = np.ascontiguousarray(ids, dtype=np.int64)
        idp = _ptr(ids)
    out = np.zeros(n, dtype=np.int32)
    lib().or_msv_db(p.M, _ptr(p.cost), p.bias, p.tbm, p.tec, _ptr(dsq), _ptr(off), idp, n,
                    nthreads or os.cpu_count() or 1, _ptr(out))
    return out


def vit_db(p: VitProfile, dsq: np.ndarray, off: np.ndarray, ids=None, nthreads: int | None = None) -> np.ndarray:
    dsq = np.ascontiguousarray(dsq, dtype=np.uint8)
    off = np.ascontiguousarray(off, dtype=np.int64)
    n = len(off) - 1 if ids is None else len(ids)
    idp = None
    if ids is not None:
        ids = np.ascontiguousarray(ids, dtype=np.int64)
        idp = _ptr(ids)
    out = np.zeros(n, dtype=np.int32)
    lib().or_vit_db(p.M, _ptr(p.rsc), _ptr(p.tr), _ptr(dsq), _ptr(off), idp, n,
                    nthreads or os.cpu_count() or 1, _ptr(out))
    return out


def fwd_seq(msc: np.ndarray, tsc: np.ndarray, dsq: np.ndarray) -> float:
    """Forward score in nats ("total log-likelihood ratios summed over
    all possible alignments", Fig 1), double precision log space."""
    msc = np.ascontiguousarray(msc, dtype=np.float32)
    tsc = np.ascontiguousarray(tsc, dtype=np.float32)
    d = np.ascontiguousarray(dsq, dtype=np.uint8)
    M = msc.shape[0]
    scratch = np.zeros(6 * (M + 1), dtype=np.float64)
    return lib().or_fwd_seq(M, _ptr(msc), _ptr(tsc), _ptr(d), len(d), _ptr(scratch))


def fwd_db(msc, tsc, dsq, off, ids=None, nthreads: int | None = None) -> np.ndarray:
    msc = np.ascontiguousarray(msc, dtype=np.float32)
    tsc = np.ascontiguousarray(tsc, dtype=np.float32)
    dsq = np.ascontiguousarray(dsq, dtype=np.uint8)
    off = np.ascontiguousarray(off, dtype=np.int64)
    n = len(off) - 1 if ids is None else len(ids)
    idp = None
    if ids is not None:
        ids = np.ascontiguousarray(ids, dtype=np.int64)
        idp = _ptr(ids)
    out = np.zeros(n, dtype=np.float64)
    lib().or_fwd_db(msc.shape[0], _ptr(msc), _ptr(tsc), _ptr(dsq), _ptr(off), idp, n,
                    nthreads or os.cpu_count() or 1, _ptr(out))
    return out


# ---------------------------------------------------------------- statistics
def msv_nats(raw: int, L: int) -> float: return lib().or_msv_nats(int(raw), int(L))
def vit_nats(raw: int, L: int) -> float: return lib().or_vit_nats(int(raw), int(L))
def null1(L: int) -> float: return lib().or_null1(int(L))
def gumbel_surv(x: float, mu: float, lam: float) -> float: return lib().or_gumbel_surv(x, mu, lam)
def pvalue(nats: float, L: int, mu: float, lam: float) -> float: return lib().or_pvalue(nats, int(L), mu, lam)
def bits(nats: float, L: int) -> float: return lib().or_bits(nats, int(L))


def msv_pass(raw: int, L: int, mu: float, lam: float, F: float) -> int:
    return lib().or_msv_pass(int(raw), int(L), mu, lam, F)


def vit_pass(raw: int, L: int, mu: float, lam: float, F: float) -> int:
    return lib().or_vit_pass(int(raw), int(L), mu, lam, F)


def fit_mu(bit_scores: np.ndarray, lam: float) -> float:
    """ML location of a Gumbel with known lambda (P:41-45 fixes lambda = log 2):
    mu = -log(mean(exp(-lambda*x)))/lambda."""
    x = np.asarray(bit_scores, dtype=np.float64)
    return float(-np.log(np.mean(np.exp(-lam * x))) / lam)
