"""Independent pins for the oracle (pure Python / numpy, tiny inputs only).

None of this is used by the product path.  Each function re-derives a result
by a route different from the oracle's row-by-row DP:

* ``msv_brute`` / ``vit_brute``: enumerate every alignment (path) of the
  model explicitly and apply the saturating per-step arithmetic along it; the
  filter score is the max over paths.  This is the definition the DP computes
  (every step is a monotone map, so max over paths == DP), P:209-214 (MSV:
  multiple ungapped segments joined through J) and Fig 3 P:294-330 (Plan 7).
* ``msv_wide`` / ``vit_wide``: the recurrences of Alg 1 / Alg 2 recomputed in
  numpy int64 with an explicit clamp after every operation.
* ``vit_lazyf``: the Viterbi filter with HMMER's Lazy-F: D->D is
  resolved only on rows where Dmax + ddbound > xB, and then by iterating until
  nothing improves -- it must equal the full closure the oracle performs.
* ``vit_ungapped``: the Viterbi filter with no I and no D states written as its
  own 20-line DP.
* ``fwd_brute``: the Forward score ("summed over all possible
  alignments") as an explicit sum over every state path of the Plan-7
  multihit model with its N/J/C length model, in float64 (fsum of exp).
"""
from __future__ import annotations

import sys

import numpy as np

NEG = -32768


def u8(v):
    return 0 if v < 0 else (255 if v > 255 else v)


def s16(v):
    return NEG if v < NEG else (32767 if v > 32767 else v)


# ----------------------------------------------------------------------------- MSV
def msv_brute(cost, bias, tbm, tec, tjb, dsq, reenter=True):
    """Max over ordered lists of row-disjoint ungapped diagonal segments.

    A segment enters at row i, node k from B (value 190 - tjb from N, or
    J - tjb from the previous segment's J value), loses tbm (B->M_k), and
    walks the diagonal (i, k), (i+1, k+1), ...; each cell adds bias then
    subtracts cost[x_i][k] (u8 saturating).  Leaving at any cell gives
    E = cell, J = E - tec.  Returns 255 if any cell reaches 255 - bias.
    ``reenter=False`` drops the J entries (every segment from N): the pins use it only to
    show that a case really chains a later segment through J."""
    M = cost.shape[1]
    L = len(dsq)
    best = [0, False]  # raw, overflow

    def segments_from(row_min, J):
        for i in range(row_min, L + 1):
            entries = [u8(190 - tjb)]
            if J is not None and reenter:
                entries.append(u8(J - tjb))
            for k in range(1, M + 1):
                for entry in entries:
                    v = u8(entry - tbm)
                    t = 0
                    while i + t <= L and k + t <= M:
                        v = u8(v + bias)
                        v = u8(v - int(cost[dsq[i + t - 1], k + t - 1]))
                        if v >= 255 - bias:
                            best[1] = True
                        Jn = u8(v - tec)
                        if Jn > best[0]:
                            best[0] = Jn
                        segments_from(i + t + 1, Jn)
                        t += 1

    sys.setrecursionlimit(10000)
    segments_from(1, None)
    return 255 if best[1] else best[0]


def msv_wide(cost, bias, tbm, tec, tjb, dsq):
    """Alg 1 in numpy int64, explicit clamp after every op (vectorised over k)."""
    M = cost.shape[1]
    c = cost.astype(np.int64)
    prev = np.zeros(M + 1, dtype=np.int64)
    xJ = 0
    xB = np.clip(190 - tjb, 0, 255)
    for x in dsq:
        xBp = np.clip(xB - tbm, 0, 255)
        s = np.maximum(prev[:-1], xBp)
        s = np.clip(s + bias, 0, 255)
        s = np.clip(s - c[x], 0, 255)
        xE = int(s.max()) if M else 0
        if xE >= 255 - bias:
            return 255
        xJ = max(xJ, int(np.clip(xE - tec, 0, 255)))
        xB = np.clip(max(xJ, 190) - tjb, 0, 255)
        prev = np.concatenate([[0], s])
    return xJ


# ----------------------------------------------------------------------------- Viterbi
def vit_brute(rsc, tr, move, dsq, xw_e=-500):
    """Max over Plan-7 local multihit paths (Fig 3) with s16 saturation per step.

    States: M_k (emits), I_k (emits, score 0), D_k (silent).  A domain enters
    B->M_k (value max(J, 12000) + move via J or N), walks the core model,
    leaves M_j->E; E->C / E->J cost xw_e; C->T is folded into the final
    conversion, so the raw score is xC = max over domain lists of E + xw_e."""
    tBM, tMM, tIM, tDM, tMD, tMI, tII, tDD = [tr[t].astype(np.int64) for t in range(8)]
    M = rsc.shape[1]
    L = len(dsq)
    out = {"xC": NEG, "ovf": False}

    def em(i, k):  # M_k emitting residue i (1-based)
        return int(rsc[dsq[i - 1], k - 1])

    def walk(state, k, i, v):
        # state at node k, having consumed residues up to i (M/I emitted residue i; D at row i)
        if state == "M":
            if v >= 32767:
                out["ovf"] = True
            e = v + xw_e
            if e > out["xC"]:
                out["xC"] = e
            domains(i + 1, e)                                  # E -> J -> next domain
            if k < M and i < L:                                # M_k -> M_{k+1}
                walk("M", k + 1, i + 1, s16(s16(v + int(tMM[k])) + em(i + 1, k + 1)))
            if i < L:                                          # M_k -> I_k
                walk("I", k, i + 1, s16(v + int(tMI[k - 1])))
            if k < M:                                          # M_k -> D_{k+1}
                walk("D", k + 1, i, s16(v + int(tMD[k - 1])))
        elif state == "I":
            if i < L:
                walk("I", k, i + 1, s16(v + int(tII[k - 1])))
            if k < M and i < L:
                walk("M", k + 1, i + 1, s16(s16(v + int(tIM[k])) + em(i + 1, k + 1)))
        else:  # D
            if k < M:
                walk("D", k + 1, i, s16(v + int(tDD[k - 1])))
            if k < M and i < L:
                walk("M", k + 1, i + 1, s16(s16(v + int(tDM[k])) + em(i + 1, k + 1)))

    def domains(row_min, J):
        for i in range(row_min, L + 1):
            xBs = [12000 + move]
            if J is not None:
                xBs.append(J + move)
            for xB in xBs:
                for k in range(1, M + 1):
                    walk("M", k, i, s16(s16(xB + int(tBM[k - 1])) + em(i, k)))

    sys.setrecursionlimit(100000)
    domains(1, None)
    return 32767 if out["ovf"] else max(out["xC"], NEG)


def vit_wide(rsc, tr, move, dsq, xw_e=-500):
    """Alg 2 in numpy int64 with explicit clamps, D->D closure by a k loop."""
    M = rsc.shape[1]
    T = tr.astype(np.int64)
    tBM, tMM, tIM, tDM, tMD, tMI, tII, tDD = T
    Mp = np.full(M + 1, NEG, dtype=np.int64)
    Ip = Mp.copy()
    Dp = Mp.copy()
    xN, xJ, xC = 12000, NEG, NEG
    xB = xN + move
    sat = lambda a: np.clip(a, NEG, 32767)
    for x in dsq:
        r = rsc[x].astype(np.int64)
        Mn = np.full(M + 1, NEG, dtype=np.int64)
        In = Mn.copy()
        Dn = Mn.copy()
        m = np.maximum.reduce([sat(xB + tBM), sat(Mp[:-1] + tMM), sat(Ip[:-1] + tIM), sat(Dp[:-1] + tDM)])
        Mn[1:] = sat(m + r)
        In[1:] = np.maximum(sat(Mp[1:] + tMI), sat(Ip[1:] + tII))
        Dn[2:] = sat(Mn[1:-1] + tMD[:-1])
        xE = int(Mn[1:].max())
        if xE >= 32767:
            return 32767
        xC = max(xC, xE + xw_e)
        xJ = max(xJ, xE + xw_e)
        xB = max(xJ, xN) + move
        for k in range(2, M + 1):
            Dn[k] = max(Dn[k], int(sat(Dn[k - 1] + tDD[k - 2])))
        Mp, Ip, Dp = Mn, In, Dn
    return int(xC)


def vit_lazyf(rsc, tr, move, ddbound, dsq, xw_e=-500, stats=None):
    """Viterbi filter with Lazy-F (Farrar ref [19]): D->D resolved only on
    rows where Dmax + ddbound > xB, by repeated sweeps until no D cell improves."""
    M = rsc.shape[1]
    T = tr.astype(np.int64)
    tBM, tMM, tIM, tDM, tMD, tMI, tII, tDD = T
    Mp = [NEG] * (M + 1)
    Ip = [NEG] * (M + 1)
    Dp = [NEG] * (M + 1)
    xN, xJ, xC = 12000, NEG, NEG
    xB = xN + move
    for x in dsq:
        Mn = [NEG] * (M + 1)
        In = [NEG] * (M + 1)
        Dn = [NEG] * (M + 1)
        for k in range(1, M + 1):
            m = max(s16(xB + tBM[k - 1]), s16(Mp[k - 1] + tMM[k - 1]), s16(Ip[k - 1] + tIM[k - 1]),
                    s16(Dp[k - 1] + tDM[k - 1]))
            Mn[k] = s16(m + int(rsc[x, k - 1]))
            In[k] = max(s16(Mp[k] + tMI[k - 1]), s16(Ip[k] + tII[k - 1]))
            if k >= 2:
                Dn[k] = s16(Mn[k - 1] + tMD[k - 2])
        xE = max(Mn[1:])
        if xE >= 32767:
            return 32767
        xC = max(xC, xE + xw_e)
        xJ = max(xJ, xE + xw_e)
        xB = max(xJ, xN) + move
        Dmax = max(Dn[2:]) if M >= 2 else NEG
        if Dmax + ddbound > xB:
            if stats is not None:
                stats["rows_lazyf"] = stats.get("rows_lazyf", 0) + 1
            changed = True
            while changed:
                changed = False
                for k in range(2, M + 1):
                    dd = s16(Dn[k - 1] + tDD[k - 2])
                    if dd > Dn[k]:
                        Dn[k] = dd
                        changed = True
        Mp, Ip, Dp = Mn, In, Dn
    return xC


def vit_ungapped(rsc, tbm, tmm, move, dsq, xw_e=-500):
    """Viterbi filter of a model with no I / D states: the M cells follow only
    B->M_k and M_{k-1}->M_k (an ungapped word-scale local multihit DP)."""
    M = rsc.shape[1]
    prev = [NEG] * (M + 1)
    xJ = xC = NEG
    xB = 12000 + move
    for x in dsq:
        cur = [NEG] * (M + 1)
        for k in range(1, M + 1):
            cur[k] = s16(max(s16(xB + int(tbm[k - 1])), s16(prev[k - 1] + int(tmm[k - 1]))) + int(rsc[x, k - 1]))
        xE = max(cur[1:])
        if xE >= 32767:
            return 32767
        xC = max(xC, xE + xw_e)
        xJ = max(xJ, xE + xw_e)
        xB = max(xJ, 12000) + move
        prev = cur
    return xC


def fwd_brute(msc, tsc, dsq, stats=False):
    """log of the sum over ALL state paths S->N->B->(M|I|D)->E->(J->B..)->C->T of the path's
    odds (emission odds exp(msc) for M, 1 for I/N/J/C; transition probabilities exp(tsc);
    local entry B->M_k, local exit M_k->E and D_k->E with probability 1, E->C = E->J = 1/2,
    N->N = J->J = C->C = L/(L+3), N->B = J->B = C->T = 3/(L+3)).  Depth-first enumeration,
    tiny M and L only."""
    import math
    M, L = msc.shape[0], len(dsq)
    loop, move = math.log(L / (L + 3.0)), math.log(3.0 / (L + 3.0))
    half = math.log(0.5)
    T = lambda k, t: float(tsc[k - 1, t])       # node k = 1..M
    terms = []
    sys.setrecursionlimit(10000)

    def go(state, k, i, v):                      # i residues emitted so far, v log-odds so far
        if v == -math.inf:
            return
        if state == "N":
            if i < L:
                go("N", 0, i + 1, v + loop)      # N loop emits residue i+1
            go("B", 0, i, v + move)
        elif state == "B":
            if i < L:
                for kk in range(1, M + 1):
                    go("M", kk, i + 1, v + T(kk, 0) + float(msc[kk - 1, dsq[i]]))
        elif state == "M":
            go("E", 0, i, v)                     # local exit
            if k < M:
                if i < L:
                    go("M", k + 1, i + 1, v + T(k + 1, 1) + float(msc[k, dsq[i]]))
                    go("I", k, i + 1, v + T(k, 5))
                go("D", k + 1, i, v + T(k, 4))
        elif state == "I":
            if i < L:
                go("M", k + 1, i + 1, v + T(k + 1, 2) + float(msc[k, dsq[i]]))
                go("I", k, i + 1, v + T(k, 6))
        elif state == "D":
            go("E", 0, i, v)                     # local exit
            if k < M:
                if i < L:
                    go("M", k + 1, i + 1, v + T(k + 1, 3) + float(msc[k, dsq[i]]))
                go("D", k + 1, i, v + T(k, 7))
        elif state == "E":
            go("C", 0, i, v + half)
            go("J", 0, i, v + half)
        elif state == "J":
            if i < L:
                go("J", 0, i + 1, v + loop)
            go("B", 0, i, v + move)
        elif state == "C":
            if i < L:
                go("C", 0, i + 1, v + loop)
            else:
                terms.append(v + move)           # C -> T after the last residue

    go("N", 0, 0, 0.0)
    if not terms:
        return (-math.inf, -math.inf, 0) if stats else -math.inf
    top = max(terms)
    lse = top + math.log(math.fsum(math.exp(t - top) for t in terms))
    return (lse, top, len(terms)) if stats else lse
