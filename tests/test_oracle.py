"""Pins for the CPU oracle (runs without a GPU).

Every test fixes the oracle against something other than itself: closed-form
constants (SURVEY Appendix B / tests/golden/closed_forms.json), brute-force
path enumeration, a wide-integer recomputation, the Lazy-F shortcut, a
special-case model with its own DP, invariants the recurrences imply, a
textbook Gumbel, and a statistical check of the pass fraction.
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
from paper_conf_ipps_jiangg15_b200 import synth
from tests import _pins

GOLD = os.path.join(os.path.dirname(__file__), "golden", "closed_forms.json")


def _tiny_profile(rng, M, lo=-4.0, hi=2.0):
    """Random float profile with a 3-letter effective alphabet for brute force."""
    msc = rng.uniform(lo, hi, size=(M, 29)).astype(np.float32)
    tsc = np.log(rng.uniform(0.05, 1.0, size=(M, 8))).astype(np.float32)
    tsc[0, 1:4] = -np.inf
    tsc[M - 1, 4:8] = -np.inf
    return msc, tsc


# ------------------------------------------------------------------ constants
def test_closed_form_constants_golden():
    """Appendix B values (HMMER 3.0 formulas, float32 + roundf) -- reading R1-R10."""
    g = json.load(open(GOLD))
    for M, v in g["tbm_b"].items():
        assert oracle.tbm_b(int(M)) == v, M
    for L, v in g["tjb_b"].items():
        assert oracle.tjb_b(int(L)) == v, L
    for L, v in g["move_w"].items():
        assert oracle.move_w(int(L)) == v, L
    for L, v in g["null1"].items():
        assert abs(oracle.null1(int(L)) - v) < 2e-5, L
    assert oracle.tec_b() == g["tec_b"] == 3
    assert oracle.xw_e() == g["xw_e"] == -500


def _round_half_away(x):
    return math.copysign(math.floor(abs(x) + 0.5), x)


@pytest.mark.parametrize("M", [1, 2, 3, 17, 48, 64, 100, 400, 1000, 2048, 2405, 5000])
def test_tbm_closed_form(M):
    """tbm_b = -round(3/ln2 * ln(2/(M(M+1)))): uniform MSV entry."""
    x = (3.0 / math.log(2)) * math.log(2.0 / (M * (M + 1.0)))
    if abs(abs(x) - math.floor(abs(x)) - 0.5) > 1e-3:  # not at a rounding tie
        assert oracle.tbm_b(M) == min(255, int(-_round_half_away(x)))


@pytest.mark.parametrize("L", [1, 2, 5, 10, 99, 100, 360, 999, 35213, 100000])
def test_length_params_closed_form(L):
    xb = (3.0 / math.log(2)) * math.log(3.0 / (L + 3))
    xw = (500.0 / math.log(2)) * math.log(3.0 / (L + 3))
    if abs(abs(xb) % 1 - 0.5) > 1e-3:
        assert oracle.tjb_b(L) == int(-_round_half_away(xb))
    if abs(abs(xw) % 1 - 0.5) > 1e-2:
        assert oracle.move_w(L) == int(_round_half_away(xw))
    p1 = L / (L + 1.0)
    assert abs(oracle.null1(L) - (L * math.log(p1) + math.log(1 - p1))) < 1e-5 * max(1.0, abs(oracle.null1(L)))


def test_quantiser_clamps():
    """Byte/word clamps (readings R3-R6): -inf -> 255 / -32768, caps, bias rule."""
    M = 6
    msc = np.zeros((M, 29), np.float32)
    msc[:, :20] = -1.0
    msc[2, 5] = 2.0                      # the canonical maximum sets the bias
    msc[3, 21] = 3.0                     # non-canonical column above it: cost floored at 0
    msc[:, 27] = -np.inf
    msc[4, 0] = -200.0                   # far below: 255 (byte) and -32768 (word)
    p = oracle.MSVProfile(msc)
    assert p.bias == oracle.ub(-2.0) == 9   # round(4.328*2) = 9
    assert p.cost[5, 2] == 0
    assert p.cost[21, 3] == 0
    assert (p.cost[27] == 255).all()
    assert p.cost[0, 4] == 255
    assert p.cost[0, 0] == 4 + 9             # round(4.328) = 4
    tsc = np.full((M, 8), np.log(0.5), np.float32)
    tsc[:, 6] = 0.0                          # II = log 1 -> clamped to -1
    tsc[0, 1:4] = -np.inf
    v = oracle.VitProfile(msc, tsc)
    assert v.rsc[0, 4] == -32768 and (v.rsc[27] == -32768).all()
    assert v.rsc[5, 2] == 1443                # round(721.3475*2)
    assert (v.tr[6] == -1).all()
    assert (v.tr[1:4, 0] == -32768).all()
    assert v.tr[0, 0] == -500


def test_ddbound_definition():
    rng = np.random.default_rng(3)
    msc, tsc = _tiny_profile(rng, 9)
    v = oracle.VitProfile(msc, tsc)
    w = [[oracle.w(float(tsc[k, t])) for t in range(8)] for k in range(9)]
    ref = max(w[k - 1][7] + w[k + 1][3] - w[k + 1][0] for k in range(2, 8))
    assert v.ddbound == ref
    assert oracle.VitProfile(msc[:3], tsc[:3]).ddbound == -32768


# ------------------------------------------------------------------ MSV pins
@pytest.mark.parametrize("seed", range(40))
def test_msv_brute_force(seed):
    """Alg 1 DP == max over explicitly enumerated multi-segment ungapped alignments."""
    rng = np.random.default_rng(100 + seed)
    M = int(rng.integers(1, 5))
    L = int(rng.integers(1, 6))
    msc, _ = _tiny_profile(rng, M, lo=-3.0, hi=3.0 if seed % 4 else 25.0)
    p = oracle.MSVProfile(msc)
    dsq = rng.integers(0, 3, size=L).astype(np.uint8)   # 3-letter sub-alphabet
    tjb = int(rng.integers(1, 30))
    got = oracle.msv_seq(p, dsq, tjb=tjb)
    want = _pins.msv_brute(p.cost, p.bias, p.tbm, p.tec, tjb, dsq)
    assert got == want


@pytest.mark.parametrize("seed", range(20))
def test_msv_wide_int(seed):
    rng = np.random.default_rng(200 + seed)
    M = int(rng.integers(1, 300))
    prof = synth.make_profile(M, seed, stress=bool(seed % 3 == 0))
    p = oracle.MSVProfile(prof.msc)
    dsq = synth.random_dsq(rng, int(rng.integers(1, 400)))
    tjb = oracle.tjb_b(len(dsq))
    assert oracle.msv_seq(p, dsq) == _pins.msv_wide(p.cost, p.bias, p.tbm, p.tec, tjb, dsq)


def test_msv_invariants():
    rng = np.random.default_rng(7)
    prof = synth.make_profile(120, 5)
    p = oracle.MSVProfile(prof.msc)
    dsq = synth.random_dsq(rng, 300, alphabet=20)
    tjb = oracle.tjb_b(300)
    # appending residues (length params fixed) never lowers the score; xJ only grows
    prev = 0
    for n in range(1, 300, 7):
        r = oracle.msv_seq(p, dsq[:n], tjb=tjb)
        assert r >= prev
        prev = r
    # legit raw <= 251 - bias
    assert prev <= 251 - p.bias
    # all-255 cost rows -> raw 0 (no alignment has positive value)
    msc = np.full((50, 29), -np.inf, np.float32)
    q = oracle.MSVProfile(msc)
    assert (q.cost == 255).all() and oracle.msv_seq(q, dsq) == 0


def test_msv_closed_form_L1():
    """One residue: raw = max(0, max_k(((190 - tjb - tbm) + bias) - cost) - 3)."""
    for seed in range(20):
        prof = synth.make_profile(30 + seed, seed)
        p = oracle.MSVProfile(prof.msc)
        for x in range(29):
            tjb = oracle.tjb_b(1)
            v = max(0, 190 - tjb - p.tbm)
            cells = [max(0, min(255, v + p.bias) - int(c)) for c in p.cost[x]]
            want = 255 if max(cells) >= 255 - p.bias else max(0, max(cells) - 3)
            assert oracle.msv_seq(p, np.array([x], np.uint8)) == want


def test_msv_saturation_maps_to_pass():
    """msc = +20 nats -> bias 87, cells saturate -> raw 255 -> P = 0 -> pass (R13)."""
    msc = np.full((40, 29), 20.0, np.float32)
    p = oracle.MSVProfile(msc)
    assert p.bias == 87
    dsq = np.zeros(50, np.uint8)
    assert oracle.msv_seq(p, dsq) == 255
    assert oracle.msv_nats(255, 50) == math.inf
    assert oracle.msv_pass(255, 50, -10.0, math.log(2), 1e-30) == 1


# ------------------------------------------------------------------ Viterbi pins
@pytest.mark.parametrize("seed", range(40))
def test_vit_brute_force(seed):
    """Alg 2 DP (full D->D closure) == max over enumerated Plan-7 local multihit paths."""
    rng = np.random.default_rng(300 + seed)
    M = int(rng.integers(1, 4))
    L = int(rng.integers(1, 5))
    hi = 2.0 if seed % 5 else 45.0   # some overflow cases
    msc, tsc = _tiny_profile(rng, M, lo=-3.0, hi=hi)
    if seed % 7 == 0:
        msc[:, :3] = -60.0           # deep negatives: saturation at -32768 and recovery
        msc[:, 1] = 5.0
    p = oracle.VitProfile(msc, tsc)
    dsq = rng.integers(0, 3, size=L).astype(np.uint8)
    move = -int(rng.integers(100, 7000))
    got = oracle.vit_seq(p, dsq, move=move)
    want = _pins.vit_brute(p.rsc, p.tr, move, dsq)
    assert got == want


@pytest.mark.parametrize("seed", range(12))
def test_vit_wide_int(seed):
    rng = np.random.default_rng(400 + seed)
    M = int(rng.integers(1, 120))
    prof = synth.make_profile(M, seed, stress=bool(seed % 3 == 0), dd=(1.0, 9.0) if seed % 2 else (7.0, 3.0))
    p = oracle.VitProfile(prof.msc, prof.tsc)
    dsq = synth.random_dsq(rng, int(rng.integers(1, 200)))
    move = oracle.move_w(len(dsq))
    assert oracle.vit_seq(p, dsq) == _pins.vit_wide(p.rsc, p.tr, move, dsq)


@pytest.mark.parametrize("seed", range(8))
def test_vit_lazyf_equals_full_closure(seed):
    """Lazy-F is an exact shortcut: same raw score as the full closure."""
    rng = np.random.default_rng(500 + seed)
    M = int(rng.integers(4, 90))
    prof = synth.make_profile(M, 50 + seed, dd=(1.0, 9.0) if seed % 2 else (7.0, 3.0))
    p = oracle.VitProfile(prof.msc, prof.tsc)
    dsq = synth.random_dsq(rng, int(rng.integers(1, 150)), alphabet=20)
    move = oracle.move_w(len(dsq))
    st = {}
    assert oracle.vit_seq(p, dsq) == _pins.vit_lazyf(p.rsc, p.tr, move, p.ddbound, dsq, stats=st)


def test_vit_ungapped_special_case():
    """tMI = tMD = -inf: the Viterbi filter reduces to an ungapped word-scale DP."""
    rng = np.random.default_rng(9)
    for M in (1, 2, 7, 40):
        prof = synth.make_profile(M, M)
        tsc = prof.tsc.copy()
        tsc[:, 4] = -np.inf   # MD
        tsc[:, 5] = -np.inf   # MI
        p = oracle.VitProfile(prof.msc, tsc)
        for _ in range(5):
            dsq = synth.random_dsq(rng, int(rng.integers(1, 120)))
            move = oracle.move_w(len(dsq))
            assert oracle.vit_seq(p, dsq) == _pins.vit_ungapped(p.rsc, p.tr[0], p.tr[1], move, dsq)


def test_vit_no_path_and_overflow():
    M = 5
    msc = np.full((M, 29), -np.inf, np.float32)
    tsc = np.full((M, 8), np.log(0.3), np.float32)
    p = oracle.VitProfile(msc, tsc)
    # -inf emissions quantise to -32768, which is a floor, not an absorbing -inf:
    # sat(xB + tBM - 32768) stays finite (reading R35); the brute-force paths agree.
    d = np.zeros(3, np.uint8)
    assert oracle.vit_seq(p, d) == _pins.vit_brute(p.rsc, p.tr, oracle.move_w(3), d) < -20000
    msc[:] = 60.0
    p = oracle.VitProfile(msc, tsc)
    assert oracle.vit_seq(p, np.zeros(10, np.uint8)) == 32767
    assert oracle.vit_nats(32767, 10) == math.inf
    assert oracle.vit_nats(-32768, 10) == -math.inf


# ------------------------------------------------------------------ statistics
def test_nats_closed_form():
    g = json.load(open(GOLD))
    for raw, v in g["msv_nats_L300"].items():
        assert abs(oracle.msv_nats(int(raw), 300) - v) < 0.01
    for raw in (0, 50, 170, 251):
        for L in (1, 77, 300, 20000):
            want = ((raw - oracle.tjb_b(L)) - 190.0) / (3.0 / math.log(2)) - 3.0
            assert abs(oracle.msv_nats(raw, L) - want) < 1e-5 * max(1, abs(want))
    for raw in (-32000, -5, 0, 7000, 32000):
        for L in (1, 300, 35213):
            want = (raw + oracle.move_w(L) - 12000.0) / (500.0 / math.log(2)) - 3.0
            assert abs(oracle.vit_nats(raw, L) - want) < 1e-5 * max(1, abs(want))


def test_gumbel_textbook():
    """Gumbel survival 1 - exp(-exp(-lambda (x - mu)))."""
    for x in np.linspace(-20, 40, 61):
        for mu, lam in ((-10.0, math.log(2)), (3.0, 0.7)):
            want = -math.expm1(-math.exp(-lam * (x - mu)))
            got = oracle.gumbel_surv(float(x), mu, lam)
            assert abs(got - want) <= 1e-12 + 1e-9 * want


def test_mu_fit_recovers_location():
    rng = np.random.default_rng(1)
    lam, mu = math.log(2), -9.5
    x = mu - np.log(-np.log(rng.uniform(size=200000))) / lam
    assert abs(oracle.fit_mu(x, lam) - mu) < 0.02


def test_msv_pass_fraction_near_F1():
    """Statistical pin (~2.2% pass MSV): with mu calibrated at lambda = ln 2
    on background sequences, the MSV pass fraction at F1 = 0.02 is within 2x of F1."""
    prof = synth.make_profile(100, 1100)
    p = oracle.MSVProfile(prof.msc)
    cal = synth.Database(np.full(1000, 200, np.int32), seed=7)
    dsq, off = cal.materialize()
    raw = oracle.msv_db(p, dsq, off)
    bits = [oracle.bits(oracle.msv_nats(int(r), 200), 200) for r in raw]
    mu = oracle.fit_mu(np.array(bits), math.log(2))
    db = synth.make_db(12000, 5.6, 0.75, seed=21)
    dsq, off = db.materialize()
    raw = oracle.msv_db(p, dsq, off)
    npass = sum(oracle.msv_pass(int(r), int(L), mu, math.log(2), 0.02) for r, L in zip(raw, db.lengths))
    frac = npass / db.N
    assert 0.01 <= frac <= 0.04, frac


def _gap_forcing(rng, M):
    """Entry only at node 1, node 1 likes residue 0, node M likes residue 1, the
    middle nodes dislike everything: the best alignments must walk D or I states,
    so every transition index of Alg 2 l.15-17 and Lazy-F is exercised."""
    msc = np.full((M, 29), -6.0, np.float32)
    msc[:, 2] = rng.uniform(-2.0, -0.5)
    msc[0, 0] = 4.0
    msc[M - 1, 1] = 4.0
    tsc = np.log(rng.uniform(0.05, 1.0, size=(M, 8))).astype(np.float32)
    tsc[1:, 0] = -np.inf
    tsc[0, 1:4] = -np.inf
    tsc[M - 1, 4:8] = -np.inf
    return msc, tsc


@pytest.mark.parametrize("seed", range(40))
def test_vit_brute_force_gap_paths(seed):
    rng = np.random.default_rng(900 + seed)
    M = int(rng.integers(2, 5))
    msc, tsc = _gap_forcing(rng, M)
    p = oracle.VitProfile(msc, tsc)
    L = int(rng.integers(2, 5 if M < 4 else 4))
    dsq = np.concatenate([[0], rng.integers(0, 3, size=L - 2), [1]]).astype(np.uint8)
    move = -int(rng.integers(100, 4000))
    assert oracle.vit_seq(p, dsq, move=move) == _pins.vit_brute(p.rsc, p.tr, move, dsq)


@pytest.mark.parametrize("seed", range(10))
def test_vit_wide_int_glocal_entry(seed):
    """Entry only at node 1 (tBM = -inf elsewhere): D->D chains decide the score."""
    rng = np.random.default_rng(950 + seed)
    M = int(rng.integers(3, 80))
    prof = synth.make_profile(M, 77 + seed, dd=(1.0, 9.0) if seed % 2 else (7.0, 3.0))
    tsc = prof.tsc.copy()
    tsc[1:, 0] = -np.inf
    p = oracle.VitProfile(prof.msc, tsc)
    dsq = synth.random_dsq(rng, int(rng.integers(2, 150)), alphabet=20)
    move = oracle.move_w(len(dsq))
    want = _pins.vit_wide(p.rsc, p.tr, move, dsq)
    assert oracle.vit_seq(p, dsq) == want == _pins.vit_lazyf(p.rsc, p.tr, move, p.ddbound, dsq)


def test_msv_overflow_boundary():
    """Overflow test of R13 is xE >= 255 - bias: sweep a one-node model across the boundary."""
    hit = set()
    for s100 in range(500, 900):
        s = s100 / 100.0
        msc = np.full((1, 29), -1.0, np.float32)
        msc[0, 0] = 9.24      # canonical max: bias 40
        msc[0, 1] = s
        p = oracle.MSVProfile(msc)
        v = max(0, 190 - oracle.tjb_b(1) - p.tbm)
        cell = max(0, min(255, v + p.bias) - int(p.cost[1, 0]))
        want = 255 if cell >= 255 - p.bias else max(0, cell - 3)
        assert oracle.msv_seq(p, np.array([1], np.uint8)) == want
        hit.add(cell - (255 - p.bias))
    assert 0 in hit and -1 in hit and 1 in hit


@pytest.mark.parametrize("seed", range(10))
def test_vit_long_delete_chain(seed):
    """Node 1 and node M are the only good matches: [0, ..., 1] must cross M-2 deletes
    (D->D chain) or insert; wide-int, Lazy-F and the oracle agree."""
    rng = np.random.default_rng(990 + seed)
    M = int(rng.integers(4, 60))
    msc, tsc = _gap_forcing(rng, M)
    p = oracle.VitProfile(msc, tsc)
    for L in (2, 3, 5):
        dsq = np.concatenate([[0], rng.integers(0, 3, size=L - 2), [1]]).astype(np.uint8)
        move = oracle.move_w(L)
        want = _pins.vit_wide(p.rsc, p.tr, move, dsq)
        assert oracle.vit_seq(p, dsq) == want == _pins.vit_lazyf(p.rsc, p.tr, move, p.ddbound, dsq)


# ------------------------------------------------------------------ Forward (f2)
@pytest.mark.parametrize("seed", range(6))
def test_fwd_brute_force(seed):
    """Forward = log of the sum over every Plan-7 path, enumerated explicitly; includes
    I self-loops, D chains with D->E exits, multihit J and the N/C loops."""
    rng = np.random.default_rng(400 + seed)
    M = int(rng.integers(1, 4))
    msc = rng.uniform(-3.0, 2.5, size=(M, 29)).astype(np.float32)
    msc[:, 20] = -np.inf
    tsc = np.log(rng.uniform(0.05, 0.9, size=(M, 8))).astype(np.float32)
    tsc[0, 1:4] = -np.inf
    tsc[M - 1, 4:8] = -np.inf
    for L in (1, 2, 3, 4):
        d = rng.integers(0, 20, size=L).astype(np.uint8)
        want = _pins.fwd_brute(msc, tsc, d)
        got = oracle.fwd_seq(msc, tsc, d)
        assert got == pytest.approx(want, rel=1e-12, abs=1e-12), (M, L)


def test_fwd_closed_form_one_node():
    """M = 1, L = 1: the only path is N->B->M_1->E->C->T, so
    fwd = 2 log(3/4) + tBM + msc[x] + log(1/2)."""
    msc = np.full((1, 29), -1.0, np.float32)
    msc[0, 7] = 1.25
    tsc = np.full((1, 8), -np.inf, np.float32)
    tsc[0, 0] = np.log(0.3)
    got = oracle.fwd_seq(msc, tsc, np.array([7], np.uint8))
    want = 2 * math.log(0.75) + float(np.float32(np.log(0.3))) + 1.25 + math.log(0.5)
    assert got == pytest.approx(want, rel=1e-12)


def test_fwd_bounds_best_path():
    """A sum of path odds lies between its largest term (the unquantised Viterbi path) and that
    term times the number of paths; the oracle's DP must respect both bounds."""
    rng = np.random.default_rng(9)
    for M in (1, 2, 3):
        msc = rng.uniform(-2.0, 2.0, size=(M, 29)).astype(np.float32)
        tsc = np.log(rng.uniform(0.1, 0.9, size=(M, 8))).astype(np.float32)
        tsc[0, 1:4] = -np.inf
        tsc[M - 1, 4:8] = -np.inf
        d = rng.integers(0, 20, size=4).astype(np.uint8)
        _, best, npath = _pins.fwd_brute(msc, tsc, d, stats=True)
        f = oracle.fwd_seq(msc, tsc, d)
        assert best - 1e-12 <= f <= best + math.log(npath) + 1e-12


# ------------------------------------------------------------------ round-2 pins (VERDICT r01 "What's weak" 1)
_SHAPES_J = [(1, 5), (1, 6), (1, 7), (1, 8), (2, 5), (2, 6), (2, 7), (3, 5), (3, 6), (4, 5)]


def test_msv_brute_force_multisegment_J_reentry():
    """MSV's multiple segments joined through J ("Multiple Segment"; Alg 1 l.20-21):
    one strong residue (+3.5 .. +6 nats at every node, below overflow) lifts xJ above the
    base 190, so a later segment entering from J (xB = max(190, xJ) - tjb) beats one entering
    from N.  Brute force over segment lists must equal the DP, and at least a quarter of the
    cases must be ones where dropping the J entry changes the score (so the pin exercises it)."""
    chained = 0
    for seed in range(40):
        rng = np.random.default_rng(5000 + seed)
        M, L = _SHAPES_J[int(rng.integers(len(_SHAPES_J)))]
        msc = rng.uniform(-3.0, 1.0, size=(M, 29)).astype(np.float32)
        msc[:, 0] = rng.uniform(3.5, 6.0, size=M)
        p = oracle.MSVProfile(msc)
        dsq = rng.choice(3, size=L, p=[0.35, 0.4, 0.25]).astype(np.uint8)
        tjb = int(rng.integers(1, 12))
        want = _pins.msv_brute(p.cost, p.bias, p.tbm, p.tec, tjb, dsq)
        assert oracle.msv_seq(p, dsq, tjb=tjb) == want, seed
        if 190 < want < 255 and want != _pins.msv_brute(p.cost, p.bias, p.tbm, p.tec, tjb, dsq, reenter=False):
            chained += 1
    assert chained >= 10, chained


def test_msv_J_reentry_closed_form():
    """Two isolated one-residue segments (residue 0 scores s at every node, residue 1 is -inf):
    the first gives xJ1 = B1 + bias - c - tec with B1 = 190 - tjb - tbm; the second enters from
    J when xJ1 > 190: xJ2 = (xJ1 - tjb - tbm) + bias - c - tec.  Closed form, Alg 1 l.15/20-21."""
    n = 0
    for s in (4.0, 4.5, 5.0, 5.5, 6.0):
        for tjb in (1, 3, 6):
            msc = np.full((3, 29), -np.inf, np.float32)
            msc[:, 0] = s
            msc[:, 2:20] = -1.0
            p = oracle.MSVProfile(msc)
            c = int(p.cost[0, 0])
            gain = p.bias - c
            x1 = max(0, 190 - tjb - p.tbm + gain - p.tec)
            x2 = max(x1, max(190, x1) - tjb - p.tbm + gain - p.tec)
            if x2 + p.tec >= 255 - p.bias:
                continue                                 # would overflow (R13): not this pin
            dsq = np.array([0, 1, 1, 0], np.uint8)
            assert oracle.msv_seq(p, dsq, tjb=tjb) == x2, (s, tjb)
            n += x1 > 190
    assert n >= 6, n


def test_vit_nats_golden():
    """Viterbi-filter raw -> nats against tests/golden/vit_nats.json (written by
    tests/golden/make_vit_nats.py from the c.3 conversion and Appendix-B constants)."""
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "vit_nats.json")))
    n = 0
    for L, row in g.items():
        if L.startswith("_"):
            continue
        for raw, v in row.items():
            assert abs(oracle.vit_nats(int(raw), int(L)) - v) <= 2e-6 * max(1.0, abs(v)), (L, raw)
            n += 1
    assert n == 9 * 15


def _py_pass(nats, L, mu, lam, F):
    """pass <=> not (P > F), P = Gumbel survival of (nats - null1(L)) / ln 2 (c.4),
    written out in Python doubles: independent of the oracle's C."""
    if nats == math.inf:
        return True, 0.0
    if nats == -math.inf:
        return F >= 1.0, 1.0
    p1 = L / (L + 1.0)
    null1 = L * math.log(p1) + math.log(1.0 - p1)
    bits = (nats - null1) / math.log(2)
    P = -math.expm1(-math.exp(-lam * (bits - mu)))
    return not (P > F), P


def test_vit_pass_direct():
    """The Viterbi pass decision (c.4): Gumbel survival of the Viterbi bits,
    evaluated here from the golden conversion table, over a (raw, L, mu, F) grid."""
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "vit_nats.json")))
    lam = math.log(2)
    seen = set()
    for L, row in g.items():
        if L.startswith("_"):
            continue
        for raw, v in row.items():
            for mu in (-14.0, -11.0, -7.0, 0.0, 6.0):
                for F in (0.02, 1e-3, 0.3):
                    want, P = _py_pass(v, int(L), mu, lam, F)
                    if abs(P - F) <= 1e-4 * F:
                        continue
                    assert oracle.vit_pass(int(raw), int(L), mu, lam, F) == int(want), (L, raw, mu, F)
                    seen.add(want)
    assert seen == {True, False}
    for L in (1, 300, 35213):                          # sentinels (R17)
        assert oracle.vit_pass(32767, L, -11.0, lam, 1e-30) == 1
        assert oracle.vit_pass(-32768, L, -11.0, lam, 0.999) == 0


def test_msv_pass_direct():
    """The MSV pass decision (c.4) from the golden L = 300 conversion values."""
    g = json.load(open(GOLD))
    lam = math.log(2)
    seen = set()
    for raw, v in g["msv_nats_L300"].items():
        for mu in (-12.0, -9.0, -5.0, 0.0):
            for F in (0.02, 1e-3, 0.3):
                want, P = _py_pass(v, 300, mu, lam, F)
                if abs(P - F) <= 0.05 * F:              # golden values carry 2 decimals
                    continue
                assert oracle.msv_pass(int(raw), 300, mu, lam, F) == int(want), (raw, mu, F)
                seen.add(want)
    assert seen == {True, False}
    assert oracle.msv_pass(255, 300, -9.0, lam, 1e-30) == 1
    # F = 1 passes everything (pass <=> not P > F, c.4): the lowest scores reach P == 1.0 exactly
    for raw in (0, 1, 40):
        assert _py_pass(oracle.msv_nats(raw, 300), 300, -9.0, lam, 1.0) == (True, 1.0)
        assert oracle.msv_pass(raw, 300, -9.0, lam, 1.0) == 1
    assert oracle.vit_pass(-32768, 300, -11.0, lam, 1.0) == 1


@pytest.mark.parametrize("M,pseed", [(100, 1100), (400, 1400)])
def test_vit_pass_fraction_near_F2(M, pseed):
    """Statistical pin of the Viterbi stage (0.1% of the DB reaches Forward).
    A Gumbel (mu, lambda) fitted by maximum likelihood to the Viterbi bit scores of 2000
    background sequences of L = 200 predicts the pass fraction of 20 000 Swiss-Prot-shaped
    background sequences (lognormal lengths) at F2 within 2x.  (With lambda
    pinned to ln 2 as P:41-45 states, these synthetic profiles pass 3-5x fewer than F2: their
    Viterbi tail is steeper, lambda ~ 0.88 per bit, reading R25.)"""
    from scipy import stats
    prof = synth.make_profile(M, pseed)
    vp = oracle.VitProfile(prof.msc, prof.tsc)
    cal = synth.Database(np.full(2000, 200, np.int32), seed=7)
    dsq, off = cal.materialize()
    b = np.array([oracle.bits(oracle.vit_nats(int(r), 200), 200) for r in oracle.vit_db(vp, dsq, off)])
    loc, scale = stats.gumbel_r.fit(b)
    db = synth.make_db(20000, 5.6, 0.75, seed=21)
    dsq, off = db.materialize()
    raw = oracle.vit_db(vp, dsq, off)
    for F in (0.02, 0.01):
        frac = np.mean([oracle.vit_pass(int(r), int(L), loc, 1.0 / scale, F) for r, L in zip(raw, db.lengths)])
        assert F / 2 <= frac <= 2 * F, (F, frac, loc, 1.0 / scale)
    # length model (R10, R24): the same thresholds pass similar fractions at L = 50 and 1000
    fr = []
    for L in (50, 1000):
        d = synth.Database(np.full(8000 if L == 50 else 3000, L, np.int32), seed=33)
        dsq, off = d.materialize()
        r = oracle.vit_db(vp, dsq, off)
        fr.append(np.mean([oracle.vit_pass(int(x), L, loc, 1.0 / scale, 0.05) for x in r]))
    assert 0.5 <= fr[0] / fr[1] <= 2.0, fr
