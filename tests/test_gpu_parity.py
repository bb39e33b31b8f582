"""GPU parity: libhmg's CUDA path vs the CPU oracle, bit-exact (raw scores and flags).

Every call goes through the C ABI (paper_conf_ipps_jiangg15_b200.hmg).  Cases
span several tiles and ragged tails: model lengths around every register /
lane-group boundary, sequence lengths 1..7 and around the 6-residue word, the
adversarial profiles (saturating bias, long D->D chains, -inf emissions), and
the BASELINE configurations (config 1 in full; configs 2/3 at full size on a
sample the oracle scores one by one).
"""
import math
import os

import numpy as np
import pytest

import oracle
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _lib():
    if not torch.cuda.is_available():
        pytest.fail("GPU test run without a CUDA device")
    build.build()
    hmg.lib()


def _db_from(dsq_list):
    off = np.zeros(len(dsq_list) + 1, np.int64)
    np.cumsum([len(d) for d in dsq_list], out=off[1:])
    dsq = np.concatenate(dsq_list).astype(np.uint8) if dsq_list else np.zeros(0, np.uint8)
    return dsq, off


def _ragged_db(rng, n=70, alphabet=20, lmax=400):
    lens = list(range(1, 14)) + [17, 18, 19, 23, 24, 25, 35, 36, 37, 95, 96, 97]
    lens += rng.integers(1, lmax, size=max(0, n - len(lens))).tolist()
    return _db_from([synth.random_dsq(rng, int(L), alphabet) for L in lens])


def _msv_gpu(prof_msc, dsq, off, **kw):
    p = hmg.Profile(prof_msc, **kw)
    db = hmg.Database(dsq, off)
    raw = torch.zeros(db.nseq, dtype=torch.uint8, device="cuda")
    hmg.hmg_msv(p, db, raw)
    torch.cuda.synchronize()
    return raw.cpu().numpy().astype(np.int32), p


def _vit_gpu(msc, tsc, dsq, off, ids=None):
    p = hmg.Profile(msc, tsc)
    db = hmg.Database(dsq, off)
    raw = torch.full((db.nseq,), -12345, dtype=torch.int16, device="cuda")
    t_ids = None if ids is None else torch.as_tensor(ids, dtype=torch.int32, device="cuda")
    hmg.hmg_viterbi(p, db, raw, ids=t_ids)
    torch.cuda.synchronize()
    return raw.cpu().numpy().astype(np.int32), p


# ------------------------------------------------------------------ MSV
def test_msv_config1_full():
    prof, db = synth.config(1)
    dsq, off = db.materialize()
    got, _ = _msv_gpu(prof.msc, dsq, off)
    want = oracle.msv_db(oracle.MSVProfile(prof.msc), dsq, off)
    assert np.array_equal(got, want)


MS = [1, 2, 3, 4, 5, 7, 8, 9, 15, 16, 17, 31, 32, 33, 48, 63, 64, 65, 100, 127, 128, 129, 200, 255, 256, 257,
      400, 511, 512, 513, 700, 1000, 1024, 1025, 1528, 2048, 2049, 2405, 2560, 2561, 3000]


@pytest.mark.parametrize("M", MS)
def test_msv_model_lengths(M):
    rng = np.random.default_rng(M)
    prof = synth.make_profile(M, 7000 + M)
    dsq, off = _ragged_db(rng, n=60, alphabet=29)
    got, _ = _msv_gpu(prof.msc, dsq, off)
    want = oracle.msv_db(oracle.MSVProfile(prof.msc), dsq, off)
    assert np.array_equal(got, want)


@pytest.mark.parametrize("G", [4, 8, 16, 32])
@pytest.mark.parametrize("M", [60, 333, 900])
def test_msv_every_lane_group(G, M, tune):
    tune("MSV_G", str(G))
    rng = np.random.default_rng(G * 1000 + M)
    prof = synth.make_profile(M, M + G, stress=True)
    dsq, off = _ragged_db(rng, n=90, alphabet=29)
    got, p = _msv_gpu(prof.msc, dsq, off)
    q = p.quant()
    assert q["msv_lanes"] >= G or q["msv_regs"] == 0
    assert np.array_equal(got, oracle.msv_db(oracle.MSVProfile(prof.msc), dsq, off))


@pytest.mark.parametrize("score", [20.0, 21.5, 22.0, 22.5, 23.0, 30.0, 45.0])
def test_msv_overflow_and_exact_kernel(score):
    """msc = +20 nats: bias 87 < 66 + tbm -> fast kernel, cells saturate -> raw 255 (R13);
    msc >= +30 nats: bias >= 66 + tbm -> the exact kernel (fast-kernel precondition)."""
    rng = np.random.default_rng(1)
    msc = np.full((40, 29), score, np.float32)
    msc[:, 25:] = -np.inf
    msc[::3, 4] = -3.0
    dsq, off = _ragged_db(rng, n=30, alphabet=29)
    got, p = _msv_gpu(msc, dsq, off)
    om = oracle.MSVProfile(msc)
    assert p.quant()["msv_fast"] == int(om.bias < 66 + om.tbm)     # 20 -> fast, 23+ -> exact
    assert np.array_equal(got, oracle.msv_db(om, dsq, off))
    assert (got == 255).sum() > 0


def test_msv_high_scores_fast_path():
    """Strong hits: planted homologs and a high-scoring profile drive the J->B update
    (vote fires) and the in-kernel overflow test of the fast kernel."""
    rng = np.random.default_rng(3)
    prof = synth.make_profile(150, 99)
    msc = prof.msc.copy()
    msc[:, :20] *= 1.9          # higher bias, still fast
    p_or = oracle.MSVProfile(msc)
    seqs = []
    for i in range(80):
        L = int(rng.integers(20, 600))
        d = synth.random_dsq(rng, L)
        seg = np.argmax(msc[:, :20], axis=1)[: min(L, 150 - (i % 40))].astype(np.uint8)
        a = int(rng.integers(0, L - len(seg) + 1))
        if i % 3:
            d[a:a + len(seg)] = seg
        seqs.append(d)
    dsq, off = _db_from(seqs)
    got, p = _msv_gpu(msc, dsq, off)
    assert p.quant()["msv_fast"] == 1
    want = oracle.msv_db(p_or, dsq, off)
    assert np.array_equal(got, want)
    assert (want == 255).sum() > 0 and (want >= 190).sum() > 0


@pytest.mark.parametrize("M,G", [(400, 8), (100, 8), (200, 16), (60, 16), (200, 8), (512, 16), (256, 8)])
@pytest.mark.parametrize("top", [8.0, 10.0, 10.6, 10.9, 11.2, 13.0])
def test_msv_int8_remainder_bound(M, G, top, tune):
    """Lane geometries with int8 emissions (G = 8 / 16 with a 2-register remainder, Q % 4 in {2, 3})
    and without (M = 256 / 400 / 512 fill 2GQ = M exactly, so node M's cell is the carry the running
    max takes): raising the profile's top score moves 3 + tjb(Lmax) + tbm + bias across 128 -- below it
    the fast kernel with the clamped int8 chunk, above it the exact kernel -- with planted hits so the
    J->B re-entry and overflow paths run on both sides (tjb(~3000) = 30: at M = 400, tbm = 49, the
    bound is bias <= 46, i.e. top <= 10.6 nats; at M = 200 top <= 12).  Bit-exact against the oracle."""
    tune("MSV_G", str(G))
    rng = np.random.default_rng(int(M * 10 + top * 7))
    prof = synth.make_profile(M, 4000 + M, stress=True)
    msc = prof.msc.copy()
    best = np.argmax(msc[:, :20], axis=1)
    msc[np.arange(M), best] = np.maximum(msc[np.arange(M), best], 2.0)
    msc[M // 3, best[M // 3]] = top                     # sets the bias byte
    seqs = []
    for i in range(120):
        L = int(rng.integers(1, 900)) if i % 10 else int(rng.integers(2000, 3100))
        d = synth.random_dsq(rng, L, 29 if i % 7 == 0 else 20)
        if i % 4 == 0 and L > 8:
            seg = best[: min(L, M)].astype(np.uint8)[: int(rng.integers(3, min(L, M) + 1))]
            a = int(rng.integers(0, L - len(seg) + 1))
            d[a:a + len(seg)] = seg
        seqs.append(d)
    dsq, off = _db_from(seqs)
    got, p = _msv_gpu(msc, dsq, off)
    q = p.quant()
    assert q["msv_lanes"] == G
    om = oracle.MSVProfile(msc)
    want = oracle.msv_db(om, dsq, off)
    assert np.array_equal(got, want)
    assert (want >= 190).sum() > 0                             # hits chain through J


def test_msv_all_minus_inf_redo_path():
    """Gap-only sequences: every cell <= B', the fast kernel defers to the exact kernel."""
    prof = synth.make_profile(77, 5)
    seqs = [np.full(L, 20, np.uint8) for L in (1, 2, 6, 7, 50)] + [np.array([27, 28, 20], np.uint8)]
    dsq, off = _db_from(seqs)
    got, _ = _msv_gpu(prof.msc, dsq, off)
    assert np.array_equal(got, oracle.msv_db(oracle.MSVProfile(prof.msc), dsq, off))


def test_empty_db():
    prof = synth.make_profile(10, 1)
    p = hmg.Profile(prof.msc, prof.tsc, ev=(-9, math.log(2), -9, math.log(2)))
    db = hmg.Database(np.zeros(0, np.uint8), np.zeros(1, np.int64))
    out = hmg.alloc_outputs(0)
    hmg.hmg_pipeline(p, db, **out)
    torch.cuda.synchronize()
    assert int(out["n_survivors"].item()) == 0


# ------------------------------------------------------------------ Viterbi
def test_vit_config1_full():
    prof, db = synth.config(1)
    dsq, off = db.materialize()
    got, _ = _vit_gpu(prof.msc, prof.tsc, dsq, off)
    want = oracle.vit_db(oracle.VitProfile(prof.msc, prof.tsc), dsq, off)
    assert np.array_equal(got, want)


VMS = [1, 2, 3, 4, 5, 8, 9, 16, 17, 31, 32, 33, 63, 64, 65, 100, 127, 128, 129, 200, 255, 256, 257, 400, 511,
       512, 513, 1000, 2048]


@pytest.mark.parametrize("M", VMS)
@pytest.mark.parametrize("dd", [(7.0, 3.0), (1.0, 9.0)])
@pytest.mark.parametrize("pair", [True, False])
def test_vit_model_lengths(M, dd, pair, tune):
    """pair: the s16x2 pair kernel (+ s32 re-scoring of what leaves its window); otherwise the
    s32 kernels alone (tuning NO_VIT_PAIR)."""
    if not pair:
        tune("NO_VIT_PAIR", "1")
    rng = np.random.default_rng(M + int(dd[0]))
    prof = synth.make_profile(M, 8000 + M, dd=dd)
    n = 40 if M <= 600 else 12
    dsq, off = _ragged_db(rng, n=n, alphabet=29, lmax=300)
    got, _ = _vit_gpu(prof.msc, prof.tsc, dsq, off)
    assert np.array_equal(got, oracle.vit_db(oracle.VitProfile(prof.msc, prof.tsc), dsq, off))


@pytest.mark.parametrize("M", [3, 20, 64, 130, 300, 500, 700])
def test_vit_long_delete_chains(M):
    """Entry only at node 1, good matches only at nodes 1 and M: the score depends on
    D->D chains that cross every lane boundary (Lazy-F carries, Fig 7)."""
    rng = np.random.default_rng(M)
    msc = np.full((M, 29), -6.0, np.float32)
    msc[0, 0] = 4.0
    msc[M - 1, 1] = 4.0
    tsc = np.log(rng.uniform(0.05, 1.0, size=(M, 8))).astype(np.float32)
    tsc[:, 7] = np.log(rng.uniform(0.8, 0.999, size=M))
    tsc[1:, 0] = -np.inf
    tsc[0, 1:4] = -np.inf
    tsc[M - 1, 4:8] = -np.inf
    seqs = [np.array([0, 1], np.uint8), np.array([0, 2, 1], np.uint8), np.array([0, 1, 0, 1], np.uint8)]
    seqs += [synth.random_dsq(rng, int(L), 3) for L in rng.integers(1, 60, size=30)]
    dsq, off = _db_from(seqs)
    got, _ = _vit_gpu(msc, tsc, dsq, off)
    assert np.array_equal(got, oracle.vit_db(oracle.VitProfile(msc, tsc), dsq, off))


@pytest.mark.parametrize("pair", [True, False])
def test_vit_long_delete_chains_s32(pair, tune):
    """The delete-chain profiles above have -inf entry below node 1, so the pair kernel does not
    apply; here entry is finite everywhere but weak, so the pair kernel's Lazy-F (carries through
    both halves of every register, lane G-1 low -> lane 0 high) decides the score."""
    if not pair:
        tune("NO_VIT_PAIR", "1")
    for M in (3, 20, 64, 130, 300, 500, 700, 1000):
        rng = np.random.default_rng(M + 17)
        msc = np.full((M, 29), -6.0, np.float32)
        msc[0, 0] = 4.0
        msc[M - 1, 1] = 4.0
        msc[M // 2, 2] = 3.0
        tsc = np.log(rng.uniform(0.05, 1.0, size=(M, 8))).astype(np.float32)
        tsc[:, 7] = np.log(rng.uniform(0.8, 0.999, size=M))
        tsc[:, 0] = np.log(1e-4 / M)
        tsc[0, 0] = np.log(0.5)
        tsc[0, 1:4] = -np.inf
        tsc[M - 1, 4:8] = -np.inf
        seqs = [np.array([0, 1], np.uint8), np.array([0, 2, 1], np.uint8), np.array([0, 1, 0, 1], np.uint8)]
        seqs += [synth.random_dsq(rng, int(L), 3) for L in rng.integers(1, 60, size=30)]
        dsq, off = _db_from(seqs)
        got, p = _vit_gpu(msc, tsc, dsq, off)
        assert (p.quant()["vit_pair_lanes"] > 0) == (pair and M <= 1024), M
        assert np.array_equal(got, oracle.vit_db(oracle.VitProfile(msc, tsc), dsq, off)), M


@pytest.mark.parametrize("G", [8, 16, 32])
@pytest.mark.parametrize("M", [10, 100, 257, 600])
def test_vit_pair_every_lane_group(G, M, tune):
    tune("VIT_PAIR_G", str(G))
    rng = np.random.default_rng(G + M)
    prof = synth.make_profile(M, 300 + M + G, dd=(1.0, 9.0))
    dsq, off = _ragged_db(rng, n=70, alphabet=29, lmax=350)
    got, p = _vit_gpu(prof.msc, prof.tsc, dsq, off)
    q = p.quant()
    assert q["vit_pair_lanes"] >= G and 2 * q["vit_pair_lanes"] * q["vit_pair_regs"] >= M
    assert np.array_equal(got, oracle.vit_db(oracle.VitProfile(prof.msc, prof.tsc), dsq, off))


def test_vit_pair_window_exits():
    """Sequences the pair kernel hands to the s32 kernel: strong planted hits (cells above the
    16-bit window), overflow, gap-only sequences (every row floored); and long sequences whose
    floor F is low.  Scores stay bit-exact and some sequences are re-scored."""
    rng = np.random.default_rng(8)
    M = 180
    prof = synth.make_profile(M, 818)
    msc = prof.msc.copy()
    best = np.argmax(msc[:, :20], axis=1).astype(np.uint8)
    seqs = []
    for i in range(120):
        L = int(rng.integers(5, 900)) if i % 10 else int(rng.integers(3000, 9000))
        d = synth.random_dsq(rng, L)
        if i % 4 == 0:                         # best-path prefixes: below, inside and above the window
            seg = best[: min(L, int(rng.integers(5, M + 1)))]
            a = int(rng.integers(0, L - len(seg) + 1))
            d[a:a + len(seg)] = seg
        seqs.append(d)
    seqs += [np.full(L, 20, np.uint8) for L in (1, 5, 40)] + [np.array([27, 28, 20, 27], np.uint8)]
    dsq, off = _db_from(seqs)
    hmg.hmg_set_stage_timing(True)
    try:
        got, p = _vit_gpu(msc, prof.tsc, dsq, off)
        redo = hmg.hmg_stage_counts()["vit_pair_redo"]
    finally:
        hmg.hmg_set_stage_timing(False)
    want = oracle.vit_db(oracle.VitProfile(msc, prof.tsc), dsq, off)
    assert p.quant()["vit_pair_lanes"] > 0
    assert np.array_equal(got, want)
    assert (want == 32767).sum() > 0 and redo >= 4


def test_vit_overflow_and_minus_inf():
    rng = np.random.default_rng(4)
    M = 50
    msc = np.full((M, 29), 60.0, np.float32)
    msc[:, 10:] = -np.inf
    tsc = np.full((M, 8), np.log(0.3), np.float32)
    tsc[0, 1:4] = -np.inf
    tsc[-1, 4:] = -np.inf
    dsq, off = _ragged_db(rng, n=30, alphabet=29, lmax=100)
    got, _ = _vit_gpu(msc, tsc, dsq, off)
    want = oracle.vit_db(oracle.VitProfile(msc, tsc), dsq, off)
    assert np.array_equal(got, want)
    assert (want == 32767).any() and (want < 0).any()


def test_vit_ids_subset_untouched_elsewhere():
    prof, db = synth.config(1)
    dsq, off = db.materialize()
    ids = np.array([5, 3, 3, 999, 0, 512], np.int32)
    got, _ = _vit_gpu(prof.msc, prof.tsc, dsq, off, ids=ids)
    want = oracle.vit_db(oracle.VitProfile(prof.msc, prof.tsc), dsq, off, ids=ids)
    assert np.array_equal(got[ids], want)
    mask = np.ones(len(got), bool)
    mask[ids] = False
    assert (got[mask] == -12345).all()


# ------------------------------------------------------------------ pipeline + flags
def _calibrate(prof):
    """mu for lambda = ln 2 fitted by the ORACLE on 1000 background sequences of L = 200."""
    cal = synth.Database(np.full(1000, 200, np.int32), seed=7)
    dsq, off = cal.materialize()
    mp, vp = oracle.MSVProfile(prof.msc), oracle.VitProfile(prof.msc, prof.tsc)
    lam = math.log(2)
    mb = [oracle.bits(oracle.msv_nats(int(r), 200), 200) for r in oracle.msv_db(mp, dsq, off)]
    vb = [oracle.bits(oracle.vit_nats(int(r), 200), 200) for r in oracle.vit_db(vp, dsq, off)]
    return (oracle.fit_mu(np.array(mb), lam), lam, oracle.fit_mu(np.array(vb), lam), lam)


@pytest.mark.parametrize("M", [64, 200, 700])
def test_calibrate_matches_oracle_fit(M):
    """hmg_calibrate (library RNG, GPU scoring) vs the oracle's fit on other background
    sequences: the ML location for known lambda has SD ~ 1/(lambda sqrt(n)) = 0.046 bits at
    n = 1000, so two independent fits agree within 0.3 bits (> 4.5 SD of the difference)."""
    prof = synth.make_profile(M, 100 + M)
    p = hmg.Profile(prof.msc, prof.tsc)
    mu_m, lam_m, mu_v, lam_v = p.calibrate(n=1000, L=200, seed=11)
    want = _calibrate(prof)
    assert lam_m == lam_v == pytest.approx(math.log(2))
    assert abs(mu_m - want[0]) < 0.3 and abs(mu_v - want[2]) < 0.3
    # deterministic in the seed
    assert p.calibrate(n=1000, L=200, seed=11) == (mu_m, lam_m, mu_v, lam_v)


@pytest.mark.parametrize("M,lens", [(64, "fixed"), (400, "fixed"), (1500, "mixed")])
def test_calibrate_db_equals_oracle_fit(M, lens):
    """SURVEY 8(f) f3 parity: hmg_calibrate_db on a background DB vs the oracle's fit of the SAME
    sequences (oracle raw scores -> nats -> bits with each sequence's null1 -> closed-form ML
    location for lambda = ln 2).  The raw scores are bit-exact, so the two fits differ
    only in the order of a double sum: 1e-9 relative."""
    prof = synth.make_profile(M, 300 + M)
    if lens == "fixed":
        cal = synth.Database(np.full(1000, 200, np.int32), seed=7)
    else:
        cal = synth.make_db(1500, 5.4, 0.7, seed=19)
    dsq, off = cal.materialize()
    p = hmg.Profile(prof.msc, prof.tsc)
    db = hmg.Database(dsq, off)
    mu_m, lam_m, mu_v, lam_v = p.calibrate_db(db)
    L = np.diff(off)
    mraw = oracle.msv_db(oracle.MSVProfile(prof.msc), dsq, off)
    vraw = oracle.vit_db(oracle.VitProfile(prof.msc, prof.tsc), dsq, off)
    mb = np.array([oracle.bits(oracle.msv_nats(int(r), int(l)), int(l)) for r, l in zip(mraw, L)])
    vb = np.array([oracle.bits(oracle.vit_nats(int(r), int(l)), int(l)) for r, l in zip(vraw, L)])
    lam = math.log(2)
    want_m = oracle.fit_mu(mb[np.isfinite(mb)], lam)
    want_v = oracle.fit_mu(vb[np.isfinite(vb)], lam)
    assert lam_m == lam_v == pytest.approx(lam)
    assert mu_m == pytest.approx(want_m, rel=1e-9, abs=1e-9)
    assert mu_v == pytest.approx(want_v, rel=1e-9, abs=1e-9)


def _check_pipeline(prof, dsq, off, F1, F2, sample=None):
    ev = _calibrate(prof)
    p = hmg.Profile(prof.msc, prof.tsc, ev=ev)
    db = hmg.Database(dsq, off)
    out = hmg.alloc_outputs(db.nseq)
    hmg.hmg_pipeline(p, db, F1=F1, F2=F2, **out)
    torch.cuda.synchronize()
    mraw = out["msv_raw"].cpu().numpy().astype(np.int32)
    vraw = out["vit_raw"].cpu().numpy().astype(np.int32)
    flags = out["flags"].cpu().numpy()
    ns = int(out["n_survivors"].item())
    surv = out["survivor_ids"].cpu().numpy()[:ns]
    lens = np.diff(off)
    mp, vp = oracle.MSVProfile(prof.msc), oracle.VitProfile(prof.msc, prof.tsc)
    idx = np.arange(db.nseq) if sample is None else np.asarray(sample)
    want_m = oracle.msv_db(mp, dsq, off, ids=idx)
    assert np.array_equal(mraw[idx], want_m)
    want_pass = np.array([oracle.msv_pass(int(r), int(lens[s]), ev[0], ev[1], F1) for r, s in zip(want_m, idx)])
    assert np.array_equal(flags[idx] & 1, want_pass)
    # survivors: exactly the MSV-passing sequences, length-descending, stable (caller order on ties)
    passing = np.nonzero(flags & 1)[0]
    assert sorted(surv.tolist()) == passing.tolist()
    order = np.lexsort((np.arange(db.nseq), -lens))
    assert surv.tolist() == [s for s in order if flags[s] & 1]
    # Viterbi ran on every survivor and only there
    assert np.array_equal((flags >> 2) & 1, flags & 1)
    assert (vraw[flags & 1 == 0] == -32768).all()
    vs = surv if sample is None else np.intersect1d(surv, idx)
    want_v = oracle.vit_db(vp, dsq, off, ids=vs)
    assert np.array_equal(vraw[vs], want_v)
    want_vp = np.array([oracle.vit_pass(int(r), int(lens[s]), ev[2], ev[3], F2) for r, s in zip(want_v, vs)])
    assert np.array_equal((flags[vs] >> 1) & 1, want_vp.astype(np.uint8))
    return ns


def test_pipeline_config1():
    prof, db = synth.config(1)
    dsq, off = db.materialize()
    ns = _check_pipeline(prof, dsq, off, F1=0.02, F2=1e-3)
    assert 0 < ns < 200


def test_pipeline_loose_thresholds():
    """F1 = 0.5 sends about half the DB to the Viterbi stage; F = 1 passes everything."""
    prof, db = synth.config(1)
    dsq, off = db.materialize()
    ns = _check_pipeline(prof, dsq, off, F1=0.5, F2=0.5)
    assert ns > 300
    assert _check_pipeline(prof, dsq, off, F1=1.0, F2=1.0) == db.N


def test_pipeline_config3_full_size_sampled():
    """BASELINE config 3 at full size (550k sequences, M=400, planted homologs) in the
    bench launch configuration; the oracle checks a length-stratified sample plus
    every survivor in it."""
    prof, db = synth.config(3)
    dsq, off = db.materialize()
    rng = np.random.default_rng(0)
    sample = np.unique(np.concatenate([rng.choice(db.N, 3000, replace=False), db.planted_ids,
                                       np.argsort(-db.lengths)[:50]]))
    _check_pipeline(prof, dsq, off, F1=0.02, F2=1e-3, sample=sample)


def test_msv_config2_full_size_sampled():
    prof, db = synth.config(2)
    dsq, off = db.materialize()
    got, _ = _msv_gpu(prof.msc, dsq, off)
    rng = np.random.default_rng(1)
    sample = np.unique(np.concatenate([rng.choice(db.N, 4000, replace=False), np.argsort(-db.lengths)[:40],
                                       np.argsort(db.lengths)[:40]]))
    want = oracle.msv_db(oracle.MSVProfile(prof.msc), dsq, off, ids=sample)
    assert np.array_equal(got[sample], want)


def _stratified(lengths, n, rng):
    """n sequence ids spread over the length distribution (equal counts per length decile)."""
    order = np.argsort(lengths, kind="stable")
    parts = np.array_split(order, 10)
    return np.unique(np.concatenate([rng.choice(pp, n // 10, replace=False) for pp in parts]))


@pytest.mark.parametrize("kernel", ["wide_tm", "cpair2"])
def test_viterbi_config4_full_size_sampled(kernel, tune):
    """BASELINE config 4 at full size in the bench launch configuration: the Viterbi filter
    (Lazy-F) over every one of the 550k Swiss-Prot-shaped sequences at M = 2048 (M up
    to 2405 P:816-818), with the bench's kernel (one warp per sequence, transitions in tensor
    memory) and the two-warp one.  The oracle checks a 2k length-stratified sample, the 50 longest
    sequences (L up to 35,213) and the pass flags there; planted homologs (strong hits that re-base
    the 16-bit window) are checked on a second 20k-sequence DB."""
    if kernel == "cpair2":
        tune("VIT_WIDE", 0)
    c = synth.CONFIGS[4]
    prof = synth.make_profile(c["M"], c["pseed"])
    db = synth.make_db(c["N"], c["mu_ln"], c["sigma"], c["dseed"])
    dsq, off = db.materialize()
    ev = _calibrate(prof)
    p = hmg.Profile(prof.msc, prof.tsc, ev=ev)
    assert p.quant()["vit_pair_kernel"] == (5 if kernel == "wide_tm" else 3)
    D = hmg.Database(dsq, off)
    raw = torch.full((D.nseq,), -12345, dtype=torch.int16, device="cuda")
    pas = torch.zeros(D.nseq, dtype=torch.uint8, device="cuda")
    hmg.hmg_viterbi(p, D, raw, pass_=pas, F2=1e-3)
    torch.cuda.synchronize()
    got = raw.cpu().numpy().astype(np.int32)
    gp = pas.cpu().numpy()
    assert (got != -12345).all()
    rng = np.random.default_rng(4)
    sample = np.unique(np.concatenate([_stratified(db.lengths, 2000, rng), np.argsort(-db.lengths)[:50]]))
    assert db.lengths[sample].max() > 30000
    vp = oracle.VitProfile(prof.msc, prof.tsc)
    want = oracle.vit_db(vp, dsq, off, ids=sample)
    assert np.array_equal(got[sample], want)
    wp = [oracle.vit_pass(int(r), int(db.lengths[s]), ev[2], ev[3], 1e-3) for r, s in zip(want, sample)]
    assert np.array_equal(gp[sample], np.array(wp, np.uint8))
    # planted homologs: strong hits
    db2 = synth.make_db(20000, c["mu_ln"], c["sigma"], 44, planted=0.01, profile=prof)
    dsq2, off2 = db2.materialize()
    D2 = hmg.Database(dsq2, off2)
    raw2 = torch.zeros(D2.nseq, dtype=torch.int16, device="cuda")
    hmg.hmg_viterbi(p, D2, raw2)
    torch.cuda.synchronize()
    ids = np.unique(np.concatenate([db2.planted_ids, rng.choice(db2.N, 300, replace=False)]))
    w2 = oracle.vit_db(vp, dsq2, off2, ids=ids)
    assert np.array_equal(raw2.cpu().numpy().astype(np.int32)[ids], w2)
    assert (w2[np.isin(ids, db2.planted_ids)] > 10000).mean() > 0.5     # they are hits


@pytest.mark.parametrize("which", [0, 1, 2])
def test_pipeline_config5_shard_full_size_sampled(which):
    """BASELINE config 5 as one rank of the 8-way run holds it: the 1/8 snake shard (1.25 M
    sequences) of the 10 M-sequence UniProt-shaped DB at M = 100 / 500 / 1000, the pipeline in the
    bench launch configuration; the oracle checks a 3k length-stratified sample, the 40 longest and
    every survivor among them (_check_pipeline) plus 2000 random survivors' Viterbi scores."""
    from paper_conf_ipps_jiangg15_b200 import dist as hdist
    c = synth.CONFIGS[5]
    prof = synth.make_profile(c["M"][which], c["pseed"][which])
    db = synth.make_db(c["N"], c["mu_ln"], c["sigma"], c["dseed"])
    ids = hdist.snake_shard(db.lengths, 8, 0)
    dsq, off = db.materialize(ids)
    L = np.diff(off)
    rng = np.random.default_rng(50 + which)
    sample = np.unique(np.concatenate([_stratified(L, 3000, rng), np.argsort(-L)[:40]]))
    _check_pipeline(prof, dsq, off, F1=0.02, F2=1e-3, sample=sample)
    ev = _calibrate(prof)
    p = hmg.Profile(prof.msc, prof.tsc, ev=ev)
    D = hmg.Database(dsq, off)
    out = hmg.alloc_outputs(D.nseq)
    hmg.hmg_pipeline(p, D, F1=0.02, F2=1e-3, **out)
    torch.cuda.synchronize()
    ns = int(out["n_survivors"].item())
    surv = out["survivor_ids"].cpu().numpy()[:ns]
    pick = rng.choice(surv, min(2000, ns), replace=False)
    want = oracle.vit_db(oracle.VitProfile(prof.msc, prof.tsc), dsq, off, ids=pick)
    assert np.array_equal(out["vit_raw"].cpu().numpy().astype(np.int32)[pick], want)


@pytest.mark.parametrize("M", [2, 3, 64, 255, 300, 513, 700, 1024, 1025, 1500, 2048, 2600, 4000])
@pytest.mark.parametrize("dd", [(7.0, 3.0), (1.0, 9.0)])
def test_vit_block_kernel(M, dd, tune):
    """Block-per-sequence Viterbi (W warps per row, cross-warp Lazy-F through shared memory);
    forced for small M with tuning VIT_CTA, used by default above M = 512."""
    tune("VIT_CTA", "1")
    tune("NO_VIT_PAIR", "1")
    rng = np.random.default_rng(M * 3 + int(dd[1]))
    prof = synth.make_profile(M, 9000 + M, dd=dd)
    n = 30 if M <= 1100 else 10
    dsq, off = _ragged_db(rng, n=n, alphabet=29, lmax=250)
    got, p = _vit_gpu(prof.msc, prof.tsc, dsq, off)
    q = p.quant()
    assert q["vit_lanes"] >= 256 or M > 3072       # beyond: general kernel (table > 227 KB)
    assert np.array_equal(got, oracle.vit_db(oracle.VitProfile(prof.msc, prof.tsc), dsq, off))


@pytest.mark.parametrize("M", [40, 300, 700, 2000])
def test_vit_block_kernel_delete_chains(M, tune):
    """D->D chains that cross every warp boundary of the block (cross-warp Lazy-F rounds)."""
    tune("VIT_CTA", "1")
    tune("NO_VIT_PAIR", "1")
    rng = np.random.default_rng(M + 5)
    msc = np.full((M, 29), -6.0, np.float32)
    msc[0, 0] = 4.0
    msc[M - 1, 1] = 4.0
    msc[M // 2, 2] = 3.0
    tsc = np.log(rng.uniform(0.05, 1.0, size=(M, 8))).astype(np.float32)
    tsc[:, 7] = np.log(rng.uniform(0.9, 0.9999, size=M))
    tsc[1:, 0] = -np.inf
    tsc[0, 1:4] = -np.inf
    tsc[M - 1, 4:8] = -np.inf
    seqs = [np.array([0, 1], np.uint8), np.array([0, 2, 1], np.uint8), np.array([0, 1, 0, 2, 1], np.uint8)]
    seqs += [synth.random_dsq(rng, int(L), 3) for L in rng.integers(1, 40, size=12)]
    dsq, off = _db_from(seqs)
    got, _ = _vit_gpu(msc, tsc, dsq, off)
    assert np.array_equal(got, oracle.vit_db(oracle.VitProfile(msc, tsc), dsq, off))


@pytest.mark.parametrize("chunk,sms,M,lane", [(1032, "0", 120, "s32"), (60, "0", 120, "s32"),
                                               (1032, "0", 100, "pair"), (60, "2", 64, "pair"),
                                               (1032, "2", 120, "s32"), (1032, "0", 300, "pair"),
                                               (60, "3", 300, "s32"), (1032, "0", 700, "pair"),
                                               (200, "2", 1000, "pair")])
def test_pipeline_long_lane(chunk, sms, M, lane, tune):
    """The pipeline long lane: sequences longer than max(1500, 8 x mean) get chunked MSV (rows
    from the empty state M rows early) and whole-warp Viterbi on SMs held alone (the s32 latency
    lane, or the s16x2 pair lane for models of 129..1024 nodes).  Strong planted hits in some
    long sequences force the sequential fallback (a chunk sees a J->B row).  Models of <= 128
    nodes ("pair" at M = 64 / 100) run the pair lane on tables of their own (G = 32)."""
    tune("PIPE_CHUNK", str(chunk))
    if sms != "0":
        tune("PIPE_LONG_SMS", sms)
    if lane == "s32":
        tune("LONG_S32", "1")
    rng = np.random.default_rng(42)
    prof = synth.make_profile(M, 4242 + M)
    best = np.argmax(prof.msc[:, :20], axis=1).astype(np.uint8)
    seqs = []
    for i in range(300):
        L = int(rng.integers(1600, 7000)) if i < 40 else int(rng.integers(20, 400))
        d = synth.random_dsq(rng, L, 20)
        if i % 5 == 0:                      # plant a strong hit somewhere
            seg = best[: min(len(best), L)]
            a = int(rng.integers(0, L - len(seg) + 1))
            d[a:a + len(seg)] = seg
        seqs.append(d)
    dsq, off = _db_from(seqs)
    ns = _check_pipeline(prof, dsq, off, F1=0.02, F2=1e-3)
    assert ns >= 10


@pytest.mark.parametrize("M", [130, 300, 451, 641, 1000])
def test_pipeline_many_survivors(M):
    """Pipeline with the pair Viterbi kernel at every MSV lane-group geometry: loose F1 sends many
    sequences to the Viterbi stage; planted hits and gap-only sequences take the overflow /
    re-score paths."""
    rng = np.random.default_rng(M + 77)
    prof = synth.make_profile(M, 5000 + M)
    best = np.argmax(prof.msc[:, :20], axis=1).astype(np.uint8)
    seqs = []
    for i in range(700):
        L = int(rng.integers(1, 900))
        d = synth.random_dsq(rng, L, 20)
        if i % 37 == 0:
            seg = best[: min(L, int(rng.integers(5, M + 1)))]
            a = int(rng.integers(0, L - len(seg) + 1))
            d[a:a + len(seg)] = seg
        seqs.append(d)
    seqs += [np.full(L, 20, np.uint8) for L in (3, 60)]
    dsq, off = _db_from(seqs)
    ns = _check_pipeline(prof, dsq, off, F1=0.3, F2=0.05)
    assert ns > 100


@pytest.mark.parametrize("M", [2, 3, 64, 300, 513, 1024, 1025, 1500, 2048, 2600, 4000])
@pytest.mark.parametrize("W", [2, 4, 8, 16, "2b", "2t", "wide", "wide_tm"])
def test_vit_block_pair_kernel(M, W, tune):
    """Block-per-sequence pair kernel (W warps per row, 2 cells per register, closed-form carries
    across virtual warps); forced for small M with tuning VIT_PAIR_CTA, used by default above 1024.
    W = 2 runs the kernel without a per-row barrier (vit_cpair2.cuh); "2b" the barrier kernel;
    "2t" the barrier-free kernel with four transition vectors in shared memory (3 sequences/block);
    "wide" / "wide_tm" one warp per sequence with the transitions in shared / tensor memory
    (vit_wide.cuh, the default above 1024 nodes)."""
    tune("VIT_PAIR_CTA", "1")
    if W in ("2b", "2t"):
        tune("VIT_CPAIR2", "0" if W == "2b" else "23")
        W = 2
    if W in ("wide", "wide_tm"):                     # one warp, transitions in shared / tensor memory (vit_wide.cuh)
        tune("VIT_WIDE", 1 if W == "wide" else 2)
        W = 1
    else:
        tune("VIT_WIDE", 0)
    tune("VIT_PAIR_W", str(W))
    rng = np.random.default_rng(M * 7 + W)
    for dd in [(7.0, 3.0), (1.0, 9.0)]:
        prof = synth.make_profile(M, 9100 + M + W, dd=dd)
        n = 24 if M <= 1100 else 8
        dsq, off = _ragged_db(rng, n=n, alphabet=29, lmax=250)
        got, p = _vit_gpu(prof.msc, prof.tsc, dsq, off)
        q = p.quant()
        assert q["vit_pair_lanes"] >= 32 * W and 2 * q["vit_pair_lanes"] * q["vit_pair_regs"] >= M
        assert np.array_equal(got, oracle.vit_db(oracle.VitProfile(prof.msc, prof.tsc), dsq, off)), dd


@pytest.mark.parametrize("W", [2, 4, 8, 16, "2b", "2t", "wide", "wide_tm"])
def test_vit_block_pair_delete_chains_and_exits(W, tune):
    """D->D chains across every virtual-warp boundary (low halves -> high halves), strong hits that
    re-base the window or overflow, and gap-only sequences handed to the s32 kernel."""
    tune("VIT_PAIR_CTA", "1")
    if W in ("2b", "2t"):
        tune("VIT_CPAIR2", "0" if W == "2b" else "23")
        W = 2
    if W in ("wide", "wide_tm"):                     # one warp, transitions in shared / tensor memory (vit_wide.cuh)
        tune("VIT_WIDE", 1 if W == "wide" else 2)
        W = 1
    else:
        tune("VIT_WIDE", 0)
    tune("VIT_PAIR_W", str(W))
    for M in (40, 700, 2000):
        rng = np.random.default_rng(M + W)
        msc = np.full((M, 29), -6.0, np.float32)
        msc[0, 0] = 4.0
        msc[M - 1, 1] = 4.0
        msc[M // 2, 2] = 3.0
        msc[:, 3] = 2.5                              # residue 3 scores everywhere: strong hits
        tsc = np.log(rng.uniform(0.05, 1.0, size=(M, 8))).astype(np.float32)
        tsc[:, 7] = np.log(rng.uniform(0.9, 0.9999, size=M))
        tsc[:, 0] = np.log(1e-4 / M)
        tsc[0, 0] = np.log(0.5)
        tsc[0, 1:4] = -np.inf
        tsc[M - 1, 4:8] = -np.inf
        seqs = [np.array([0, 1], np.uint8), np.array([0, 2, 1], np.uint8), np.array([0, 1, 0, 2, 1], np.uint8)]
        seqs += [synth.random_dsq(rng, int(L), 3) for L in rng.integers(1, 40, size=12)]
        seqs += [np.full(L, 3, np.uint8) for L in (5, 30, 200)] + [np.full(7, 20, np.uint8)]
        dsq, off = _db_from(seqs)
        got, p = _vit_gpu(msc, tsc, dsq, off)
        assert p.quant()["vit_pair_lanes"] >= 32 * W
        want = oracle.vit_db(oracle.VitProfile(msc, tsc), dsq, off)
        assert np.array_equal(got, want), M


@pytest.mark.parametrize("M", [129, 300, 700, 1000])
def test_vit_pair_maxplus_scan(M, tune):
    """the cross-lane D->D carries of the pair kernel resolved by one max-plus
    prefix scan (tuning VIT_SCAN) instead of vote-terminated passes: identical raw scores on the
    typical and the long-D-chain (Dir(1, 9)) profiles and on chains crossing every lane."""
    tune("VIT_SCAN", "1")
    rng = np.random.default_rng(M + 31)
    for dd in [(7.0, 3.0), (1.0, 9.0)]:
        prof = synth.make_profile(M, 600 + M, dd=dd)
        dsq, off = _ragged_db(rng, n=40, alphabet=29, lmax=300)
        got, p = _vit_gpu(prof.msc, prof.tsc, dsq, off)
        assert p.quant()["vit_pair_lanes"] == 32
        assert np.array_equal(got, oracle.vit_db(oracle.VitProfile(prof.msc, prof.tsc), dsq, off)), dd
    msc = np.full((M, 29), -6.0, np.float32)
    msc[0, 0] = 4.0
    msc[M - 1, 1] = 4.0
    tsc = np.log(rng.uniform(0.05, 1.0, size=(M, 8))).astype(np.float32)
    tsc[:, 7] = np.log(rng.uniform(0.9, 0.9999, size=M))
    tsc[:, 0] = np.log(1e-4 / M)
    tsc[0, 0] = np.log(0.5)
    tsc[0, 1:4] = -np.inf
    tsc[M - 1, 4:8] = -np.inf
    seqs = [np.array([0, 1], np.uint8), np.array([0, 2, 1], np.uint8)]
    seqs += [synth.random_dsq(rng, int(L), 3) for L in rng.integers(1, 40, size=20)]
    dsq, off = _db_from(seqs)
    got, _ = _vit_gpu(msc, tsc, dsq, off)
    assert np.array_equal(got, oracle.vit_db(oracle.VitProfile(msc, tsc), dsq, off))


@pytest.mark.parametrize("cfg,sched", [(1, None), (3, None), (3, (12, 700)), (3, (2, 1500)),
                                       (3, (6, 1000)), (1, (12, 1000)), (3, (6, 1000, 2)), (3, (3, 1000, 2))])
def test_pipeline_upload_overlapped_equals_pipeline(cfg, sched, tune):
    """hmg_pipeline_upload (packed image re-sent from pinned host memory in length-ordered parts,
    MSV per part as it lands, long lane alongside) gives hmg_pipeline's outputs exactly; the device
    image is scrubbed first so every residue read must come from this call's upload.  `sched`
    overrides the part schedule (tuning UPLOAD_PARTS, UPLOAD_GROW: shrinking / growing parts)."""
    if sched is not None:
        tune("UPLOAD_PARTS", sched[0])
        tune("UPLOAD_GROW", sched[1])
        if len(sched) > 2:
            tune("UPLOAD_MSV_STREAMS", sched[2])     # parts' MSV kernels on two alternating streams
    prof, db = synth.config(cfg)
    dsq, off = db.materialize()
    ev = _calibrate(prof) if cfg == 1 else (-9.5, math.log(2), -9.0, math.log(2))
    p = hmg.Profile(prof.msc, prof.tsc, ev=ev)
    D = hmg.Database(dsq, off)
    ref = hmg.alloc_outputs(D.nseq)
    hmg.hmg_pipeline(p, D, **ref)
    img = torch.empty(D.packed_bytes // 4, dtype=torch.int32, pin_memory=True)
    D.image(img)
    D.upload(torch.zeros_like(img).pin_memory())          # scrub the device copy
    out = hmg.alloc_outputs(D.nseq)
    hmg.hmg_pipeline_upload(p, D, img, **out)
    torch.cuda.synchronize()
    ns = int(ref["n_survivors"].item())
    assert int(out["n_survivors"].item()) == ns
    for k in ("msv_raw", "flags"):
        assert torch.equal(out[k], ref[k]), k
    assert torch.equal(out["survivor_ids"][:ns], ref["survivor_ids"][:ns])
    sv = ref["survivor_ids"][:ns].long()
    assert torch.equal(out["vit_raw"][sv], ref["vit_raw"][sv])


def test_pipeline_in_cuda_graph():
    """The bench replays hmg_pipeline (and hmg_pipeline_upload) from a CUDA graph captured once:
    replays give the eager call's outputs exactly (scratch allocations, memsets, the long lane's
    programmatic launch and the side-stream upload are all capturable)."""
    prof, db = synth.config(1)
    dsq, off = db.materialize()
    rng = np.random.default_rng(8)
    extra = [synth.random_dsq(rng, L, 20) for L in (3000, 4100, 5200)]          # long-lane sequences
    dsq2, off2 = _db_from([dsq[off[i]:off[i + 1]] for i in range(len(off) - 1)] + extra)
    ev = _calibrate(prof)
    p = hmg.Profile(prof.msc, prof.tsc, ev=ev)
    D = hmg.Database(dsq2, off2)
    assert D.long_lane()[0] >= 3
    ref = hmg.alloc_outputs(D.nseq)
    hmg.hmg_pipeline(p, D, F1=0.3, F2=0.3, **ref)
    torch.cuda.synchronize()
    img = torch.empty(D.packed_bytes // 4, dtype=torch.int32, pin_memory=True)
    D.image(img)
    for upload in (False, True):
        out = hmg.alloc_outputs(D.nseq)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, capture_error_mode="thread_local"):
            if upload:
                hmg.hmg_pipeline_upload(p, D, img, F1=0.3, F2=0.3, stream=torch.cuda.current_stream(), **out)
            else:
                hmg.hmg_pipeline(p, D, F1=0.3, F2=0.3, stream=torch.cuda.current_stream(), **out)
        for _ in range(2):
            g.replay()
        torch.cuda.synchronize()
        ns = int(ref["n_survivors"].item())
        assert int(out["n_survivors"].item()) == ns
        assert torch.equal(out["msv_raw"], ref["msv_raw"]) and torch.equal(out["flags"], ref["flags"])
        sv = ref["survivor_ids"][:ns].long()
        assert torch.equal(out["survivor_ids"][:ns], ref["survivor_ids"][:ns])
        assert torch.equal(out["vit_raw"][sv], ref["vit_raw"][sv])


def test_graph_survives_new_thresholds():
    """Threshold tables are never freed while the profile lives: a graph captured with
    one (F1, F2) still replays its outputs after eager calls built tables for other F; a fresh
    profile prepared with hmg_prepare_thresholds captures on its first call."""
    prof, db = synth.config(1)
    dsq, off = db.materialize()
    ev = _calibrate(prof)
    p = hmg.Profile(prof.msc, prof.tsc, ev=ev)
    D = hmg.Database(dsq, off)
    ref = hmg.alloc_outputs(D.nseq)
    hmg.hmg_pipeline(p, D, F1=0.2, F2=0.1, **ref)
    out = hmg.alloc_outputs(D.nseq)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, capture_error_mode="thread_local"):
        hmg.hmg_pipeline(p, D, F1=0.2, F2=0.1, stream=torch.cuda.current_stream(), **out)
    other = hmg.alloc_outputs(D.nseq)
    for F1, F2 in ((0.05, 0.01), (0.5, 0.5), (0.9, 0.02)):          # new tables (a larger set each)
        hmg.hmg_pipeline(p, D, F1=F1, F2=F2, **other)
    g.replay()
    torch.cuda.synchronize()
    for k in ("msv_raw", "flags", "n_survivors"):
        assert torch.equal(out[k], ref[k]), k
    assert int(other["n_survivors"].item()) != int(ref["n_survivors"].item())
    # first call under capture: tables prepared ahead
    p2 = hmg.Profile(prof.msc, prof.tsc, ev=ev)
    hmg.hmg_prepare_thresholds(p2, 0.2, 0.1, Lmax=int(np.diff(off).max()))
    out2 = hmg.alloc_outputs(D.nseq)
    g2 = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g2, capture_error_mode="thread_local"):
        hmg.hmg_pipeline(p2, D, F1=0.2, F2=0.1, stream=torch.cuda.current_stream(), **out2)
    g2.replay()
    torch.cuda.synchronize()
    for k in ("msv_raw", "flags", "n_survivors"):
        assert torch.equal(out2[k], ref[k]), k

