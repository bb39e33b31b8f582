"""GPU parity of the Forward stage against the fp64 log-space oracle.

The CUDA path computes in float32 odds space, so parity is a tolerance, not bit-exactness.
Tolerance: a Forward score is the log of a sum of products of positive
terms -- no cancellation -- so its float32 relative error is bounded by the number of roundings
along the paths that carry the score times u = 2^-24.  Per row a path meets at most ~40
roundings (5 for the M cell, the E reduction over nodes and warps, 2 per special state, the
length-model loops) and a D->D chain adds 2 per node it crosses, so

    |gpu - oracle| <= 2^-24 (40 L + 4 M) + 1e-6   nats.

Both sides give -inf exactly when no path has non-zero odds.
"""
import math

import numpy as np
import pytest

import oracle
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

U = 2.0 ** -24


@pytest.fixture(scope="module", autouse=True)
def _lib():
    if not torch.cuda.is_available():
        pytest.fail("GPU test run without a CUDA device")
    build.build()
    hmg.lib()


def _tol(L, M):
    return U * (40.0 * np.asarray(L, np.float64) + 4.0 * M) + 1e-6


def _db_from(dsq_list):
    off = np.zeros(len(dsq_list) + 1, np.int64)
    np.cumsum([len(d) for d in dsq_list], out=off[1:])
    dsq = np.concatenate(dsq_list).astype(np.uint8) if dsq_list else np.zeros(0, np.uint8)
    return dsq, off


def _ragged(rng, n=60, lmax=500, alphabet=29):
    lens = list(range(1, 14)) + [17, 18, 19, 35, 36, 37, 191, 192, 193]
    lens += rng.integers(1, lmax, size=max(0, n - len(lens))).tolist()
    return _db_from([synth.random_dsq(rng, int(L), alphabet) for L in lens])


def _fwd_gpu(msc, tsc, dsq, off, ids=None):
    p = hmg.Profile(msc, tsc)
    db = hmg.Database(dsq, off)
    out = torch.full((db.nseq,), float("nan"), dtype=torch.float32, device="cuda")
    t_ids = None if ids is None else torch.as_tensor(ids, dtype=torch.int32, device="cuda")
    hmg.hmg_forward(p, db, out, ids=t_ids)
    torch.cuda.synchronize()
    return out.cpu().numpy().astype(np.float64), p


def _assert_close(got, want, lens, M):
    got = np.asarray(got, np.float64)
    want = np.asarray(want, np.float64)
    inf = np.isneginf(want)
    assert np.array_equal(np.isneginf(got), inf), "-inf pattern differs"
    assert np.isfinite(got[~inf]).all()
    err = np.abs(got[~inf] - want[~inf])
    tol = _tol(np.asarray(lens)[~inf], M)
    bad = np.nonzero(err > tol)[0]
    assert bad.size == 0, "max err %.3g (tol %.3g) at %d of %d" % (err.max(), tol[bad[0]], bad.size, err.size)
    return err.max() if err.size else 0.0


def test_fwd_config1_full():
    prof, db = synth.config(1)
    dsq, off = db.materialize()
    got, _ = _fwd_gpu(prof.msc, prof.tsc, dsq, off)
    want = oracle.fwd_db(prof.msc, prof.tsc, dsq, off)
    _assert_close(got, want, np.diff(off), prof.M)


FMS = [1, 2, 3, 31, 63, 64, 65, 127, 128, 129, 255, 256, 257, 384, 385, 400, 416, 417, 448, 449, 511, 512, 513,
       1000, 1024, 1025, 2047, 2048, 2049, 3000, 4096]


@pytest.mark.parametrize("M", FMS)
@pytest.mark.parametrize("dd", [(7.0, 3.0), (1.0, 9.0)])
def test_fwd_model_lengths(M, dd):
    """Every geometry (W warps x Q nodes) and its boundaries, ragged sequence lengths around the
    6-residue word and the 32-word residue chunk, all 29 codes, and long D->D chains."""
    rng = np.random.default_rng(M)
    prof = synth.make_profile(M, 9000 + M, dd=dd)
    n = 40 if M > 1500 else 60
    dsq, off = _ragged(rng, n=n, lmax=300 if M > 1500 else 500)
    got, p = _fwd_gpu(prof.msc, prof.tsc, dsq, off)
    q = p.quant()
    assert q["fwd_lanes"] * q["fwd_nodes"] >= M
    want = oracle.fwd_db(prof.msc, prof.tsc, dsq, off)
    _assert_close(got, want, np.diff(off), M)


@pytest.mark.parametrize("M", [64, 700, 2048])
def test_fwd_stress_profiles(M):
    """Unmixed emissions (log-odds down to ~-45 nats) exercise tiny odds and denormal ranges."""
    rng = np.random.default_rng(M + 1)
    prof = synth.make_profile(M, 9100 + M, stress=True)
    dsq, off = _ragged(rng, n=40, lmax=400)
    got, _ = _fwd_gpu(prof.msc, prof.tsc, dsq, off)
    want = oracle.fwd_db(prof.msc, prof.tsc, dsq, off)
    _assert_close(got, want, np.diff(off), M)


@pytest.mark.parametrize("boost", [3.0, 8.0, 20.0, 40.0])
def test_fwd_rescaling(boost):
    """Strongly positive emissions grow the row by up to e^boost per residue: the kernel's exact
    power-of-two rescaling (E > 2^40) fires on most rows of long sequences."""
    rng = np.random.default_rng(int(boost))
    M = 300
    prof = synth.make_profile(M, 9200)
    msc = prof.msc.copy()
    msc[:, :20] = np.minimum(msc[:, :20] + np.float32(boost), np.float32(40.0))
    dsq, off = _db_from([synth.random_dsq(rng, L, 20) for L in (1, 5, 100, 1000, 3000, 6001)])
    got, _ = _fwd_gpu(msc, prof.tsc, dsq, off)
    want = oracle.fwd_db(msc, prof.tsc, dsq, off)
    _assert_close(got, want, np.diff(off), M)
    assert want[-1] > 1000.0


def test_fwd_minus_inf_and_range_check():
    """Sequences made only of gap codes (-inf emissions everywhere) have no path: -inf on both
    sides.  Emission log-odds above +40 nats are outside float odds space: EUNSUPPORTED."""
    prof = synth.make_profile(100, 9300)
    dsq, off = _db_from([np.full(L, 20, np.uint8) for L in (1, 7, 50)] + [np.arange(20, dtype=np.uint8)])
    got, _ = _fwd_gpu(prof.msc, prof.tsc, dsq, off)
    want = oracle.fwd_db(prof.msc, prof.tsc, dsq, off)
    assert np.isneginf(want[:3]).all() and np.isneginf(got[:3]).all()
    _assert_close(got, want, np.diff(off), 100)
    msc = prof.msc.copy()
    msc[5, 3] = 41.0
    with pytest.raises(hmg.HmgError) as ei:
        _fwd_gpu(msc, prof.tsc, dsq, off)
    assert ei.value.status == hmg.HMG_EUNSUPPORTED
    big = synth.make_profile(4097, 9301)
    with pytest.raises(hmg.HmgError) as ei:
        _fwd_gpu(big.msc, big.tsc, dsq, off)
    assert ei.value.status == hmg.HMG_EUNSUPPORTED


def test_fwd_ids_subset_untouched_elsewhere():
    rng = np.random.default_rng(5)
    prof = synth.make_profile(200, 9400)
    dsq, off = _ragged(rng, n=80)
    ids = np.array([3, 70, 0, 41, 41, 12], np.int32)
    got, _ = _fwd_gpu(prof.msc, prof.tsc, dsq, off, ids=ids)
    mask = np.zeros(len(off) - 1, bool)
    mask[ids] = True
    assert np.isnan(got[~mask]).all()
    want = oracle.fwd_db(prof.msc, prof.tsc, dsq, off, ids=np.unique(ids))
    _assert_close(got[np.unique(ids)], want, np.diff(off)[np.unique(ids)], 200)


def test_fwd_empty_db():
    prof = synth.make_profile(50, 9500)
    p = hmg.Profile(prof.msc, prof.tsc)
    db = hmg.Database(np.zeros(0, np.uint8), np.zeros(1, np.int64))
    out = torch.zeros(1, dtype=torch.float32, device="cuda")
    hmg.hmg_forward(p, db, out)
    torch.cuda.synchronize()


def _check_pipeline_forward(prof, dsq, off, F1, F2, sample=None):
    ev = synth_ev(prof)
    p = hmg.Profile(prof.msc, prof.tsc, ev=ev)
    db = hmg.Database(dsq, off)
    out = hmg.alloc_outputs(db.nseq)
    fo = hmg.alloc_forward_outputs(db.nseq)
    hmg.hmg_pipeline_forward(p, db, F1=F1, F2=F2, **out, **fo)
    torch.cuda.synchronize()
    flags = out["flags"].cpu().numpy()
    nf = int(fo["n_fwd"].item())
    fids = fo["fwd_ids"].cpu().numpy()[:nf]
    fn = fo["fwd_nats"].cpu().numpy().astype(np.float64)
    lens = np.diff(off)
    # the Forward list is exactly the Viterbi passes, length-descending, stable
    order = np.lexsort((np.arange(db.nseq), -lens))
    assert fids.tolist() == [s for s in order if flags[s] & 2]
    assert np.array_equal((flags >> 3) & 1, (flags >> 1) & 1)
    assert np.isnan(fn[(flags & 2) == 0]).all()
    chk = fids if sample is None else fids[: sample]
    want = oracle.fwd_db(prof.msc, prof.tsc, dsq, off, ids=chk)
    _assert_close(fn[chk], want, lens[chk], prof.M)
    # the MSV / Viterbi outputs of the same call equal the oracle's on the Forward list
    mraw = out["msv_raw"].cpu().numpy().astype(np.int32)
    vraw = out["vit_raw"].cpu().numpy().astype(np.int32)
    assert np.array_equal(mraw[chk], oracle.msv_db(oracle.MSVProfile(prof.msc), dsq, off, ids=chk))
    assert np.array_equal(vraw[chk], oracle.vit_db(oracle.VitProfile(prof.msc, prof.tsc), dsq, off, ids=chk))
    return nf


def synth_ev(prof):
    """mu for lambda = ln 2 fitted by the ORACLE on 1000 background sequences of L = 200."""
    cal = synth.Database(np.full(1000, 200, np.int32), seed=7)
    dsq, off = cal.materialize()
    mp, vp = oracle.MSVProfile(prof.msc), oracle.VitProfile(prof.msc, prof.tsc)
    lam = math.log(2)
    mb = [oracle.bits(oracle.msv_nats(int(r), 200), 200) for r in oracle.msv_db(mp, dsq, off)]
    vb = [oracle.bits(oracle.vit_nats(int(r), 200), 200) for r in oracle.vit_db(vp, dsq, off)]
    return (oracle.fit_mu(np.array(mb), lam), lam, oracle.fit_mu(np.array(vb), lam), lam)


def test_pipeline_forward_config1():
    prof, db = synth.config(1)
    dsq, off = db.materialize()
    nf = _check_pipeline_forward(prof, dsq, off, F1=0.5, F2=0.2)
    assert nf > 50


def test_pipeline_forward_config3_full_size():
    """BASELINE config 3 at full size (550k sequences, M = 400, planted homologs) through the
    whole Fig 1 pipeline; the oracle re-scores the first 400 Forward sequences (longest first)."""
    prof, db = synth.config(3)
    dsq, off = db.materialize()
    nf = _check_pipeline_forward(prof, dsq, off, F1=0.02, F2=1e-3, sample=400)
    assert nf >= 400


@pytest.mark.parametrize("M,S,qmax", [(10, 4, 16), (10, 32, 16), (30, 8, 16), (30, 16, 16), (32, 32, 16),
                                      (40, 2, 16), (40, 4, 16), (40, 8, 16), (40, 12, 16), (100, 2, 16),
                                      (128, 12, 16), (200, 2, 16),
                                      (200, 12, 16), (200, 4, 16), (300, 1, 8), (300, 2, 8), (300, 4, 8), (300, 6, 8),
                                      (700, 1, 8), (700, 2, 8), (700, 3, 8), (300, 2, 16), (300, 4, 16),
                                      (300, 8, 16), (700, 1, 16), (700, 2, 16), (700, 4, 16)])
def test_fwd_every_block_shape(M, S, qmax, tune):
    """Every instantiated (W, Q, S): S sequences per block share the staged table and take
    sequences from the queue independently (named barriers per sequence group)."""
    tune("FWD_S", str(S))
    tune("FWD_QMAX", str(qmax))
    rng = np.random.default_rng(M * 100 + S)
    prof = synth.make_profile(M, 9600 + M, dd=(1.0, 9.0))
    dsq, off = _ragged(rng, n=90, lmax=400)
    got, p = _fwd_gpu(prof.msc, prof.tsc, dsq, off)
    assert p.quant()["fwd_seqs_per_block"] == S
    want = oracle.fwd_db(prof.msc, prof.tsc, dsq, off)
    _assert_close(got, want, np.diff(off), M)


@pytest.mark.parametrize("M", [100, 257, 400, 449, 512, 513, 1000, 2048, 3000])
def test_fwd_lean_sixteen_nodes(M, tune):
    """The register-lean 16-nodes-per-thread variant (tuning FWD_QMAX=16: one warp up to M = 512, no
    per-row barrier; D = Dloc + c_in P applied as two 8-node product chains); one-warp models of
    257 ... 448 nodes take 12 / 13 / 14 nodes per thread instead."""
    tune("FWD_QMAX", "16")
    rng = np.random.default_rng(M + 77)
    prof = synth.make_profile(M, 9700 + M, dd=(1.0, 9.0))
    dsq, off = _ragged(rng, n=50, lmax=400)
    got, p = _fwd_gpu(prof.msc, prof.tsc, dsq, off)
    q = p.quant()
    assert q["fwd_nodes"] == 16 or M <= 256 or (M <= 448 and q["fwd_nodes"] in (12, 13, 14))
    want = oracle.fwd_db(prof.msc, prof.tsc, dsq, off)
    _assert_close(got, want, np.diff(off), M)
