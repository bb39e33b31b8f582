"""Randomised GPU-vs-oracle parity sweep: seeded random model lengths, transition mixes (typical,
long D->D chains, stress emissions), databases with every residue code and lengths from 1 to
3000, F thresholds; every case checks MSV and Viterbi raw scores bit-exactly, pass flags of the
pipeline, the batch call on the same DB, and Forward scores within the float32 bound of
DESIGN.md 4.7 on a subset."""
import math

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


def _db(rng, n):
    lens = rng.integers(1, 400, size=n)
    lens[: max(1, n // 20)] = rng.integers(400, 3000, size=max(1, n // 20))
    seqs = []
    for L in lens:
        alpha = int(rng.choice([20, 21, 29]))
        seqs.append(synth.random_dsq(rng, int(L), alpha))
    off = np.zeros(n + 1, np.int64)
    np.cumsum([len(s) for s in seqs], out=off[1:])
    return np.concatenate(seqs).astype(np.uint8), off


@pytest.mark.parametrize("case", range(60))
def test_fuzz_case(case):
    rng = np.random.default_rng(10_000 + case)
    M = int(rng.choice([int(rng.integers(1, 64)), int(rng.integers(64, 700)), int(rng.integers(700, 2600))]))
    dd = [(7.0, 3.0), (1.0, 9.0), (5.0, 5.0)][case % 3]
    prof = synth.make_profile(M, 20_000 + case, stress=bool(case % 4 == 3), dd=dd)
    dsq, off = _db(rng, 80)
    lam = math.log(2)
    ev = (float(rng.uniform(-10, -6)), lam, float(rng.uniform(-10, -6)), lam)
    F1, F2 = float(rng.choice([0.02, 0.2, 1.0])), float(rng.choice([1e-3, 0.1, 1.0]))
    p = hmg.Profile(prof.msc, prof.tsc, ev=ev)
    D = hmg.Database(dsq, off)
    out = hmg.alloc_outputs(D.nseq)
    hmg.hmg_pipeline(p, D, F1=F1, F2=F2, **out)
    allv = torch.full((D.nseq,), -12345, dtype=torch.int16, device="cuda")
    hmg.hmg_viterbi(p, D, allv)
    braw = torch.zeros((2, D.nseq), dtype=torch.uint8, device="cuda")
    hmg.hmg_msv_batch([p, p], D, braw)
    torch.cuda.synchronize()
    lens = np.diff(off)
    want_m = oracle.msv_db(oracle.MSVProfile(prof.msc), dsq, off)
    want_v = oracle.vit_db(oracle.VitProfile(prof.msc, prof.tsc), dsq, off)
    mraw = out["msv_raw"].cpu().numpy().astype(np.int32)
    assert np.array_equal(mraw, want_m), "MSV"
    assert np.array_equal(braw.cpu().numpy().astype(np.int32), np.stack([want_m, want_m])), "batch MSV"
    assert np.array_equal(allv.cpu().numpy().astype(np.int32), want_v), "Viterbi"
    flags = out["flags"].cpu().numpy()
    wp = np.array([oracle.msv_pass(int(r), int(L), ev[0], ev[1], F1) for r, L in zip(want_m, lens)], np.uint8)
    assert np.array_equal(flags & 1, wp), "MSV pass"
    sv = np.nonzero(wp)[0]
    wv = np.array([oracle.vit_pass(int(want_v[s]), int(lens[s]), ev[2], ev[3], F2) for s in sv], np.uint8)
    assert np.array_equal((flags[sv] >> 1) & 1, wv), "Viterbi pass"
    if case % 3 == 0 and prof.msc.max() <= 40.0:     # Forward on a subset (the fp64 oracle is slow)
        ids = np.arange(0, D.nseq, 4, dtype=np.int32)
        f = torch.full((D.nseq,), float("nan"), dtype=torch.float32, device="cuda")
        hmg.hmg_forward(p, D, f, ids=torch.as_tensor(ids, device="cuda"))
        torch.cuda.synchronize()
        got = f.cpu().numpy().astype(np.float64)[ids]
        want = oracle.fwd_db(prof.msc, prof.tsc, dsq, off, ids=ids)
        fin = np.isfinite(want)
        assert np.array_equal(np.isneginf(got), np.isneginf(want))
        tol = 2.0 ** -24 * (40.0 * lens[ids] + 4.0 * M) + 1e-6
        assert (np.abs(got[fin] - want[fin]) <= tol[fin]).all(), "Forward"
