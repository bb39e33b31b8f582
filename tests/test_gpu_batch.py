"""GPU parity of the many-profile MSV batch against the oracle, bit-exact.

hmg_msv_batch scores every (profile, sequence) pair in one call: profiles are bucketed by lane
geometry and padded, work items are (DB chunk, profile).  Every row must equal the oracle's MSV
of that profile (and hmg_msv's) exactly; pass flags equal the oracle's pass decisions.
"""
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


def _db_from(dsq_list):
    off = np.zeros(len(dsq_list) + 1, np.int64)
    np.cumsum([len(d) for d in dsq_list], out=off[1:])
    return np.concatenate(dsq_list).astype(np.uint8), off


def _ragged(rng, n=300, lmax=600, alphabet=29):
    lens = list(range(1, 14)) + [23, 24, 25, 95, 96, 97, 1500, 3100]
    lens += rng.integers(1, lmax, size=n - len(lens)).tolist()
    seqs = [synth.random_dsq(rng, int(L), alphabet) for L in lens]
    seqs += [np.full(L, 20, np.uint8) for L in (1, 4, 30)]        # all-gap: the exact re-score path
    return _db_from(seqs)


def _batch(profs, dsq, off, F1=0.02, evs=None):
    P = [hmg.Profile(p.msc, p.tsc, ev=None if evs is None else evs[i]) for i, p in enumerate(profs)]
    db = hmg.Database(dsq, off)
    raw = torch.full((len(P), db.nseq), 77, dtype=torch.uint8, device="cuda")
    pas = torch.full((len(P), db.nseq), 9, dtype=torch.uint8, device="cuda") if evs is not None else None
    hmg.hmg_msv_batch(P, db, raw, pas, F1=F1)
    torch.cuda.synchronize()
    return (raw.cpu().numpy().astype(np.int32), None if pas is None else pas.cpu().numpy()), P, db


MIX = [1, 5, 40, 64, 79, 80, 100, 149, 150, 200, 255, 300, 400, 450, 451, 513, 640, 641, 700, 1000, 1300, 2048]


def test_batch_mixed_lengths_bit_exact():
    """22 model lengths across every lane geometry and bucket boundary, one duplicate, a saturating
    profile outside the fast precondition (all its pairs on the exact pair kernel), ragged and
    all-gap sequences: every row equals the oracle's MSV of that profile."""
    rng = np.random.default_rng(4)
    profs = [synth.make_profile(M, 5000 + M) for M in MIX]
    profs.append(profs[7])                                          # duplicate
    sat = synth.make_profile(120, 5999)
    sat.msc = sat.msc.copy()
    sat.msc[:, :20] = np.float32(30.0)                              # bias >= 66 + tbm: exact kernel
    profs.append(sat)
    dsq, off = _ragged(rng)
    (raw, _), P, db = _batch(profs, dsq, off)
    assert P[-1].quant()["msv_fast"] == 0
    for i, pr in enumerate(profs):
        want = oracle.msv_db(oracle.MSVProfile(pr.msc), dsq, off)
        assert np.array_equal(raw[i], want), "profile %d (M=%d)" % (i, pr.M)


def test_batch_equals_single_calls_config1():
    """BASELINE config-1 DB against 40 Pfam-like profiles (M ~ lognormal, median ~180): the batch
    equals 40 hmg_msv calls and the oracle."""
    prof1, dbs = synth.config(1)
    dsq, off = dbs.materialize()
    rng = np.random.default_rng(11)
    Ms = np.clip(np.round(rng.lognormal(math.log(180), 0.6, size=40)), 20, 1500).astype(int)
    profs = [synth.make_profile(int(M), 6000 + i) for i, M in enumerate(Ms)]
    (raw, _), P, db = _batch(profs, dsq, off)
    one = torch.zeros(db.nseq, dtype=torch.uint8, device="cuda")
    for i, (pr, p) in enumerate(zip(profs, P)):
        hmg.hmg_msv(p, db, one)
        torch.cuda.synchronize()
        assert np.array_equal(raw[i], one.cpu().numpy().astype(np.int32))
        if i % 8 == 0:
            assert np.array_equal(raw[i], oracle.msv_db(oracle.MSVProfile(pr.msc), dsq, off))


def _mu_msv(pr, lam=math.log(2)):
    """MSV Gumbel location fitted by the ORACLE on 1000 background sequences of L = 200."""
    cal = synth.Database(np.full(1000, 200, np.int32), seed=7)
    dsq, off = cal.materialize()
    b = [oracle.bits(oracle.msv_nats(int(r), 200), 200) for r in oracle.msv_db(oracle.MSVProfile(pr.msc), dsq, off)]
    return oracle.fit_mu(np.array(b), lam)


def test_batch_pass_flags():
    """Pass flags of every pair equal the oracle's decisions under each profile's own calibrated
    thresholds (F1 = 0.05 on background sequences: a few % pass)."""
    rng = np.random.default_rng(21)
    profs = [synth.make_profile(M, 6100 + M) for M in (60, 200, 333, 800)]
    dsq, off = _ragged(rng, n=400, alphabet=20)
    lam = math.log(2)
    evs = [(_mu_msv(pr), lam, 0.0, lam) for pr in profs]
    (raw, pas), _, _ = _batch(profs, dsq, off, F1=0.05, evs=evs)
    lens = np.diff(off)
    for i, pr in enumerate(profs):
        want = oracle.msv_db(oracle.MSVProfile(pr.msc), dsq, off)
        assert np.array_equal(raw[i], want)
        ev = evs[i]
        wp = [oracle.msv_pass(int(r), int(L), ev[0], ev[1], 0.05) for r, L in zip(want, lens)]
        assert np.array_equal(pas[i], np.array(wp, np.uint8))
        assert 0 < pas[i].sum() < len(lens)


def test_batch_config2_full_size_sampled():
    """BASELINE config-2 DB at full size (550k sequences) against 6 profiles in one call (3 lane
    geometries); the oracle checks a length-stratified sample of every row."""
    _, dbs = synth.config(2)
    dsq, off = dbs.materialize()
    profs = [synth.make_profile(M, 6200 + M) for M in (64, 100, 200, 220, 400, 1000)]
    (raw, _), _, _ = _batch(profs, dsq, off)
    rng = np.random.default_rng(3)
    sample = np.unique(np.concatenate([rng.choice(dbs.N, 1500, replace=False), np.argsort(-dbs.lengths)[:20]]))
    for i, pr in enumerate(profs):
        want = oracle.msv_db(oracle.MSVProfile(pr.msc), dsq, off, ids=sample)
        assert np.array_equal(raw[i][sample], want), "M=%d" % pr.M


def test_batch_invalid_and_empty():
    pr = synth.make_profile(50, 6300)
    p = hmg.Profile(pr.msc, pr.tsc)
    db = hmg.Database(np.zeros(0, np.uint8), np.zeros(1, np.int64))
    hmg.hmg_msv_batch([p], db, torch.zeros((1, 1), dtype=torch.uint8, device="cuda"))
    dsq, off = _db_from([np.arange(20, dtype=np.uint8)])
    db2 = hmg.Database(dsq, off)
    out = torch.zeros((1, 1), dtype=torch.uint8, device="cuda")
    with pytest.raises(hmg.HmgError) as ei:       # pass flags need ev
        hmg.hmg_msv_batch([p], db2, out, torch.zeros((1, 1), dtype=torch.uint8, device="cuda"))
    assert ei.value.status == hmg.HMG_EINVAL
    with pytest.raises(hmg.HmgError):
        hmg.hmg_msv_batch([], db2, out)


def test_pipeline_batch_equals_per_profile_pipelines():
    """hmg_pipeline_batch (MSV batch -> per-profile compaction + Viterbi + Forward on side streams)
    equals one hmg_pipeline_forward call per profile on every output, and the oracle on the
    survivors of two rows."""
    prof1, dbs = synth.config(1)
    dsq, off = dbs.materialize()
    lam = math.log(2)
    Ms = (64, 150, 200, 420, 700, 1100, 64)
    profs = [synth.make_profile(M, 6400 + i) for i, M in enumerate(Ms)]
    evs = [(_mu_msv(pr), lam, _mu_msv(pr) - 1.0, lam) for pr in profs]
    P = [hmg.Profile(pr.msc, pr.tsc, ev=ev) for pr, ev in zip(profs, evs)]
    db = hmg.Database(dsq, off)
    out = hmg.alloc_batch_outputs(len(P), db.nseq)
    fo = hmg.alloc_batch_forward_outputs(len(P), db.nseq)
    hmg.hmg_pipeline_batch(P, db, F1=0.1, F2=0.05, **out, **fo)
    torch.cuda.synchronize()
    for i, p in enumerate(P):
        one = hmg.alloc_outputs(db.nseq)
        f1 = hmg.alloc_forward_outputs(db.nseq)
        hmg.hmg_pipeline_forward(p, db, F1=0.1, F2=0.05, **one, **f1)
        torch.cuda.synchronize()
        nf = int(f1["n_fwd"].item())
        assert int(fo["n_fwd"][i].item()) == nf
        assert torch.equal(fo["fwd_ids"][i][:nf], f1["fwd_ids"][:nf])
        assert torch.equal(fo["fwd_nats"][i].isnan(), f1["fwd_nats"].isnan())
        fi = f1["fwd_ids"][:nf].long()
        assert torch.equal(fo["fwd_nats"][i][fi], f1["fwd_nats"][fi])   # same kernel, same inputs
        ns = int(one["n_survivors"].item())
        assert int(out["n_survivors"][i].item()) == ns > 0
        assert torch.equal(out["msv_raw"][i], one["msv_raw"])
        assert torch.equal(out["flags"][i], one["flags"])
        assert torch.equal(out["survivor_ids"][i][:ns], one["survivor_ids"][:ns])
        assert torch.equal(out["vit_raw"][i], one["vit_raw"])
        if i in (0, 4):
            sv = one["survivor_ids"][:ns].cpu().numpy()
            want = oracle.vit_db(oracle.VitProfile(profs[i].msc, profs[i].tsc), dsq, off, ids=sv)
            assert np.array_equal(out["vit_raw"][i].cpu().numpy().astype(np.int32)[sv], want)
