"""The sharded (multi-GPU) path proven on one GPU: SURVEY 8(c.6) "gathered W-GPU results ==
1-GPU results, byte-for-byte" (the database is split "without any dependencies").

Each test plays every rank of a W-way run in turn on cuda:0 -- its snake shard
(dist.snake_shard) as its own hmg_db, the same calls bench.py times -- takes the padded slices
dist.Gatherer hands to all_gather_into_tensor (Gatherer.local), concatenates them in rank order
(exactly what the collective returns), reassembles with dist.assemble and compares with one call
over the whole DB: MSV raw, Viterbi raw, flags and the survivor set, byte for byte.  The NCCL /
gloo collective itself is covered by tests/test_dist_cpu.py (world_size 2 and 3).
"""
import numpy as np
import pytest

from paper_conf_ipps_jiangg15_b200 import build, dist as hdist, hmg, synth

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _lib():
    if not torch.cuda.is_available():
        pytest.fail("GPU test run without a CUDA device")
    build.build()
    hmg.lib()


def _emulate(gdb, P, run, world, n_global):
    """Run every rank's shard; return what all_gather + assemble give rank 0."""
    pads, svs, nss, gps = [], [], [], []
    for r in range(world):
        ids = hdist.snake_shard(gdb.lengths, world, r)
        D = hmg.Database(*gdb.materialize(ids))
        o = hmg.alloc_outputs(D.nseq)
        run(P, D, o)
        g = hdist.Gatherer(n_global, world, torch.as_tensor(ids, device="cuda"), exchange=False)
        pad, sv, ns = g.local(o["msv_raw"], o["vit_raw"], o["flags"], o["survivor_ids"], o["n_survivors"])
        pads.append(pad.clone()); svs.append(sv.clone()); nss.append(ns.clone()); gps.append(g.gid_pad.clone())
        # each rank's survivor list is in its schedule order: length-descending
        n = int(ns.item())
        assert (np.diff(gdb.lengths[sv[:n].cpu().numpy()]) <= 0).all()
    torch.cuda.synchronize()
    nmax = pads[0].numel()
    words = torch.cat(pads).view(world, nmax).cpu().numpy()
    gids = torch.cat(gps).view(world, nmax).cpu().numpy()
    counts = torch.cat(nss).cpu().numpy()
    surv = torch.cat(svs).view(world, nmax).cpu().numpy()
    return hdist.assemble(words, gids, counts, surv, n_global)


def _whole(gdb, P, run):
    D = hmg.Database(*gdb.materialize())
    o = hmg.alloc_outputs(D.nseq)
    run(P, D, o)
    torch.cuda.synchronize()
    ns = int(o["n_survivors"].item())
    return (o["msv_raw"].cpu().numpy().astype(np.int32), o["vit_raw"].cpu().numpy().astype(np.int32),
            o["flags"].cpu().numpy(), o["survivor_ids"][:ns].cpu().numpy().astype(np.int64))


def _pipeline(P, D, o):
    hmg.hmg_pipeline(P, D, F1=0.02, F2=1e-3, **o)


@pytest.mark.parametrize("world", [2, 4, 8])
def test_config3_sharded_equals_unsharded(world):
    """Config 3 at full size (M = 400, 550k Swiss-Prot-shaped sequences, 0.1% planted)."""
    prof, gdb = synth.config(3)
    P, _ = hmg.calibrated_profile(prof.msc, prof.tsc)
    msv, vit, flags, surv = _whole(gdb, P, _pipeline)
    gm, gv, gf, sl = _emulate(gdb, P, _pipeline, world, gdb.N)
    assert np.array_equal(gm, msv)
    assert np.array_equal(gf, flags)
    run = (flags & 4) != 0                               # Viterbi ran (survivors): raw defined there
    assert np.array_equal(gv[run], vit[run])
    assert np.array_equal(np.sort(np.concatenate(sl)), np.sort(surv))
    assert len(surv) > 1000


@pytest.mark.parametrize("which,world", [(0, 8), (2, 4)])
def test_config5_sharded_equals_unsharded(which, world):
    """Config-5 shape (UniProt-like lognormal(5.55, 0.80), M = 100 / 1000) on a 400k-sequence DB."""
    prof, gdb = synth.config(5, which=which, N=400_000)
    P, _ = hmg.calibrated_profile(prof.msc, prof.tsc)
    msv, vit, flags, surv = _whole(gdb, P, _pipeline)
    gm, gv, gf, sl = _emulate(gdb, P, _pipeline, world, gdb.N)
    assert np.array_equal(gm, msv) and np.array_equal(gf, flags)
    run = (flags & 4) != 0
    assert np.array_equal(gv[run], vit[run])
    assert np.array_equal(np.sort(np.concatenate(sl)), np.sort(surv))


def test_config4_viterbi_sharded_equals_unsharded():
    """Config 4's Viterbi-only stage (M = 2048, every sequence) on 60k sequences, 8 shards."""
    prof = synth.make_profile(2048, 3048)
    gdb = synth.make_db(60_000, 5.6, 0.75, 12)
    P, _ = hmg.calibrated_profile(prof.msc, prof.tsc)

    def vit_all(P, D, o):
        hmg.hmg_viterbi(P, D, o["vit_raw"], pass_=o["flags"], F2=1e-3)

    _, vit, flags, _ = _whole(gdb, P, vit_all)
    _, gv, gf, _ = _emulate(gdb, P, vit_all, 8, gdb.N)
    assert np.array_equal(gv, vit) and np.array_equal(gf, flags)
