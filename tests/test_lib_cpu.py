"""libhmg host-side tests that need no GPU.

* the C-ABI library loads and exports every function include/hmg.h declares;
* the library's quantiser (host-only handle, device = -1) produces the same
  tables as the oracle's independent quantiser, byte for byte;
* the DB packer: 6 residues x 5 bits per word, pad 31, 16-byte aligned runs,
  length-descending stable order (Fig 6);
* score conversion helpers agree with the oracle within 1e-6 relative;
* invalid inputs return HMG_EINVAL with no handle created.
"""
import ctypes
import math
import os
import re

import numpy as np
import pytest

import oracle
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    build.build()
    return hmg.lib()


def test_exports_every_declared_symbol(L):
    hdr = open(os.path.join(ROOT, "include", "hmg.h")).read()
    declared = set(re.findall(r"\b(hmg_[a-z0-9_]+)\s*\(", hdr))
    assert len(declared) >= 19
    for name in declared:
        assert hasattr(L, name), name
    assert set(hmg.SIGNATURES) == declared


@pytest.mark.parametrize("M,seed,stress", [(1, 1, False), (2, 2, True), (17, 3, False), (64, 1064, False),
                                           (200, 1200, True), (400, 1400, False), (1000, 2000, False),
                                           (2048, 3048, True)])
def test_quantiser_matches_oracle(L, M, seed, stress):
    prof = synth.make_profile(M, seed, stress=stress)
    p = hmg.Profile(prof.msc, prof.tsc, device=-1)
    q = p.quant()
    om = oracle.MSVProfile(prof.msc)
    ov = oracle.VitProfile(prof.msc, prof.tsc)
    assert (q["bias_b"], q["tbm_b"], q["tec_b"], q["base_b"]) == (om.bias, om.tbm, om.tec, 190)
    assert np.array_equal(q["cost"], om.cost)
    assert np.array_equal(q["rsc"], ov.rsc)
    assert np.array_equal(q["tsc"], ov.tr)
    assert q["ddbound_w"] == ov.ddbound
    assert q["xw_e"] == oracle.xw_e() == -500
    assert q["base_w"] == 12000
    assert q["msv_fast"] == 1


def test_quantiser_extreme_values(L):
    rng = np.random.default_rng(5)
    msc = rng.uniform(-60, 8, size=(33, 29)).astype(np.float32)
    msc[3, 7] = -np.inf
    msc[5, 2] = 25.0
    tsc = np.log(rng.uniform(1e-9, 1, size=(33, 8))).astype(np.float32)
    tsc[0, 1:4] = -np.inf
    tsc[-1, 4:] = -np.inf
    q = hmg.Profile(msc, tsc, device=-1).quant()
    assert np.array_equal(q["cost"], oracle.MSVProfile(msc).cost)
    v = oracle.VitProfile(msc, tsc)
    assert np.array_equal(q["rsc"], v.rsc) and np.array_equal(q["tsc"], v.tr)
    assert q["msv_fast"] == int(q["bias_b"] < 66 + q["tbm_b"])


def test_invalid_inputs(L):
    msc = np.zeros((4, 29), np.float32)
    for bad in (np.nan, np.inf):
        m = msc.copy()
        m[1, 1] = bad
        with pytest.raises(hmg.HmgError) as e:
            hmg.Profile(m, device=-1)
        assert e.value.status == hmg.HMG_EINVAL
    tsc = np.full((4, 8), -1.0, np.float32)
    tsc[2, 3] = 0.5   # a log-probability above 0
    with pytest.raises(hmg.HmgError):
        hmg.Profile(msc, tsc, device=-1)
    h = ctypes.c_void_p()
    assert L.hmg_profile_create(0, msc.ctypes.data_as(ctypes.c_void_p), None, None, -1, ctypes.byref(h)) == 1
    assert not h.value
    dsq = np.array([0, 1, 29], np.uint8)       # code 29 is not a residue
    with pytest.raises(hmg.HmgError):
        hmg.Database(dsq, np.array([0, 3]), device=-1)
    with pytest.raises(hmg.HmgError):         # zero-length sequence
        hmg.Database(np.array([0, 1], np.uint8), np.array([0, 0, 2]), device=-1)
    assert L.hmg_strerror(1) == b"invalid argument"


def _unpack(img, start_word, L):
    out = []
    w = start_word
    while len(out) < L:
        v = int(img[w])
        assert v >> 30 == 0
        for j in range(6):
            out.append((v >> (5 * j)) & 31)
        w += 1
    return out


def test_packer_roundtrip(L):
    rng = np.random.default_rng(2)
    lens = rng.integers(1, 40, size=200).astype(np.int64)
    lens[5] = lens[9] = lens[77] = 13  # ties keep caller order (stable)
    off = np.zeros(len(lens) + 1, np.int64)
    np.cumsum(lens, out=off[1:])
    dsq = rng.integers(0, 29, size=int(off[-1])).astype(np.uint8)
    db = hmg.Database(dsq, off, device=-1)
    order = db.order()
    assert sorted(order.tolist()) == list(range(len(lens)))
    sl = lens[order]
    assert (np.diff(sl) <= 0).all()
    ties = [s for s in order if lens[s] == 13]
    assert ties == sorted(ties)
    img = db.image()
    w = 0
    for s in order:
        Ls = int(lens[s])
        got = _unpack(img, w, Ls)
        assert got[:Ls] == dsq[off[s]:off[s + 1]].tolist()
        assert all(c == 31 for c in got[Ls:])          # pad slots = 31
        w += ((Ls + 5) // 6 + 3) // 4 * 4                # 16-byte aligned runs
    assert db.residues == int(lens.sum())


def test_conversions_match_oracle(L):
    for L_ in (1, 2, 17, 300, 35213, 100000):
        assert abs(hmg.hmg_null1_nats(L_) - oracle.null1(L_)) <= 1e-6 * abs(oracle.null1(L_))
        for raw in (0, 1, 77, 190, 251, 255):
            a, b = hmg.hmg_msv_nats(raw, L_), oracle.msv_nats(raw, L_)
            assert a == b or abs(a - b) <= 1e-6 * abs(b)
        for raw in (-32768, -30000, -1, 0, 5000, 32766, 32767):
            a, b = hmg.hmg_vit_nats(raw, L_), oracle.vit_nats(raw, L_)
            assert a == b or abs(a - b) <= 1e-6 * abs(b)
    for x in (-30.0, -5.0, 0.0, 3.3, 40.0):
        a, b = hmg.hmg_gumbel_surv(x, -9.0, math.log(2)), oracle.gumbel_surv(x, -9.0, math.log(2))
        assert a == b or abs(a - b) <= 1e-6 * abs(b)


def test_host_only_handles_rejected_by_compute_calls(L):
    """Compute entry points (incl. Forward and the batch calls) reject host-only handles and bad
    arguments with HMG_EINVAL before touching a device (no GPU needed)."""
    msc = np.zeros((8, 29), np.float32)
    tsc = np.full((8, 8), -1.0, np.float32)
    p = hmg.Profile(msc, tsc, device=-1)
    d = hmg.Database(np.zeros(12, np.uint8), np.array([0, 5, 12]), device=-1)
    q = p.quant()
    assert q["fwd_lanes"] == 8 and q["fwd_nodes"] == 2 and q["fwd_rows_smem"] == 29
    vp = ctypes.c_void_p
    assert L.hmg_forward(p.handle, d.handle, None, 0, None, vp(1)) == hmg.HMG_EINVAL
    assert L.hmg_pipeline_forward(p.handle, d.handle, 0.02, 1e-3, None, vp(1), vp(1), vp(1), vp(1), vp(1),
                                  vp(1), vp(1), vp(1)) == hmg.HMG_EINVAL
    arr = (vp * 1)(p.handle)
    assert L.hmg_msv_batch(arr, 1, d.handle, 0.02, None, vp(1), None) == hmg.HMG_EINVAL
    assert L.hmg_msv_batch(arr, 0, d.handle, 0.02, None, vp(1), None) == hmg.HMG_EINVAL
    assert L.hmg_pipeline_batch(arr, 1, d.handle, 0.02, 2.0, None, vp(1), vp(1), vp(1), vp(1),
                                vp(1), None, None, None) == hmg.HMG_EINVAL
    assert L.hmg_pipeline_batch(arr, 1, d.handle, 0.02, 1e-3, None, vp(1), vp(1), vp(1), vp(1),
                                vp(1), vp(1), None, None) == hmg.HMG_EINVAL     # Forward outputs: all or none


def test_forward_geometry_host_only(L):
    """Forward kernel geometry: 8-lane groups up to M = 32, then the
    fewest warps at 16 nodes per thread and the fewest nodes (one warp: 12 / 13 / 14 before 16);
    unsupported above 4096 nodes."""
    for M, (T, Qn) in {1: (8, 2), 16: (8, 2), 17: (8, 4), 32: (8, 4), 33: (32, 2), 64: (32, 2), 65: (32, 4),
                       128: (32, 4), 129: (32, 8), 256: (32, 8), 257: (32, 12), 384: (32, 12), 385: (32, 13),
                       400: (32, 13), 416: (32, 13), 417: (32, 14), 448: (32, 14), 449: (32, 16), 512: (32, 16),
                       513: (64, 16), 1000: (64, 16), 2048: (128, 16), 4096: (256, 16)}.items():
        p = hmg.Profile(np.zeros((M, 29), np.float32), np.full((M, 8), -1.0, np.float32), device=-1)
        q = p.quant()
        assert (q["fwd_lanes"], q["fwd_nodes"], q["fwd_warps"]) == (T, Qn, max(1, T // 32)), M
    p = hmg.Profile(np.zeros((4097, 29), np.float32), np.full((4097, 8), -1.0, np.float32), device=-1)
    assert p.quant()["fwd_warps"] == 0


def test_tuning_api():
    """hmg_set_tuning accepts the documented knobs only (the library reads no environment
    variables); clearing restores the defaults."""
    hmg.lib()
    for k in ("MSV_G", "VIT_PAIR_W", "VIT_CPAIR2", "UPLOAD_PARTS", "PIPE_LLONG"):
        hmg.set_tuning(k, 4)
        hmg.clear_tuning(k)
    with pytest.raises(hmg.HmgError):
        hmg.set_tuning("NOT_A_KNOB", 1)
    with pytest.raises(hmg.HmgError):
        hmg.clear_tuning("NOT_A_KNOB")
    hmg.clear_tuning()
    src = open(os.path.join(os.path.dirname(__file__), "..", "paper_conf_ipps_jiangg15_b200", "csrc", "host.cu")).read()
    assert "getenv" not in src


def test_tuning_knobs_documented():
    """Every knob the library accepts is listed in include/hmg.h (hmg_set_tuning's contract)."""
    here = os.path.dirname(__file__)
    src = open(os.path.join(here, "..", "paper_conf_ipps_jiangg15_b200", "csrc", "host.cu")).read()
    names = re.findall(r'"([A-Z0-9_]+)"', src[src.index("kTuneNames[]"):src.index("};", src.index("kTuneNames[]"))])
    hdr = open(os.path.join(here, "..", "include", "hmg.h")).read()
    doc = hdr[hdr.index("hmg_set_tuning") - 2000:hdr.index("hmg_set_tuning")]
    assert len(names) > 20
    for n in names:
        assert n in doc, n
        hmg.set_tuning(n, 0)
    hmg.clear_tuning()


@pytest.mark.parametrize("M,kind", [(40, 1), (400, 1), (1024, 1), (1100, 4), (1500, 5), (2048, 5), (3000, 2)])
def test_viterbi_kernel_choice(M, kind):
    """Which s16x2 Viterbi kernel a profile gets (hmg_quant.vit_pair_kernel, DESIGN.md 4.3b-d):
    lane groups up to 1024 nodes, one warp per sequence above (transitions in shared memory up to
    1280 nodes, in tensor memory to 2048), warps joined per row beyond; VIT_WIDE = 0 restores the
    two-warp kernel."""
    prof = synth.make_profile(M, 77 + M)
    q = hmg.Profile(prof.msc, prof.tsc, device=-1).quant()
    assert q["vit_pair_kernel"] == kind
    assert 2 * q["vit_pair_lanes"] * q["vit_pair_regs"] >= M
    if kind in (4, 5):
        assert q["vit_pair_lanes"] == 32
        hmg.set_tuning("VIT_WIDE", 0)
        try:
            assert hmg.Profile(prof.msc, prof.tsc, device=-1).quant()["vit_pair_kernel"] in (2, 3)
        finally:
            hmg.clear_tuning()

