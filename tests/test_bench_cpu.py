"""bench.py host logic without a GPU: the roofline record and the workload / sharding choices."""
import json
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def test_kernel_roofline_msv_lds_bound():
    ev = bench.load_evidence()
    cells, ms = 78.03e9, 5.95
    r = bench.kernel_roofline(ev, "msv_fast_kernel", cells, ms, 18.612, 0.75, "msv", lds_bound=True)
    assert r["bound"] == "lds" and r["unit"] == "TB/s"
    assert r["achieved"] == pytest.approx(2.0 * cells / (ms * 1e-3) / 1e12, rel=1e-3)   # algorithmic bytes
    assert r["frac"] == pytest.approx(r["achieved"] / ev["lds_peak_tbs"], rel=1e-3)
    assert r["lds"]["measured_frac"] > r["frac"]                 # measured 2.31 B/cell > design 2.0
    assert r["alu"]["frac"] == pytest.approx(0.75 * cells / (ms * 1e-3) / 1e12 / 18.612, rel=1e-3)
    assert 1.0 < r["alu"]["executed_over_essential"] < 1.2
    json.dumps(r)


def test_kernel_roofline_viterbi_alu_bound():
    ev = bench.load_evidence()
    r = bench.kernel_roofline(ev, "vit_cpair2_kernel", 405e9, 188.0, 18.612, 4.25, "vit")
    assert r["bound"] == "alu" and 0.3 < r["frac"] < 1.0
    assert r["lds"]["bytes_per_cell"] > 0
    r2 = bench.kernel_roofline(ev, "no-such-kernel", 1e9, 1.0, 18.612, 0.75, "x", lds_bound=True)
    assert r2["bound"] == "alu" and "lds" not in r2          # no evidence: the live ALU fraction only


@pytest.mark.parametrize("cfg,stage,scaling", [(1, "pipeline", "weak"), (2, "msv", "weak"), (3, "pipeline", "weak"),
                                               (4, "vit", "strong"), (5, "pipeline", "strong")])
def test_config_defaults(cfg, stage, scaling):
    assert bench.STAGE_OF[cfg] == stage and bench.SCALING_OF[cfg] == scaling


@pytest.mark.parametrize("scaling,world,n", [("weak", 4, 1000), ("strong", 4, 1000), ("strong", 1, 1000)])
def test_workload_sharding(scaling, world, n):
    class A:
        config, which, nseq = 3, 0, n
    A.scaling = scaling
    c, prof, db = bench.workload(A, world)
    assert prof.M == 400
    assert db.N == (n * world if scaling == "weak" else n)


def test_bench_names_the_viterbi_kernel():
    """hmg_quant.vit_pair_kernel picks the evidence entry and the label of the Viterbi roofline."""
    for kind in range(1, 6):
        key, label = bench.vit_kernel({"vit_pair_kernel": kind, "vit_pair_lanes": 32, "vit_pair_regs": 32})
        assert key == bench.VIT_KERNELS[kind][0] and "32 lanes" in label
    assert bench.vit_kernel({"vit_pair_kernel": 0, "vit_pair_lanes": 0, "vit_pair_regs": 0})[0] == "-"
