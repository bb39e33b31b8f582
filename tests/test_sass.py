"""SASS check of the hot kernels (north_star: "saturating add/max whose emulated-
versus-native cost is verified in SASS").  CPU-only: cuobjdump disassembles the sm_100a code of
libhmg.so here.  For every kernel of the measured path (BASELINE configs 2-5 and f4):

* the cell updates are native DPX: VIADDMNMX.S16x2 (saturating add + max of two 16-bit cells) in
  the unrolled row body, VIMNMX3.S16x2 for the row maximum;
* no emulated byte-SIMD: the compiler's __vmaxu4 / __vaddus4 / __vsubus4 emulation is built from
  LOP3 with the byte-lane masks 0x7f7f7f7f / 0x80808080 and PRMT sign spreads (0xba98) -- none may
  appear (the MSV int8 table's PRMT 0x9180 / 0xb3a2 widenings are one op per two cells, by design).
"""
import os
import re
import shutil
import subprocess

import pytest

from paper_conf_ipps_jiangg15_b200 import build

CUOBJDUMP = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"

# kernel (mangled) -> minimum static VIADDMNMX.S16x2 / VIMNMX3.S16x2 counts
KERNELS = {
    "_ZN3hmg18msv_fast_kernel_mbILi8ELi25ELi3EEEvNS_7MsvArgsE": (150, 60),      # config 3 MSV (M = 400, Q = 25)
    "_ZN3hmg15msv_fast_kernelILi8ELi13EEEvNS_7MsvArgsE": (60, 30),             # config 2 MSV (M = 200)
    "_ZN3hmg15vit_pair_kernelILi32ELi7ELb0EEEvNS_7VitArgsE": (40, 3),           # config 3 Viterbi stage
    "_ZN3hmg17vit_cpair2_kernelILi16ELi2ELi0EEEvNS_7VitArgsE": (120, 5),        # two-warp Viterbi (M <= 2048)
    "_ZN3hmg15vit_wide_kernelILi32ELb1EEEvNS_7VitArgsE": (300, 10),            # config 4 Viterbi (M = 2048, TMEM)
    "_ZN3hmg15vit_wide_kernelILi20ELb0EEEvNS_7VitArgsE": (300, 10),            # 1024 < M <= 1280 (shared memory)
    "_ZN3hmg19msv_multi_kernel_mbILi8ELi25ELi3EEEvNS_12MsvMultiArgsE": (100, 50),  # f4 batch MSV
    "_ZN3hmg22pipe_long_vpair_kernelILi7EEEvNS_8LongArgsE": (40, 3),           # config 3 long lane
}
EMULATION = [re.compile(r"LOP3\.LUT.*0x7f7f7f7f"), re.compile(r"LOP3\.LUT.*0x80808080"),
             re.compile(r"PRMT\s+R\d+, R\d+, 0xba98")]


@pytest.fixture(scope="module")
def lib_path():
    if not os.path.exists(CUOBJDUMP):
        pytest.skip("cuobjdump not available")
    return build.build()


def _sass(lib, fn):
    r = subprocess.run([CUOBJDUMP, "-sass", "-fun", fn, lib], capture_output=True, text=True)
    return [l for l in r.stdout.splitlines() if re.search(r"/\*[0-9a-f]{4,}\*/", l)]


@pytest.mark.parametrize("fn", sorted(KERNELS))
def test_hot_kernel_is_native_dpx(lib_path, fn):
    lines = _sass(lib_path, fn)
    assert lines, "kernel %s not found in libhmg.so" % fn
    add_max = sum("VIADDMNMX" in l and ".S16x2" in l for l in lines)
    max3 = sum("VIMNMX3.S16x2" in l for l in lines)
    lo, lo3 = KERNELS[fn]
    assert add_max >= lo, (fn, add_max)
    assert max3 >= lo3, (fn, max3)
    bad = [l.strip() for l in lines if any(p.search(l) for p in EMULATION)]
    assert not bad, bad[:5]


def test_wide_kernel_reads_transitions_from_tensor_memory(lib_path):
    """vit_wide_kernel<Q, true> streams the transition vectors with tcgen05.ld
    (SASS LDTM), two loads per chunk of four registers in the M / I sweep and one in the D chain,
    and allocates / frees its TMEM columns (UTCATOMSWS)."""
    lines = _sass(lib_path, "_ZN3hmg15vit_wide_kernelILi32ELb1EEEvNS_7VitArgsE")
    ldtm = sum("LDTM" in l for l in lines)
    assert ldtm >= 3 * 8, ldtm
    assert any("UTCATOMSWS" in l for l in lines)
    smem = _sass(lib_path, "_ZN3hmg15vit_wide_kernelILi32ELb0EEEvNS_7VitArgsE")
    assert not any("LDTM" in l for l in smem)
