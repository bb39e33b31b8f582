"""Static SASS opcode counts of the hot kernels in libhmg.so (cuobjdump -sass, sm_100a): the
native-DPX evidence tests/test_sass.py asserts, as a table.
usage: python tools/sass_static.py > profiles/sass_static_<tag>.md"""
import collections
import os
import re
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from tests.test_sass import EMULATION, KERNELS  # noqa: E402

from paper_conf_ipps_jiangg15_b200 import build  # noqa: E402

lib = build.build()
print("# static SASS of the hot kernels (cuobjdump -sass, sm_100a)\n")
print("| kernel | instructions | VIADDMNMX.S16x2 | VIMNMX3.S16x2 | VIMNMX.S16x2 | PRMT | LOP3 | emulated byte-SIMD |")
print("|---|---|---|---|---|---|---|---|")
for fn in sorted(KERNELS):
    out = subprocess.run(["cuobjdump", "-sass", "-fun", fn, lib], capture_output=True, text=True).stdout
    lines = [l for l in out.splitlines() if re.search(r"/\*[0-9a-f]{4,}\*/", l)]
    c = collections.Counter()
    for l in lines:
        m = re.search(r"\*/\s+(?:@!?U?P\w+\s+)?([A-Z0-9]+(?:\.[A-Za-z0-9]+)*)", l)
        if m:
            op = m.group(1)
            c[op.split(".")[0] + (".S16x2" if ".S16x2" in op else "")] += 1
    emu = sum(any(p.search(l) for p in EMULATION) for l in lines)
    print("| `%s` | %d | %d | %d | %d | %d | %d | %d |" % (fn, len(lines), c["VIADDMNMX.S16x2"], c["VIMNMX3.S16x2"],
                                                        c["VIMNMX.S16x2"], c["PRMT"], c["LOP3"], emu))
