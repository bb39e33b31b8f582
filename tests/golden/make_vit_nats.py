"""Writes tests/golden/vit_nats.json: Viterbi-filter raw score -> nats (SURVEY 8(c) c.3,
reading R14/R17: nats = (xC + move_w(L) - 12000) / scale_w - 3, HMMER 3.0's word score
system) at the lengths of SURVEY Appendix B.

Independent of oracle/ and of the CUDA library: it takes move_w(L) from the Appendix-B
table in closed_forms.json (itself the closed form -round(500/ln2 * ln(3/(L+3)))),
scale_w = float32(500/ln2) = 721.3475341796875 (Appendix B), and evaluates the
conversion in numpy float32 in the order c.3 writes it.  Run:
    python tests/golden/make_vit_nats.py
"""
import json
import math
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
g = json.load(open(os.path.join(HERE, "closed_forms.json")))
scale_w = np.float32(500.0 / math.log(2))
assert float(scale_w) == 721.3475341796875            # Appendix B
RAWS = [-32767, -30000, -20000, -12000, -5000, -1, 0, 1, 2500, 8671, 12000, 15329, 20000, 25000, 32266]
out = {"_source": "tests/golden/make_vit_nats.py: c.3 conversion (float32) with Appendix-B move_w(L), "
                  "scale_w = float32(500/ln2); raw -32768 -> -inf and 32767 -> +inf are the sentinels (R17)"}
for L, mv in g["move_w"].items():
    row = {}
    for r in RAWS:
        sc = (np.float32(r + mv) - np.float32(12000.0)) / scale_w
        row[str(r)] = round(float(np.float32(float(sc) - 3.0)), 6)
    out[L] = row
json.dump(out, open(os.path.join(HERE, "vit_nats.json"), "w"), indent=1)
print("wrote vit_nats.json:", len(out) - 1, "lengths x", len(RAWS), "raw scores")
