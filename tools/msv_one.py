"""One MSV call on the config-2 DB for a given M (for ncu captures): python tools/msv_one.py M [reps]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
M = int(sys.argv[1])
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
_, db = synth.config(2)
dsq, off = db.materialize()
D = hmg.Database(dsq, off)
P = hmg.Profile(synth.make_profile(M, 1000 + M).msc)
raw = torch.zeros(D.nseq, dtype=torch.uint8, device="cuda")
for _ in range(reps):
    hmg.hmg_msv(P, D, raw)
torch.cuda.synchronize()
print("ok", P.quant()["msv_lanes"], P.quant()["msv_regs"])
