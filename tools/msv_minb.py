"""MSV kernel time per model length (config-2 DB, 200k sequences) for the current libhmg build."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
db = synth.make_db(200000, 5.60, 0.75, 12)
dsq, off = db.materialize()
D = hmg.Database(dsq, off)
raw = torch.zeros(D.nseq, dtype=torch.uint8, device="cuda")
hmg.hmg_set_stage_timing(True)
tag = sys.argv[1] if len(sys.argv) > 1 else ""
for M in (64, 100, 150, 200, 300, 400, 450, 500, 640, 700, 1000, 1500):
    prof = synth.make_profile(M, 1000 + M)
    P = hmg.Profile(prof.msc, prof.tsc)
    ts = []
    for _ in range(4):
        hmg.hmg_msv(P, D, raw)
        ts.append(hmg.hmg_stage_times()["msv_kernel"])
    q = P.quant()
    t = min(ts[1:])
    print(json.dumps({"tag": tag, "M": M, "G": q["msv_lanes"], "Q": q["msv_regs"], "ms": round(t, 4),
                      "gcups": round(M * D.residues / t / 1e6, 1)}), flush=True)
