"""MSV kernel time vs lane-group size G on the config-2 DB (550k Swiss-Prot-shaped sequences)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
_, db = synth.config(2)
dsq, off = db.materialize()
D = hmg.Database(dsq, off)
raw = torch.zeros(D.nseq, dtype=torch.uint8, device="cuda")
hmg.hmg_set_stage_timing(True)
Ms = [int(m) for m in sys.argv[1].split(",")] if len(sys.argv) > 1 else [64, 100, 200, 400, 500, 1000, 2048]
for M in Ms:
    prof = synth.make_profile(M, 1000 + M)
    for G in (4, 8, 16, 32):
        hmg.set_tuning("MSV_G", G)
        P = hmg.Profile(prof.msc)
        q = P.quant()
        if q["msv_lanes"] != G:
            continue
        ts = []
        for _ in range(4):
            hmg.hmg_msv(P, D, raw)
            ts.append(hmg.hmg_stage_times()["msv_kernel"])
        t = min(ts[1:])
        print(json.dumps({"M": M, "G": G, "Q": q["msv_regs"], "ms": round(t, 3),
                          "gcups": round(M * D.residues / t / 1e6, 1),
                          "cells_per_clk_sm": round(M * D.residues / (t * 1e-3) / 148 / 1.965e9, 1)}), flush=True)
        P.close()
