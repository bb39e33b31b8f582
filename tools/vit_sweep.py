"""Pair Viterbi kernel: time vs lane-group size G per model length (config-2-shaped DB, all
sequences).  python tools/vit_sweep.py [N] [M,M,...]"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
N = int(sys.argv[1]) if len(sys.argv) > 1 else 100000
Ms = [int(m) for m in sys.argv[2].split(",")] if len(sys.argv) > 2 else [64, 128, 200, 256, 400, 512, 700, 1000]
db = synth.make_db(N, 5.60, 0.75, 12)
dsq, off = db.materialize()
D = hmg.Database(dsq, off)
hmg.hmg_set_stage_timing(True)
for M in Ms:
    prof = synth.make_profile(M, 1000 + M)
    ref = None
    for G in (8, 16, 32):
        hmg.set_tuning("VIT_PAIR_G", G)
        P = hmg.Profile(prof.msc, prof.tsc)
        q = P.quant()
        raw = torch.zeros(D.nseq, dtype=torch.int16, device="cuda")
        best = None
        for _ in range(3):
            hmg.hmg_viterbi(P, D, raw)
            t = hmg.hmg_stage_times()["vit_kernel"]
            best = t if best is None else min(best, t)
        ref = raw.clone() if ref is None else ref
        print(json.dumps({"M": M, "G": q["vit_pair_lanes"], "Q": q["vit_pair_regs"], "ms": round(best, 3),
                          "gcups": round(M * D.residues / best / 1e6, 1), "same": bool(torch.equal(ref, raw))}),
              flush=True)
