"""Block pair Viterbi kernel vs the s32 block kernel on the config-4 shape (M=2048 by default):
time per W (warps per sequence).  python tools/vit_cpair_sweep.py [N] [M]"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
N = int(sys.argv[1]) if len(sys.argv) > 1 else 50000
M = int(sys.argv[2]) if len(sys.argv) > 2 else 2048
db = synth.make_db(N, 5.60, 0.75, 12)
dsq, off = db.materialize()
D = hmg.Database(dsq, off)
prof = synth.make_profile(M, 1000 + M)
hmg.hmg_set_stage_timing(True)
ref = None
for mode in ("s32", "W2S2", "W2S4", "W4S1", "W4S3", "W8S1", "W8S2"):
    for k in ("NO_VIT_PAIR", "VIT_PAIR_W", "VIT_PAIR_SG", "VIT_CPAIR2"):
        hmg.clear_tuning(k)
    if mode == "s32":
        hmg.set_tuning("NO_VIT_PAIR", 1)
    else:
        w, sg = mode[1:].split("S")
        hmg.set_tuning("VIT_PAIR_W", int(w))
        hmg.set_tuning("VIT_PAIR_SG", int(sg))
    P = hmg.Profile(prof.msc, prof.tsc)
    q = P.quant()
    raw = torch.zeros(D.nseq, dtype=torch.int16, device="cuda")
    best = None
    for _ in range(3):
        hmg.hmg_viterbi(P, D, raw)
        t = hmg.hmg_stage_times()["vit_kernel"]
        c = hmg.hmg_stage_counts()["vit_pair_redo"]
        best = t if best is None else min(best, t)
    ref = raw.clone() if ref is None else ref
    print(json.dumps({"M": M, "mode": mode, "lanes": q["vit_pair_lanes"], "regs": q["vit_pair_regs"],
                      "ms": round(best, 3), "gcups": round(M * D.residues / best / 1e6, 1), "redo": c,
                      "same": bool(torch.equal(ref, raw))}), flush=True)
