"""Config-4 shape (M = 2048 by default): the two-warp Viterbi kernel without a per-row barrier
(vit_cpair2.cuh, SG sequences per block) vs the barrier kernel (vit_cpair.cuh) -- time, GCUPS and
identical outputs.  python tools/cpair2_bench.py [N] [M] > profiles/cpair2_<tag>.jsonl"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
N = int(sys.argv[1]) if len(sys.argv) > 1 else 100000
M = int(sys.argv[2]) if len(sys.argv) > 2 else 2048
db = synth.make_db(N, 5.60, 0.75, 12)
dsq, off = db.materialize()
D = hmg.Database(dsq, off)
prof = synth.make_profile(M, 1000 + M)
hmg.hmg_set_stage_timing(True)
ref = None
for sg in ("0", "2", "wide", "wide_tm"):
    hmg.clear_tuning()
    if sg in ("wide", "wide_tm"):
        hmg.set_tuning("VIT_WIDE", 1 if sg == "wide" else 2)
    else:
        hmg.set_tuning("VIT_WIDE", 0)
        hmg.set_tuning("VIT_CPAIR2", int(sg))
    P = hmg.Profile(prof.msc, prof.tsc)
    raw = torch.zeros(D.nseq, dtype=torch.int16, device="cuda")
    ts = []
    for _ in range(4):
        hmg.hmg_viterbi(P, D, raw)
        ts.append(hmg.hmg_stage_times()["vit_kernel"])
    best = min(ts[1:])
    ref = raw.clone() if ref is None else ref
    print(json.dumps({"M": M, "N": N, "kernel": "cpair (barrier)" if sg == "0" else "wide (one warp, smem)" if sg == "wide" else "wide (one warp, TMEM)" if sg == "wide_tm" else "cpair2 var=%s (10 TSM + SG)" % sg,
                      "ms": round(best, 3), "gcups": round(M * D.residues / best / 1e6, 1),
                      "redo": hmg.hmg_stage_counts()["vit_pair_redo"], "same": bool(torch.equal(ref, raw))}), flush=True)
