"""Forward stage on the Viterbi passes of BASELINE config 3 (the bench's Forward leg): lengths of
the Forward list and the stage time per geometry (tuning FWD_W / FWD_S).
usage: python tools/fwd_latency.py"""
import os, sys, json, subprocess
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth, dist as hdist

build.build()
prof, db = synth.config(3)
dsq, off = db.materialize()
D = hmg.Database(dsq, off)
P, ev = hmg.calibrated_profile(prof.msc, prof.tsc)
out = hmg.alloc_outputs(D.nseq)
fo = hmg.alloc_forward_outputs(D.nseq)
hmg.hmg_pipeline_forward(P, D, **out, **fo)
torch.cuda.synchronize()
nf = int(fo["n_fwd"].item())
ids = fo["fwd_ids"][:nf].clone()
L = D.lengths[ids.cpu().numpy()]
print(json.dumps({"n_fwd": nf, "residues": int(L.sum()), "top_lengths": sorted(L.tolist())[::-1][:12]}), flush=True)
res = torch.zeros(D.nseq, dtype=torch.float32, device="cuda")
hmg.hmg_set_stage_timing(True)
for W in (1, 2, 4, 8, 16):
    hmg.set_tuning("FWD_W", W)
    try:
        Pw = hmg.Profile(prof.msc, prof.tsc)
    except hmg.HmgError:
        continue
    q = Pw.quant()
    if q["fwd_warps"] != W:
        continue
    ts = []
    for _ in range(4):
        hmg.hmg_forward(Pw, D, res, ids=ids)
        ts.append(hmg.hmg_stage_times()["fwd"])
    t = min(ts)
    print(json.dumps({"W": W, "Q": q["fwd_nodes"], "S": q["fwd_seqs_per_block"], "ms": round(t, 4),
                      "gcups": round(prof.M * int(L.sum()) / t / 1e6, 1),
                      "us_per_row_longest": round(1e3 * t / int(L.max()), 4)}), flush=True)
