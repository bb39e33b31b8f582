"""Viterbi stage of config 3: time of the survivor list split by length (tail analysis)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth, dist as hdist
build.build()
prof, db = synth.config(3)
dsq, off = db.materialize()
P, ev = hmg.calibrated_profile(prof.msc, prof.tsc)
D = hmg.Database(dsq, off)
out = hmg.alloc_outputs(D.nseq)
hmg.hmg_pipeline(P, D, **out)
torch.cuda.synchronize()
ns = int(out["n_survivors"].item())
sv = out["survivor_ids"][:ns].cpu().numpy()
L = D.lengths[sv]
nlong, _ = D.long_lane()
print(json.dumps({"survivors": ns, "max_L": int(L.max()), "L>1500": int((L > 1500).sum()), "L>1000": int((L > 1000).sum()),
                  "L>2880": int((L > 2880).sum())}))
raw = torch.zeros(D.nseq, dtype=torch.int16, device="cuda")
hmg.hmg_set_stage_timing(True)
for cut in (10**9, 2880, 2000, 1500, 1000, 700):
    for side in ("short", "long"):
        ids = sv[L <= cut] if side == "short" else sv[L > cut]
        if len(ids) == 0:
            continue
        t = torch.as_tensor(ids, dtype=torch.int32, device="cuda")
        ts = []
        for _ in range(4):
            hmg.hmg_viterbi(P, D, raw, ids=t)
            ts.append(hmg.hmg_stage_times()["vit_kernel"])
        print(json.dumps({"cut": cut, "side": side, "n": len(ids), "residues": int(D.lengths[ids].sum()),
                          "ms": round(min(ts), 4), "Lmax": int(D.lengths[ids].max())}), flush=True)
