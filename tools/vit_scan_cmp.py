"""f1: pair Viterbi kernel with vote-terminated Lazy-F passes vs the max-plus scan, on typical
(D->D Dir(7,3)) and long-chain (Dir(1,9)) profiles.  python tools/vit_scan_cmp.py [N]"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
N = int(sys.argv[1]) if len(sys.argv) > 1 else 100000
db = synth.make_db(N, 5.60, 0.75, 12)
dsq, off = db.materialize()
D = hmg.Database(dsq, off)
hmg.hmg_set_stage_timing(True)
for M in (200, 400, 700, 1000):
    for dd in ((7.0, 3.0), (1.0, 9.0)):
        prof = synth.make_profile(M, 1000 + M, dd=dd)
        res = {"M": M, "dd": dd}
        outs = []
        for mode in ("passes", "scan"):
            if mode == "scan":
                hmg.set_tuning("VIT_SCAN", 1)
            P = hmg.Profile(prof.msc, prof.tsc)
            hmg.clear_tuning("VIT_SCAN")
            raw = torch.zeros(D.nseq, dtype=torch.int16, device="cuda")
            best = None
            for _ in range(3):
                hmg.hmg_viterbi(P, D, raw)
                t = hmg.hmg_stage_times()["vit_kernel"]
                best = t if best is None else min(best, t)
            outs.append(raw.clone())
            res[mode] = {"ms": round(best, 3), "gcups": round(M * D.residues / best / 1e6, 1)}
        res["identical"] = bool(torch.equal(outs[0], outs[1]))
        print(json.dumps(res), flush=True)
