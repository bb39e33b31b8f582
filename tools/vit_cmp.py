"""Viterbi-filter kernel comparison on a config-2-shaped DB (all sequences scored):
s16x2 pair kernel (+ s32 re-scoring) vs the s32 kernels alone, per model length.
python tools/vit_cmp.py [N] [M,M,...]"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
N = int(sys.argv[1]) if len(sys.argv) > 1 else 100000
Ms = [int(m) for m in sys.argv[2].split(",")] if len(sys.argv) > 2 else [64, 128, 200, 400, 512, 700, 1000]
db = synth.make_db(N, 5.60, 0.75, 12)
dsq, off = db.materialize()
D = hmg.Database(dsq, off)
hmg.hmg_set_stage_timing(True)
for M in Ms:
    prof = synth.make_profile(M, 1000 + M)
    res = {"M": M, "nseq": D.nseq, "residues": D.residues}
    outs = {}
    for mode in ("pair", "s32"):
        if mode == "s32":
            hmg.set_tuning("NO_VIT_PAIR", 1)
        P = hmg.Profile(prof.msc, prof.tsc)
        hmg.clear_tuning("NO_VIT_PAIR")
        q = P.quant()
        raw = torch.zeros(D.nseq, dtype=torch.int16, device="cuda")
        best = None
        for _ in range(3):
            hmg.hmg_viterbi(P, D, raw)
            st = hmg.hmg_stage_times()
            c = hmg.hmg_stage_counts()
            t = st["vit_kernel"]
            best = t if best is None else min(best, t)
        outs[mode] = raw.clone()
        res[mode] = {"ms": round(best, 3), "gcups": round(M * D.residues / best / 1e6, 1),
                     "geom": [q["vit_pair_lanes"], q["vit_pair_regs"]] if mode == "pair" else [q["vit_lanes"], q["vit_nodes"]],
                     "redo": c["vit_pair_redo"]}
    res["identical"] = bool(torch.equal(outs["pair"], outs["s32"]))
    print(json.dumps(res), flush=True)
