"""Models of 513-1024 nodes: the lane-group pair kernel (vit_pair.cuh, the default there) vs the
one-warp kernel with the transitions in tensor / shared memory (vit_wide.cuh, forced with
VIT_PAIR_CTA + VIT_WIDE) -- time, GCUPS and identical outputs.
python tools/wide_mid_bench.py [N] M... > profiles/wide_mid_<tag>.jsonl"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
N = int(sys.argv[1]) if len(sys.argv) > 1 else 100000
Ms = [int(m) for m in sys.argv[2:]] or [600, 800, 1000]
db = synth.make_db(N, 5.60, 0.75, 12)
dsq, off = db.materialize()
D = hmg.Database(dsq, off)
hmg.hmg_set_stage_timing(True)
for M in Ms:
    prof = synth.make_profile(M, 1000 + M)
    ref = None
    for mode in ("default", "wide_tm", "wide"):
        hmg.clear_tuning()
        if mode != "default":
            hmg.set_tuning("VIT_PAIR_CTA", 1)
            hmg.set_tuning("VIT_WIDE", 2 if mode == "wide_tm" else 1)
        P = hmg.Profile(prof.msc, prof.tsc)
        q = P.quant()
        raw = torch.zeros(D.nseq, dtype=torch.int16, device="cuda")
        ts = []
        for _ in range(4):
            hmg.hmg_viterbi(P, D, raw)
            ts.append(hmg.hmg_stage_times()["vit_kernel"])
        best = min(ts[1:])
        ref = raw.clone() if ref is None else ref
        print(json.dumps({"M": M, "N": N, "mode": mode, "kernel": q["vit_pair_kernel"], "lanes": q["vit_pair_lanes"],
                          "regs": q["vit_pair_regs"], "ms": round(best, 3), "gcups": round(M * D.residues / best / 1e6, 1),
                          "same": bool(torch.equal(ref, raw))}), flush=True)
hmg.clear_tuning()
