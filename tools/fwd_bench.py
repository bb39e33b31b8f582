"""Forward-stage throughput (f2) on one GPU: hmg_forward over N sequences of a config-2-shaped
DB for each M, timed by the library's stage events (development aid and ncu target).
usage: python tools/fwd_bench.py [M,M,...] [nseq] [reps]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth

Ms = [int(m) for m in (sys.argv[1] if len(sys.argv) > 1 else "64,200,400,1000,2048").split(",")]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 100000
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
build.build()
db = synth.make_db(N, 5.60, 0.75, 12)
dsq, off = db.materialize()
D = hmg.Database(dsq, off)
out = torch.zeros(D.nseq, dtype=torch.float32, device="cuda")
hmg.hmg_set_stage_timing(True)
for M in Ms:
    prof = synth.make_profile(M, 1000 + M)
    P = hmg.Profile(prof.msc, prof.tsc)
    q = P.quant()
    ts = []
    for _ in range(reps):
        hmg.hmg_forward(P, D, out)
        ts.append(hmg.hmg_stage_times()["fwd"])
    t = min(ts)
    print(json.dumps({"M": M, "nseq": D.nseq, "residues": D.residues, "W": q["fwd_warps"], "Q": q["fwd_nodes"], "S": q["fwd_seqs_per_block"],
                      "rows_smem": q["fwd_rows_smem"], "ms": round(t, 3),
                      "gcups": round(M * D.residues / t / 1e6, 1)}), flush=True)
