"""Per-row latency of the pipeline long lane's Viterbi: one long sequence that passes MSV (F1 = 1),
scored by hmg_pipeline (chunked MSV on the whole GPU, then the long-lane Viterbi on one warp).
usage: python tools/long_latency.py [L] [KNOB=V ...]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
L = int(sys.argv[1]) if len(sys.argv) > 1 else 30000
for kv in sys.argv[2:]:                      # tuning knobs NAME=V (hmg_set_tuning)
    k, v = kv.split("=")
    hmg.set_tuning(k, int(v))
rng = np.random.default_rng(0)
for M in (100, 400, 500):
    prof = synth.make_profile(M, 1000 + M)
    P = hmg.Profile(prof.msc, prof.tsc, ev=(-9.0, 0.6931, -8.0, 0.6931))
    # the long sequence plus enough short ones that the DB has a long lane (L > 8 x mean)
    lens = [L] + [200] * 2000
    dsq = np.concatenate([synth.random_dsq(rng, n) for n in lens]).astype(np.uint8)
    off = np.zeros(len(lens) + 1, np.int64)
    np.cumsum(lens, out=off[1:])
    D = hmg.Database(dsq, off)
    out = hmg.alloc_outputs(D.nseq)
    hmg.hmg_set_stage_timing(True)
    ts = []
    for r in range(4):
        hmg.hmg_pipeline(P, D, F1=1.0, F2=1.0, **out)
        st = hmg.hmg_stage_times()
        torch.cuda.synchronize()
        ts.append(st["msv_kernel"])
    ms = min(ts[1:])
    raw = torch.zeros(D.nseq, dtype=torch.uint8, device="cuda")
    tm = []
    for r in range(4):                       # MSV alone: chunked long-lane MSV (+ sequential fallback)
        hmg.hmg_msv(P, D, raw)
        st = hmg.hmg_stage_times()
        torch.cuda.synchronize()
        tm.append(st["msv_kernel"])
    msv_ms = min(tm[1:])
    print(json.dumps({"M": M, "L": L, "msv_stage_ms": round(ms, 3), "cycles_per_row": round(ms * 1e-3 * 1.965e9 / L, 1),
                      "msv_only_ms": round(msv_ms, 3), "msv_cycles_per_row": round(msv_ms * 1e-3 * 1.965e9 / L, 1),
                      "survivors": int(out["n_survivors"].item()), "long_lane": D.long_lane() if hasattr(D, "long_lane") else None}))
