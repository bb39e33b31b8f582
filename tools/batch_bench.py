"""Many-profile MSV (f4) throughput: hmg_msv_batch vs one hmg_msv call per profile.
P Pfam-like profiles (M ~ lognormal, median 180, clipped to [20, 1500]) against a config-1-sized
DB (hmmscan-like: few targets, many models) and the config-2 DB (550k sequences).
usage: python tools/batch_bench.py [P] [reps]"""
import os, sys, json, math
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth

P = int(sys.argv[1]) if len(sys.argv) > 1 else 64
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
build.build()
rng = np.random.default_rng(11)
Ms = np.clip(np.round(rng.lognormal(math.log(180), 0.6, size=P)), 20, 1500).astype(int)
profs = [hmg.Profile(*(lambda p: (p.msc, p.tsc))(synth.make_profile(int(M), 6000 + i))) for i, M in enumerate(Ms)]
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def timed(fn):
    ts = []
    for _ in range(reps + 1):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return min(ts[1:])


for name, cfg in (("config1-db", 1), ("config2-db", 2)):
    _, dbs = synth.config(cfg)
    dsq, off = dbs.materialize()
    D = hmg.Database(dsq, off)
    raw = torch.zeros((P, D.nseq), dtype=torch.uint8, device="cuda")
    cells = int(Ms.sum()) * D.residues
    t_b = timed(lambda: hmg.hmg_msv_batch(profs, D, raw))
    def loop():
        for i, p in enumerate(profs):
            hmg.hmg_msv(p, D, raw[i])
    t_l = timed(loop)
    print(json.dumps({"db": name, "nseq": D.nseq, "residues": D.residues, "profiles": P,
                      "sum_M": int(Ms.sum()), "cells": cells, "batch_ms": round(t_b, 3),
                      "batch_gcups": round(cells / t_b / 1e6, 1), "loop_ms": round(t_l, 3),
                      "loop_gcups": round(cells / t_l / 1e6, 1), "speedup": round(t_l / t_b, 2)}), flush=True)

# Fig 1 pipeline for every profile (hmg_pipeline_batch) vs one hmg_pipeline call per profile
evs = [p.calibrate() for p in profs]
pprofs = [hmg.Profile(*(lambda q: (q.msc, q.tsc))(synth.make_profile(int(M), 6000 + i)), ev=evs[i])
          for i, M in enumerate(Ms)]
for name, cfg in (("config1-db", 1), ("config2-db", 2)):
    _, dbs = synth.config(cfg)
    dsq, off = dbs.materialize()
    D = hmg.Database(dsq, off)
    out = hmg.alloc_batch_outputs(P, D.nseq)
    ones = [hmg.alloc_outputs(D.nseq) for _ in range(min(P, 8))]
    cells = int(Ms.sum()) * D.residues
    t_b = timed(lambda: hmg.hmg_pipeline_batch(pprofs, D, **out))
    def loop():
        for i, p in enumerate(pprofs):
            hmg.hmg_pipeline(p, D, **ones[i % len(ones)])
    t_l = timed(loop)
    ns = out["n_survivors"].cpu().numpy()
    print(json.dumps({"pipeline": True, "db": name, "nseq": D.nseq, "profiles": P, "cells": cells,
                      "survivors_mean": float(ns.mean()), "batch_ms": round(t_b, 3),
                      "batch_gcups": round(cells / t_b / 1e6, 1), "loop_ms": round(t_l, 3),
                      "loop_gcups": round(cells / t_l / 1e6, 1), "speedup": round(t_l / t_b, 2)}), flush=True)
