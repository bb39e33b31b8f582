"""Quick stage timing of the pipeline on one GPU (development aid, not the bench contract).
usage: python tools/stage_bench.py [config] [reps]"""
import os, sys, time, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth, dist as hdist

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 3
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
build.build()
prof, db = synth.config(cfg)
t = time.time(); dsq, off = db.materialize(); tm = time.time() - t
P, ev = hmg.calibrated_profile(prof.msc, prof.tsc)
t = time.time(); D = hmg.Database(dsq, off); tp = time.time() - t
out = hmg.alloc_outputs(D.nseq)
M = prof.M
print(json.dumps({"config": cfg, "M": M, "nseq": D.nseq, "residues": D.residues, "materialize_s": round(tm, 2),
                  "pack_upload_s": round(tp, 2), "quant": {k: v for k, v in P.quant().items() if k in
                  ("bias_b", "msv_lanes", "msv_regs", "vit_lanes", "vit_nodes", "msv_fast")}}))
hmg.hmg_set_stage_timing(True)
for r in range(reps):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    hmg.hmg_pipeline(P, D, **out)
    b.record()
    st = hmg.hmg_stage_times()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b)
    ns = int(out["n_survivors"].item())
    sv = out["survivor_ids"][:ns].cpu().numpy()
    sres = int(D.lengths[sv].sum())
    st = {k: round(v, 3) for k, v in st.items()}
    print(json.dumps({"rep": r, "ms": round(ms, 3), "gcups": round(M * D.residues / ms / 1e6, 1),
                      "msv_gcups": round(M * D.residues / st["msv_kernel"] / 1e6, 1),
                      "vit_gcups": round(M * sres / max(st["vit_kernel"], 1e-9) / 1e6, 1),
                      "survivors": ns, "surv_Lmax": int(D.lengths[sv].max()) if ns else 0, **st}))
# MSV-only (config-2-like: all sequences, raw only)
raw = torch.zeros(D.nseq, dtype=torch.uint8, device="cuda")
for r in range(3):
    hmg.hmg_msv(P, D, raw)
    st = hmg.hmg_stage_times()
    print(json.dumps({"msv_only_ms": round(st["msv_kernel"], 3), "gcups": round(M * D.residues / st["msv_kernel"] / 1e6, 1)}))
