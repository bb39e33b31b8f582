"""Per-row latency of one long sequence (a single warp alone on the GPU)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
rng = np.random.default_rng(0)
for M in (64, 200, 400):
    prof = synth.make_profile(M, 1000 + M)
    P = hmg.Profile(prof.msc, prof.tsc)
    for nseq in (1, 4):
        L = 30000
        dsq = rng.integers(0, 20, size=L * nseq).astype(np.uint8)
        off = np.arange(nseq + 1, dtype=np.int64) * L
        D = hmg.Database(dsq, off)
        raw = torch.zeros(nseq, dtype=torch.uint8, device="cuda")
        vraw = torch.zeros(nseq, dtype=torch.int16, device="cuda")
        hmg.hmg_set_stage_timing(True)
        res = {}
        for name, fn in (("msv", lambda: hmg.hmg_msv(P, D, raw)), ("vit", lambda: hmg.hmg_viterbi(P, D, vraw))):
            for _ in range(2):
                fn()
                st = hmg.hmg_stage_times()
            ms = st["msv_kernel"] if name == "msv" else st["vit_kernel"]
            res[name + "_ms"] = round(ms, 3)
            res[name + "_cycles_per_row"] = round(ms * 1e-3 * 1.965e9 / L, 1)
        print(json.dumps({"M": M, "nseq": nseq, "L": L, **res, "q": {k: v for k, v in P.quant().items() if k in ("msv_lanes", "msv_regs", "vit_lanes", "vit_nodes")}}))
