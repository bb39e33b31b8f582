"""GCUPS of every BASELINE.json configuration on one GPU (development / evidence table).

config 1: M=64 vs 1000 sequences, MSV + Viterbi on all (latency-bound, parity case)
config 2: M=200 vs 550k Swiss-Prot-shaped sequences, MSV only
config 3: M=400 pipeline (MSV -> compaction -> Viterbi on survivors) on the config-2 DB + planted
config 4: M=2048 Viterbi filter (Lazy-F) over all 550k sequences
config 5: M=100/500/1000 pipeline on one rank's 1/8 snake shard of the 10M-sequence UniProt-shaped DB

usage: python tools/configs_bench.py [configs, e.g. 1,2,3,4,5] > profiles/configs_<tag>.jsonl
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_ipps_jiangg15_b200 import build, dist as hdist, hmg, synth

build.build()
hmg.hmg_set_stage_timing(True)
which = [int(c) for c in (sys.argv[1] if len(sys.argv) > 1 else "1,2,3,4,5").split(",")]
peaks = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                    "MEASURED_PEAKS.json"))) if os.path.exists("MEASURED_PEAKS.json") else {}
f_sm = float(peaks.get("sm_max_mhz", 1965.0)) * 1e6
P_INT = 64 * 148 * f_sm          # ALU-pipe lane-ops/s
msv_roof = P_INT / 0.75          # cells/s at 0.75 ALU ops per cell
vit_roof = P_INT / 4.25          # cells/s at 4.25 ALU ops per cell (s16x2 pair encoding, DESIGN 4.6)


def timed(fn, reps=3):
    ts, st = [], None
    for _ in range(reps + 1):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        st = hmg.hmg_stage_times()
        torch.cuda.synchronize()
        ts.append((a.elapsed_time(b), st))
    ts = ts[1:]
    best = min(ts, key=lambda t: t[0])
    return best


def report(cfg, M, D, ms, st, extra):
    cells = M * D.residues
    line = {"config": cfg, "M": M, "nseq": D.nseq, "residues": D.residues, "ms": round(ms, 3),
            "gcups": round(cells / ms / 1e6, 1)}
    if st.get("msv_kernel", -1) > 0:
        g = cells / (st["msv_kernel"] * 1e-3)
        line.update(msv_kernel_ms=round(st["msv_kernel"], 3), msv_gcups=round(g / 1e9, 1),
                    msv_roof_frac=round(g / msv_roof, 3))
    line.update(extra)
    line["stages_ms"] = {k: round(v, 3) for k, v in st.items() if v >= 0}
    print(json.dumps(line), flush=True)


def pipeline(cfg, prof, dsq, off):
    P, ev = hmg.calibrated_profile(prof.msc, prof.tsc)
    D = hmg.Database(dsq, off)
    out = hmg.alloc_outputs(D.nseq)
    ms, st = timed(lambda: hmg.hmg_pipeline(P, D, **out))
    ns = int(out["n_survivors"].item())
    sv = out["survivor_ids"][:ns].cpu().numpy()
    sres = int(D.lengths[sv].sum()) if ns else 0
    extra = {"survivors": ns, "survivor_frac": round(ns / D.nseq, 5)}
    if st.get("vit_kernel", -1) > 0 and sres:
        g = prof.M * sres / (st["vit_kernel"] * 1e-3)
        extra.update(vit_gcups=round(g / 1e9, 1), vit_roof_frac=round(g / vit_roof, 3))
    report(cfg, prof.M, D, ms, st, extra)


for cfg in which:
    t0 = time.time()
    if cfg == 1:
        prof, db = synth.config(1)
        dsq, off = db.materialize()
        P = hmg.Profile(prof.msc, prof.tsc)
        D = hmg.Database(dsq, off)
        raw = torch.zeros(D.nseq, dtype=torch.uint8, device="cuda")
        vraw = torch.zeros(D.nseq, dtype=torch.int16, device="cuda")
        ms, st = timed(lambda: hmg.hmg_msv(P, D, raw))
        report(1, 64, D, ms, st, {"stage": "msv_all"})
        ms, st = timed(lambda: hmg.hmg_viterbi(P, D, vraw))
        g = 64 * D.residues / (st["vit_kernel"] * 1e-3)
        report(1, 64, D, ms, st, {"stage": "viterbi_all", "vit_gcups": round(g / 1e9, 1),
                                  "vit_roof_frac": round(g / vit_roof, 3)})
    elif cfg == 2:
        prof, db = synth.config(2)
        dsq, off = db.materialize()
        P = hmg.Profile(prof.msc)
        D = hmg.Database(dsq, off)
        raw = torch.zeros(D.nseq, dtype=torch.uint8, device="cuda")
        ms, st = timed(lambda: hmg.hmg_msv(P, D, raw))
        report(2, 200, D, ms, st, {"stage": "msv_all"})
    elif cfg == 3:
        prof, db = synth.config(3)
        dsq, off = db.materialize()
        pipeline(3, prof, dsq, off)
    elif cfg == 4:
        prof, db = synth.config(4)
        dsq, off = db.materialize()
        P = hmg.Profile(prof.msc, prof.tsc)
        D = hmg.Database(dsq, off)
        vraw = torch.zeros(D.nseq, dtype=torch.int16, device="cuda")
        ms, st = timed(lambda: hmg.hmg_viterbi(P, D, vraw), reps=2)
        g = 2048 * D.residues / (st["vit_kernel"] * 1e-3)
        q = P.quant()
        report(4, 2048, D, ms, st, {"stage": "viterbi_all", "vit_gcups": round(g / 1e9, 1),
                                    "vit_roof_frac": round(g / vit_roof, 3),
                                    "kernel": ("vit_cpair_kernel<W=%d, Q=%d>" % (q["vit_pair_lanes"] // 32, q["vit_pair_regs"])
                                               if q["vit_pair_lanes"] else
                                               "vit_cta_kernel<%d,%d>" % (q["vit_lanes"] // 32, q["vit_nodes"]))})
    elif cfg == 5:
        c = synth.CONFIGS[5]
        L = synth.make_lengths(c["N"], c["mu_ln"], c["sigma"], c["dseed"])
        ids = hdist.snake_shard(L, 8, 0)
        db = synth.Database(L, c["dseed"])
        dsq, off = db.materialize(ids)
        for M, ps in zip(c["M"], c["pseed"]):
            pipeline("5/8-shard", synth.make_profile(M, ps), dsq, off)
    print(json.dumps({"config": cfg, "wall_s": round(time.time() - t0, 1)}), file=sys.stderr, flush=True)
