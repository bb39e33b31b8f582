#!/usr/bin/env python
"""Benchmark of the hmmsearch filter hot path on B200 (BASELINE.json metric:
MSV / P7Viterbi / pipeline GCUPS, fraction of the integer-SIMD roofline).

One step = one pass of the whole hot path over the workload:
MSV over every sequence -> pass flags -> on-device survivor compaction ->
Viterbi filter (Lazy-F) over the survivors -> (N > 1) NCCL gather of the
per-sequence results and survivor lists.  Workload (N=1): BASELINE config 3,
profile M=400 against the Swiss-Prot-shaped DB (550k sequences, mean length
~360, 0.1% planted homologs).  With N GPUs each rank holds a 550k-sequence
length-balanced shard of an N x 550k DB (weak scaling, the default).

Other BASELINE configs as the headline (each a bench line of its own):
    --config 2               MSV only (stage msv), M = 200
    --config 4               Viterbi filter only over every sequence (stage vit), M = 2048,
                             the 550k DB split over the N ranks (strong scaling)
    --config 5 --which k     pipeline, M = 100 / 500 / 1000, the 10 M-sequence UniProt-shaped
                             DB split over the N ranks (strong scaling)
    --scaling weak|strong    override: every rank a full DB / the config's DB split over ranks

    python bench.py [--gpus N --steps K --warmup W] [--impl reference]
    torchrun --nproc-per-node N bench.py --gpus N ...   (--gpus must equal WORLD_SIZE)

Prints ONE JSON line on rank 0.  --impl reference runs the CPU oracle (the
reference arm of this tier) on a bounded sample of the same workload.

The pipeline is captured once in a CUDA graph and replayed per timed step (--no-graph: eager).
Beside the 8(a) headline the line carries (N = 1): `e2e` (hmg_pipeline_upload: the packed DB
re-sent from pinned host memory, overlapped with the filter, plus the D2H of the results),
`forward` (Fig 1 with the Forward stage, with its FP32 roofline), `batch` (the
f4 many-profile leg), `configs` (BASELINE configs 2, 4 and the config-5 shards, stage GCUPS and
roofline fractions), `cpu_baseline` (the oracle on the host cores) and `roofline` (the dominant
kernel: ALU fraction on essential ops, shared-memory fraction, executed/essential op ratio from the
committed SASS mix, DRAM traffic from the committed ncu capture).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "MSV / P7Viterbi / pipeline GCUPS at 1/2/4/8 B200; fraction of int-SIMD roofline"
ALU_LANES_PER_CLK_SM = 64        # measured: VIADDMNMX/VIMNMX3 issue at 64 lanes/clk/SM (profiles/intpeak)
MSV_ALU_OPS_PER_CELL = 0.75      # VIADDMNMX.S16x2 (1 per 2 cells) + VIMNMX3.S16x2 (1 per 4 cells)
VIT_ALU_OPS_PER_CELL = 4.25      # s16x2 pair kernel: M 4, I 2, D 2, R 1/2 per cell pair
FP32_LANES_PER_CLK_SM = 128      # B200 FP32 FMA lanes per SM per clock (4 SMSPs x 32)
FWD_FLOPS_PER_CELL = 16          # Forward recurrence: M 4 mul + 3 add + 1 mul, I 2 mul + 1 add,
                                 # D 2 mul + 1 add, E 2 add


def load_traffic(kernel):
    try:
        t = json.load(open(os.path.join(ROOT, "profiles", "traffic_r01.json")))[kernel]
        return t["bytes"], t["source"]
    except Exception:
        return None, None


def load_evidence():
    try:
        return json.load(open(os.path.join(ROOT, "profiles", "kernel_evidence_r02.json")))
    except Exception:
        return {}


STAGE_OF = {1: "pipeline", 2: "msv", 3: "pipeline", 4: "vit", 5: "pipeline"}
# hmg_quant.vit_pair_kernel -> (evidence key in profiles/kernel_evidence_r02.json, kernel name)
VIT_KERNELS = {1: ("vit_pair_kernel", "vit_pair_kernel"), 2: ("vit_cpair_kernel", "vit_cpair_kernel"),
               3: ("vit_cpair2_kernel", "vit_cpair2_kernel"), 4: ("vit_wide_kernel_smem", "vit_wide_kernel<Q,0>"),
               5: ("vit_wide_kernel", "vit_wide_kernel<Q,1> (TMEM transitions)")}


def vit_kernel(q):
    key, name = VIT_KERNELS.get(q["vit_pair_kernel"], ("-", "s32 Viterbi kernel"))
    return key, "%s, %d lanes x %d registers" % (name, q["vit_pair_lanes"], q["vit_pair_regs"])
SCALING_OF = {1: "weak", 2: "weak", 3: "weak", 4: "strong", 5: "strong"}


def env_rank():
    return (int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)),
            int(os.environ.get("LOCAL_RANK", 0)))


def load_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu):
        self.gpu = gpu
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), "--query-gpu=" + self.Q,
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            t0 = time.time()                       # nvidia-smi takes ~0.5 s to start: wait until it
            while not self.rows and time.time() - t0 < 5.0:   # samples, so the region is covered
                time.sleep(0.01)
        except Exception:
            self.proc = None
        self.n0 = max(len(self.rows) - 1, 0)      # the latest pre-region sample onwards
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        rows = self.rows[getattr(self, "n0", 0):]
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({n for r in rows for n, v in zip(names, r[5:9]) if v.strip().lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


def workload(args, world):
    """(config dict, profile, global DB).  Weak scaling: every rank holds args.nseq (default the
    config's N) sequences of an N x larger DB; strong: the config's DB split over the ranks."""
    from paper_conf_ipps_jiangg15_b200 import synth
    c = dict(synth.CONFIGS[args.config])
    if isinstance(c["M"], tuple):
        c["M"], c["pseed"] = c["M"][args.which], c["pseed"][args.which]
    n_rank = args.nseq or c["N"]
    n_glob = n_rank * world if args.scaling == "weak" else n_rank
    prof = synth.make_profile(c["M"], c["pseed"])
    db = synth.make_db(n_glob, c["mu_ln"], c["sigma"], c["dseed"], planted=c["planted"], profile=prof)
    return c, prof, db


# ------------------------------------------------------------------------------------------ reference
def run_reference(args):
    """The oracle (reference arm of this tier), timed on the host cores on a bounded
    sample of the same workload and stage: pipeline = MSV on every sampled sequence and Viterbi
    on its MSV survivors; msv = MSV only; vit = Viterbi on every sampled sequence."""
    rank, world, _ = env_rank()
    if rank != 0:
        return
    import oracle
    c, prof, db = workload(args, 1)
    oracle.build()
    mp, vp = oracle.MSVProfile(prof.msc), oracle.VitProfile(prof.msc, prof.tsc)
    ev = oracle_calibrate(oracle, prof)
    rng = np.random.default_rng(0)
    ncores = os.cpu_count() or 1
    nsamp = args.ref_sample if args.stage != "vit" else max(200, args.ref_sample * 64 // c["M"] // 4)
    times, cells = [], []
    for step in range(args.warmup + args.steps):
        ids = np.sort(rng.choice(db.N, size=min(nsamp, db.N), replace=False))
        dsq, off = db.materialize(ids)
        lens = np.diff(off)
        t0 = time.perf_counter()
        if args.stage in ("pipeline", "msv"):
            m = oracle.msv_db(mp, dsq, off, nthreads=ncores)
        if args.stage == "pipeline":
            sv = np.array([j for j, (r, L) in enumerate(zip(m, lens))
                           if oracle.msv_pass(int(r), int(L), ev[0], ev[1], args.F1)], dtype=np.int64)
            if len(sv):
                oracle.vit_db(vp, dsq, off, ids=sv, nthreads=ncores)
        if args.stage == "vit":
            oracle.vit_db(vp, dsq, off, nthreads=ncores)
        t = time.perf_counter() - t0
        if step >= args.warmup:
            times.append(t)
            cells.append(c["M"] * int(lens.sum()))
    v = sum(cells) / sum(times) / 1e9
    what = {"pipeline": "MSV all, Viterbi on MSV survivors", "msv": "MSV all", "vit": "Viterbi all"}[args.stage]
    line = {"impl": "reference", "metric": METRIC, "value": round(v, 4), "unit": "GCUPS", "n_gpus": 0,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(1e3 * sum(times) / len(times), 3),
            "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "u8/s16",
            "data": "synthetic",
            "config": {"workload": "config%d sample (stage %s)" % (args.config, args.stage), "M": c["M"],
                       "sample_seqs": int(min(nsamp, db.N))},
            "cpu_baseline": {"value": round(v, 4), "unit": "GCUPS", "cores": ncores, "kind": "oracle",
                             "sample": "%d random sequences per step of the config-%d DB (%s)"
                                       % (min(nsamp, db.N), args.config, what)},
            "e2e": {"value": round(v, 4), "unit": "GCUPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def oracle_calibrate(oracle, prof, n=1000, L=200):
    from paper_conf_ipps_jiangg15_b200 import synth
    cal = synth.Database(np.full(n, L, np.int32), seed=7)
    dsq, off = cal.materialize()
    lam = math.log(2)
    mb = [oracle.bits(oracle.msv_nats(int(r), L), L) for r in oracle.msv_db(oracle.MSVProfile(prof.msc), dsq, off)]
    vb = [oracle.bits(oracle.vit_nats(int(r), L), L)
          for r in oracle.vit_db(oracle.VitProfile(prof.msc, prof.tsc), dsq, off)]
    return (oracle.fit_mu(np.array(mb), lam), lam, oracle.fit_mu(np.array(vb), lam), lam)


def cpu_baseline(prof, dsq, off, ev, F1, M, sample_every, stage="pipeline"):
    """Oracle as it stands on this box's host cores, on a bounded sample (every k-th sequence),
    same stage as the headline (pipeline: MSV on all + Viterbi on MSV survivors)."""
    import oracle
    oracle.build()
    mp, vp = oracle.MSVProfile(prof.msc), oracle.VitProfile(prof.msc, prof.tsc)
    n = len(off) - 1
    ids = np.arange(0, n, sample_every, dtype=np.int64)
    ncores = os.cpu_count() or 1
    lens = (off[ids + 1] - off[ids])
    t0 = time.perf_counter()
    sv = np.zeros(0, np.int64)
    if stage in ("pipeline", "msv"):
        m = oracle.msv_db(mp, dsq, off, ids=ids, nthreads=ncores)
    if stage == "pipeline":
        sv = np.array([s for s, r, L in zip(ids, m, lens) if oracle.msv_pass(int(r), int(L), ev[0], ev[1], F1)],
                      dtype=np.int64)
        if len(sv):
            oracle.vit_db(vp, dsq, off, ids=sv, nthreads=ncores)
    if stage == "vit":
        oracle.vit_db(vp, dsq, off, ids=ids, nthreads=ncores)
    t = time.perf_counter() - t0
    what = {"pipeline": "MSV on all, Viterbi on %d MSV survivors" % len(sv), "msv": "MSV on all",
            "vit": "Viterbi on all"}[stage]
    return {"value": round(M * int(lens.sum()) / t / 1e9, 4), "unit": "GCUPS", "cores": ncores, "kind": "oracle",
            "sample": "every %d-th sequence of rank 0's shard (%d seqs, %d residues): %s; %.1f s"
                      % (sample_every, len(ids), int(lens.sum()), what, t)}


def alu_peak(nsm, f_hz):
    """ALU-pipe peak in T lane-ops/s: 64 lanes/clk/SM (VIADDMNMX / VIMNMX3, profiles/intpeak_r01.txt)."""
    return ALU_LANES_PER_CLK_SM * nsm * f_hz / 1e12


def kernel_roofline(ev, key, cells, ms, p_int, ops_per_cell, label, lds_bound=False):
    """Roofline of one kernel launch from its live time.  Two resources bound these kernels
    (DESIGN.md 4.2, 4.3c): the ALU pipe (DPX ops, 64 lanes/clk/SM) and the shared-memory data
    path (LDS, 37.1 TB/s measured).  `bound` names the one ncu shows busiest for the kernel
    (lds_bound: the MSV kernel, L1 99% vs ALU 84%, profiles/ncu_full_r02zo.md); `achieved` is ALGORITHMIC work per launch
    (design bytes or essential ops per cell x cells) / live time.  Both resources are reported,
    each with the measured counterpart from the committed ncu capture / SASS mix."""
    e = ev.get(key, {})
    alu = ops_per_cell * cells / (ms * 1e-3) / 1e12
    a = {"achieved": round(alu, 3), "peak": round(p_int, 3), "unit": "T int-lane-ops/s",
         "frac": round(alu / p_int, 4), "essential_ops_per_cell": ops_per_cell}
    if "executed_dpx_ops_per_cell" in e:
        a["executed_ops_per_cell"] = e["executed_dpx_ops_per_cell"]
        a["executed_over_essential"] = round(e["executed_dpx_ops_per_cell"] / ops_per_cell, 3)
        a["executed_frac"] = round(alu * e["executed_dpx_ops_per_cell"] / ops_per_cell / p_int, 4)
        a["executed_lane_instructions_per_cell"] = e.get("executed_lane_instructions_per_cell")
        a["mix_source"] = e.get("mix_source")
    lds = None
    if "lds_bytes_per_cell" in e:
        design = e.get("lds_bytes_per_cell_design", e["lds_bytes_per_cell"])
        la = design * cells / (ms * 1e-3) / 1e12
        lm = e["lds_bytes_per_cell"] * cells / (ms * 1e-3) / 1e12
        lds = {"achieved": round(la, 3), "peak": ev.get("lds_peak_tbs"), "unit": "TB/s",
               "frac": round(la / ev["lds_peak_tbs"], 4), "bytes_per_cell": design,
               "measured_bytes_per_cell": e["lds_bytes_per_cell"],
               "measured_frac": round(lm / ev["lds_peak_tbs"], 4), "peak_source": ev.get("lds_peak_source")}
        for k_src, k_dst in (("lds_bytes_per_cell_source", "measured_source"), ("lds_design_note", "note")):
            if k_src in e:
                lds[k_dst] = e[k_src]
    if lds_bound and lds:
        r = {"bound": "lds", "kernel": label, "achieved": lds["achieved"], "peak": lds["peak"], "unit": "TB/s",
             "frac": lds["frac"], "algorithmic_bytes_per_cell": lds["bytes_per_cell"], "lds": lds, "alu": a}
    else:
        r = {"bound": "alu", "kernel": label, "achieved": a["achieved"], "peak": a["peak"], "unit": a["unit"],
             "frac": a["frac"], "essential_alu_ops_per_cell": ops_per_cell, "alu": a}
        if lds:
            r["lds"] = lds
    r.update({"kernel_cells": int(cells), "kernel_ms": round(ms, 4), "pipes": e.get("ncu_pipes")})
    return r


def timed_ms(fn, stream, flush, reps):
    """Mean device time of fn() over reps calls (CUDA events on the launching stream, L2 flushed
    before each call outside the events), after one untimed call."""
    import torch
    ts = []
    for i in range(reps + 1):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        fn()
        b.record(stream)
        b.synchronize()
        if i:
            ts.append(a.elapsed_time(b))
    return statistics.mean(ts)


def configs_leg(args, dev, stream, flush, p_int, ev_file):
    """The other BASELINE configs on this GPU, each a short timed run of its own stage:
    config 2 (MSV only, M = 200, the 550k DB), config 4 (Viterbi filter over every sequence,
    M = 2048, the same DB) and config 5 (pipeline, M = 100 / 500 / 1000, one rank's 1/8 snake
    shard of the 10 M-sequence DB).  Stage times from the library's events."""
    import torch

    from paper_conf_ipps_jiangg15_b200 import dist as hdist
    from paper_conf_ipps_jiangg15_b200 import hmg, synth
    out = []
    c2 = synth.CONFIGS[2]
    db2 = synth.make_db(c2["N"], c2["mu_ln"], c2["sigma"], c2["dseed"])
    D2 = hmg.Database(*db2.materialize(), device=dev.index)
    hmg.hmg_set_stage_timing(True)
    try:
        for cfg in (2, 4):
            c = synth.CONFIGS[cfg]
            prof = synth.make_profile(c["M"], c["pseed"])
            P = hmg.Profile(prof.msc, prof.tsc, device=dev.index)
            P = hmg.Profile(prof.msc, prof.tsc, ev=P.calibrate(), device=dev.index)
            n = D2.nseq
            if cfg == 2:
                raw = torch.empty(n, dtype=torch.uint8, device=dev)
                pas = torch.empty(n, dtype=torch.uint8, device=dev)
                fn = lambda: hmg.hmg_msv(P, D2, raw, pas, F1=args.F1, stream=stream)
                key, ops, stage = "msv_fast_kernel<8,13>", MSV_ALU_OPS_PER_CELL, "msv_kernel"   # no mix: ALU only
            else:
                raw = torch.empty(n, dtype=torch.int16, device=dev)
                pas = torch.empty(n, dtype=torch.uint8, device=dev)
                fn = lambda: hmg.hmg_viterbi(P, D2, raw, pass_=pas, F2=args.F2, stream=stream)
                key, ops, stage = None, VIT_ALU_OPS_PER_CELL, "vit_kernel"
            ms = timed_ms(fn, stream, flush, 3 if cfg == 2 else 2)
            kms = hmg.hmg_stage_times()[stage]
            cells = c["M"] * D2.residues
            q = P.quant()
            if key is None:
                key, vlabel = vit_kernel(q)
            out.append({"config": cfg, "stage": "msv" if cfg == 2 else "vit", "M": c["M"], "nseq": n,
                        "residues": D2.residues, "ms": round(ms, 3), "gcups": round(cells / ms / 1e6, 1),
                        "kernel_ms": round(kms, 3), "kernel_gcups": round(cells / kms / 1e6, 1),
                        "roofline": kernel_roofline(ev_file, key, cells, kms, p_int, ops,
                                                    ("msv_fast_kernel G=%d Q=%d" % (q["msv_lanes"], q["msv_regs"]))
                                                    if cfg == 2 else vlabel)})
            print("configs leg: config %d %.3f ms" % (cfg, ms), file=sys.stderr, flush=True)
        del D2
        c5 = synth.CONFIGS[5]
        db5 = synth.make_db(c5["N"], c5["mu_ln"], c5["sigma"], c5["dseed"])
        ids = hdist.snake_shard(db5.lengths, 8, 0)
        D5 = hmg.Database(*db5.materialize(ids), device=dev.index)
        o = hmg.alloc_outputs(D5.nseq, dev.index)
        for k, (M, ps) in enumerate(zip(c5["M"], c5["pseed"])):
            prof = synth.make_profile(M, ps)
            P = hmg.Profile(prof.msc, prof.tsc, device=dev.index)
            P = hmg.Profile(prof.msc, prof.tsc, ev=P.calibrate(), device=dev.index)
            fn = lambda: hmg.hmg_pipeline(P, D5, F1=args.F1, F2=args.F2, stream=stream, **o)
            ms = timed_ms(fn, stream, flush, 3)
            st = hmg.hmg_stage_times()
            ns = int(o["n_survivors"].item())
            sres = int(D5.lengths[o["survivor_ids"][:ns].cpu().numpy()].sum()) if ns else 0
            cells = M * D5.residues
            out.append({"config": 5, "which": k, "stage": "pipeline", "M": M, "nseq": D5.nseq,
                        "residues": D5.residues, "shard": "rank 0 of 8 (snake) of the 10 M-sequence DB",
                        "ms": round(ms, 3), "gcups": round(cells / ms / 1e6, 1),
                        "msv_kernel_ms": round(st["msv_kernel"], 3),
                        "msv_gcups": round(cells / st["msv_kernel"] / 1e6, 1),
                        "msv_alu_frac": round(MSV_ALU_OPS_PER_CELL * cells / (st["msv_kernel"] * 1e-3) / 1e12 / p_int, 4),
                        "vit_kernel_ms": round(st["vit_kernel"], 3), "survivors": ns,
                        "vit_gcups": round(M * sres / st["vit_kernel"] / 1e6, 1) if st["vit_kernel"] > 0 else None})
            print("configs leg: config 5/%d %.3f ms" % (k, ms), file=sys.stderr, flush=True)
    finally:
        hmg.hmg_set_stage_timing(False)
    return out


# ------------------------------------------------------------------------------------------ main arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="hmg", choices=["hmg", "reference"])
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--which", type=int, default=0, help="profile index for config 5")
    ap.add_argument("--stage", default=None, choices=["pipeline", "msv", "vit"],
                    help="default: the config's (2 msv, 4 vit, else pipeline)")
    ap.add_argument("--scaling", default=None, choices=["weak", "strong"],
                    help="default: weak for configs 1-3, strong for 4 and 5")
    ap.add_argument("--nseq", type=int, default=0, help="sequences per rank (weak) / in all (strong)")
    ap.add_argument("--F1", type=float, default=0.02)
    ap.add_argument("--F2", type=float, default=1e-3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-forward", action="store_true")
    ap.add_argument("--no-configs", action="store_true", help="skip the configs 2/4/5 leg (N = 1)")
    ap.add_argument("--no-graph", action="store_true", help="launch the step eagerly in the timed region")
    ap.add_argument("--batch", type=int, default=64, help="profiles of the f4 batch leg (0 = skip)")
    ap.add_argument("--cpu-sample-every", type=int, default=0, help="default: 1 (pipeline, msv), 23 (vit)")
    ap.add_argument("--ref-sample", type=int, default=100000)
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo + --one-device: exercise the N > 1 path with every rank on cuda:0 (tests only)")
    ap.add_argument("--one-device", action="store_true", help="every rank on cuda:0 (tests of the N > 1 path)")
    ap.add_argument("--tune", action="append", default=[], metavar="NAME=V",
                    help="libhmg performance knob (hmg_set_tuning; sweeps only, results never depend on it)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    args.stage = args.stage or STAGE_OF[args.config]
    args.scaling = args.scaling or SCALING_OF[args.config]
    if not args.cpu_sample_every:
        args.cpu_sample_every = 23 if args.stage == "vit" else 1   # ~6-10 s of oracle work on 16 cores

    rank, world, local = env_rank()
    if args.one_device:
        local = 0
    if args.gpus != world and not (args.impl == "reference" and world == 1):
        sys.exit("bench.py: --gpus %d but WORLD_SIZE %d (launch N > 1 with torchrun, one process per GPU)"
                 % (args.gpus, world))
    if args.impl == "reference":
        run_reference(args)
        return

    import torch
    import torch.distributed as dist

    from paper_conf_ipps_jiangg15_b200 import build, hmg
    from paper_conf_ipps_jiangg15_b200 import dist as hdist

    if world > 1:
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group("gloo")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if rank == 0:
        build.build()
    if world > 1:
        dist.barrier()
    hmg.lib()
    for kv in args.tune:
        k, v = kv.split("=")
        hmg.set_tuning(k, int(v))

    c, prof, gdb = workload(args, world)
    M = c["M"]
    ids = hdist.snake_shard(gdb.lengths, world, rank)
    dsq, off = gdb.materialize(ids)
    P0 = hmg.Profile(prof.msc, prof.tsc, device=local)
    ev = P0.calibrate()                               # hmg_calibrate: mu of both filters on the GPU
    P0.close()
    P = hmg.Profile(prof.msc, prof.tsc, ev=ev, device=local)
    D = hmg.Database(dsq, off, device=local)
    n = D.nseq
    res_local = D.residues
    out = hmg.alloc_outputs(n, local)
    vraw = torch.zeros(n, dtype=torch.int16, device=dev) if args.stage == "vit" else out["vit_raw"]
    gids = torch.as_tensor(ids, device=dev)
    gather = hdist.Gatherer(gdb.N, world, gids, stage_host=args.backend == "gloo") if world > 1 else None
    stream = torch.cuda.current_stream()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)   # > 126 MB L2

    def run_stage(st):
        if args.stage == "pipeline":
            hmg.hmg_pipeline(P, D, F1=args.F1, F2=args.F2, stream=st, **out)
        elif args.stage == "msv":
            hmg.hmg_msv(P, D, out["msv_raw"], out["flags"], F1=args.F1, stream=st)
        else:
            hmg.hmg_viterbi(P, D, vraw, pass_=out["flags"], F2=args.F2, stream=st)

    def gather_step():
        if gather is not None:
            gather(out["msv_raw"], vraw, out["flags"], out["survivor_ids"], out["n_survivors"])

    for _ in range(args.warmup):                       # eager warm-up (threshold tables, module load)
        run_stage(stream)
        gather_step()
    torch.cuda.synchronize()

    # The stage is captured once in a CUDA graph (its launches, scratch allocation and memsets
    # become one graph launch: no host launch gaps between the stages); the NCCL gather stays eager.
    graph, launches_per_step = None, None
    if not args.no_graph:
        graph = torch.cuda.CUDAGraph()
        n0 = hmg.hmg_kernel_launches()
        with torch.cuda.graph(graph, capture_error_mode="thread_local"):
            run_stage(torch.cuda.current_stream())
        launches_per_step = hmg.hmg_kernel_launches() - n0

    def step():
        if graph is not None:
            graph.replay()
        else:
            run_stage(stream)
        gather_step()

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    # ---------------------------------------------------------------- timed region (device-resident inputs)
    launches0 = hmg.hmg_kernel_launches()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        for i in range(args.steps):
            flush.zero_()                              # L2 flush between timed steps (outside the events)
            evs[i][0].record(stream)
            step()
            evs[i][1].record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches = hmg.hmg_kernel_launches() - launches0
    if graph is not None:
        launches += launches_per_step * args.steps     # graph replays launch the captured kernels
    # stage times: the same stage eagerly, with the library's stage events (not in the timed region)
    hmg.hmg_set_stage_timing(True)
    stages = []
    for i in range(args.steps):
        flush.zero_()
        run_stage(stream)
        stages.append(hmg.hmg_stage_times())           # waits for this call's last stage event
        redo = hmg.hmg_stage_counts()["vit_pair_redo"]
    hmg.hmg_set_stage_timing(False)
    if graph is not None:
        graph.replay()                                 # leave the outputs of a timed-path step
    torch.cuda.synchronize()
    ms = [a.elapsed_time(b) for a, b in evs]
    t_step = sum(ms) / len(ms)
    rdev = dev if args.backend == "nccl" else torch.device("cpu")        # gloo tests: host reductions
    t_max = torch.tensor([t_step], dtype=torch.float64, device=rdev)
    if world > 1:
        dist.all_reduce(t_max, op=dist.ReduceOp.MAX)
    t_step = float(t_max.item())

    if args.stage == "pipeline":
        ns = int(out["n_survivors"].item())
        surv = out["survivor_ids"][:ns].cpu().numpy()
        surv_res = int(D.lengths[surv].sum()) if ns else 0
    else:
        ns, surv_res = (n, res_local) if args.stage == "vit" else (0, 0)
    tot = torch.tensor([res_local, surv_res, ns, n], dtype=torch.float64, device=rdev)
    if world > 1:
        dist.all_reduce(tot)
    res_all, surv_all, ns_all, n_all = [float(x) for x in tot.tolist()]
    cells_all = M * res_all
    value = cells_all / (t_step * 1e-3) / 1e9

    st = {k: statistics.mean([s[k] for s in stages]) for k in stages[0]}
    msv_ms, vit_ms = st["msv_kernel"], st["vit_kernel"]
    nlong, res_long = D.long_lane()            # long lane: runs concurrently inside the MSV stage
    msv_gcups = M * res_local / (msv_ms * 1e-3) / 1e9 if msv_ms > 0 else None
    vit_gcups = (M * surv_res / (vit_ms * 1e-3) / 1e9) if vit_ms > 0 else None
    peaks, src = load_peaks()
    clock = clk.summary()
    f_peak = float(peaks.get("sm_max_mhz", 1965.0)) * 1e6
    nsm = torch.cuda.get_device_properties(dev).multi_processor_count
    p_int = alu_peak(nsm, f_peak)
    evf = load_evidence()
    q = P.quant()
    if args.stage == "vit":
        vkey, vlabel = vit_kernel(q)
        roofline = kernel_roofline(evf, vkey, M * surv_res, vit_ms, p_int, VIT_ALU_OPS_PER_CELL, vlabel)
        roofline["kernel_share_of_step"] = round(vit_ms / t_step, 4)
    else:
        roofline = kernel_roofline(evf, "msv_fast_kernel", M * res_local, msv_ms, p_int, MSV_ALU_OPS_PER_CELL,
                                   "msv_fast_kernel (+ concurrent long lane, one MSV stage)", lds_bound=True)
        roofline["kernel_share_of_step"] = round(msv_ms / t_step, 4)
        roofline["long_lane"] = {"sequences": nlong, "residues": res_long}
        # SURVEY 8(d)'s literal MSV roofline, P_int / 2 cells/s (2 lane-ops per cell), is exceeded:
        # those op counts were not lower bounds
        roofline["survey_8d_msv_roofline_gcups"] = round(p_int * 1e12 / 2 / 1e9, 1)
        roofline["survey_8d_msv_ratio"] = round(msv_gcups * 1e9 / (p_int * 1e12 / 2), 3) if msv_gcups else None
    roofline["alu"]["peak_source"] = "%s sm_max_mhz x %d SMs x %d lanes/clk (ALU pipe, measured profiles/intpeak_r01.txt)" \
                                     % (src, nsm, ALU_LANES_PER_CLK_SM)
    # DRAM traffic of the captured launch: only for the workloads the ncu captures ran (config 3's
    # MSV kernel, config 4's Viterbi kernel); other workloads report null
    ek = evf.get(vit_kernel(q)[0] if args.stage == "vit" and args.config == 4
                 else "msv_fast_kernel" if args.stage != "vit" and args.config == 3 else "-", {})
    tb, tsrc = ek.get("dram_bytes_per_launch"), ek.get("dram_source")
    roofline["traffic"] = tb
    roofline["traffic_unit"] = "bytes/launch (ncu dram__bytes_read.sum + dram__bytes_write.sum)"
    roofline["traffic_source"] = tsrc

    forward = batch = e2e = cpu = configs = None
    single = world == 1 and args.stage == "pipeline" and args.config == 3

    # ---------------------------------------------------------------- Fig 1 with the Forward stage
    # The same step followed by compaction of the Viterbi passes and the Forward kernel on them
    # (hmg_pipeline_forward), timed the same way; reported beside the 8(a) headline, not in it.
    if not args.no_forward and single and q["fwd_warps"] > 0:
        fo = hmg.alloc_forward_outputs(n, local)
        hmg.hmg_set_stage_timing(True)
        f_ms, f_stage = [], []
        for i in range(args.warmup + args.steps):
            flush.zero_()
            hmg.hmg_pipeline_forward(P, D, F1=args.F1, F2=args.F2, stream=stream, **out, **fo)
            sf = hmg.hmg_stage_times()["fwd"]
            if i >= args.warmup:
                f_stage.append(sf)
        hmg.hmg_set_stage_timing(False)
        torch.cuda.synchronize()
        fwd_graph = None
        if graph is not None:
            fwd_graph = torch.cuda.CUDAGraph()
            with torch.cuda.graph(fwd_graph, capture_error_mode="thread_local"):
                hmg.hmg_pipeline_forward(P, D, F1=args.F1, F2=args.F2, stream=torch.cuda.current_stream(),
                                         **out, **fo)
        for i in range(args.warmup + args.steps):
            flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            if fwd_graph is not None:
                fwd_graph.replay()
            else:
                hmg.hmg_pipeline_forward(P, D, F1=args.F1, F2=args.F2, stream=stream, **out, **fo)
            b.record(stream)
            torch.cuda.synchronize()
            if i >= args.warmup:
                f_ms.append(a.elapsed_time(b))
        nf = int(fo["n_fwd"].item())
        fres = int(D.lengths[fo["fwd_ids"][:nf].cpu().numpy()].sum()) if nf else 0
        tf, tfs = statistics.mean(f_ms), statistics.mean(f_stage)
        fp_peak = FP32_LANES_PER_CLK_SM * 2 * nsm * f_peak / 1e12                # TFLOP/s (FMA = 2)
        f_ach = FWD_FLOPS_PER_CELL * M * fres / (tfs * 1e-3) / 1e12 if tfs > 0 else 0.0
        forward = {"sequences": nf, "residues": fres, "stage_ms": round(tfs, 4),
                   "gcups": round(M * fres / (tfs * 1e-3) / 1e9, 2) if tfs > 0 else None,
                   "fig1_pipeline_ms": round(tf, 4),
                   "fig1_pipeline_gcups": round(M * res_local / (tf * 1e-3) / 1e9, 3),
                   "kernel": "fwd_kernel<%d, %d, %d>" % (q["fwd_warps"], q["fwd_nodes"], q["fwd_seqs_per_block"]),
                   "roofline": {"bound": "fp32", "achieved": round(f_ach, 3), "peak": round(fp_peak, 3),
                                "unit": "TFLOP/s", "frac": round(f_ach / fp_peak, 4),
                                "traffic": load_traffic("fwd_kernel")[0],
                                "algorithmic_flops_per_cell": FWD_FLOPS_PER_CELL,
                                "peak_source": "%s sm_max_mhz x %d SMs x %d FP32 lanes x 2 (FMA)"
                                               % (src, nsm, FP32_LANES_PER_CLK_SM),
                                "note": "stage = Viterbi-pass compaction + Forward kernel on %d sequences "
                                        "(latency-bound at this size: see throughput)" % nf}}
        # the same kernel over every sequence of the DB (hmg_forward, no list): its throughput
        # roofline, where the Fig 1 stage above is bounded by the row latency of its longest sequence
        fall = torch.empty(n, dtype=torch.float32, device=dev)
        t_all = timed_ms(lambda: hmg.hmg_forward(P, D, fall, stream=stream), stream, flush, 2)
        a_all = FWD_FLOPS_PER_CELL * M * res_local / (t_all * 1e-3) / 1e12
        forward["throughput"] = {"sequences": n, "residues": int(res_local), "ms": round(t_all, 3),
                                 "gcups": round(M * res_local / (t_all * 1e-3) / 1e9, 1),
                                 "achieved_tflops": round(a_all, 3), "frac": round(a_all / fp_peak, 4),
                                 "note": "hmg_forward over every sequence of the workload (throughput mode)"}

    # ---------------------------------------------------------------- many-profile batch
    if args.batch > 0 and single:
        from paper_conf_ipps_jiangg15_b200 import synth as _synth
        brng = np.random.default_rng(11)
        bMs = np.clip(np.round(brng.lognormal(math.log(180), 0.6, size=args.batch)), 20, 1500).astype(int)
        bprofs = [hmg.Profile(*(lambda pr: (pr.msc, pr.tsc))(_synth.make_profile(int(m), 6000 + i)), device=local)
                  for i, m in enumerate(bMs)]
        braw = torch.empty((args.batch, n), dtype=torch.uint8, device=dev)
        tb_ = timed_ms(lambda: hmg.hmg_msv_batch(bprofs, D, braw, stream=stream), stream, flush, 3)

        def loop():
            for i, bp in enumerate(bprofs):
                hmg.hmg_msv(bp, D, braw[i], stream=stream)

        tl = timed_ms(loop, stream, flush, 2)
        bcells = int(bMs.sum()) * res_local
        batch = {"profiles": args.batch, "sum_M": int(bMs.sum()), "cells": bcells, "ms": round(tb_, 3),
                 "gcups": round(bcells / (tb_ * 1e-3) / 1e9, 2), "per_profile_calls_ms": round(tl, 3),
                 "per_profile_calls_gcups": round(bcells / (tl * 1e-3) / 1e9, 2),
                 "speedup_vs_calls": round(tl / tb_, 3),
                 "workload": "hmg_msv_batch: %d Pfam-like profiles (M ~ lognormal median 180, 20..1500, seeds "
                             "6000+i) x this DB; L2 flushed before each timed call" % args.batch}
        del bprofs, braw

    # ---------------------------------------------------------------- end to end through the C ABI (host buffers)
    if not args.no_e2e and single:
        img = torch.empty(D.packed_bytes // 4, dtype=torch.int32, pin_memory=True)
        D.image(img)
        h_msv = torch.empty(n, dtype=torch.uint8, pin_memory=True)
        h_vit = torch.empty(n, dtype=torch.int16, pin_memory=True)
        h_flags = torch.empty(n, dtype=torch.uint8, pin_memory=True)
        h_ns = torch.empty(1, dtype=torch.int64, pin_memory=True)
        e_ms = []

        def e2e_step(st_):
            # H2D of the packed DB in length-ordered parts overlapped with the filter
            hmg.hmg_pipeline_upload(P, D, img, F1=args.F1, F2=args.F2, stream=st_, **out)
            h_msv.copy_(out["msv_raw"], non_blocking=True)                 # D2H of the results
            h_vit.copy_(out["vit_raw"], non_blocking=True)
            h_flags.copy_(out["flags"], non_blocking=True)
            h_ns.copy_(out["n_survivors"], non_blocking=True)

        e2e_graph = None
        if graph is not None:                                              # same launch mode as the timed step
            e2e_step(stream)
            torch.cuda.synchronize()
            e2e_graph = torch.cuda.CUDAGraph()
            with torch.cuda.graph(e2e_graph, capture_error_mode="thread_local"):
                e2e_step(torch.cuda.current_stream())
        for i in range(args.warmup + args.steps):
            flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            if e2e_graph is not None:
                e2e_graph.replay()
            else:
                e2e_step(stream)
            b.record(stream)
            b.synchronize()
            if i >= args.warmup:
                e_ms.append(a.elapsed_time(b))
        te = sum(e_ms) / len(e_ms)
        dimg = torch.empty_like(img, device=dev)                           # the PCIe floor: H2D alone
        h_ms = []
        for i in range(4):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            with torch.cuda.stream(stream):
                dimg.copy_(img, non_blocking=True)
            b.record(stream)
            b.synchronize()
            h_ms.append(a.elapsed_time(b))
        del dimg
        th = min(h_ms[1:])
        e2e = {"value": round(M * res_local / (te * 1e-3) / 1e9, 3), "unit": "GCUPS",
               "h2d_bytes_per_step": int(D.packed_bytes), "d2h_bytes_per_step": int(n * 4 + 8),
               "ms_per_step": round(te, 3), "h2d_alone_ms": round(th, 3),
               "h2d_alone_gbs": round(D.packed_bytes / (th * 1e-3) / 1e9, 2)}

    if not args.no_configs and single:
        configs = configs_leg(args, dev, stream, flush, p_int, evf)

    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(prof, dsq, off, ev, args.F1, M, args.cpu_sample_every, args.stage)

    if rank == 0:
        wl = {"pipeline": "MSV -> on-device compaction -> P7Viterbi (Lazy-F)", "msv": "MSV filter only",
              "vit": "P7Viterbi filter (Lazy-F) over every sequence"}[args.stage]
        line = {
            "metric": METRIC, "value": round(value, 3), "unit": "GCUPS", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(t_step, 4), "higher_is_better": True,
            "scaling": args.scaling, "vs_baseline": None, "dtype": "u8/s16", "data": "synthetic",
            "config": {"workload": "config%d: M=%d %s, %s DB" % (args.config, M, wl,
                                                                  "UniProt-shaped" if args.config == 5 else "Swiss-Prot-shaped"),
                       "stage": args.stage, "M": M, "nseq_per_rank": n, "residues_per_rank": res_local,
                       "nseq_total": int(n_all), "residues_total": int(res_all), "F1": args.F1, "F2": args.F2,
                       "l2": "flushed (256 MiB write) before every timed step, outside its events",
                       "launch": "CUDA graph of the stage (captured once), replayed per step" if graph is not None
                                 else "eager calls",
                       "parallelism": "db-shard x%d (snake length-balanced, %s scaling), %s all_gather of results"
                                      % (world, args.scaling, "NCCL" if args.backend == "nccl" else
                                         "gloo (host-staged, test of the N > 1 path)"),
                       "tuning": args.tune or None},
            "stages": {"msv_kernel_ms": round(msv_ms, 4) if msv_ms > 0 else None,
                       "msv_gcups": round(msv_gcups, 2) if msv_gcups else None,
                       "msv_redo_ms": round(st["msv_redo"], 4) if st["msv_redo"] > 0 else None,
                       "flags_compaction_ms": round(st["msv_flags_compaction"], 4) if st["msv_flags_compaction"] > 0 else None,
                       "vit_kernel_ms": round(vit_ms, 4) if vit_ms > 0 else None,
                       "vit_gcups": round(vit_gcups, 2) if vit_gcups else None,
                       "vit_alu_frac": (round(vit_gcups * 1e9 * VIT_ALU_OPS_PER_CELL / (p_int * 1e12), 4)
                                        if vit_gcups else None),
                       "vit_alu_note": "vs the ALU-pipe peak at %.2f essential ops/cell (s16x2 pair encoding)"
                                       % VIT_ALU_OPS_PER_CELL,
                       "vit_flags_ms": round(st["vit_flags"], 4) if st["vit_flags"] > 0 else None,
                       "vit_s32_rescored": int(redo),
                       "survivors": int(ns_all), "survivor_frac": round(ns_all / max(n_all, 1), 5),
                       "survivor_residues": int(surv_all)},
            "roofline": roofline,
            "forward": forward,
            "batch": batch,
            "configs": configs,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": int(launches),
            "clocks": clock,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
