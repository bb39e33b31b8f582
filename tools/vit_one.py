"""One Viterbi-filter call over a config-2-shaped DB for a given M (for ncu captures):
python tools/vit_one.py M [nseq] [KNOB=VALUE ...]  (tuning knobs, include/hmg.h)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
M = int(sys.argv[1])
N = int(sys.argv[2]) if len(sys.argv) > 2 else 100000
for kv in sys.argv[3:]:
    k, v = kv.split("=")
    hmg.set_tuning(k, int(v))
prof = synth.make_profile(M, 1000 + M)
db = synth.make_db(N, 5.60, 0.75, 12)
dsq, off = db.materialize()
D = hmg.Database(dsq, off)
P = hmg.Profile(prof.msc, prof.tsc)
raw = torch.zeros(D.nseq, dtype=torch.int16, device="cuda")
hmg.hmg_set_stage_timing(True)
for _ in range(2):
    hmg.hmg_viterbi(P, D, raw)
    print(hmg.hmg_stage_times(), P.quant()["vit_lanes"], P.quant()["vit_nodes"], flush=True)
