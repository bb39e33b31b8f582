"""Viterbi stage of config 3 split in two concurrent calls (long survivors / the rest) on two
streams: does running the longest survivors beside the rest shorten the stage?"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth, dist as hdist
build.build()
prof, db = synth.config(3)
dsq, off = db.materialize()
P, ev = hmg.calibrated_profile(prof.msc, prof.tsc)
D = hmg.Database(dsq, off)
out = hmg.alloc_outputs(D.nseq)
hmg.hmg_pipeline(P, D, **out)
torch.cuda.synchronize()
ns = int(out["n_survivors"].item())
sv = out["survivor_ids"][:ns].cpu().numpy()
L = D.lengths[sv]
sv = sv[L <= 2880]; L = L[L <= 2880]          # the long lane's survivors are scored during MSV
raw = torch.zeros(D.nseq, dtype=torch.int16, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def run(ids_a, ids_b):
    ta = torch.as_tensor(ids_a, dtype=torch.int32, device="cuda")
    tb = torch.as_tensor(ids_b, dtype=torch.int32, device="cuda") if len(ids_b) else None
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(4):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        s1.wait_stream(torch.cuda.current_stream()); s2.wait_stream(torch.cuda.current_stream())
        hmg.hmg_viterbi(P, D, raw, ids=ta, stream=s1)
        if tb is not None:
            hmg.hmg_viterbi(P, D, raw, ids=tb, stream=s2)
        torch.cuda.current_stream().wait_stream(s1); torch.cuda.current_stream().wait_stream(s2)
        b.record(); torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b))
    return best
print(json.dumps({"all_one_call_ms": round(run(sv, []), 4), "n": int(len(sv))}), flush=True)
for cut in (2000, 1500, 1000, 700):
    A, B = sv[L > cut], sv[L <= cut]
    print(json.dumps({"cut": cut, "nA": int(len(A)), "split_ms": round(run(A, B), 4)}), flush=True)
