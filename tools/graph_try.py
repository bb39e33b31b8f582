"""Capture hmg_pipeline (config 3) in a CUDA graph and compare replay time / outputs with eager calls."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth, dist as hdist
build.build()
prof, db = synth.config(3)
dsq, off = db.materialize()
P, ev = hmg.calibrated_profile(prof.msc, prof.tsc)
D = hmg.Database(dsq, off)
out = hmg.alloc_outputs(D.nseq)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for _ in range(3):
    hmg.hmg_pipeline(P, D, **out)
torch.cuda.synchronize()
ref = {k: v.clone() for k, v in out.items()}
def timeit(fn, k=10):
    ts = []
    for _ in range(k):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
    return sum(ts) / len(ts), min(ts)
te = timeit(lambda: hmg.hmg_pipeline(P, D, **out))
for k in ("msv_raw", "flags", "survivor_ids", "n_survivors"):
    out[k].zero_()
g = torch.cuda.CUDAGraph()
n0 = hmg.hmg_kernel_launches()
with torch.cuda.graph(g):
    hmg.hmg_pipeline(P, D, stream=torch.cuda.current_stream(), **out)
nl = hmg.hmg_kernel_launches() - n0
g.replay(); torch.cuda.synchronize()
ns = int(ref["n_survivors"].item())
sv = ref["survivor_ids"][:ns].long()
same = (torch.equal(ref["msv_raw"], out["msv_raw"]) and torch.equal(ref["flags"], out["flags"]) and
        torch.equal(ref["n_survivors"], out["n_survivors"]) and
        torch.equal(ref["survivor_ids"][:ns], out["survivor_ids"][:ns]) and
        torch.equal(ref["vit_raw"][sv], out["vit_raw"][sv]))
tg = timeit(lambda: g.replay())
print(json.dumps({"eager_ms": te, "graph_ms": tg, "launches_per_step": nl, "outputs_equal": same}))
