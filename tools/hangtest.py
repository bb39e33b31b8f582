"""Small long-lane pipeline run (diagnostics): a DB with a few long sequences."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
rng = np.random.default_rng(1)
prof = synth.make_profile(120, 4242)
nlong = int(sys.argv[1]) if len(sys.argv) > 1 else 5
seqs = [synth.random_dsq(rng, int(rng.integers(1600, 4000)), 20) for _ in range(nlong)]
seqs += [synth.random_dsq(rng, int(rng.integers(20, 300)), 20) for _ in range(200)]
off = np.zeros(len(seqs) + 1, np.int64); np.cumsum([len(s) for s in seqs], out=off[1:])
dsq = np.concatenate(seqs)
P = hmg.Profile(prof.msc, prof.tsc, ev=(-9.0, 0.6931, -9.0, 0.6931))
D = hmg.Database(dsq, off)
out = hmg.alloc_outputs(D.nseq)
t = time.time()
hmg.hmg_pipeline(P, D, F1=0.5, F2=0.5, **out)
print("enqueued", time.time() - t, flush=True)
torch.cuda.synchronize()
print("done", time.time() - t, int(out["n_survivors"].item()), flush=True)
