"""Small end-to-end case for compute-sanitizer: every kernel of the library runs at least once
(MSV fast + exact + chunked long lane, pipeline with long-lane Viterbi, register / block /
generic Viterbi kernels, compaction)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_jiangg15_b200 import build, hmg, synth
build.build()
rng = np.random.default_rng(0)
lens = [int(x) for x in rng.integers(5, 300, size=120)] + [1700, 2100]   # two long-lane sequences
dsq = np.concatenate([synth.random_dsq(rng, L, 29) for L in lens]).astype(np.uint8)
off = np.zeros(len(lens) + 1, np.int64); np.cumsum(lens, out=off[1:])
for M, env in ((60, {}), (300, {}), (700, {}), (1500, {}), (2048, {"VIT_CPAIR2": 23}), (3500, {}),
               (90, {"VIT_CTA": 1}), (400, {}), (100, {}), (64, {}), (512, {"MSV_G": 16}), (2048, {})):
    for k, v in env.items():
        hmg.set_tuning(k, v)
    prof = synth.make_profile(M, M, dd=(1.0, 9.0))
    P = hmg.Profile(prof.msc, prof.tsc, ev=(-9.0, 0.693, -9.0, 0.693))
    D = hmg.Database(dsq, off)
    out = hmg.alloc_outputs(D.nseq)
    hmg.hmg_pipeline(P, D, F1=0.5, F2=0.5, **out)
    raw = torch.zeros(D.nseq, dtype=torch.uint8, device="cuda")
    hmg.hmg_msv(P, D, raw)
    vr = torch.zeros(D.nseq, dtype=torch.int16, device="cuda")
    hmg.hmg_viterbi(P, D, vr)
    torch.cuda.synchronize()
    hmg.clear_tuning()
    print("M", M, "ok", int(out["n_survivors"].item()))
msc = np.full((40, 29), 30.0, np.float32)       # exact MSV kernel (bias >= 66 + tbm)
P = hmg.Profile(msc)
D = hmg.Database(dsq, off)
raw = torch.zeros(D.nseq, dtype=torch.uint8, device="cuda")
hmg.hmg_msv(P, D, raw)
torch.cuda.synchronize()
print("exact ok")
# Forward stage (every group width W with its block shape S) and the Fig 1 pipeline with Forward
for M in (60, 300, 700, 1500):
    prof = synth.make_profile(M, 50 + M, dd=(1.0, 9.0))
    P = hmg.Profile(prof.msc, prof.tsc, ev=(-9.0, 0.693, -9.0, 0.693))
    D = hmg.Database(dsq, off)
    f = torch.zeros(D.nseq, dtype=torch.float32, device="cuda")
    hmg.hmg_forward(P, D, f)
    out = hmg.alloc_outputs(D.nseq)
    fo = hmg.alloc_forward_outputs(D.nseq)
    hmg.hmg_pipeline_forward(P, D, F1=0.5, F2=0.5, **out, **fo)
    torch.cuda.synchronize()
    print("forward M", M, "ok", int(fo["n_fwd"].item()))
# many-profile batch (two buckets, a profile outside the fast precondition) and its pipeline
profs = [synth.make_profile(M, 70 + M) for M in (40, 64, 300, 310)]
Ps = [hmg.Profile(p.msc, p.tsc, ev=(-9.0, 0.693, -9.0, 0.693)) for p in profs]
Ps.append(hmg.Profile(np.full((40, 29), 30.0, np.float32), np.full((40, 8), -1.0, np.float32),
                      ev=(-9.0, 0.693, -9.0, 0.693)))
D = hmg.Database(dsq, off)
raw = torch.zeros((len(Ps), D.nseq), dtype=torch.uint8, device="cuda")
pas = torch.zeros((len(Ps), D.nseq), dtype=torch.uint8, device="cuda")
hmg.hmg_msv_batch(Ps, D, raw, pas, F1=0.5)
ob = hmg.alloc_batch_outputs(len(Ps), D.nseq)
hmg.hmg_pipeline_batch(Ps, D, F1=0.5, F2=0.5, **ob)
torch.cuda.synchronize()
print("batch ok", ob["n_survivors"].tolist())
# overlapped upload (parts on two MSV streams) at the 2GQ = M and int8-remainder geometries
for M in (400, 100):
    prof = synth.make_profile(M, 90 + M)
    P = hmg.Profile(prof.msc, prof.tsc, ev=(-9.0, 0.693, -9.0, 0.693))
    D = hmg.Database(dsq, off)
    img = torch.empty(D.packed_bytes // 4, dtype=torch.int32, pin_memory=True)
    D.image(img)
    out = hmg.alloc_outputs(D.nseq)
    hmg.hmg_pipeline_upload(P, D, img, F1=0.5, F2=0.5, **out)
    torch.cuda.synchronize()
    print("upload M", M, "ok", int(out["n_survivors"].item()))
