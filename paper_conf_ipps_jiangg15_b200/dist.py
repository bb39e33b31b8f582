"""Multi-GPU shard / gather layer (the database is split across devices
"without any dependencies"; combined results on the host).

One process per GPU (torchrun).  Each rank builds its own hmg_db over a
length-balanced shard of the global database and runs the whole filter
pipeline locally; the only exchange step is gathering per-sequence results
and survivor lists over NCCL (NVLink / NVSwitch).  Sharding is a snake over
the global length-descending order: rank r takes positions r, 2W-1-r, 2W+r,
... so every rank gets the same length histogram and (to within one
sequence) the same residue count, i.e. the same MSV cells.

Everything here is plumbing: numpy for shard index bookkeeping,
torch.distributed for the collectives.  All scoring happens in libhmg.
"""
from __future__ import annotations

import math

import numpy as np


def snake_shard(lengths: np.ndarray, world: int, rank: int) -> np.ndarray:
    """Global caller indices owned by ``rank`` (ascending), length-balanced snake order."""
    lengths = np.asarray(lengths)
    order = np.argsort(-lengths.astype(np.int64), kind="stable")
    pos = np.arange(len(order))
    rnd, k = pos // world, pos % world
    owner = np.where(rnd % 2 == 0, k, world - 1 - k)
    return np.sort(order[owner == rank]).astype(np.int64)


def shard_sizes(n: int, world: int) -> list[int]:
    """Number of sequences each rank owns under snake_shard (independent of lengths)."""
    pos = np.arange(n)
    rnd, k = pos // world, pos % world
    owner = np.where(rnd % 2 == 0, k, world - 1 - k)
    return np.bincount(owner, minlength=world).tolist()


def pack_results(msv_raw, vit_raw, flags):
    """Per-sequence result word: msv_raw | flags << 8 | (vit_raw & 0xffff) << 16 (int32)."""
    import torch
    return (msv_raw.to(torch.int32) | (flags.to(torch.int32) << 8) |
            ((vit_raw.to(torch.int32) & 0xFFFF) << 16))


def unpack_results(words: np.ndarray):
    w = np.asarray(words).astype(np.int64) & 0xFFFFFFFF
    msv = (w & 0xFF).astype(np.int32)
    flags = ((w >> 8) & 0xFF).astype(np.uint8)
    vit = ((w >> 16) & 0xFFFF).astype(np.uint16).view(np.int16).astype(np.int32)
    return msv, vit, flags


def gather(packed, survivor_ids, n_survivors, global_ids, world: int, group=None):
    """All-gather per-sequence result words and survivor lists (global caller ids).

    packed        : device int32 [n_local] (pack_results)
    survivor_ids  : device int32 [>= n_local] local caller indices, schedule order
    n_survivors   : device int64 [1]
    global_ids    : device int64 [n_local] global caller index of each local sequence
    Returns device tensors: words [world, nmax], gids [world, nmax], counts [world],
    surv [world, nmax] (global ids, first counts[r] valid per row).
    """
    import torch
    import torch.distributed as dist
    n_local = packed.numel()
    nmax_t = torch.tensor([n_local], dtype=torch.int64, device=packed.device)
    dist.all_reduce(nmax_t, op=dist.ReduceOp.MAX, group=group)
    nmax = int(nmax_t.item())
    pad = torch.zeros(nmax, dtype=torch.int32, device=packed.device)
    pad[:n_local] = packed
    words = torch.empty(world * nmax, dtype=torch.int32, device=packed.device)
    dist.all_gather_into_tensor(words, pad, group=group)
    gid = torch.full((nmax,), -1, dtype=torch.int64, device=packed.device)
    gid[:n_local] = global_ids
    gids = torch.empty(world * nmax, dtype=torch.int64, device=packed.device)
    dist.all_gather_into_tensor(gids, gid, group=group)
    counts = torch.empty(world, dtype=torch.int64, device=packed.device)
    dist.all_gather_into_tensor(counts, n_survivors.reshape(1), group=group)
    sv = torch.full((nmax,), -1, dtype=torch.int64, device=packed.device)
    sv[:n_local] = global_ids[survivor_ids[:n_local].to(torch.int64).clamp_(0, max(n_local - 1, 0))]
    surv = torch.empty(world * nmax, dtype=torch.int64, device=packed.device)
    dist.all_gather_into_tensor(surv, sv, group=group)
    return words.view(world, nmax), gids.view(world, nmax), counts, surv.view(world, nmax)


def assemble(words, gids, counts, surv, n_global: int):
    """Host-side reassembly of gathered results into global caller order."""
    words = np.asarray(words)
    gids = np.asarray(gids)
    out = np.zeros(n_global, dtype=np.int64)
    m = gids >= 0
    out[gids[m]] = words[m]
    msv, vit, flags = unpack_results(out)
    sl = [np.asarray(surv)[r, :int(c)] for r, c in enumerate(np.asarray(counts))]
    return msv, vit, flags, sl


def calibrate(msc, tsc, device: int = 0, n: int = 1000, L: int = 200, seed: int = 7):
    """Gumbel location mu for lambda = ln 2 of both filters, fitted on ``n``
    background sequences of length ``L`` scored by the GPU kernels themselves
    (closed-form ML location for known lambda).  Returns the hmg_evparams tuple."""
    import torch

    from . import hmg, synth
    cal = synth.Database(np.full(n, L, np.int32), seed=seed)
    dsq, off = cal.materialize()
    p = hmg.Profile(msc, tsc, device=device)
    db = hmg.Database(dsq, off, device=device)
    dev = torch.device("cuda", device)
    mraw = torch.zeros(n, dtype=torch.uint8, device=dev)
    vraw = torch.zeros(n, dtype=torch.int16, device=dev)
    hmg.hmg_msv(p, db, mraw)
    hmg.hmg_viterbi(p, db, vraw)
    torch.cuda.synchronize(dev)
    lam = math.log(2)
    null = hmg.hmg_null1_nats(L)
    mb = np.array([(hmg.hmg_msv_nats(int(r), L) - null) / lam for r in mraw.cpu().numpy()])
    vb = np.array([(hmg.hmg_vit_nats(int(r), L) - null) / lam for r in vraw.cpu().numpy()])
    mu = lambda x: float(-np.log(np.mean(np.exp(-lam * x[np.isfinite(x)]))) / lam)
    return (mu(mb), lam, mu(vb), lam)
