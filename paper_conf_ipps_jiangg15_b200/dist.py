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


class Gatherer:
    """All-gather of per-sequence result words and survivor lists (global caller ids) with
    static shapes: every buffer is allocated once, padded to the largest snake shard
    (``shard_sizes``), so a step issues its collectives with no host synchronisation and no
    allocation (it can sit inside a CUDA graph or a timed loop).

    n_global   : sequences in the whole database; world / rank as torch.distributed
    global_ids : device int64 [n_local] global caller index of each local sequence
    exchange   : False builds the static buffers without any collective (one process playing
                 every rank in turn: ``local`` gives the slices all_gather_into_tensor would
                 concatenate in rank order -- the one-GPU proof of the sharded path)
    stage_host : run the collectives on host copies (gloo tests of the N > 1 path with several
                 ranks on one GPU; NCCL is the product path)
    """

    def __init__(self, n_global: int, world: int, global_ids, group=None, exchange: bool = True,
                 stage_host: bool = False):
        import torch
        self.world, self.group = world, group
        self.nmax = max(shard_sizes(n_global, world))
        dev = global_ids.device
        self.n_local = global_ids.numel()
        self.gid_local = global_ids.to(torch.int64)
        self.pad = torch.zeros(self.nmax, dtype=torch.int32, device=dev)
        self.words = torch.empty(world * self.nmax, dtype=torch.int32, device=dev)
        self.counts = torch.empty(world, dtype=torch.int64, device=dev)
        self.sv = torch.full((self.nmax,), -1, dtype=torch.int64, device=dev)
        self.surv = torch.empty(world * self.nmax, dtype=torch.int64, device=dev)
        self.gid_pad = torch.full((self.nmax,), -1, dtype=torch.int64, device=dev)
        self.gid_pad[:self.n_local] = self.gid_local
        self.gids = torch.empty(world * self.nmax, dtype=torch.int64, device=dev)
        self.exchange = exchange
        self.stage_host = stage_host
        if world > 1 and exchange:
            self._all_gather(self.gids, self.gid_pad)   # once: the shard map is static
        else:
            self.gids[:self.nmax].copy_(self.gid_pad)

    def _all_gather(self, out, inp):
        import torch.distributed as dist
        if self.stage_host:
            o = out.cpu()
            dist.all_gather_into_tensor(o, inp.cpu(), group=self.group)
            out.copy_(o)
        else:
            dist.all_gather_into_tensor(out, inp, group=self.group)

    def local(self, msv_raw, vit_raw, flags, survivor_ids, n_survivors):
        """This rank's padded slices (device ops only): result words and global survivor ids."""
        import torch
        n = self.n_local
        self.pad[:n] = pack_results(msv_raw[:n], vit_raw[:n], flags[:n])
        ids = survivor_ids[:n].to(torch.int64).clamp_(0, max(n - 1, 0))
        self.sv[:n] = self.gid_local[ids]
        return self.pad, self.sv, n_survivors.reshape(1)

    def __call__(self, msv_raw, vit_raw, flags, survivor_ids, n_survivors):
        """Gather every rank's results; returns device views words [world, nmax],
        gids [world, nmax], counts [world], surv [world, nmax] (first counts[r] valid)."""
        if not self.exchange:
            raise RuntimeError("Gatherer(exchange=False) has no collective step")
        pad, sv, ns = self.local(msv_raw, vit_raw, flags, survivor_ids, n_survivors)
        if self.world > 1:
            self._all_gather(self.words, pad)
            self._all_gather(self.counts, ns)
            self._all_gather(self.surv, sv)
        else:
            self.words.copy_(pad)
            self.counts.copy_(ns)
            self.surv.copy_(sv)
        return (self.words.view(self.world, self.nmax), self.gids.view(self.world, self.nmax), self.counts,
                self.surv.view(self.world, self.nmax))


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
