"""Spatial decomposition of the grid-binned Boids step over ranks (SURVEY.md
8(f) #3; the thesis names spatial data structures and multiple devices as
future work).

Rank g owns the agents whose search-cell layer z lies in its slab and holds
only them and its halo (the layers within the search radius of its slab); see
csrc/k_spatial.cu and include/boids.h ("Spatial decomposition").  Each step:

    boids_step_spatial(h, dt)      owned agents: search + steer + modify, then
                                   pack halo copies / migrants per destination
    exchange                       every rank's records for destination d go
                                   into d's inboxes (NCCL point-to-point
                                   sends/receives here; device copies in
                                   `emulated_step`)
    boids_spatial_unpack(h, ...)   apply them

Only boundary layers and migrants cross ranks, instead of the all-gather of
all n agents of the index-sharded mode (shard.py).  The library does all the
arithmetic; this module only moves record buffers (zero-copy torch views of
the library's device memory) and computes where they land.
"""
from __future__ import annotations

import numpy as np

from . import abi
from .shard import device_view


def inbox_layout(counts: np.ndarray):
    """counts[s, d] = records rank s sends to rank d.  Returns (offsets, totals):
    source s's records for d land at offsets[s, d] of d's inbox (sources in rank
    order, contiguous), and totals[d] records arrive at d."""
    counts = np.asarray(counts, np.int64)
    offsets = np.zeros_like(counts)
    offsets[1:] = np.cumsum(counts[:-1], axis=0)
    return offsets, counts.sum(axis=0)


def _views(h, world, dev):
    hc, mc, ho, mo, cap_h, cap_m = abi.boids_spatial_outbox(h, world)
    hi, mi, cap_hi, cap_mi = abi.boids_spatial_inbox(h)
    hf, mf = abi.SPATIAL_HALO_F4 * 4, abi.SPATIAL_MIG_F4 * 4  # floats per record
    return dict(hc=hc, mc=mc,
                hout=device_view(ho, world * cap_h * hf * 4, dev).view(world, cap_h, hf),
                mout=device_view(mo, world * cap_m * mf * 4, dev).view(world, cap_m, mf),
                hin=device_view(hi, cap_hi * hf * 4, dev).view(cap_hi, hf),
                min=device_view(mi, cap_mi * mf * 4, dev).view(cap_mi, mf))


def emulated_step(handles, dt: float):
    """One step of G spatial handles living on ONE device (tests, per-rank timing):
    the exchange is done by device copies between the handles' buffers."""
    import torch

    world = len(handles)
    dev = torch.device("cuda", torch.cuda.current_device())
    for h in handles:
        abi.boids_step_spatial(h, dt)
    vs = [_views(h, world, dev) for h in handles]
    hcnt = np.stack([v["hc"] for v in vs])
    mcnt = np.stack([v["mc"] for v in vs])
    hoff, htot = inbox_layout(hcnt)
    moff, mtot = inbox_layout(mcnt)
    for d, vd in enumerate(vs):
        for s, vsrc in enumerate(vs):
            k = int(hcnt[s, d])
            if k:
                vd["hin"][hoff[s, d]:hoff[s, d] + k].copy_(vsrc["hout"][d, :k])
            k = int(mcnt[s, d])
            if k:
                vd["min"][moff[s, d]:moff[s, d] + k].copy_(vsrc["mout"][d, :k])
    for d, h in enumerate(handles):
        abi.boids_spatial_unpack(h, int(htot[d]), int(mtot[d]))


def gather_owned(handles, n: int):
    """Merge the owned rows of every rank: state dict (n rows), lists, owner rank."""
    keys = ("pos", "fwd", "up", "side", "speed")
    out = {k: None for k in keys}
    idx = np.full((n, 7), -1, np.int32)
    cnt = np.full(n, -1, np.int32)
    owner = np.full(n, -1, np.int32)
    for r, h in enumerate(handles):
        own = abi.boids_spatial_owned(h)
        assert not (own & (owner >= 0)).any(), "agent owned by two ranks"
        owner[own] = r
        st = abi.boids_get_state(h)
        for k in keys:
            if out[k] is None:
                out[k] = np.zeros_like(st[k])
            out[k][own] = st[k][own]
        i7, c = abi.boids_get_neighbors(h)
        idx[own], cnt[own] = i7[own], c[own]
    assert (owner >= 0).all(), "agent owned by no rank"
    return out, idx, cnt, owner


def route(dist, group, rank: int, world: int, inputs, outputs):
    """inputs[d] -> rank d's outputs[rank], for every pair of ranks: point-to-point
    sends and receives (NCCL or gloo), a copy for d == rank; empty pieces skipped."""
    ops = []
    for d in range(world):
        if d == rank:
            if inputs[d].numel():
                outputs[rank].copy_(inputs[d])
        elif inputs[d].numel():
            ops.append(dist.P2POp(dist.isend, inputs[d].contiguous(), d, group))
    for s in range(world):
        if s != rank and outputs[s].numel():
            ops.append(dist.P2POp(dist.irecv, outputs[s], s, group))
    if ops:
        for w in dist.batch_isend_irecv(ops):
            w.wait()


class SpatialFlock:
    """One rank of a spatially decomposed flock (one process per GPU, NCCL)."""

    def __init__(self, n: int, params=None, seed: int = 1, group=None):
        import torch
        import torch.distributed as dist

        self.dist, self.group = dist, group
        self.rank, self.world = dist.get_rank(group), dist.get_world_size(group)
        self.device = torch.device("cuda", torch.cuda.current_device())
        self.params = params or abi.boids_default_params(search_mode=abi.BOIDS_GRID)
        self.h = abi.boids_create_spatial(n, self.params, seed, self.rank, self.world)
        abi.boids_set_stream(self.h, torch.cuda.current_stream().cuda_stream)
        self.n = n

    def exchange(self):
        """Halo and migrant records to their destinations (counts all-gathered,
        records sent point to point: only slab neighbours exchange anything)."""
        import torch

        v = _views(self.h, self.world, self.device)
        mine = torch.tensor(np.stack([v["hc"], v["mc"]]), device=self.device, dtype=torch.int64)
        allc = [torch.empty_like(mine) for _ in range(self.world)]
        self.dist.all_gather(allc, mine, group=self.group)  # counts[s] of every source s
        counts = torch.stack(allc).cpu().numpy()  # [s, kind, d]
        got = []
        for kind, (src, dst) in enumerate((("hout", "hin"), ("mout", "min"))):
            c = counts[:, kind, :]
            off, tot = inbox_layout(c)
            inputs = [v[src][d, :int(c[self.rank, d])] for d in range(self.world)]
            outputs = [v[dst][off[s, self.rank]:off[s, self.rank] + int(c[s, self.rank])] for s in range(self.world)]
            try:
                route(self.dist, self.group, self.rank, self.world, inputs, outputs)
            except Exception as e:  # surface as the ABI's NCCL error code
                raise abi.BoidsError(abi.BOIDS_ENCCL, f"record exchange failed: {e}") from e
            got.append(int(tot[self.rank]))
        abi.boids_spatial_unpack(self.h, got[0], got[1])

    def step(self, dt: float, steps: int = 1):
        for _ in range(steps):
            abi.boids_step_spatial(self.h, dt)
            self.exchange()
        return self

    def close(self):
        if getattr(self, "h", None):
            abi.boids_sync(self.h)
            abi.boids_destroy(self.h)
            self.h = None
