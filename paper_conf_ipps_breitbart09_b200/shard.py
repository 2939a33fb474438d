"""Multi-GPU Boids: agents sharded by index, one process per GPU.

SURVEY.md 8(e): rank g owns agents [g*m, min((g+1)*m, n)) with the slice
m = ceil(n / world) rounded up to 256 (libboids pads each slice with phantom
agents whose positions are NaN, so every rank's send buffer has the same size).
Every step is

    all_gather(full <- send)      # NCCL over NVLink/NVSwitch via torch.distributed
    boids_step_shard(h, dt)       # search this rank's slice against all n agents,
                                  # steer + modify it, write the new slice into send

The exchanged record is [pos4(m) | fwd4(m)] (32 B per agent): alignment needs
the neighbours' forward vectors (Listing 5.5), positions alone are not
enough.  The result is bit-identical to the single-GPU step because every
agent's arithmetic is identical and the neighbour order is the (d2, index) key.

torch.distributed is plumbing only: the device buffers are owned by the C
library and wrapped (no copy) as torch tensors through __cuda_array_interface__.
"""
from __future__ import annotations

import numpy as np

from . import abi

SLICE_ALIGN = 256  # == boids::TILE in csrc/internal.h


def partition(n: int, world: int, rank: int):
    """(lo, hi, m) of `rank` -- the same rule as create_impl in csrc/api.cu."""
    per = (n + world - 1) // world
    m = (per + SLICE_ALIGN - 1) // SLICE_ALIGN * SLICE_ALIGN
    lo = min(rank * m, n)
    hi = min((rank + 1) * m, n)
    return lo, hi, m


def pack_slice(pos: np.ndarray, fwd: np.ndarray, speed: np.ndarray, lo: int, hi: int, m: int) -> np.ndarray:
    """Host image of one rank's send buffer: float32 (2m, 4) = [pos4 | fwd4], NaN phantoms."""
    buf = np.zeros((2 * m, 4), np.float32)
    k = hi - lo
    buf[:m, :3] = np.nan
    buf[:k, :3] = pos[lo:hi]
    buf[m:m + k, :3] = fwd[lo:hi]
    buf[m:m + k, 3] = speed[lo:hi]
    return buf


def unpack_full(full: np.ndarray, n: int, m: int, world: int):
    """Inverse of the gathered layout: (pos (n,3), fwd (n,3), speed (n,))."""
    f = full.reshape(world, 2, m, 4)
    pos = f[:, 0, :, :3].reshape(world * m, 3)[:n]
    fwd = f[:, 1, :, :3].reshape(world * m, 3)[:n]
    speed = f[:, 1, :, 3].reshape(world * m)[:n]
    return pos, fwd, speed


class _CudaArray:
    """Zero-copy view of a device pointer for torch.as_tensor (CUDA array interface v3)."""

    def __init__(self, ptr: int, nfloats: int):
        self.__cuda_array_interface__ = {"shape": (nfloats,), "typestr": "<f4", "data": (ptr, False),
                                         "version": 3, "strides": None, "stream": None}


def device_view(ptr: int, nbytes: int, device):
    import torch

    return torch.as_tensor(_CudaArray(ptr, nbytes // 4), device=device)


class _SymViews:
    """Zero-copy float32 views of a handle's sym-shard exchange buffers (bits are moved, never read)."""

    def __init__(self, h: int, world: int, m: int, device):
        b = abi.boids_symshard_buffers(h)
        cap = b["hits_cap"]
        self.lim_send = device_view(b["lim_send"], m * 4, device)
        self.lim_full = device_view(b["lim_full"], world * m * 4, device)
        self.hits = device_view(b["hits"], world * m * cap * 8, device)  # u64 keys as 2 float32 each
        self.hitcnt = device_view(b["hitcnt"], world * m * 4, device)
        self.recv = device_view(b["recv"], world * m * cap * 8, device)
        self.rcnt = device_view(b["rcnt"], world * m * 4, device)
        self.block_keys = m * cap * 2  # float32 words per rank block
        self.block_cnt = m


def emulated_symshard_step(handles, views, dt: float, warm: bool):
    """One step of G sym-shard handles on ONE device (tests, per-rank timing): both
    exchanges (and the position all-gather) done by device copies."""
    world = len(handles)
    sends = views["pos"]
    for r, (send, _, nf) in enumerate(sends):  # all-gather of the [pos4 | fwd4] slices
        for (_, full, _) in sends:
            full[r * nf:(r + 1) * nf].copy_(send)
    if not warm:
        for h in handles:
            abi.boids_step_shard(h, dt)
        return
    sv = views["sym"]
    m = sv[0].block_cnt
    for h in handles:
        abi.boids_symshard_prep(h)
    for r, v in enumerate(sv):  # all-gather of the limits
        for w in sv:
            w.lim_full[r * m:(r + 1) * m].copy_(v.lim_send)
    for h in handles:
        abi.boids_symshard_search(h)
    for d, vd in enumerate(sv):  # all-to-all of the hit blocks
        for s_, vs in enumerate(sv):
            k = vd.block_keys
            vd.recv[s_ * k:(s_ + 1) * k].copy_(vs.hits[d * k:(d + 1) * k])
            vd.rcnt[s_ * m:(s_ + 1) * m].copy_(vs.hitcnt[d * m:(d + 1) * m])
    for h in handles:
        abi.boids_symshard_finish(h, dt)


class ShardedFlock:
    """One rank of an index-sharded flock.  Call inside an initialised process group.

    sym=True (brute force): warm steps split the global unordered-pair triangle
    over the ranks (boids_symshard_*): two more collectives per step (the limits'
    all-gather, the hits' all-to-all) instead of n/G x n ordered pairs per rank."""

    def __init__(self, n: int, params=None, seed: int = 1, group=None, kernel: int | None = None,
                 record_steering: bool = False, profile: bool = False, sym: bool = False):
        import torch
        import torch.distributed as dist

        self.dist = dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.device = torch.device("cuda", torch.cuda.current_device())
        self.params = params or abi.boids_default_params()
        self.h = abi.boids_create_shard(n, self.params, seed, self.rank, self.world)
        abi.boids_set_stream(self.h, torch.cuda.current_stream().cuda_stream)
        if kernel is not None:
            abi.boids_set_option(self.h, abi.BOIDS_OPT_KERNEL, kernel)
        if record_steering:
            abi.boids_set_option(self.h, abi.BOIDS_OPT_RECORD_STEERING, 1)
        if profile:
            abi.boids_set_option(self.h, abi.BOIDS_OPT_PROFILE, 1)
        send, full, nbytes = abi.boids_shard_buffers(self.h)
        self.slice_bytes = nbytes
        self.send = device_view(send, nbytes, self.device)
        self.full = device_view(full, nbytes * self.world, self.device)
        self.n = n
        info = abi.boids_info(self.h)
        self.lo, self.hi, self.m = info.lo, info.hi, info.slice
        self.sym = (sym and self.params.search_mode == abi.BOIDS_BRUTE and self.params.think_every == 1
                    and kernel in (None, abi.BOIDS_KERNEL_FUSED))
        self.sv = _SymViews(self.h, self.world, self.m, self.device) if self.sym else None
        self.steps_done = 0

    def exchange(self):
        """a1: all-gather every rank's [pos4 | fwd4] slice into the full buffer (NCCL)."""
        try:
            self.dist.all_gather_into_tensor(self.full, self.send, group=self.group)
        except Exception as e:  # surface as the ABI's NCCL error code
            raise abi.BoidsError(abi.BOIDS_ENCCL, f"all_gather_into_tensor failed: {e}") from e

    def step(self, dt: float, steps: int = 1):
        for _ in range(steps):
            self.exchange()
            if self.sym and self.steps_done > 0:
                self._sym_step(dt)
            else:
                abi.boids_step_shard(self.h, dt)
            self.steps_done += 1
        return self

    def _sym_step(self, dt: float):
        d, v = self.dist, self.sv
        try:
            abi.boids_symshard_prep(self.h)
            d.all_gather_into_tensor(v.lim_full, v.lim_send, group=self.group)
            abi.boids_symshard_search(self.h)
            d.all_to_all_single(v.recv, v.hits, group=self.group)
            d.all_to_all_single(v.rcnt, v.hitcnt, group=self.group)
        except abi.BoidsError:
            raise
        except Exception as e:  # surface as the ABI's NCCL error code
            raise abi.BoidsError(abi.BOIDS_ENCCL, f"sym-shard collective failed: {e}") from e
        abi.boids_symshard_finish(self.h, dt)

    def state(self):
        return abi.boids_get_state(self.h)

    def set_state(self, state: dict):
        abi.boids_set_state(self.h, state)

    def neighbors(self):
        return abi.boids_get_neighbors(self.h)

    def steering(self):
        return abi.boids_get_steering(self.h)

    def profile(self, reset: bool = True):
        return abi.boids_get_profile(self.h, reset)

    def close(self):
        if getattr(self, "h", None):
            abi.boids_sync(self.h)
            self.send = self.full = None
            abi.boids_destroy(self.h)
            self.h = None
