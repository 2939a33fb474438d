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


class ShardedFlock:
    """One rank of an index-sharded flock.  Call inside an initialised process group."""

    def __init__(self, n: int, params=None, seed: int = 1, group=None, kernel: int | None = None,
                 record_steering: bool = False, profile: bool = False):
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

    def exchange(self):
        """a1: all-gather every rank's [pos4 | fwd4] slice into the full buffer (NCCL)."""
        try:
            self.dist.all_gather_into_tensor(self.full, self.send, group=self.group)
        except Exception as e:  # surface as the ABI's NCCL error code
            raise abi.BoidsError(abi.BOIDS_ENCCL, f"all_gather_into_tensor failed: {e}") from e

    def step(self, dt: float, steps: int = 1):
        for _ in range(steps):
            self.exchange()
            abi.boids_step_shard(self.h, dt)
        return self

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
