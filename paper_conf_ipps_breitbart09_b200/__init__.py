"""B200-native OpenSteer Boids step (Breitbart, CuPP thesis, ch. 5-6).

The product is ``libboids.so`` (CUDA, sm_100a) behind the C ABI of
``include/boids.h``; ``abi`` is its thin ctypes binding (same names),
``Flock`` a convenience handle, ``shard`` the multi-GPU driver (agents
sharded by index, NCCL all-gather of positions each step through
torch.distributed).  PyTorch is used only for device memory, streams and
process groups.  There is no CPU fallback.
"""
from __future__ import annotations

from . import abi
from .abi import (BOIDS_BRUTE, BOIDS_GRID, BOIDS_INIT_OPENSTEER, BOIDS_INIT_WORLD, BOIDS_KERNEL_FUSED,
                  BOIDS_KERNEL_SIMPLE, BoidsError, boids_default_params)

__all__ = ["abi", "Flock", "BoidsError", "boids_default_params", "BOIDS_BRUTE", "BOIDS_GRID",
           "BOIDS_INIT_OPENSTEER", "BOIDS_INIT_WORLD", "BOIDS_KERNEL_FUSED", "BOIDS_KERNEL_SIMPLE"]


def _torch_stream():
    try:
        import torch

        if torch.cuda.is_available():
            return torch.cuda.current_stream().cuda_stream
    except Exception:  # pragma: no cover - torch is plumbing only
        pass
    return None


class Flock:
    """One single-rank handle: ``Flock(n, params, seed).step(dt, steps)``."""

    def __init__(self, n: int, params=None, seed: int = 1, *, stream=None, kernel: int | None = None,
                 record_steering: bool = False, cluster: int = 0, profile: bool = False,
                 symmetric: bool | None = None):
        self.params = params or boids_default_params()
        self.h = abi.boids_create(n, self.params, seed)
        abi.boids_set_stream(self.h, stream if stream is not None else _torch_stream())
        if kernel is not None:
            abi.boids_set_option(self.h, abi.BOIDS_OPT_KERNEL, kernel)
        if record_steering:
            abi.boids_set_option(self.h, abi.BOIDS_OPT_RECORD_STEERING, 1)
        if cluster:
            abi.boids_set_option(self.h, abi.BOIDS_OPT_CLUSTER, cluster)
        if profile:
            abi.boids_set_option(self.h, abi.BOIDS_OPT_PROFILE, 1)
        if symmetric is not None:
            abi.boids_set_option(self.h, abi.BOIDS_OPT_SYMMETRIC, int(symmetric))
        self.n = n

    def step(self, dt: float, steps: int = 1):
        abi.boids_step(self.h, dt, steps)
        return self

    def state(self) -> dict:
        return abi.boids_get_state(self.h)

    def set_state(self, state: dict):
        abi.boids_set_state(self.h, state)

    def neighbors(self):
        return abi.boids_get_neighbors(self.h)

    def steering(self):
        return abi.boids_get_steering(self.h)

    def info(self):
        return abi.boids_info(self.h)

    def profile(self, reset: bool = True):
        return abi.boids_get_profile(self.h, reset)

    def sync(self):
        abi.boids_sync(self.h)

    def close(self):
        if getattr(self, "h", None):
            abi.boids_destroy(self.h)
            self.h = None

    def __del__(self):  # pragma: no cover
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()
