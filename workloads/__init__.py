"""Seeded synthetic inputs shared by the tests, the bench and smoke().

This module holds NONE of the method's arithmetic (no search, steering,
modification or Appendix-B init); it only draws numbers with numpy and names
the BASELINE.json configurations.  Both the oracle side and the CUDA side may
be fed from it; neither side imports the other.

Recipe:
  * ``ball_flock``: positions uniform in a ball (the thesis scenario is the
    OpenSteer Boids flock, P:345 / P:418; OpenSteer resets boids inside a
    ball of radius 20 [ext]); forwards uniform on the unit sphere; up vectors
    a random unit vector (not necessarily orthogonal -- the step regenerates
    the local space, so any up is a valid input); speeds uniform in
    [0, max_speed].
  * ``lattice_flock``: integer lattice points -> many exactly equal d2, the
    adversarial tie case for reading Q4 (total order on (d2, index)).
  * ``coincident_flock``: clusters of agents at identical positions (Q6).
  * ``radius_shell_flock``: agents exactly at distance r and at the float just
    inside it along an axis (Q2: strict d2 < r2).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

DT = np.float32(1.0 / 60.0)  # OpenSteerDemo frame time -- proposed, the paper is silent (Table C1)


@dataclass(frozen=True)
class Config:
    name: str
    n: int
    steps: int
    search_mode: int  # 0 brute, 1 grid
    init_mode: int    # 0 ball r=init_radius (20), 1 ball r=world_radius (50)
    desc: str


# BASELINE.json "configs", in order.
CONFIGS = {
    "c1": Config("c1", 1024, 10, 0, 0, "Boids n=1024, 10 steps, thesis default radius/weights, fixed seed"),
    "c2": Config("c2", 4096, 100, 0, 0, "Boids n=4096, 100 steps, brute-force neighbour search, 1 B200"),
    "c3": Config("c3", 16384, 100, 0, 0, "Boids n=16384 (thesis max scale), 100 steps, 1 B200"),
    "c4": Config("c4", 131072, 10, 0, 1, "Boids n=131072, brute force sharded by agent index, all-gather"),
    "c5": Config("c5", 1048576, 10, 1, 1, "Boids n=1048576, grid-binned neighbour search (identical sets)"),
}


def _unit(rng: np.random.Generator, n: int) -> np.ndarray:
    v = rng.standard_normal((n, 3))
    nrm = np.linalg.norm(v, axis=1, keepdims=True)
    nrm[nrm == 0] = 1.0
    return (v / nrm).astype(np.float32)


def ball_flock(n: int, seed: int = 1, radius: float = 20.0, max_speed: float = 9.0) -> dict:
    rng = np.random.default_rng(seed)
    d = _unit(rng, n).astype(np.float64)
    r = radius * rng.random(n) ** (1.0 / 3.0)
    pos = (d * r[:, None]).astype(np.float32)
    return dict(pos=pos, fwd=_unit(rng, n), up=_unit(rng, n), side=_unit(rng, n),
                speed=(rng.random(n) * max_speed).astype(np.float32))


def lattice_flock(side: int, spacing: float = 1.0, seed: int = 1, jitter_perm: bool = True) -> dict:
    """side^3 agents on an integer lattice (exactly representable; many equal d2)."""
    rng = np.random.default_rng(seed)
    g = np.arange(side, dtype=np.float32) - np.float32(side // 2)
    X, Y, Z = np.meshgrid(g, g, g, indexing="ij")
    pos = (np.stack([X.ravel(), Y.ravel(), Z.ravel()], 1) * np.float32(spacing)).astype(np.float32)
    if jitter_perm:
        pos = pos[rng.permutation(pos.shape[0])]
    n = pos.shape[0]
    return dict(pos=np.ascontiguousarray(pos), fwd=_unit(rng, n), up=_unit(rng, n),
                side=_unit(rng, n), speed=(rng.random(n) * 9.0).astype(np.float32))


def coincident_flock(n: int, groups: int = 4, seed: int = 1) -> dict:
    """n agents stacked on `groups` distinct points (d2 = 0 between members)."""
    rng = np.random.default_rng(seed)
    centers = (rng.random((groups, 3)) * 6.0 - 3.0).astype(np.float32)
    pos = centers[rng.integers(0, groups, n)]
    return dict(pos=np.ascontiguousarray(pos), fwd=_unit(rng, n), up=_unit(rng, n),
                side=_unit(rng, n), speed=(rng.random(n) * 9.0).astype(np.float32))


def radius_shell_flock(radius: float = 9.0, seed: int = 1) -> dict:
    """Agent 0 at the origin; others exactly at r and at nextafter(r, 0) on each axis."""
    rng = np.random.default_rng(seed)
    r = np.float32(radius)
    r_in = np.nextafter(r, np.float32(0))
    pts = [[0, 0, 0]]
    for v in (r, r_in, -r, -r_in):
        pts += [[v, 0, 0], [0, v, 0], [0, 0, v]]
    pos = np.array(pts, np.float32)
    n = pos.shape[0]
    return dict(pos=pos, fwd=_unit(rng, n), up=_unit(rng, n), side=_unit(rng, n),
                speed=(rng.random(n) * 9.0).astype(np.float32))


def jitter(state: dict, scale: float, seed: int = 11) -> dict:
    """Copy of a state dict with every position moved by a seeded normal offset
    (std `scale` per axis): a new input that keeps the spatial structure, so a
    handle stepped on the old state has neighbour lists that are stale but close
    (the warm path's realistic case)."""
    rng = np.random.default_rng(seed)
    out = {k: np.array(v, dtype=np.float32, copy=True) for k, v in state.items()}
    out["pos"] = (out["pos"] + scale * rng.standard_normal(out["pos"].shape)).astype(np.float32)
    return out


def sample_agents(n: int, m: int, seed: int = 7) -> np.ndarray:
    """Seeded sample of m distinct agent indices (always includes 0 and n-1)."""
    rng = np.random.default_rng(seed)
    m = min(m, n)
    s = rng.choice(n, size=m, replace=False)
    s[0] = 0
    if m > 1:
        s[1] = n - 1
    return np.unique(s).astype(np.int64)


def random_forces(n: int, seed: int = 13, scale: float = 30.0) -> np.ndarray:
    """Seeded steering vectors (n, 3) float32, Gaussian with per-axis std `scale`:
    a stored-steering input for think-frequency checks (no method arithmetic)."""
    rng = np.random.default_rng(seed)
    return (rng.standard_normal((n, 3)) * scale).astype(np.float32)
