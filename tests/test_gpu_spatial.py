"""Spatial decomposition against the CPU oracle.

G spatial shards (boids_create_spatial, ranks 0..G-1) of one flock live on one
GPU (the pool gives one GPU per call); spatial.emulated_step moves every
rank's halo and migrant records into the destination ranks' inboxes by device
copies -- the same buffers an NCCL all-to-all fills (spatial.SpatialFlock).
Every agent must be owned by exactly one rank after every step, and the merged
owned rows (state, neighbour lists) must equal the oracle's bit for bit: the
owner sees every candidate within the radius (its own agents and its halo
layers), so lists, steering and modification are the single-GPU ones.
"""
import os
import socket

import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu
KEYS = ("pos", "fwd", "up", "side", "speed")
DT = float(W.DT)


def _op(orc, p):
    return orc.default_params(**{name: getattr(p, name) for name, _ in p._fields_})


@pytest.mark.parametrize("world,n,R,steps", [(1, 3000, 15.0, 3), (2, 20000, 20.0, 5), (3, 20000, 20.0, 5),
                                             (4, 20000, 20.0, 5), (8, 30000, 25.0, 4)])
def test_spatial_emulated_trajectory(boidslib, orc, world, n, R, steps):
    import paper_conf_ipps_breitbart09_b200 as pk
    from paper_conf_ipps_breitbart09_b200 import abi
    from paper_conf_ipps_breitbart09_b200.spatial import emulated_step, gather_owned

    p = pk.boids_default_params(search_mode=1, init_mode=1, world_radius=R)
    op = _op(orc, p)
    hs = [abi.boids_create_spatial(n, p, 1, r, world) for r in range(world)]
    try:
        zb, reach = abi.boids_spatial_bounds(hs[0], world)
        assert zb[0] == 0 and (np.diff(zb) >= 0).all() and reach >= 1
        o = orc.init(n, op, seed=1)
        moved = 0
        for t in range(steps):
            before = [abi.boids_spatial_owned(h) for h in hs]
            emulated_step(hs, DT)
            after = [abi.boids_spatial_owned(h) for h in hs]
            moved += sum(int((b & ~a).sum()) for b, a in zip(before, after))
            o, o_idx, o_cnt, _ = orc.step(o, DT, op)
            g, g_idx, g_cnt, owner = gather_owned(hs, n)
            np.testing.assert_array_equal(g_cnt, o_cnt, err_msg=f"step {t}")
            np.testing.assert_array_equal(g_idx, o_idx, err_msg=f"step {t}")
            for k in KEYS:
                assert np.array_equal(g[k], o[k]), (t, k)
        if world > 1:
            assert moved > 0, "no agent crossed a slab boundary: the migration path was not exercised"
    finally:
        for h in hs:
            abi.boids_destroy(h)


def test_spatial_4m_sampled(boidslib, orc):
    """n = 4M (beyond C5): 2, 4 and 8 emulated spatial shards.  Step 1 (cold)
    from the Appendix-B init, then every rank uploads the same jittered copy of
    the init state (workloads.jitter; the stale lists only seed the bound) and
    step 2 runs warm with migrations and halos rebuilt from the upload; 512
    sampled agents of each step checked one by one against oracle.step_sample."""
    import paper_conf_ipps_breitbart09_b200 as pk
    from paper_conf_ipps_breitbart09_b200 import abi
    from paper_conf_ipps_breitbart09_b200.spatial import emulated_step, gather_owned

    n = 4 * 1024 * 1024
    p = pk.boids_default_params(search_mode=1, init_mode=1)
    op = _op(orc, p)
    ag = W.sample_agents(n, 512, seed=17)
    s0 = orc.init(n, op, seed=1)
    s1 = W.jitter({k: s0[k] for k in KEYS}, 0.05, seed=18)
    o1, o1_idx, _, _ = orc.step_sample(s0, ag, DT, op)
    o2, o2_idx, _, _ = orc.step_sample(orc.State(s1), ag, DT, op)
    for world in (2, 4, 8):
        hs = [abi.boids_create_spatial(n, p, 1, r, world) for r in range(world)]
        try:
            emulated_step(hs, DT)
            g, g_idx, _, _ = gather_owned(hs, n)
            np.testing.assert_array_equal(g_idx[ag], o1_idx, err_msg=f"world {world} step 1")
            for k in KEYS:
                assert np.array_equal(g[k][ag], o1[k]), (world, 1, k)
            for h in hs:
                abi.boids_set_state(h, s1)
            emulated_step(hs, DT)
            g, g_idx, _, _ = gather_owned(hs, n)
            np.testing.assert_array_equal(g_idx[ag], o2_idx, err_msg=f"world {world} step 2")
            for k in KEYS:
                assert np.array_equal(g[k][ag], o2[k]), (world, 2, k)
        finally:
            for h in hs:
                abi.boids_destroy(h)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def test_spatial_flock_nccl_single_rank(boidslib, orc):
    """SpatialFlock over a real NCCL group of one rank (all_gather of the counts,
    all_to_all of the records on zero-copy views), against the oracle."""
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_breitbart09_b200 as pk
    from paper_conf_ipps_breitbart09_b200.spatial import SpatialFlock, gather_owned

    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ["MASTER_PORT"] = str(_free_port())
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        n = 4000
        p = pk.boids_default_params(search_mode=1, init_mode=1, world_radius=15.0)
        sf = SpatialFlock(n, p, seed=3)
        sf.step(DT, 3)
        g, g_idx, _, _ = gather_owned([sf.h], n)
        sf.close()
        op = _op(orc, p)
        o = orc.init(n, op, seed=3)
        for _ in range(3):
            o, o_idx, _, _ = orc.step(o, DT, op)
        assert np.array_equal(g_idx, o_idx)
        for k in KEYS:
            assert np.array_equal(g[k], o[k]), k
    finally:
        dist.destroy_process_group()
