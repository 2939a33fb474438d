"""Multi-GPU path on one GPU (the pool gives one GPU per call).

* Shard emulation: G shard handles (boids_create_shard, ranks
  0..G-1) in one process; the per-step NCCL all-gather is emulated by device
  copies of every rank's send slice into every rank's full buffer (the exact
  layout all_gather_into_tensor produces).  The gathered state after k steps
  and the last step's neighbour lists must be bit-identical to the CPU
  oracle's k steps from its own Appendix-B init (same per-agent arithmetic,
  same (d2, index) order, whatever the partition).
* ShardedFlock over a real NCCL process group of size 1 (torch.distributed,
  all_gather_into_tensor on zero-copy views of the library's buffers), against
  the oracle the same way.
"""
import os
import socket

import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu
KEYS = ("pos", "fwd", "up", "side", "speed")
DT = float(W.DT)


def _emulated_run(pk, n, world, params, steps, seed=1):
    import torch

    from paper_conf_ipps_breitbart09_b200 import abi
    from paper_conf_ipps_breitbart09_b200.shard import device_view

    dev = torch.device("cuda", 0)
    hs = [abi.boids_create_shard(n, params, seed, r, world) for r in range(world)]
    try:
        stream = torch.cuda.current_stream().cuda_stream
        views = []
        for h in hs:
            abi.boids_set_stream(h, stream)
            send, full, nbytes = abi.boids_shard_buffers(h)
            views.append((device_view(send, nbytes, dev), device_view(full, nbytes * world, dev), nbytes // 4))
        for _ in range(steps):
            for r, (send, _, nf) in enumerate(views):  # all-gather: rank r's slice -> every full buffer
                for (_, full, _) in views:
                    full[r * nf:(r + 1) * nf].copy_(send)
            for h in hs:
                abi.boids_step_shard(h, DT)
        torch.cuda.synchronize()
        parts = [abi.boids_get_state(h) for h in hs]
        nbrs = [abi.boids_get_neighbors(h)[0] for h in hs]
        return {k: np.concatenate([p[k] for p in parts]) for k in KEYS}, np.concatenate(nbrs)
    finally:
        for h in hs:
            abi.boids_destroy(h)


@pytest.mark.parametrize("mode,n,world,steer", [(0, 3000, 2, 0), (0, 5000, 3, 0), (0, 1000, 8, 0), (1, 20000, 4, 0),
                                                (1, 777, 2, 0), (0, 3000, 3, 1), (1, 5000, 2, 1)])
def test_shard_emulation_bitidentical(boidslib, orc, mode, n, world, steer):
    """steer = 1: OpenSteer steering, whose smoothed accelerations live with the owner."""
    import paper_conf_ipps_breitbart09_b200 as pk

    p = pk.boids_default_params(init_mode=1, search_mode=mode, world_radius=20.0, steer_mode=steer)
    steps = 4
    got, got_nbr = _emulated_run(pk, n, world, p, steps)
    ref, ref_nbr = _oracle_run(orc, n, p, steps, seed=1)
    assert np.array_equal(got_nbr, ref_nbr)
    for k in KEYS:
        assert np.array_equal(got[k], ref[k]), k


def _oracle_run(orc, n, p, steps, seed):
    """The oracle's `steps` synchronous steps from its own Appendix-B init; returns
    the state and the last step's neighbour lists."""
    op = orc.default_params(**{name: getattr(p, name) for name, _ in p._fields_})
    o = orc.init(n, op, seed=seed)
    idx = None
    for _ in range(steps):
        o, idx, _, _ = orc.step(o, DT, op)
    return o, idx


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_sharded_flock_nccl_single_rank(boidslib, orc):
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_breitbart09_b200 as pk
    from paper_conf_ipps_breitbart09_b200.shard import ShardedFlock

    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ["MASTER_PORT"] = str(_free_port())
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        p = pk.boids_default_params(init_mode=1)
        n = 4000
        sf = ShardedFlock(n, p, seed=3)
        sf.step(DT, 5)
        got = sf.state()
        got_nbr = sf.neighbors()[0]
        sf.close()
        ref, ref_nbr = _oracle_run(orc, n, p, 5, seed=3)
        assert np.array_equal(got_nbr, ref_nbr)
        for k in KEYS:
            assert np.array_equal(got[k], ref[k]), k
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("n,world,steps", [(9000, 2, 5), (20000, 3, 4), (20000, 4, 4), (30001, 8, 3), (6000, 3, 12)])
def test_symshard_emulation_oracle(boidslib, orc, n, world, steps):
    """Sym-shards: the unordered-pair triangle split over `world` index shards
    (boids_symshard_*), both exchanges emulated by device copies; the gathered
    lists and states after `steps` steps equal the oracle's bit for bit."""
    import torch

    import paper_conf_ipps_breitbart09_b200 as pk
    from paper_conf_ipps_breitbart09_b200 import abi
    from paper_conf_ipps_breitbart09_b200.shard import _SymViews, device_view, emulated_symshard_step

    p = pk.boids_default_params(init_mode=1, world_radius=25.0)
    dev = torch.device("cuda", 0)
    hs = [abi.boids_create_shard(n, p, 1, r, world) for r in range(world)]
    try:
        stream = torch.cuda.current_stream().cuda_stream
        pos = []
        for h in hs:
            abi.boids_set_stream(h, stream)
            send, full, nbytes = abi.boids_shard_buffers(h)
            pos.append((device_view(send, nbytes, dev), device_view(full, nbytes * world, dev), nbytes // 4))
        m = abi.boids_info(hs[0]).slice
        views = {"pos": pos, "sym": [_SymViews(h, world, m, dev) for h in hs]}
        for t in range(steps):
            emulated_symshard_step(hs, views, DT, warm=t > 0)
        torch.cuda.synchronize()
        assert abi.boids_info(hs[0]).last_path == abi.BOIDS_PATH_SYM
        got = {k: np.concatenate([abi.boids_get_state(h)[k] for h in hs]) for k in KEYS}
        got_nbr = np.concatenate([abi.boids_get_neighbors(h)[0] for h in hs])
    finally:
        for h in hs:
            abi.boids_destroy(h)
    ref, ref_nbr = _oracle_run(orc, n, p, steps, seed=1)
    assert np.array_equal(got_nbr, ref_nbr)
    for k in KEYS:
        assert np.array_equal(got[k], ref[k]), k
