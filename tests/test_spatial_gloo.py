"""Host logic of the spatial decomposition's record exchange (spatial.py) on
CPU: the inbox layout and the point-to-point routing, world sizes 2 and 3 over
gloo (the same calls SpatialFlock makes over NCCL)."""
import os
import socket

import numpy as np
import pytest


def test_inbox_layout():
    from paper_conf_ipps_breitbart09_b200.spatial import inbox_layout

    c = np.array([[0, 3, 1], [2, 0, 0], [5, 4, 0]])
    off, tot = inbox_layout(c)
    assert tot.tolist() == [7, 7, 1]
    assert off[:, 0].tolist() == [0, 0, 2] and off[:, 1].tolist() == [0, 3, 3] and off[:, 2].tolist() == [0, 1, 1]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_breitbart09_b200.spatial import inbox_layout, route

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        rng = np.random.default_rng(7)
        counts = rng.integers(0, 5, size=(world, world))  # the same table on every rank
        # record k from s to d: 2 float4 = [s, d, k, 0] x 2 (stands in for a halo record)
        outbox = torch.zeros(world, 8, 8)
        for d in range(world):
            for k in range(counts[rank, d]):
                outbox[d, k, :4] = torch.tensor([rank, d, k, 0.0])
                outbox[d, k, 4:] = torch.tensor([rank, d, k, 1.0])
        off, tot = inbox_layout(counts)
        inbox = torch.full((int(counts.sum()), 8), -1.0)
        inputs = [outbox[d, :counts[rank, d]] for d in range(world)]
        outputs = [inbox[off[s, rank]:off[s, rank] + counts[s, rank]] for s in range(world)]
        route(dist, None, rank, world, inputs, outputs)
        got = inbox[:tot[rank]]
        want = [[s, rank, k, 0.0] for s in range(world) for k in range(counts[s, rank])]
        q.put((rank, got[:, :4].tolist() == want and bool((got[:, 7] == 1).all())))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_route_gloo(world):
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    assert all(res[r] for r in range(world)), res
