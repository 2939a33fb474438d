"""Multi-process (world size 2 and 3) checks of the sharded step's host logic on CPU/gloo.

The GPU data path (ShardedFlock: NCCL all-gather + boids_step_shard) cannot run
here; these tests exercise everything around it with the same helpers
(paper_conf_ipps_breitbart09_b200.shard): the partition rule, the padded
[pos4 | fwd4] send-slice image with NaN phantoms, all_gather_into_tensor's
layout, and its inverse -- and that an index-sharded step computed from the
gathered state equals the unsharded step (here with the oracle as the per-rank
compute, since there is no GPU).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import oracle
        import workloads as W
        from paper_conf_ipps_breitbart09_b200.shard import pack_slice, partition, unpack_full

        s = oracle.init(n, seed=4)
        lo, hi, m = partition(n, world, rank)
        send = torch.from_numpy(pack_slice(s["pos"], s["fwd"], s["speed"], lo, hi, m).ravel())
        full = torch.empty(world * send.numel(), dtype=torch.float32)
        dist.all_gather_into_tensor(full, send)
        pos, fwd, speed = unpack_full(full.numpy(), n, m, world)
        assert np.array_equal(pos, s["pos"]) and np.array_equal(fwd, s["fwd"]) and np.array_equal(speed, s["speed"])
        phantoms = full.numpy().reshape(world, 2, m, 4)[:, 0, :, :3].reshape(-1, 3)[n:]
        assert np.isnan(phantoms).all()
        # per-rank step of the owned agents from the gathered state
        mine = np.arange(lo, hi, dtype=np.int64)
        gathered = oracle.State(pos=pos.copy(), fwd=fwd.copy(), up=s["up"], side=s["side"], speed=speed.copy())
        out, idx, cnt, F = oracle.step_sample(gathered, mine, float(W.DT)) if hi > lo else (None,) * 4
        res = np.zeros((m, 4), np.float32)
        res[:, :] = np.nan
        if hi > lo:
            res[: hi - lo, :3] = out["pos"]
            res[: hi - lo, 3] = out["speed"]
        allres = torch.empty(world * m * 4, dtype=torch.float32)
        dist.all_gather_into_tensor(allres, torch.from_numpy(res.ravel()))
        if rank == 0:
            r = allres.numpy().reshape(world * m, 4)[:n]
            ref, _, _, _ = oracle.step(s, float(W.DT))
            assert np.array_equal(r[:, :3], ref["pos"]) and np.array_equal(r[:, 3], ref["speed"])
        dist.barrier()
        dist.destroy_process_group()
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        import traceback

        q.put((rank, traceback.format_exc() + repr(e)))


@pytest.mark.parametrize("world,n", [(2, 1000), (2, 513), (3, 700), (2, 100)])
def test_sharded_step_matches_unsharded(orc, world, n):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert all(v == "ok" for v in res.values()), res
