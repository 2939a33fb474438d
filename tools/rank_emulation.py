"""Per-rank step times of the G-rank sharded step, emulated on ONE GPU (the pool
gives one GPU per call), and the G-GPU step time they project.

    python tools/rank_emulation.py --workload c5 --ranks 1 2 4 8 [--steps 5 --warmup 3] [--spatial | --symshard]

For each G: G shard handles (boids_create_shard, ranks 0..G-1) live in this
process; every step the NCCL all-gather is replaced by device copies of every
rank's [pos4 | fwd4] send slice into every rank's full buffer (the exact layout
all_gather_into_tensor produces), then each rank's boids_step_shard runs alone,
bracketed by CUDA events with the L2 flushed before it (as the bench's steps).
Reported per G: the max over ranks of the mean rank step time (what one GPU of
a G-GPU job would spend per step on compute) and the all-gather payload per
rank.  The projected G-GPU step = max rank time + all-gather time, the latter
estimated as the received bytes ((G-1)/G x 32 B x n) at NVLink 5's 900 GB/s per
direction plus a fixed 15 us of NCCL latency (an assumption, stated in the
output: no multi-GPU box was available to measure it).  The 1-GPU reference
is the single-rank handle's own step (boids_create, k_sym / k_grid), so the
projected scaling is against the best 1-GPU path, not against a 1-rank shard.

--spatial (grid workloads): spatial shards instead (boids_create_spatial, slab
ownership + halo layers; spatial.py).  Rank time = its boids_step_spatial +
boids_spatial_unpack of the records it received; the exchange is estimated
from the records actually sent (halo 32 B, migrant 128 B) at the same link rate
plus latency, point to point (a rank receives from its slab neighbours).

--symshard (brute-force workloads): sym-shards (shard.py ShardedFlock(sym=True)):
warm steps split the global unordered-pair triangle over the ranks.  Rank time =
its boids_symshard_prep + _search + _finish (each timed alone, L2 flushed before
the search); the exchange estimate adds the limits' all-gather ((G-1) x 4 B x
n/G) and the hit blocks' all-to-all ((G-1) x n/G x (hits_cap x 8 + 4) B, the fixed-size
blocks all_to_all_single moves) to the position all-gather, with one latency per
collective.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
import workloads as W  # noqa: E402
from paper_conf_ipps_breitbart09_b200 import abi  # noqa: E402
from paper_conf_ipps_breitbart09_b200.shard import device_view  # noqa: E402

NVLINK_GBS = 900.0   # NVLink 5 per direction per GPU (B200 spec)
NCCL_LAT_US = 15.0   # assumed fixed all-gather latency


def single_gpu_ms(cfg, params, steps, warmup, flush):
    with pk.Flock(cfg.n, params, seed=1) as f:
        f.step(float(W.DT), warmup)
        torch.cuda.synchronize()
        ts = []
        for k in range(steps):
            flush.fill_(float(k))
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            f.step(float(W.DT), 1)
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        return float(np.mean(ts)), int(f.info().last_path)


def emulate(cfg, params, G, steps, warmup, flush):
    dev = torch.device("cuda", 0)
    hs = [abi.boids_create_shard(cfg.n, params, 1, r, G) for r in range(G)]
    try:
        stream = torch.cuda.current_stream().cuda_stream
        views = []
        for h in hs:
            abi.boids_set_stream(h, stream)
            send, full, nbytes = abi.boids_shard_buffers(h)
            views.append((device_view(send, nbytes, dev), device_view(full, nbytes * G, dev), nbytes // 4))

        def gather():
            for r, (send, _, nf) in enumerate(views):
                for (_, full, _) in views:
                    full[r * nf:(r + 1) * nf].copy_(send)

        for _ in range(warmup):
            gather()
            for h in hs:
                abi.boids_step_shard(h, float(W.DT))
        torch.cuda.synchronize()
        per_rank = np.zeros((steps, G))
        for k in range(steps):
            gather()
            for r, h in enumerate(hs):
                flush.fill_(float(k * G + r))
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                abi.boids_step_shard(h, float(W.DT))
                b.record()
                torch.cuda.synchronize()
                per_rank[k, r] = a.elapsed_time(b)
        slice_bytes = views[0][2] * 4
        return per_rank.mean(0), slice_bytes, int(abi.boids_info(hs[0]).last_path)
    finally:
        for h in hs:
            abi.boids_destroy(h)


def emulate_spatial(cfg, params, G, steps, warmup, flush):
    from paper_conf_ipps_breitbart09_b200.spatial import _views, inbox_layout

    dev = torch.device("cuda", 0)
    hs = [abi.boids_create_spatial(cfg.n, params, 1, r, G) for r in range(G)]
    try:
        stream = torch.cuda.current_stream().cuda_stream
        for h in hs:
            abi.boids_set_stream(h, stream)
        per_rank = np.zeros((steps, G))
        recv_bytes = np.zeros((steps, G))
        for k in range(warmup + steps):
            ts = []
            for r, h in enumerate(hs):
                flush.fill_(float(k * G + r))
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                abi.boids_step_spatial(h, float(W.DT))
                b.record()
                ts.append((a, b))
            vs = [_views(h, G, dev) for h in hs]
            hc = np.stack([v["hc"] for v in vs])
            mc = np.stack([v["mc"] for v in vs])
            hoff, htot = inbox_layout(hc)
            moff, mtot = inbox_layout(mc)
            for d, vd in enumerate(vs):
                for s_, vs_ in enumerate(vs):
                    if hc[s_, d]:
                        vd["hin"][hoff[s_, d]:hoff[s_, d] + hc[s_, d]].copy_(vs_["hout"][d, :hc[s_, d]])
                    if mc[s_, d]:
                        vd["min"][moff[s_, d]:moff[s_, d] + mc[s_, d]].copy_(vs_["mout"][d, :mc[s_, d]])
            us = []
            for d, h in enumerate(hs):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                abi.boids_spatial_unpack(h, int(htot[d]), int(mtot[d]))
                b.record()
                us.append((a, b))
            torch.cuda.synchronize()
            if k >= warmup:
                for r in range(G):
                    per_rank[k - warmup, r] = ts[r][0].elapsed_time(ts[r][1]) + us[r][0].elapsed_time(us[r][1])
                    recv_bytes[k - warmup, r] = htot[r] * 32 + mtot[r] * 128
        return per_rank.mean(0), recv_bytes.mean(0)
    finally:
        for h in hs:
            abi.boids_destroy(h)


def emulate_symshard(cfg, params, G, steps, warmup, flush):
    from paper_conf_ipps_breitbart09_b200.shard import _SymViews, emulated_symshard_step

    dev = torch.device("cuda", 0)
    hs = [abi.boids_create_shard(cfg.n, params, 1, r, G) for r in range(G)]
    try:
        stream = torch.cuda.current_stream().cuda_stream
        pos = []
        for h in hs:
            abi.boids_set_stream(h, stream)
            send, full, nbytes = abi.boids_shard_buffers(h)
            pos.append((device_view(send, nbytes, dev), device_view(full, nbytes * G, dev), nbytes // 4))
        m = abi.boids_info(hs[0]).slice
        sv = [_SymViews(h, G, m, dev) for h in hs]
        views = {"pos": pos, "sym": sv}
        for k in range(warmup):
            emulated_symshard_step(hs, views, float(W.DT), warm=k > 0)
        torch.cuda.synchronize()

        def timed(fn, r, k):
            flush.fill_(float(k * G + r))
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            return (a, b)

        per_rank = np.zeros((steps, G))
        phases = np.zeros((steps, G, 3))
        for k in range(steps):
            for r, (send, _, nf) in enumerate(pos):
                for (_, full, _) in pos:
                    full[r * nf:(r + 1) * nf].copy_(send)
            ev = [[None] * 3 for _ in range(G)]
            for r, h in enumerate(hs):
                ev[r][0] = timed(lambda: abi.boids_symshard_prep(h), r, k)
            for r, v in enumerate(sv):
                for w in sv:
                    w.lim_full[r * m:(r + 1) * m].copy_(v.lim_send)
            for r, h in enumerate(hs):
                ev[r][1] = timed(lambda: abi.boids_symshard_search(h), r, k)
            for d, vd in enumerate(sv):
                for s_, vs in enumerate(sv):
                    kk = vd.block_keys
                    vd.recv[s_ * kk:(s_ + 1) * kk].copy_(vs.hits[d * kk:(d + 1) * kk])
                    vd.rcnt[s_ * m:(s_ + 1) * m].copy_(vs.hitcnt[d * m:(d + 1) * m])
            for r, h in enumerate(hs):
                ev[r][2] = timed(lambda: abi.boids_symshard_finish(h, float(W.DT)), r, k)
            torch.cuda.synchronize()
            for r in range(G):
                for ph in range(3):
                    phases[k, r, ph] = ev[r][ph][0].elapsed_time(ev[r][ph][1])
                per_rank[k, r] = phases[k, r].sum()
        assert int(abi.boids_info(hs[0]).last_path) == abi.BOIDS_PATH_SYM
        return per_rank.mean(0), phases.mean(0), pos[0][2] * 4, m, sv[0].block_keys * 4
    finally:
        for h in hs:
            abi.boids_destroy(h)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c5", choices=sorted(W.CONFIGS))
    ap.add_argument("--ranks", type=int, nargs="+", default=[1, 2, 4, 8])
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--spatial", action="store_true", help="spatial shards (grid workloads) instead of index shards")
    ap.add_argument("--symshard", action="store_true", help="sym-shards (brute-force workloads): triangle split")
    args = ap.parse_args()
    cfg = W.CONFIGS[args.workload]
    torch.cuda.set_device(0)
    params = pk.boids_default_params(init_mode=cfg.init_mode, search_mode=cfg.search_mode)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    t1, path1 = single_gpu_ms(cfg, params, args.steps, args.warmup, flush)
    out = {"workload": cfg.name, "n": cfg.n, "one_gpu_ms": t1, "one_gpu_path": path1,
           "assumptions": f"all-gather = (G-1)/G x 32 B x n at {NVLINK_GBS} GB/s + {NCCL_LAT_US} us",
           "ranks": {}}
    out["mode"] = "spatial shards" if args.spatial else ("sym-shards" if args.symshard else "index shards")
    for G in args.ranks:
        if args.symshard:
            per_rank, ph, slice_bytes, m, hit_block = emulate_symshard(cfg, params, G, args.steps, args.warmup, flush)
            recv = (G - 1) * (slice_bytes + m * 4 + hit_block + m * 4)
            ag_ms = 0.0 if G == 1 else (recv / (NVLINK_GBS * 1e9) * 1e3 + 3 * NCCL_LAT_US * 1e-3)
            proj = float(per_rank.max()) + ag_ms
            out["ranks"][G] = {"rank_ms_max": float(per_rank.max()), "rank_ms_min": float(per_rank.min()),
                               "phase_ms_max": {"prep": float(ph[:, 0].max()), "search": float(ph[:, 1].max()),
                                                "finish": float(ph[:, 2].max())},
                               "rank_path": abi.BOIDS_PATH_SYM, "exchange_recv_bytes": int(recv),
                               "exchange_ms_est": ag_ms, "projected_step_ms": proj,
                               "projected_speedup_vs_1gpu": t1 / proj}
            print(json.dumps({G: out["ranks"][G]}), flush=True)
            continue
        if args.spatial:
            per_rank, rb = emulate_spatial(cfg, params, G, args.steps, args.warmup, flush)
            recv, path = float(rb.max()), abi.BOIDS_PATH_GRID
            ag_ms = 0.0 if G == 1 else (recv / (NVLINK_GBS * 1e9) * 1e3 + NCCL_LAT_US * 1e-3)
            proj = float(per_rank.max()) + ag_ms
            out["ranks"][G] = {"rank_ms_max": float(per_rank.max()), "rank_ms_min": float(per_rank.min()),
                               "rank_path": path, "exchange_recv_bytes_max": int(recv), "exchange_ms_est": ag_ms,
                               "projected_step_ms": proj, "projected_speedup_vs_1gpu": t1 / proj}
            print(json.dumps({G: out["ranks"][G]}), flush=True)
            continue
        per_rank, slice_bytes, path = emulate(cfg, params, G, args.steps, args.warmup, flush)
        recv = (G - 1) * slice_bytes
        ag_ms = 0.0 if G == 1 else (recv / (NVLINK_GBS * 1e9) * 1e3 + NCCL_LAT_US * 1e-3)
        proj = float(per_rank.max()) + ag_ms
        out["ranks"][G] = {"rank_ms_max": float(per_rank.max()), "rank_ms_min": float(per_rank.min()),
                           "rank_path": path, "allgather_recv_bytes": int(recv), "allgather_ms_est": ag_ms,
                           "projected_step_ms": proj, "projected_speedup_vs_1gpu": t1 / proj}
        print(json.dumps({G: out["ranks"][G]}), flush=True)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
