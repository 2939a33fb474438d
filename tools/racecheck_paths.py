"""Exercise one kernel path for compute-sanitizer (racecheck / synccheck / memcheck).

    python tools/racecheck_paths.py sym|scan|small|fused|grid|route|gridbig|scanbig|symshard|spatial
sym:   n = 9000 brute force, 3 steps (k_fused cold, then k_sym_prep + k_sym + k_select1 + k_route warm)
scan:  n = 3000 brute force, 3 steps, k_small off (k_bound + k_scan warm)
small: n = 3000 and n = 1024, 3 steps each (k_small with 16 and 32 threads per query)
symshard: 2 emulated sym-shard ranks, n = 9000, 3 steps (k_ss_lim, cellsort, spbuild, k_sym range, k_ss_select)
spatial: 2 emulated spatial ranks, n = 6000 grid, 3 steps (slab binning, k_grid, pack / unpack)
fused: n = 3000, every step on the cluster kernel (BOIDS_KERNEL_CLUSTER), 16-CTA clusters forced
grid:  n = 5000 grid mode, 3 steps (binning + k_grid + k_grid_far)
route: n = 9000 in a small world with a long dt: agents wrap and are routed to k_route
gridbig / scanbig: denser / larger cases whose TMA rings reuse every stage many times
"""
import sys

sys.path.insert(0, '.')
import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
from paper_conf_ipps_breitbart09_b200 import abi  # noqa: E402

which = sys.argv[1]
if which == "sym":
    f = pk.Flock(9000, pk.boids_default_params(), seed=3)
    f.step(1 / 60, 3)
elif which == "scan":
    f = pk.Flock(3000, pk.boids_default_params(), seed=3)
    abi.boids_set_option(f.h, abi.BOIDS_OPT_SMALL, 0)
    f.step(1 / 60, 3)
elif which == "small":
    for n in (1024, 3000):
        g = pk.Flock(n, pk.boids_default_params(), seed=3)
        g.step(1 / 60, 3)
        g.sync()
        assert g.info().last_path == abi.BOIDS_PATH_SMALL
        g.close()
    f = pk.Flock(100, pk.boids_default_params(), seed=3)
    f.step(1 / 60, 2)
elif which == "fused":
    f = pk.Flock(3000, pk.boids_default_params(), seed=3, kernel=2, cluster=16)
    f.step(1 / 60, 2)
elif which == "grid":
    f = pk.Flock(5000, pk.boids_default_params(search_mode=1, init_mode=1, world_radius=20.0), seed=3)
    f.step(1 / 60, 3)
elif which == "gridbig":  # dense items: many tiles per item, ring stages reused
    f = pk.Flock(60000, pk.boids_default_params(search_mode=1, init_mode=1, world_radius=20.0), seed=3)
    f.step(1 / 60, 2)
elif which == "scanbig":  # n < 8192 keeps k_scan (k_small off); many tiles per CTA
    f = pk.Flock(8000, pk.boids_default_params(), seed=3)
    abi.boids_set_option(f.h, abi.BOIDS_OPT_SMALL, 0)
    f.step(1 / 60, 3)
elif which == "symshard":
    import torch
    from paper_conf_ipps_breitbart09_b200.shard import _SymViews, device_view, emulated_symshard_step
    world, n = 2, 9000
    p = pk.boids_default_params(init_mode=1, world_radius=25.0)
    dev = torch.device("cuda", 0)
    hs = [abi.boids_create_shard(n, p, 3, r, world) for r in range(world)]
    stream = torch.cuda.current_stream().cuda_stream
    pos = []
    for h in hs:
        abi.boids_set_stream(h, stream)
        send, full, nbytes = abi.boids_shard_buffers(h)
        pos.append((device_view(send, nbytes, dev), device_view(full, nbytes * world, dev), nbytes // 4))
    m = abi.boids_info(hs[0]).slice
    views = {"pos": pos, "sym": [_SymViews(h, world, m, dev) for h in hs]}
    for t in range(3):
        emulated_symshard_step(hs, views, 1 / 60, warm=t > 0)
    torch.cuda.synchronize()
    assert abi.boids_info(hs[0]).last_path == abi.BOIDS_PATH_SYM
    for h in hs:
        abi.boids_destroy(h)
    print("ok", which, flush=True)
    sys.exit(0)
elif which == "spatial":
    from paper_conf_ipps_breitbart09_b200.spatial import emulated_step
    world, n = 2, 6000
    p = pk.boids_default_params(search_mode=1, init_mode=1, world_radius=20.0)
    hs = [abi.boids_create_spatial(n, p, 3, r, world) for r in range(world)]
    for t in range(3):
        emulated_step(hs, 1 / 60)
    for h in hs:
        abi.boids_sync(h)
        abi.boids_destroy(h)
    print("ok", which, flush=True)
    sys.exit(0)
elif which == "route":
    f = pk.Flock(9000, pk.boids_default_params(init_mode=1, world_radius=12.0, max_speed=30.0), seed=5)
    f.step(0.05, 4)
f.sync()
print("ok", which, "fallbacks", f.info().fallbacks, flush=True)
f.close()
