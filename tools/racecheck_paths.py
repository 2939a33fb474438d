"""Exercise one kernel path for compute-sanitizer (racecheck / synccheck / memcheck).

    python tools/racecheck_paths.py sym|scan|fused|grid|route
sym:   n = 9000 brute force, 3 steps (k_fused cold, then k_sym_prep + k_sym + k_select1 + k_route warm)
scan:  n = 3000 brute force, 3 steps (k_bound + k_scan warm)
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
    f.step(1 / 60, 3)
elif which == "fused":
    f = pk.Flock(3000, pk.boids_default_params(), seed=3, kernel=2, cluster=16)
    f.step(1 / 60, 2)
elif which == "grid":
    f = pk.Flock(5000, pk.boids_default_params(search_mode=1, init_mode=1, world_radius=20.0), seed=3)
    f.step(1 / 60, 3)
elif which == "gridbig":  # dense items: many tiles per item, ring stages reused
    f = pk.Flock(60000, pk.boids_default_params(search_mode=1, init_mode=1, world_radius=20.0), seed=3)
    f.step(1 / 60, 2)
elif which == "scanbig":  # n < 8192 keeps k_scan; many tiles per CTA
    f = pk.Flock(8000, pk.boids_default_params(), seed=3)
    f.step(1 / 60, 3)
elif which == "route":
    f = pk.Flock(9000, pk.boids_default_params(init_mode=1, world_radius=12.0, max_speed=30.0), seed=5)
    f.step(0.05, 4)
f.sync()
print("ok", which, "fallbacks", f.info().fallbacks, flush=True)
f.close()
