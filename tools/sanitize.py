"""Drive every kernel path at small ragged sizes (run under compute-sanitizer)."""
import sys

sys.path.insert(0, '.')
import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
from paper_conf_ipps_breitbart09_b200 import abi  # noqa: E402

for n in (1, 31, 1000, 1024, 9000):
    for mode in (0, 1):
        for kernel in ((0, 1, 2) if mode == 0 and n < 9000 else (0,)):
            p = pk.boids_default_params(search_mode=mode, init_mode=1, world_radius=15.0,
                                        steer_mode=1 if n == 1000 else 0)
            with pk.Flock(n, p, seed=3, kernel=kernel, record_steering=True) as f:
                f.step(0.05, 3)
                f.set_state(f.state())
                f.step(0.05, 2)
                f.neighbors(), f.steering(), f.sync()
    print("ok", n, flush=True)
# grid with the default world: 39k search cells -> the many-CTA binning scan;
# think mode (whole-row items)
for think in (1, 3):
    p = pk.boids_default_params(search_mode=1, init_mode=1, think_every=think)
    with pk.Flock(3000, p, seed=4) as f:
        f.step(0.05, 4)
        f.sync()
print("ok grid-large")
# shard handles (emulated 2-rank all-gather is in tests; here one rank of 2)
h = abi.boids_create_shard(1000, pk.boids_default_params(), 1, 1, 2)
abi.boids_step_shard(h, 0.05)
abi.boids_sync(h)
abi.boids_destroy(h)
print("done")
