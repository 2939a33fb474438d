"""Emulated spatial decomposition: warm up, then one more step of every rank (for ncu launch lists)."""
import sys

sys.path.insert(0, '.')
import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
import workloads as W  # noqa: E402
from paper_conf_ipps_breitbart09_b200 import abi  # noqa: E402
from paper_conf_ipps_breitbart09_b200.spatial import emulated_step  # noqa: E402

G = int(sys.argv[1]) if len(sys.argv) > 1 else 8
cfg = W.CONFIGS[sys.argv[2] if len(sys.argv) > 2 else "c5"]
p = pk.boids_default_params(init_mode=cfg.init_mode, search_mode=1)
hs = [abi.boids_create_spatial(cfg.n, p, 1, r, G) for r in range(G)]
for _ in range(4):
    emulated_step(hs, float(W.DT))
for h in hs:
    abi.boids_sync(h)
print("done")
