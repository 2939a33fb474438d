"""Per-class kernel times of one rank of an emulated G-rank spatial decomposition (development aid).
    python tools/spatial_profile.py [G] [workload]"""
import sys

sys.path.insert(0, '.')
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
import workloads as W  # noqa: E402
from paper_conf_ipps_breitbart09_b200 import abi  # noqa: E402
from paper_conf_ipps_breitbart09_b200.spatial import emulated_step  # noqa: E402

G = int(sys.argv[1]) if len(sys.argv) > 1 else 8
cfg = W.CONFIGS[sys.argv[2] if len(sys.argv) > 2 else "c5"]
p = pk.boids_default_params(init_mode=cfg.init_mode, search_mode=1)
hs = [abi.boids_create_spatial(cfg.n, p, 1, r, G) for r in range(G)]
for _ in range(3):
    emulated_step(hs, float(W.DT))
f0 = [abi.boids_info(h).fallbacks for h in hs]
for h in hs:
    abi.boids_set_option(h, abi.BOIDS_OPT_PROFILE, 1)
    abi.boids_get_profile(h, reset=True)
for _ in range(5):
    emulated_step(hs, float(W.DT))
torch.cuda.synchronize()
for r, h in enumerate(hs):
    prof = abi.boids_get_profile(h, reset=True)
    own = abi.boids_spatial_owned(h).sum()
    far = (abi.boids_info(h).fallbacks - f0[r]) / 5
    print(f"rank {r} owned {own} far/step {far:.0f}: " + ", ".join(f"{k}={v[0] / 5 * 1e3:.1f}us" for k, v in prof.items() if v[1]))
