"""Per-CTA timeline of k_sym (BOIDS_OPT_PHASES): duration vs position in the item space."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import paper_conf_ipps_breitbart09_b200 as pk
from paper_conf_ipps_breitbart09_b200 import abi
import workloads as W

name = sys.argv[1] if len(sys.argv) > 1 else "c4"
cfg = W.CONFIGS[name]
p = pk.boids_default_params(init_mode=cfg.init_mode, search_mode=cfg.search_mode)
with pk.Flock(cfg.n, p, seed=1) as f:
    f.step(float(W.DT), 4)
    abi.boids_set_option(f.h, abi.BOIDS_OPT_PHASES, 1024)
    f.step(float(W.DT), 1)
    ph = abi.boids_get_phases(f.h, 1024).astype(np.int64)
ph = ph[ph[:, 1] > 0]
t0 = ph[:, 0].min()
dur = (ph[:, 1] - ph[:, 0]) / 1e3
start = (ph[:, 0] - t0) / 1e3
print(f"{name}: {len(ph)} CTAs, start spread {start.max():.1f} us, dur min/med/max {dur.min():.1f}/{np.median(dur):.1f}/{dur.max():.1f} us")
order = np.argsort(ph[:, 2])
for k in range(0, len(order), max(1, len(order) // 37)):
    i = order[k]
    print(f"  cta L0={ph[i,2]:>9d} L1={ph[i,3]:>9d} start {start[i]:7.1f} dur {dur[i]:8.1f} us slow {ph[i,4]:>6d} maxwait {ph[i,5]/1965:8.1f} maxemit {ph[i,6]/1965:8.1f} w0wait {ph[i,7]/1965:8.1f} us")
