"""Warm-path diagnostics on the GPU: vote groups that took the slow path, hit-buffer
fallbacks and per-class kernel times, for k_sym vs k_scan (sym on/off)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_breitbart09_b200 as pk
from paper_conf_ipps_breitbart09_b200 import abi
import workloads as W

for name in sys.argv[1:] or ["c3", "c4"]:
    cfg = W.CONFIGS[name]
    for sym in (1, 0):
        p = pk.boids_default_params(init_mode=cfg.init_mode, search_mode=cfg.search_mode)
        with pk.Flock(cfg.n, p, seed=1, symmetric=bool(sym)) as f:
            f.step(float(W.DT), 4)
            i0 = f.info()
            abi.boids_set_option(f.h, abi.BOIDS_OPT_PROFILE, 1)
            abi.boids_get_profile(f.h, reset=True)
            f.step(float(W.DT), 3)
            prof = abi.boids_get_profile(f.h, reset=True)
            i1 = f.info()
            sg, vg, fb = i1.slow_groups - i0.slow_groups, i1.vote_groups - i0.vote_groups, i1.fallbacks - i0.fallbacks
            print(f"{name} sym={sym}: slow {sg/3:.0f}/{vg/3:.0f} per step ({sg/max(vg,1):.4f}), fallbacks/step {fb/3:.1f}, "
                  f"ms/launch " + ", ".join(f"{k}={v[0]/max(v[1],1):.4f}" for k, v in prof.items() if v[1]), flush=True)
