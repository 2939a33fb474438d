"""Does the step's time depend on how agent ids map to space?  (development aid)

The kernels gather neighbours' pos4/fwd4 by agent id (warm bound, steering,
P:406 Listing 5.5).  With ids spatially random (the synthetic init) each gather
is a random 16 B access; if ids are renumbered in Morton order of the position
the same gathers hit sectors that nearby queries also touch.  Same state, same
n, only the numbering differs:  python tools/locality_probe.py c5 c4
"""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_ipps_breitbart09_b200 as pk
import workloads as W


def morton(pos, bits=10):
    lo, hi = pos.min(0), pos.max(0)
    q = ((pos - lo) / np.maximum(hi - lo, 1e-6) * ((1 << bits) - 1)).astype(np.uint64)
    code = np.zeros(len(pos), np.uint64)
    for b in range(bits):
        for d in range(3):
            code |= ((q[:, d] >> np.uint64(b)) & np.uint64(1)) << np.uint64(3 * b + d)
    return np.argsort(code, kind="stable")


for name in sys.argv[1:] or ["c5", "c4"]:
    c = W.CONFIGS[name]
    p = pk.boids_default_params(init_mode=c.init_mode, search_mode=c.search_mode)
    for order in ("init", "morton"):
        f = pk.Flock(c.n, p, seed=1, profile=True)
        f.step(float(W.DT), 3)
        f.sync()
        s = f.state()
        perm = morton(s["pos"]) if order == "morton" else np.arange(c.n)
        f.set_state({k: np.ascontiguousarray(v[perm]) for k, v in s.items()})
        f.step(float(W.DT), 3)
        f.sync()
        f.profile(reset=True)
        steps = 10
        i0 = f.info()
        f.step(float(W.DT), steps)
        f.sync()
        prof = f.profile()
        i1 = f.info()
        ms = sum(v[0] for v in prof.values())
        top = sorted(((v[0] / max(v[1], 1) * 1e3, k) for k, v in prof.items() if v[1]), reverse=True)[:4]
        print(f"{name} {order:6s} {ms / steps * 1e3:8.1f} us/step  agent-steps/s {c.n * steps / (ms / 1e3):.3e}  "
              f"top {[(k, round(t, 1)) for t, k in top]}  slow/vote {(i1.slow_groups - i0.slow_groups) / max(i1.vote_groups - i0.vote_groups, 1):.4f} "
              f"vote_groups/step {(i1.vote_groups - i0.vote_groups) / steps:.3e} fallbacks/step {(i1.fallbacks - i0.fallbacks) / steps:.1f}", flush=True)
        f.close()
