"""Quick device timing of the step at a few sizes (development aid)."""
import sys, time
import torch
sys.path.insert(0, '.')
import paper_conf_ipps_breitbart09_b200 as pk
from paper_conf_ipps_breitbart09_b200 import abi
import workloads as W

VOTE = int(__import__("os").environ.get("VOTE_U", "4"))
for name in sys.argv[1:] or ["c2", "c3", "c4"]:
    c = W.CONFIGS[name]
    for kernel in (0,):
        p = pk.boids_default_params(init_mode=c.init_mode)
        f = pk.Flock(c.n, p, seed=1, kernel=kernel, profile=True)
        abi.boids_set_option(f.h, abi.BOIDS_OPT_VOTE_U, VOTE)
        steps = c.steps if c.n <= 16384 else 5
        f.step(float(W.DT), 3); f.sync(); f.profile(reset=True)
        s0 = f.info()
        t0 = time.perf_counter()
        f.step(float(W.DT), steps); f.sync()
        wall = time.perf_counter() - t0
        prof = f.profile()
        i0 = f.info()
        ms = sum(v[0] for v in prof.values())
        pairs = c.n * c.n * steps
        print(f"{name} n={c.n} kernel={kernel} cluster={f.info().cluster} steps={steps} wall={wall*1e3:.2f}ms "
              f"dev={ms:.3f}ms per_step={ms/steps*1e3:.1f}us agent-steps/s={c.n*steps/(ms/1e3):.3e} "
              f"lane-op frac={8*pairs/(ms/1e3)/(148*128*1.965e9):.3f} slow={(i0.slow_groups-s0.slow_groups)/max(i0.vote_groups-s0.vote_groups,1):.4f} fallbacks={i0.fallbacks-s0.fallbacks} "
              f"prof={ {k: round(v[0]/max(v[1],1)*1e3, 1) for k, v in prof.items() if v[1]} }us", flush=True)
        f.close()
