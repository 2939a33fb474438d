"""Agents finished by the route kernels per warm step (k_sym_prep routing + hit-buffer
overflow; grid: far queries) and their cost (development aid).  python tools/route_stats.py c4 c5"""
import sys

sys.path.insert(0, '.')
import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
import workloads as W  # noqa: E402

for name in sys.argv[1:] or ["c4"]:
    c = W.CONFIGS[name]
    f = pk.Flock(c.n, pk.boids_default_params(init_mode=c.init_mode, search_mode=c.search_mode), seed=1, profile=True)
    dt = float(W.DT)
    f.step(dt, 3)
    f.sync()
    f.profile(reset=True)
    i0 = f.info()
    f.step(dt, 5)
    f.sync()
    i1 = f.info()
    prof = f.profile(reset=True)
    print(f"{name} n={c.n}: routed/step {(i1.fallbacks - i0.fallbacks) / 5:.0f} "
          f"({(i1.fallbacks - i0.fallbacks) / 5 / c.n * 100:.2f}%), per-step us: "
          + ", ".join(f"{k}={v[0] / max(v[1], 1) * 1e3 * v[1] / 5:.1f}" for k, v in prof.items() if v[1]), flush=True)
    f.close()
