"""Exercise TMA ring stage reuse (run under compute-sanitizer racecheck)."""
import sys
sys.path.insert(0, '.')
import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
which = sys.argv[1]
n = int(sys.argv[2])
mode = 1 if which == "grid" else 0
p = pk.boids_default_params(search_mode=mode, init_mode=1)
with pk.Flock(n, p, seed=3) as f:
    f.step(0.05, 2)
    f.sync()
print("ok", which, n, flush=True)
