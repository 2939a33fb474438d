"""Per-phase timing of the fused kernel from in-kernel %globaltimer stamps (development aid).

python tools/phases.py c3 [cluster ...]"""
import sys

import numpy as np

sys.path.insert(0, '.')
import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
from paper_conf_ipps_breitbart09_b200 import abi  # noqa: E402
import workloads as W  # noqa: E402

import os
SCAN = os.environ.get("SCAN") == "1"
NAMES = (["start", "setup done", "scan end", "flushed", "mbar init", "run start", "queries loaded", "tma issued"] if SCAN else
         ["start", "t0+sync", "scan end", "lists synced", "merged", "epilogue", "exit"])
cfg = W.CONFIGS[sys.argv[1]]
clusters = [int(x) for x in sys.argv[2:]] or [0]
for cl in clusters:
    f = pk.Flock(cfg.n, pk.boids_default_params(init_mode=cfg.init_mode), seed=1, cluster=cl, profile=True)
    abi.boids_set_option(f.h, abi.BOIDS_OPT_PHASES, 8192)
    f.step(float(W.DT), 4)
    f.sync()
    if SCAN:
        abi.boids_set_option(f.h, abi.BOIDS_OPT_PHASES, 0)
        abi.boids_set_option(f.h, abi.BOIDS_OPT_PHASES, 8192)
    f.profile(reset=True)
    f.step(float(W.DT), 1)
    prof = f.profile()
    ph = abi.boids_get_phases(f.h, 8192).astype(np.int64)
    used = ph[:, 0] > 0
    ph = ph[used]
    t0 = ph[:, 0].min()
    rel = (ph - t0) / 1e3  # us
    info = f.info()
    print(f"{cfg.name} n={cfg.n} cluster={info.cluster} ctas={used.sum()} kernel={prof['fused_or_search'][0]*1e3:.1f}us "
          f"binning={prof['binning'][0]*1e3:.1f}us")
    for k, nm in enumerate(NAMES):
        col = rel[:, k]
        ok = ph[:, k] > 0
        if ok.any():
            c = col[ok]
            print(f"  {nm:14s} min {c.min():8.1f}  med {np.median(c):8.1f}  max {c.max():8.1f} us")
    dur = rel[:, 2] - rel[:, 1]
    print(f"  scan duration  min {dur.min():.1f} med {np.median(dur):.1f} max {dur.max():.1f} us")
    f.close()
