"""A/B of BOIDS_OPT_BALANCE (k_sym feedback split) on one box (development aid).
python tools/ab_balance.py c4 c3"""
import sys

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
from paper_conf_ipps_breitbart09_b200 import abi  # noqa: E402
import workloads as W  # noqa: E402

for name in sys.argv[1:] or ["c4"]:
    c = W.CONFIGS[name]
    K = 10 if c.n > 20000 else 50
    res = {0: [], 1: []}
    for rep in range(3):
        for bal in (0, 1):
            f = pk.Flock(c.n, pk.boids_default_params(init_mode=c.init_mode), seed=1)
            abi.boids_set_option(f.h, abi.BOIDS_OPT_BALANCE, bal)
            f.step(float(W.DT), 5)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            f.step(float(W.DT), K)
            e1.record()
            torch.cuda.synchronize()
            res[bal].append(e0.elapsed_time(e1) / K * 1e3)
            f.close()
    print(f"{name}: balance=0 " + " ".join(f"{v:.1f}" for v in res[0]) + " | balance=1 " +
          " ".join(f"{v:.1f}" for v in res[1]) + " us/step", flush=True)
