"""Routed / overflowed agents per rank of the emulated sym-shard step (development aid).
python tools/symshard_route.py [workload] [G ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
import workloads as W  # noqa: E402
from paper_conf_ipps_breitbart09_b200 import abi  # noqa: E402
from paper_conf_ipps_breitbart09_b200.shard import _SymViews, device_view, emulated_symshard_step  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c4"
cfg = W.CONFIGS[name]
params = pk.boids_default_params(init_mode=cfg.init_mode, search_mode=cfg.search_mode)
dev = torch.device("cuda", 0)
for G in [int(x) for x in sys.argv[2:]] or [1, 8]:
    hs = [abi.boids_create_shard(cfg.n, params, 1, r, G) for r in range(G)]
    pos = []
    for h in hs:
        send, full, nbytes = abi.boids_shard_buffers(h)
        pos.append((device_view(send, nbytes, dev), device_view(full, nbytes * G, dev), nbytes // 4))
    m = abi.boids_info(hs[0]).slice
    views = {"pos": pos, "sym": [_SymViews(h, G, m, dev) for h in hs]}
    for k in range(6):
        f0 = [abi.boids_info(h).fallbacks for h in hs]
        emulated_symshard_step(hs, views, float(W.DT), warm=k > 0)
        torch.cuda.synchronize()
        f1 = [abi.boids_info(h).fallbacks for h in hs]
        print(f"G={G} step {k}: fallbacks per rank {[b - a for a, b in zip(f0, f1)]}", flush=True)
    for h in hs:
        abi.boids_destroy(h)
