"""Emulated sym-shard steps (development aid): python tools/symshard_debug.py n world steps"""
import sys

sys.path.insert(0, '.')
import torch  # noqa: E402

import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
from paper_conf_ipps_breitbart09_b200 import abi  # noqa: E402
from paper_conf_ipps_breitbart09_b200.shard import _SymViews, device_view, emulated_symshard_step  # noqa: E402

n, world, steps = (int(x) for x in sys.argv[1:4])
p = pk.boids_default_params(init_mode=1, world_radius=25.0)
dev = torch.device("cuda", 0)
hs = [abi.boids_create_shard(n, p, 1, r, world) for r in range(world)]
stream = torch.cuda.current_stream().cuda_stream
pos = []
for h in hs:
    abi.boids_set_stream(h, stream)
    send, full, nbytes = abi.boids_shard_buffers(h)
    pos.append((device_view(send, nbytes, dev), device_view(full, nbytes * world, dev), nbytes // 4))
m = abi.boids_info(hs[0]).slice
views = {"pos": pos, "sym": [_SymViews(h, world, m, dev) for h in hs]}
for t in range(steps):
    emulated_symshard_step(hs, views, 1 / 60, warm=t > 0)
    torch.cuda.synchronize()
    print("step", t, "ok", flush=True)
