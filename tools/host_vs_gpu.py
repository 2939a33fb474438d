"""Host-bound or GPU-bound?  Per-step device time of (a) one boids_step(dt, 1)
call per step bracketed by events (the bench pattern, L2 flushed before each),
(b) one boids_step(dt, K) call, (c) K back-to-back boids_step(dt, 1) calls
(development aid).  python tools/host_vs_gpu.py c1 c2 c3"""
import sys
import time

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
import workloads as W  # noqa: E402

K = 50
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda")
for name in sys.argv[1:] or ["c1", "c2", "c3"]:
    c = W.CONFIGS[name]
    import os
    f = pk.Flock(c.n, pk.boids_default_params(init_mode=c.init_mode), seed=1, kernel=int(os.environ.get("KERNEL", "0")))
    dt = float(W.DT)
    f.step(dt, 5)
    torch.cuda.synchronize()
    s = torch.cuda.current_stream()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    for k in range(K):
        flush.fill_(float(k))
        ev[k][0].record(s)
        f.step(dt, 1)
        ev[k][1].record(s)
    torch.cuda.synchronize()
    a = sum(x.elapsed_time(y) for x, y in ev) / K * 1e3
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    f.step(dt, K)
    e1.record(s)
    torch.cuda.synchronize()
    b = e0.elapsed_time(e1) / K * 1e3
    t0 = time.perf_counter()
    e0.record(s)
    for _ in range(K):
        f.step(dt, 1)
    e1.record(s)
    host = (time.perf_counter() - t0) / K * 1e6
    torch.cuda.synchronize()
    cc = e0.elapsed_time(e1) / K * 1e3
    print(f"{name} n={c.n}: bench-pattern {a:.1f} us/step, step(dt,{K}) {b:.1f} us/step, "
          f"{K} x step(dt,1) {cc:.1f} us/step (host enqueue {host:.1f} us/step)", flush=True)
    f.close()
