"""k_sym per-CTA timing from in-kernel %globaltimer stamps + per-kernel profile (development aid).

python tools/sym_phases.py c3 [c4 ...]
Fields per CTA (k_sym a.phase): [0] start, [1] end, [2] L0, [3] L1, [4] slow groups,
[5] max wait cycles of a warp, [6] max emit cycles of a warp, [7] warp 0 wait cycles."""
import sys

import numpy as np

sys.path.insert(0, '.')
import paper_conf_ipps_breitbart09_b200 as pk  # noqa: E402
from paper_conf_ipps_breitbart09_b200 import abi  # noqa: E402
import workloads as W  # noqa: E402

for name in sys.argv[1:] or ["c3"]:
    cfg = W.CONFIGS[name]
    f = pk.Flock(cfg.n, pk.boids_default_params(init_mode=cfg.init_mode), seed=1, profile=True)
    import os
    abi.boids_set_option(f.h, abi.BOIDS_OPT_BALANCE, int(os.environ.get("BAL", "1")))
    f.step(float(W.DT), 4)
    f.sync()
    f.profile(reset=True)
    f.step(float(W.DT), 8)
    f.sync()
    prof = f.profile(reset=True)
    print(f"{name} n={cfg.n} per-step kernel means (us): "
          + ", ".join(f"{k}={v[0] / max(v[1], 1) * 1e3:.1f}x{v[1] // 8}" for k, v in prof.items() if v[1]))
    abi.boids_set_option(f.h, abi.BOIDS_OPT_PROFILE, int(os.environ.get("PROF", "1")))  # 0: timeline without events
    abi.boids_set_option(f.h, abi.BOIDS_OPT_PHASES, 1024)
    f.step(float(W.DT), 1)
    f.sync()
    raw = abi.boids_get_phases(f.h, 1024)
    spans = {}
    for nm, slot in (("k_sym_prep", 1000), ("k_select1", 1001), ("k_route", 1002)):
        b, e = int(raw[slot, 0]), int(raw[slot, 1])
        if b and e:
            spans[nm] = ((~np.uint64(b)).astype(np.int64), e)
    ph = raw[:1000].astype(np.int64)
    ph = ph[ph[:, 0] > 0]
    if len(ph):
        spans["k_sym"] = (int(ph[:, 0].min()), int(ph[:, 1].max()))
    if spans:
        z = min(v[0] for v in spans.values())
        print("  timeline (us from first start): " + "  ".join(
            f"{nm} {(b - z) / 1e3:.1f}-{(e - z) / 1e3:.1f}" for nm, (b, e) in sorted(spans.items(), key=lambda kv: kv[1][0])))
    if not len(ph):
        f.close()
        continue
    t0 = ph[:, 0].min()
    st, en = (ph[:, 0] - t0) / 1e3, (ph[:, 1] - t0) / 1e3
    dur = en - st
    work = ph[:, 3] - ph[:, 2]
    print(f"  ctas={len(ph)} start min/med/max {st.min():.1f}/{np.median(st):.1f}/{st.max():.1f} us; "
          f"end {en.min():.1f}/{np.median(en):.1f}/{en.max():.1f}; dur {dur.min():.1f}/{np.median(dur):.1f}/{dur.max():.1f}")
    print(f"  items/CTA min/med/max {work.min()}/{int(np.median(work))}/{work.max()}; slow groups "
          f"{ph[:, 4].min()}/{int(np.median(ph[:, 4]))}/{ph[:, 4].max()}; max-warp wait cyc med {int(np.median(ph[:, 5]))} "
          f"max {ph[:, 5].max()}; max-warp emit cyc med {int(np.median(ph[:, 6]))} max {ph[:, 6].max()}")
    order = np.argsort(dur)
    for i in list(order[:3]) + list(order[-5:]):
        print(f"    cta {i:4d} start {st[i]:7.1f} dur {dur[i]:7.1f} items {work[i]:8d} L0 {ph[i, 2]:10d} slow {ph[i, 4]:6d} "
              f"wait {ph[i, 5]:8d} emit {ph[i, 6]:8d}")
    f.close()
