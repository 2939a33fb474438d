"""GPU parity of the think-frequency step (skipThink; Q15)
against oracle.step_think: neighbour lists (carried for non-thinkers, -1 before
an agent's first think), stored steering vectors and the full state, bit-exact,
every step from init; brute force (cold k_fused + warm scan routing) and grid.
"""
import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu
KEYS = ("pos", "fwd", "up", "side", "speed")
DT = 0.05


def _op(orc, p):
    return orc.default_params(**{name: getattr(p, name) for name, _ in p._fields_})


@pytest.mark.parametrize("mode,k,n,steps", [(0, 3, 2000, 9), (0, 10, 3000, 14), (1, 4, 2500, 9), (0, 2, 700, 6)])
def test_think_trajectory(boidslib, orc, mode, k, n, steps):
    import paper_conf_ipps_breitbart09_b200 as pk
    from paper_conf_ipps_breitbart09_b200 import abi

    p = pk.boids_default_params(search_mode=mode, init_mode=1, world_radius=15.0, think_every=k)
    op = _op(orc, p)
    with pk.Flock(n, p, seed=6, record_steering=True) as f:
        o = orc.init(n, op, seed=6)
        idx = np.full((n, 7), -1, np.int32)
        cnt = np.full(n, -1, np.int32)
        fs = np.zeros((n, 3), np.float32)
        for t in range(steps):
            o, idx, cnt, fs, F = orc.step_think(o, DT, t, fs, idx, cnt, op)
            f.step(DT, 1)
            g_idx, g_cnt = f.neighbors()
            np.testing.assert_array_equal(g_cnt, cnt, err_msg=f"step {t}")
            np.testing.assert_array_equal(g_idx, idx, err_msg=f"step {t}")
            g = f.state()
            for key in KEYS:
                assert np.array_equal(g[key], o[key]), (t, key)
            ti, gfs = abi.boids_get_think_state(f.h)
            assert ti == t + 1 and np.array_equal(gfs, fs)
            assert np.array_equal(f.steering(), F)


def test_think_snapshot_restore(boidslib, orc):
    """get_state + get_neighbors + get_think_state is a complete snapshot: a second
    handle restored from it continues bit-identically (checkpoint / resume)."""
    import paper_conf_ipps_breitbart09_b200 as pk
    from paper_conf_ipps_breitbart09_b200 import abi

    n, k = 1500, 5
    p = pk.boids_default_params(init_mode=1, world_radius=15.0, think_every=k)
    with pk.Flock(n, p, seed=2) as a, pk.Flock(n, p, seed=99) as b:
        a.step(DT, 7)
        t, fs = abi.boids_get_think_state(a.h)
        b.set_state(a.state())
        abi.boids_set_think_state(b.h, t, fs)
        # b has its own (stale) lists: still exact -- they only seed the search bound
        a.step(DT, 6)
        b.step(DT, 6)
        sa, sb = a.state(), b.state()
        for key in KEYS:
            assert np.array_equal(sa[key], sb[key]), key
