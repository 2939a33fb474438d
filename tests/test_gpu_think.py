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


@pytest.mark.parametrize("cfg", ["c4", "c5"])
def test_think10_full_size_sampled(boidslib, orc, cfg):
    """Think 10 at the bench's full sizes (C4 brute force n = 131072, C5 grid
    n = 1M), in the bench's steady state: the handle first runs 11 think steps
    from its own init (every agent has thought once; the lists that seed the
    bounds are up to 10 steps old, so ~3 % of C4's thinkers overflow the
    128-slot hit buffer and are re-searched whole; the grid's query binning
    keeps only thinkers and items span whole rows).  Then a seeded input is
    uploaded -- the oracle's Appendix-B state, jittered (workloads.jitter), and
    seeded stored steering vectors (workloads.random_forces) through
    boids_set_think_state at step index 11 -- and one step runs.  A sample of
    512 thinkers and 256 non-thinkers is checked one by one against
    oracle.step_think_sample: thinkers' lists, every sampled agent's steering
    vector used and new state, bit-exact."""
    import paper_conf_ipps_breitbart09_b200 as pk
    from paper_conf_ipps_breitbart09_b200 import abi

    c = W.CONFIGS[cfg]
    k, t = 10, 11
    p = pk.boids_default_params(init_mode=c.init_mode, search_mode=c.search_mode, think_every=k)
    op = _op(orc, p)
    dt = float(W.DT)
    s0 = orc.init(c.n, op, seed=1)
    s1 = orc.State(W.jitter({key: s0[key] for key in KEYS}, 0.05, seed=21))
    fs = W.random_forces(c.n, seed=22)
    ag = W.sample_agents(c.n, 8192, seed=23)
    think = (ag + t) % k == 0
    ag = np.concatenate([ag[think][:512], ag[~think][:256]])
    th = (ag + t) % k == 0
    with pk.Flock(c.n, p, seed=1, record_steering=True) as f:
        f.step(dt, t)
        fb0 = f.info().fallbacks
        f.set_state(s1)
        abi.boids_set_think_state(f.h, t, fs)
        f.step(dt, 1)
        g = f.state()
        g_idx, g_cnt = f.neighbors()
        gF = f.steering()
        routed = f.info().fallbacks - fb0
    o, o_idx, o_cnt, _, o_F = orc.step_think_sample(s1, ag, dt, t, fs[ag], None, None, op)
    np.testing.assert_array_equal(g_idx[ag][th], o_idx[th])
    np.testing.assert_array_equal(g_cnt[ag][th], o_cnt[th])
    np.testing.assert_array_equal(gF[ag], o_F)
    for key in KEYS:
        np.testing.assert_array_equal(g[key][ag], o[key], err_msg=key)
    print(f"{cfg} think {k}: {routed} thinkers searched whole (hit-buffer overflow / unbounded) this step")
