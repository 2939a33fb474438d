"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

The bar (BASELINE.json north_star):
  * neighbour index lists bit-exact (same fp32 distance expression, no FMA,
    ties broken by index) -- compared as ordered lists, which is stronger;
  * steering vectors and post-step state within |g - o| <= 1e-6 + 1e-5 |o|
    (numpy allclose(rtol=1e-5, atol=1e-6)), compared per step from a shared
    state; both sides follow Appendix A, so in practice they are bit-exact and
    the tests also report that.
Every state fed to the oracle comes from the seeded generators (workloads/) or
from the oracle itself; nothing the GPU computed is ever an oracle input.
"""
import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu

DT = float(W.DT)
RTOL, ATOL = 1e-5, 1e-6
KEYS = ("pos", "fwd", "up", "side", "speed")


@pytest.fixture(scope="module")
def pk(boidslib):
    import paper_conf_ipps_breitbart09_b200 as pk

    return pk


def assert_state_close(g, o, what=""):
    for k in KEYS:
        np.testing.assert_allclose(g[k], o[k], rtol=RTOL, atol=ATOL, err_msg=f"{what} {k}")


def bitexact(g, o):
    return all(np.array_equal(g[k], o[k]) for k in KEYS)


def gpu_one_step(pk, state, params=None, kernel=None, cluster=0, dt=DT):
    with pk.Flock(state["pos"].shape[0], params, seed=1, kernel=kernel, cluster=cluster,
                  record_steering=True) as f:
        f.set_state(state)
        f.step(dt, 1)
        return f.state(), f.neighbors(), f.steering()


def check_step(pk, orc, state, params=None, kernel=None, cluster=0, dt=DT, require_bitexact=True):
    o_state, o_idx, o_cnt, o_F = orc.step(orc.State(state), dt, _oparams(orc, params))
    g_state, (g_idx, g_cnt), g_F = gpu_one_step(pk, state, params, kernel, cluster, dt)
    np.testing.assert_array_equal(g_cnt, o_cnt)
    np.testing.assert_array_equal(g_idx, o_idx)
    np.testing.assert_allclose(g_F, o_F, rtol=RTOL, atol=ATOL)
    assert_state_close(g_state, o_state)
    if require_bitexact:
        assert bitexact(g_state, o_state) and np.array_equal(g_F, o_F)


def _oparams(orc, p):
    if p is None:
        return orc.default_params()
    return orc.default_params(**{name: getattr(p, name) for name, _ in p._fields_})


# ------------------------------------------------------------------ init
@pytest.mark.parametrize("n,mode", [(1, 0), (7, 0), (1000, 0), (4096, 1), (16384, 0)])
def test_init_bitexact(pk, orc, n, mode):
    p = pk.boids_default_params(init_mode=mode)
    with pk.Flock(n, p, seed=3) as f:
        g = f.state()
    o = orc.init(n, _oparams(orc, p), seed=3)
    for k in KEYS:
        assert np.array_equal(g[k], o[k]), k


# ------------------------------------------------------------- one step
SIZES = [1, 2, 7, 8, 100, 255, 256, 257, 1000, 1024, 3000]


@pytest.mark.parametrize("kernel", [0, 1])
@pytest.mark.parametrize("n", SIZES)
def test_step_ball(pk, orc, n, kernel):
    s = W.ball_flock(n, seed=n, radius=max(2.0, 20.0 * (n / 16384) ** (1 / 3) * 2))
    check_step(pk, orc, s, kernel=kernel)


@pytest.mark.parametrize("cluster", [1, 2, 4, 8, 16])
def test_step_every_cluster(pk, orc, cluster):
    s = W.ball_flock(5000, seed=cluster, radius=15.0)
    check_step(pk, orc, s, cluster=cluster)


@pytest.mark.parametrize("kernel", [0, 1])
@pytest.mark.parametrize("side,spacing", [(6, 1.0), (8, 2.0), (10, 3.0)])
def test_step_lattice_ties(pk, orc, side, spacing, kernel):
    check_step(pk, orc, W.lattice_flock(side, spacing, seed=side), kernel=kernel)


@pytest.mark.parametrize("kernel", [0, 1])
def test_step_coincident(pk, orc, kernel):
    check_step(pk, orc, W.coincident_flock(600, groups=5, seed=2), kernel=kernel)


def test_step_radius_boundary(pk, orc):
    check_step(pk, orc, W.radius_shell_flock(9.0))


def test_step_dt_zero_and_params(pk, orc):
    s = W.ball_flock(700, seed=9, radius=12.0)
    check_step(pk, orc, s, dt=0.0)
    p = pk.boids_default_params(search_radius=4.5, w_separation=3.0, max_force=5.0, max_speed=2.0,
                                mass=2.5, world_radius=11.0)
    check_step(pk, orc, s, params=p, dt=0.1)


def test_wrap_agents_outside(pk, orc):
    s = W.ball_flock(500, seed=4, radius=60.0)  # many agents outside R = 50
    check_step(pk, orc, s, dt=0.05)


# -------------------------------------------------- trajectories (warm path)
@pytest.mark.parametrize("kernel,n,steps,sym", [(0, 1024, 30, 1), (0, 4096, 10, 1), (1, 1024, 10, 1),
                                                (2, 1024, 12, 1), (0, 20000, 3, 1), (0, 1024, 12, 0),
                                                (0, 4096, 5, 0), (0, 20000, 3, 0), (0, 1, 3, 1), (0, 2, 3, 1),
                                                (0, 8192, 4, 1), (0, 8193, 4, 1), (0, 10239, 4, 1),
                                                (0, 12289, 3, 1), (0, 9000, 3, 1), (0, 40000, 2, 1)])
def test_trajectory_from_init(pk, orc, kernel, n, steps, sym):
    """GPU steps continuously (warm thresholds active after step 1); the oracle
    runs the same steps from its own init.  Bit-exact sides stay identical.
    sym=1: warm steps evaluate each unordered pair once (k_sym, the default for
    n >= 8192); sym=0: every ordered pair (k_scan).  Sizes straddle the 2048-agent
    query blocks of k_sym (ragged diagonal and off-diagonal tiles, phantoms)."""
    with pk.Flock(n, seed=1, kernel=kernel, symmetric=bool(sym)) as f:
        o = orc.init(n, seed=1)
        for t in range(steps):
            o, o_idx, o_cnt, _ = orc.step(o, DT)
            f.step(DT, 1)
            g_idx, g_cnt = f.neighbors()
            np.testing.assert_array_equal(g_idx, o_idx, err_msg=f"step {t}")
            g = f.state()
            assert_state_close(g, o, f"step {t}")
            assert bitexact(g, o), f"step {t} not bit-exact"


@pytest.mark.parametrize("new", ["ball", "lattice", "coincident"])
def test_set_state_keeps_exact_with_stale_lists(pk, orc, new):
    """boids_set_state keeps the previous neighbour lists as the seed of the warm
    bound; it must stay exact for an unrelated new state (loose bounds, ties)."""
    n = 1000
    gen = {"ball": lambda: W.ball_flock(n, seed=77, radius=14.0),
           "lattice": lambda: W.lattice_flock(10, 1.0, seed=3),
           "coincident": lambda: W.coincident_flock(n, groups=6, seed=8)}[new]
    s = gen()
    with pk.Flock(n, seed=1, record_steering=True) as f:
        f.step(DT, 3)  # warm lists of an unrelated flock
        f.set_state(s)
        f.step(DT, 1)
        o_state, o_idx, o_cnt, o_F = orc.step(orc.State(s), DT)
        np.testing.assert_array_equal(f.neighbors()[0], o_idx)
        assert bitexact(f.state(), o_state) and np.array_equal(f.steering(), o_F)


@pytest.mark.parametrize("sym", [1, 0])
def test_trajectory_wraps_and_overflow(pk, orc, sym):
    """Small world, long dt: many agents wrap to the diametric opposite point each
    step, so their old neighbours end far away -> t0 >= r2 -> the warm
    scan's hit buffers overflow and k_select's warp re-search runs.  Bit-exact."""
    p = pk.boids_default_params(init_mode=1, world_radius=12.0, max_speed=30.0)
    op = _oparams(orc, p)
    n, dt = 3000, 0.05
    with pk.Flock(n, p, seed=5, symmetric=bool(sym)) as f:
        o = orc.init(n, op, seed=5)
        wrapped = 0
        for t in range(8):
            prev = o
            o, o_idx, _, _ = orc.step(o, dt, op)
            wrapped += int((np.linalg.norm(o["pos"] - prev["pos"], axis=1) > 10.0).sum())
            f.step(dt, 1)
            np.testing.assert_array_equal(f.neighbors()[0], o_idx, err_msg=f"step {t}")
            assert bitexact(f.state(), o), f"step {t}"
        assert wrapped > 20


# ------------------------------------------- full sizes (bench launch config)
@pytest.mark.parametrize("cfg", ["c1", "c2", "c3"])
def test_config_full_multi_step(pk, orc, cfg):
    c = W.CONFIGS[cfg]
    steps = 3
    p = pk.boids_default_params(init_mode=c.init_mode)
    with pk.Flock(c.n, p, seed=1) as f:
        o = orc.init(c.n, _oparams(orc, p), seed=1)
        for t in range(steps):
            o, o_idx, _, _ = orc.step(o, DT, _oparams(orc, p))
            f.step(DT, 1)
            np.testing.assert_array_equal(f.neighbors()[0], o_idx)
            assert bitexact(f.state(), o)


@pytest.mark.parametrize("balance", [1, 0])
def test_config_c3_feedback_split(pk, orc, balance):
    """C3 (the north_star's n = 16384 brute-force case) for 12 steps: from the
    second warm step on, k_sym cuts its work from the previous launch's measured
    CTA times (BOIDS_OPT_BALANCE = 1), so the partition changes every step.  The
    lists and states stay bit-exact with the oracle either way."""
    c = W.CONFIGS["c3"]
    p = pk.boids_default_params(init_mode=c.init_mode)
    with pk.Flock(c.n, p, seed=1) as f:
        from paper_conf_ipps_breitbart09_b200 import abi
        abi.boids_set_option(f.h, abi.BOIDS_OPT_BALANCE, balance)
        o = orc.init(c.n, _oparams(orc, p), seed=1)
        for t in range(12):
            o, o_idx, _, _ = orc.step(o, DT, _oparams(orc, p))
            f.step(DT, 1)
            np.testing.assert_array_equal(f.neighbors()[0], o_idx, err_msg=f"step {t}")
            assert bitexact(f.state(), o), f"step {t}"


def test_config_c4_sampled(pk, orc):
    """C4 (n=131072, WORLD init) at full size: GPU runs 2 steps from init in the
    bench's launch configuration; the oracle checks a seeded sample of agents of
    step 1 and 2 one by one (step 2 from the oracle's own full step-1 state is
    too slow, so step 2 is checked on properties instead)."""
    c = W.CONFIGS["c4"]
    p = pk.boids_default_params(init_mode=c.init_mode)
    op = _oparams(orc, p)
    ag = W.sample_agents(c.n, 1024)
    with pk.Flock(c.n, p, seed=1, record_steering=True) as f:
        s0 = orc.init(c.n, op, seed=1)
        f.step(DT, 1)
        g = f.state()
        g_idx, g_cnt = f.neighbors()
        o, o_idx, o_cnt, o_F = orc.step_sample(s0, ag, DT, op)
        np.testing.assert_array_equal(g_idx[ag], o_idx)
        np.testing.assert_allclose(f.steering()[ag], o_F, rtol=RTOL, atol=ATOL)
        for k in KEYS:
            np.testing.assert_array_equal(g[k][ag], o[k])
        # step 2 (warm path): invariants at full size
        f.step(DT, 1)
        g2 = f.state()
        assert (g2["speed"] <= 9.0 * (1 + 4 * 2**-23)).all()
        r = np.linalg.norm(g2["pos"].astype(np.float64), axis=1)
        assert (r <= 50.0 * (1 + 4 * 2**-23)).all()
        idx2, cnt2 = f.neighbors()
        assert (cnt2 <= 7).all() and (idx2[np.arange(c.n), 0] != np.arange(c.n)).all()


@pytest.mark.parametrize("sym", [1, 0])
def test_config_c4_warm_sampled(pk, orc, sym):
    """C4 at full size on the WARM path (the bench's steady state): a cold step on
    the oracle's initial state leaves neighbour lists; the input is then replaced
    by a jittered copy (workloads.jitter, numpy only), so the next step runs the
    warm scan (k_sym / k_scan) with stale-but-close lists as bound seeds.  A
    seeded sample of 1024 agents is checked one by one against the oracle."""
    c = W.CONFIGS["c4"]
    p = pk.boids_default_params(init_mode=c.init_mode)
    op = _oparams(orc, p)
    ag = W.sample_agents(c.n, 1024, seed=3)
    s0 = orc.init(c.n, op, seed=1)
    s1 = W.jitter({k: s0[k] for k in KEYS}, 0.05, seed=4)
    with pk.Flock(c.n, p, seed=1, record_steering=True, symmetric=bool(sym)) as f:
        f.set_state({k: s0[k] for k in KEYS})
        f.step(DT, 1)
        f.set_state(s1)
        f.step(DT, 1)
        g = f.state()
        g_idx, _ = f.neighbors()
        o, o_idx, _, o_F = orc.step_sample(orc.State(s1), ag, DT, op)
        np.testing.assert_array_equal(g_idx[ag], o_idx)
        np.testing.assert_array_equal(f.steering()[ag], o_F)
        for k in KEYS:
            np.testing.assert_array_equal(g[k][ag], o[k])


def _spatial_ids(state, cells=64):
    """Renumber the agents so ids follow space (sort by a coarse z, y, x cell,
    then x): a reindex of the seeded state, no method arithmetic.  The bench's
    ids are spatially random; here neighbours have nearby ids (measured to
    change k_sym's timing, profiles/r1j/locality_probe.txt)."""
    p = state["pos"]
    lo, hi = p.min(0), p.max(0)
    q = np.clip(((p - lo) / (hi - lo) * cells).astype(np.int64), 0, cells - 1)
    perm = np.lexsort((p[:, 0], q[:, 0], q[:, 1], q[:, 2]))
    return {k: np.ascontiguousarray(state[k][perm]) for k in KEYS}


@pytest.mark.parametrize("search", [0, 1])
def test_spatially_ordered_ids_warm_sampled(pk, orc, search):
    """C4-size flock whose ids follow space (brute force on k_sym, and the grid):
    cold step, jittered copy, warm step; 1024 sampled agents bit-exact against
    the oracle (lists, steering, state)."""
    c = W.CONFIGS["c4"]
    p = pk.boids_default_params(init_mode=c.init_mode, search_mode=search)
    op = _oparams(orc, p)
    ag = W.sample_agents(c.n, 1024, seed=11)
    s0 = _spatial_ids(orc.init(c.n, op, seed=1))
    s1 = W.jitter(s0, 0.05, seed=6)
    with pk.Flock(c.n, p, seed=1, record_steering=True) as f:
        f.set_state(s0)
        f.step(DT, 1)
        f.set_state(s1)
        f.step(DT, 1)
        g = f.state()
        o, o_idx, _, o_F = orc.step_sample(orc.State(s1), ag, DT, op)
        np.testing.assert_array_equal(f.neighbors()[0][ag], o_idx)
        np.testing.assert_array_equal(f.steering()[ag], o_F)
        for k in KEYS:
            np.testing.assert_array_equal(g[k][ag], o[k])


@pytest.mark.parametrize("n,search", [(300001, 0), (2500003, 1)])
def test_large_ragged_warm_sampled(pk, orc, n, search):
    """Beyond the bench sizes, ragged (n not a multiple of any tile or query
    block): brute force at n = 300001 on k_sym (147 query blocks, stream-K,
    feedback split) and the grid at n = 2.5M.  As in the C4 warm test: a cold
    step on the oracle's initial state leaves lists, the input is replaced by a
    jittered copy (workloads.jitter), and the warm step (bounds, window / cell
    bounds, routing) is checked on 512 sampled agents against the oracle."""
    p = pk.boids_default_params(init_mode=1, search_mode=search)
    op = _oparams(orc, p)
    ag = W.sample_agents(n, 512, seed=9)
    s0 = orc.init(n, op, seed=2)
    s1 = W.jitter({k: s0[k] for k in KEYS}, 0.05, seed=5)
    with pk.Flock(n, p, seed=1, record_steering=True) as f:
        f.set_state({k: s0[k] for k in KEYS})
        f.step(DT, 1)
        f.set_state(s1)
        f.step(DT, 1)
        g = f.state()
        o, o_idx, _, o_F = orc.step_sample(orc.State(s1), ag, DT, op)
        np.testing.assert_array_equal(f.neighbors()[0][ag], o_idx)
        np.testing.assert_array_equal(f.steering()[ag], o_F)
        for k in KEYS:
            np.testing.assert_array_equal(g[k][ag], o[k])


# --------------------------------------------------------------- edges
def test_steps_zero_is_noop(pk):
    with pk.Flock(300, seed=2) as f:
        a = f.state()
        f.step(DT, 0)
        b = f.state()
        assert all(np.array_equal(a[k], b[k]) for k in KEYS)
        assert (f.neighbors()[1] == -1).all()  # -1: never searched


def test_errors(pk):
    from paper_conf_ipps_breitbart09_b200 import abi

    with pk.Flock(64, seed=2) as f:
        for dt, steps in ((-1.0, 1), (float("nan"), 1), (0.1, -1)):
            with pytest.raises(abi.BoidsError) as e:
                f.step(dt, steps)
            assert e.value.code == abi.BOIDS_EINVAL
        with pytest.raises(abi.BoidsError):
            f.steering()  # not recorded
        with pytest.raises(abi.BoidsError):
            abi.boids_step_shard(f.h, 0.1)  # not a shard handle


def test_profile_classes_sym_step(pk):
    """A warm k_sym step records its prologue (k_sym_prep, class 5) and k_sym
    (class 0) as two launches: bench.py's search roofline is k_sym alone, with
    the prologue reported beside it."""
    from paper_conf_ipps_breitbart09_b200 import abi

    with pk.Flock(16384, seed=1) as f:
        f.step(DT, 2)
        abi.boids_set_option(f.h, abi.BOIDS_OPT_PROFILE, 1)
        abi.boids_get_profile(f.h, reset=True)
        f.step(DT, 3)
        prof = abi.boids_get_profile(f.h, reset=True)
        assert f.info().last_path == abi.BOIDS_PATH_SYM
        assert prof["search_prep"][1] == 3 and prof["fused_or_search"][1] == 3
        assert prof["fused_or_search"][0] > prof["search_prep"][0] > 0
        abi.boids_set_option(f.h, abi.BOIDS_OPT_PROFILE, 2)  # level 2: the search class only
        f.step(DT, 2)
        prof = abi.boids_get_profile(f.h, reset=True)
        assert prof["fused_or_search"][1] == 2 and prof["search_prep"][1] == 0


def test_launch_count_and_info(pk):
    with pk.Flock(16384, seed=1) as f:
        i0 = f.info().launches
        f.step(DT, 5)
        f.sync()
        info = f.info()
        # step 1 (cold): the fused cluster kernel; steps 2-5 (warm, single GPU):
        # k_sym_prep + k_sym + k_select + k_route; the spatial query order (3
        # binning kernels) is refreshed on step 1 and every 8th
        assert info.launches - i0 == 1 + 4 * 4 + 3
    with pk.Flock(16384, seed=1, symmetric=False) as f:
        i0 = f.info().launches
        f.step(DT, 5)
        f.sync()
        # warm steps on the ordered-pair path: k_bound + k_scan + k_select + k_route
        assert f.info().launches - i0 == 1 + 4 * 4 + 3
        assert info.cluster == 16 and info.slice == 16384


# ------------------------------------------------------- grid mode (BOIDS_GRID)
def _grid(pk, **kw):
    return pk.boids_default_params(search_mode=1, **kw)


@pytest.mark.parametrize("n", [1, 2, 7, 257, 1000, 3000])
def test_grid_step_ball(pk, orc, n):
    s = W.ball_flock(n, seed=n + 11, radius=max(3.0, 20.0 * (n / 16384) ** (1 / 3) * 2))
    check_step(pk, orc, s, params=_grid(pk))


@pytest.mark.parametrize("case", ["lattice9", "lattice_r", "coincident", "shell", "outside"])
def test_grid_edge_cases(pk, orc, case):
    s = {"lattice9": lambda: W.lattice_flock(10, 3.0, seed=1),   # spacing 3 -> d2 = 81 = r2 ties at cell edges
         "lattice_r": lambda: W.lattice_flock(8, 9.0, seed=2),   # neighbours exactly at r (excluded)
         "coincident": lambda: W.coincident_flock(700, groups=4, seed=3),
         "shell": lambda: W.radius_shell_flock(9.0),
         "outside": lambda: W.ball_flock(1500, seed=9, radius=70.0)}[case]()  # clamped into boundary cells
    check_step(pk, orc, s, params=_grid(pk), dt=0.05)


@pytest.mark.parametrize("n,steps,world", [(4096, 10, 50.0), (3000, 8, 12.0)])
def test_grid_trajectory(pk, orc, n, steps, world):
    p = _grid(pk, init_mode=1, world_radius=world)
    op = _oparams(orc, p)
    with pk.Flock(n, p, seed=4) as f:
        o = orc.init(n, op, seed=4)
        for t in range(steps):
            o, o_idx, _, _ = orc.step(o, 0.05, op)
            f.step(0.05, 1)
            np.testing.assert_array_equal(f.neighbors()[0], o_idx, err_msg=f"step {t}")
            assert bitexact(f.state(), o), f"step {t}"


def test_grid_equals_brute_gpu(pk):
    """Variant equivalence at scale: grid and brute force give bit-identical lists and states."""
    n = 120000
    pg = pk.boids_default_params(init_mode=1, search_mode=1)
    pb = pk.boids_default_params(init_mode=1, search_mode=0)
    with pk.Flock(n, pg, seed=2) as fg, pk.Flock(n, pb, seed=2) as fb:
        for t in range(3):
            fg.step(DT, 1)
            fb.step(DT, 1)
            assert np.array_equal(fg.neighbors()[0], fb.neighbors()[0]), f"step {t}"
            sg, sb = fg.state(), fb.state()
            assert all(np.array_equal(sg[k], sb[k]) for k in KEYS), f"step {t}"


def test_config_c5_sampled(pk, orc):
    """C5 (n = 1M, grid) at full size: one step from init, 256 sampled agents
    checked one by one against the oracle (each an O(n) brute-force search)."""
    c = W.CONFIGS["c5"]
    p = pk.boids_default_params(init_mode=c.init_mode, search_mode=c.search_mode)
    op = _oparams(orc, p)
    ag = W.sample_agents(c.n, 256)
    with pk.Flock(c.n, p, seed=1, record_steering=True) as f:
        s0 = orc.init(c.n, op, seed=1)
        f.step(DT, 1)
        g = f.state()
        g_idx, _ = f.neighbors()
        o, o_idx, _, o_F = orc.step_sample(s0, ag, DT, op)
        np.testing.assert_array_equal(g_idx[ag], o_idx)
        np.testing.assert_allclose(f.steering()[ag], o_F, rtol=RTOL, atol=ATOL)
        for k in KEYS:
            np.testing.assert_array_equal(g[k][ag], o[k])


# ----------------------------------------- double-buffered readback
def test_readback_draw_matrix_double_buffered(pk, orc):
    """boids_readback_begin packs the 4x4 draw matrices (side, up, fwd, pos) of the
    current state and copies them on a second stream while later steps run; the
    two alternating buffers must hold the oracle's states of the last two steps,
    packed as rows (x, y, z, 0|0|0|1)."""
    import torch

    from paper_conf_ipps_breitbart09_b200 import abi

    n = 5000
    p = pk.boids_default_params(init_mode=1)
    op = _oparams(orc, p)
    bufs = [torch.empty((n, 4, 4), dtype=torch.float32, pin_memory=True).numpy() for _ in range(2)]
    o = orc.init(n, op, seed=4)
    states = []
    with pk.Flock(n, p, seed=4) as f:
        for t in range(4):
            f.step(DT, 1)
            abi.boids_readback_begin(f.h, bufs[t % 2])  # waits for the previous copy only
            o, _, _, _ = orc.step(o, DT, op)
            states.append(o)
        abi.boids_readback_wait(f.h)
    for t in (2, 3):  # the two buffers hold the last two steps
        m, s = bufs[t % 2], states[t]
        expect = np.zeros((n, 4, 4), np.float32)
        expect[:, 0, :3], expect[:, 1, :3], expect[:, 2, :3], expect[:, 3, :3] = s["side"], s["up"], s["fwd"], s["pos"]
        expect[:, 3, 3] = 1.0
        assert np.array_equal(m, expect), f"step {t}"


@pytest.mark.parametrize("n", [64, 100, 300, 511, 512, 513])
def test_set_state_between_steps_small_n(pk, orc, n):
    """step, set_state, step at the sizes where boids_set_state's locality check
    samples consecutive qperm entries with stride 1 (a strided copy
    with pitch < width failed there and poisoned the next step); the second step
    must succeed and match the oracle from the uploaded state."""
    s = W.ball_flock(n, seed=n, radius=10.0)
    with pk.Flock(n, seed=1, record_steering=True) as f:
        f.step(DT, 2)
        f.set_state(s)
        f.step(DT, 1)
        f.sync()
        o_state, o_idx, _, o_F = orc.step(orc.State(s), DT)
        np.testing.assert_array_equal(f.neighbors()[0], o_idx)
        assert bitexact(f.state(), o_state) and np.array_equal(f.steering(), o_F)


@pytest.mark.parametrize("mode,n,steps", [(0, 1500, 20), (0, 20000, 12), (1, 6000, 12)])
def test_graph_steps_match_eager_and_oracle(pk, orc, mode, n, steps):
    """boids_step replays captured CUDA graphs of warm steps (BOIDS_OPT_GRAPH =
    1): the trajectory must equal the eager launches bit for bit and
    the oracle's; resort steps (every 8th) and both k_sym feedback parities are
    captured separately.  Profiling inside graphs (events retargeted per replay)
    must still report every search launch."""
    from paper_conf_ipps_breitbart09_b200 import abi

    p = pk.boids_default_params(init_mode=1, search_mode=mode, world_radius=20.0)
    op = _oparams(orc, p)
    with pk.Flock(n, p, seed=3) as fg, pk.Flock(n, p, seed=3) as fe:
        abi.boids_set_option(fg.h, abi.BOIDS_OPT_GRAPH, 1)
        abi.boids_set_option(fe.h, abi.BOIDS_OPT_GRAPH, 0)
        fg.step(DT, steps)
        fe.step(DT, steps)
        assert fg.info().graph_launches >= steps - 3 and fe.info().graph_launches == 0
        sg, se = fg.state(), fe.state()
        assert all(np.array_equal(sg[k], se[k]) for k in KEYS)
        assert np.array_equal(fg.neighbors()[0], fe.neighbors()[0])
        o = orc.run(orc.init(n, op, seed=3), DT, steps, op)
        assert bitexact(sg, o)
        abi.boids_set_option(fg.h, abi.BOIDS_OPT_PROFILE, 2)
        abi.boids_get_profile(fg.h, reset=True)
        g0 = fg.info().graph_launches
        fg.step(DT, 5)
        prof = abi.boids_get_profile(fg.h, reset=True)
        assert fg.info().graph_launches - g0 == 5
        cls = "grid_search" if mode else "fused_or_search"
        assert prof[cls][1] == 5 and prof[cls][0] > 0


@pytest.mark.parametrize("small", [1, 0])
@pytest.mark.parametrize("n,steps", [(1, 3), (2, 3), (7, 4), (100, 5), (1024, 12), (3000, 6), (8191, 4)])
def test_small_step_kernel(pk, orc, n, steps, small):
    """Warm steps of small single-rank flocks run as one kernel (k_small,
    BOIDS_OPT_SMALL = 1, the default below 8192 agents) or as the k_bound +
    k_scan + k_select1 + k_route chain (0): both bit-identical to the oracle's
    trajectory, lists included (ragged sizes, 16 and 8 threads per query)."""
    from paper_conf_ipps_breitbart09_b200 import abi

    p = pk.boids_default_params(init_mode=1, world_radius=max(4.0, 20.0 * (n / 8192) ** (1 / 3)))
    op = _oparams(orc, p)
    with pk.Flock(n, p, seed=5) as f:
        abi.boids_set_option(f.h, abi.BOIDS_OPT_SMALL, small)
        o = orc.init(n, op, seed=5)
        for t in range(steps):
            o, o_idx, _, _ = orc.step(o, DT, op)
            f.step(DT, 1)
            np.testing.assert_array_equal(f.neighbors()[0], o_idx, err_msg=f"step {t}")
            assert bitexact(f.state(), o), f"step {t}"
        want = abi.BOIDS_PATH_SMALL if small else abi.BOIDS_PATH_SCAN
        assert f.info().last_path == want
