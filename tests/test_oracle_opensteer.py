"""Pins for the oracle's steer_mode 1 -- OpenSteer 0.8.2 flocking [ext]
(the thesis's device code "is based on the CPU version of
OpenSteer"; readings DESIGN.md Q20-Q24):

  * inBoidNeighborhood filters: inside 3 * radius (1.5) always; beyond the
    behaviour's radius (5 / 7.5 / 9) never; otherwise forward . unit offset
    > cos angle (-0.707 / 0.7 / -0.15);
  * separation = n^(mean(offset / -d2)), alignment = n^(mean(f_j) - f_i),
    cohesion = n^(mean(p_j) - p_i), weighted 12 / 8 / 8;
  * adjustRawSteeringForce below 0.2 maxSpeed (cone of cos = 1 - 2 range^20
    around forward), acceleration smoothing with rate clip(9 dt, 0.15, 0.4).

Closed forms are worked by hand (exact cases) or in fp64 from the formulas
above (tolerance: a few fp32 ulps)."""
import numpy as np
import pytest

import workloads as W

DT = float(W.DT)


def close(a, b, rtol=3e-6, atol=1e-6):
    np.testing.assert_allclose(np.asarray(a, np.float64), np.asarray(b, np.float64), rtol=rtol, atol=atol)


def os_params(orc, **kw):
    return orc.default_params(steer_mode=1, **kw)


def steer(orc, pos, fwd, params):
    pos = np.array(pos, np.float32)
    fwd = np.array(fwd, np.float32)
    idx, cnt = orc.search_one(pos, 0, 9.0)
    return orc.steer_one(pos, fwd, 0, idx, cnt, params)


def test_behind_outside_min_distance_is_ignored(orc):
    # distance 4 straight behind: forwardness -1 fails every angle test -> F = 0
    F = steer(orc, [[0, 0, 0], [-4, 0, 0]], [[1, 0, 0], [1, 0, 0]], os_params(orc))
    assert np.array_equal(F, np.zeros(3, np.float32))
    # the thesis's listings (steer_mode 0) do use it
    F0 = steer(orc, [[0, 0, 0], [-4, 0, 0]], [[1, 0, 0], [1, 0, 0]], orc.default_params())
    assert np.abs(F0).sum() > 0


def test_behind_inside_min_distance_exact(orc):
    # distance 1 behind (< 1.5): in all three neighbourhoods.  sep = n^((-1,0,0)/-1) = (1,0,0);
    # ali = n^(f_j - f_i) = 0; coh = n^(p_j - p_i) = (-1,0,0)  ->  F = 12 - 8 = (4, 0, 0) exactly
    F = steer(orc, [[0, 0, 0], [-1, 0, 0]], [[1, 0, 0], [1, 0, 0]], os_params(orc))
    assert np.array_equal(F, np.array([4, 0, 0], np.float32))


def test_ahead_beyond_separation_radius(orc):
    # distance 6 ahead: outside separation (5), inside alignment (7.5, cos 1 > 0.7) and cohesion
    F = steer(orc, [[0, 0, 0], [6, 0, 0]], [[1, 0, 0], [0, 1, 0]], os_params(orc))
    r = 8 * np.array([-1, 1, 0]) / np.sqrt(2) + 8 * np.array([1, 0, 0])
    close(F, r)


def test_side_neighbour_only_cohesion(orc):
    # distance 6 to the side: forwardness 0 -> only cohesion (0 > -0.15) accepts it
    F = steer(orc, [[0, 0, 0], [0, 6, 0]], [[1, 0, 0], [0, 0, 1]], os_params(orc))
    close(F, [0, 8, 0], atol=0)


def test_radius_edges(orc):
    # alignment accepts d2 <= 7.5^2 (d2 > max^2 excludes); at exactly 7.5 ahead it is in
    F = steer(orc, [[0, 0, 0], [7.5, 0, 0]], [[1, 0, 0], [0, 1, 0]], os_params(orc))
    r = 8 * np.array([-1, 1, 0]) / np.sqrt(2) + 8 * np.array([1, 0, 0])
    close(F, r)
    # just beyond 7.5: alignment drops out, cohesion stays
    F = steer(orc, [[0, 0, 0], [np.nextafter(np.float32(7.5), np.float32(9)), 0, 0]],
              [[1, 0, 0], [0, 1, 0]], os_params(orc))
    close(F, [8, 0, 0], atol=0)


def test_averaged_behaviours_fp64(orc):
    rng = np.random.default_rng(5)
    for _ in range(30):
        pos = np.zeros((4, 3), np.float32)
        pos[1:] = rng.uniform(-3, 3, (3, 3)).astype(np.float32)
        fwd = rng.normal(size=(4, 3))
        fwd = (fwd / np.linalg.norm(fwd, axis=1, keepdims=True)).astype(np.float32)
        F = steer(orc, pos, fwd, os_params(orc))
        p = pos.astype(np.float64)
        f = fwd.astype(np.float64)
        sep, ali, coh, ns, na, nc = np.zeros(3), np.zeros(3), np.zeros(3), 0, 0, 0

        def hood(o, d2, mx, cs):
            if d2 < 1.5 ** 2:
                return True
            if d2 > mx * mx:
                return False
            return f[0] @ (o / np.sqrt(d2)) > cs

        for j in range(1, 4):
            o = p[j] - p[0]
            d2 = o @ o
            if hood(o, d2, 5.0, -0.707):
                sep += o / -d2
                ns += 1
            if hood(o, d2, 7.5, 0.7):
                ali += f[j]
                na += 1
            if hood(o, d2, 9.0, -0.15):
                coh += p[j]
                nc += 1

        def nz(v):
            n = np.linalg.norm(v)
            return v / n if n > 0 else v

        r = 12 * (nz(sep / ns) if ns else sep) + 8 * (nz(ali / na - f[0]) if na else ali) + \
            8 * (nz(coh / nc - p[0]) if nc else coh)
        close(F, r, rtol=2e-5, atol=2e-5)


def test_no_neighbours_zero(orc):
    F = steer(orc, [[0, 0, 0], [20, 0, 0]], [[1, 0, 0], [1, 0, 0]], os_params(orc))
    assert np.array_equal(F, np.zeros(3, np.float32))


# ------------------------------------------------------- modification
def _modify(orc, p, speed, F, dt, acc=None, fwd=(1, 0, 0)):
    return orc.modify_one(np.zeros(3), np.array(fwd), np.array([0, 1, 0]), np.array([0, 0, 1]), speed,
                          np.array(F, np.float32), dt, p, acc=acc)


def test_smoothing_from_rest_fast_agent(orc):
    # speed 9 > 0.2 * 9: force unchanged; smoothed acc = 0.15 F (rate clip(9/60) = 0.15)
    p = os_params(orc)
    out = _modify(orc, p, 9.0, [0, 10, 0], DT)
    close(out["acc"], [0, 1.5, 0])
    v = np.array([9.0, 0, 0]) + np.array([0, 1.5, 0]) * DT
    v = v * (9.0 / np.linalg.norm(v))
    close(out["speed"], 9.0)
    close(out["pos"], v * DT)


@pytest.mark.parametrize("dt,rate", [(0.01, 0.15), (0.03, 0.27), (0.1, 0.4)])
def test_smoothing_rate_clip(orc, dt, rate):
    p = os_params(orc)
    out = _modify(orc, p, 5.0, [2, 0, 0], dt, acc=[1, 0, 0])
    close(out["acc"], [1 + (2 - 1) * rate, 0, 0])


def test_dt_zero_keeps_acc_and_position(orc):
    p = os_params(orc)
    out = _modify(orc, p, 5.0, [0, 3, 0], 0.0, acc=[0.5, 0.25, 0])
    assert np.array_equal(out["acc"], np.array([0.5, 0.25, 0], np.float32))
    assert np.array_equal(out["pos"], np.zeros(3, np.float32))


def test_slow_agent_force_limited_to_cone(orc):
    # speed 0.9 = 0.5 * 0.2 maxSpeed: cos = 1 - 2 * 0.5^20; a sideways force is turned into
    # the cone around forward, length kept
    p = os_params(orc)
    out = _modify(orc, p, 0.9, [0, 10, 0], DT)
    c = 1 - 2 * 0.5 ** 20
    Fa = (np.array([c, 0, 0]) + np.array([0, 1, 0]) * np.sqrt(1 - c * c)) * 10
    close(out["acc"], 0.15 * Fa, rtol=2e-5)
    # a force already inside the cone is kept
    out = _modify(orc, p, 0.9, [10, 0, 0], DT)
    close(out["acc"], [1.5, 0, 0])


def test_thesis_mode_has_no_acc_state(orc):
    s = orc.init(64, orc.default_params(), seed=3)
    o, _, _, _ = orc.step(s, DT)
    assert "acc" not in o
    o1, _, _, _ = orc.step(s, DT, os_params(orc))
    assert o1["acc"].shape == (64, 3)


def test_flock_invariants_and_acc_carry(orc):
    p = os_params(orc)
    s = orc.init(300, p, seed=9)
    for t in range(40):
        s, idx, cnt, F = orc.step(s, DT, p)
        assert np.all(s["speed"] <= 9.0 * (1 + 4e-7 * 4))
        assert np.all(np.linalg.norm(s["pos"], axis=1) <= 50.0 * (1 + 4e-7 * 4))
        assert np.all(np.linalg.norm(s["acc"], axis=1) <= 27.0 * (1 + 1e-6))
    # the carried acceleration matters: restarting it from zero changes the next step
    a, _, _, _ = orc.step(s, DT, p)
    z = orc.State({k: v for k, v in s.items() if k != "acc"})
    b, _, _, _ = orc.step(z, DT, p)
    assert not np.array_equal(a["pos"], b["pos"])
