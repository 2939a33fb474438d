"""Pins for the oracle's steering (Listings 5.1, 5.3-5.5), modification
(P:345, P:497-499, P:522 + DESIGN.md Q10-Q13), synchronous update
and Appendix-B init.

Closed forms (fp64 references, tolerance = a few fp32 ulps):
  (i)   one neighbour at offset o: F = (w_c - w_s) o^ + w_a n^(f_j - f_i)
  (ii)  equilateral triangle, equal forwards: |F| = 4, F points away from the centroid
  (iii) clamp case: F = (-28,0,0) exactly, clamped to |F'| = 27
  (iv)  no neighbours: F = 0
Modification: F = 0 keeps v; speed clamp; wrap (50.5,0,0) -> (-49.5,0,0);
dt = 0 keeps p; invariants |v| <= maxSpeed, |p| <= R, orthonormal frame.
Init: the standard SplitMix64 test vector, ball/sphere invariants, exact speed.
"""
import numpy as np
import pytest

import workloads as W

DT = float(W.DT)


def unit(v):
    v = np.asarray(v, np.float64)
    n = np.linalg.norm(v)
    return v / n if n > 0 else v


def ulp_close(a, b, rel=4e-7 * 8, abs_=1e-6):
    np.testing.assert_allclose(np.asarray(a, np.float64), np.asarray(b, np.float64), rtol=rel, atol=abs_)


def steer_case(orc, pos, fwd, i=0):
    pos = np.array(pos, np.float32)
    fwd = np.array(fwd, np.float32)
    idx, cnt = orc.search_one(pos, i, 9.0)
    return orc.steer_one(pos, fwd, i, idx, cnt), idx, cnt


@pytest.mark.parametrize("seed", range(20))
def test_one_neighbour_closed_form(orc, seed):
    rng = np.random.default_rng(seed)
    o = rng.standard_normal(3)
    o = o / np.linalg.norm(o) * rng.uniform(0.5, 8.5)
    me = rng.uniform(-5, 5, 3)
    fi, fj = unit(rng.standard_normal(3)), unit(rng.standard_normal(3))
    pos = np.array([me, me + o], np.float32)
    F, idx, cnt = steer_case(orc, pos, [fi, fj])
    assert cnt == 1 and idx[0] == 1
    o32 = pos[1].astype(np.float64) - pos[0].astype(np.float64)
    f32 = np.array([fi, fj], np.float32).astype(np.float64)
    expect = (8.0 - 12.0) * unit(o32) + 8.0 * unit(f32[1] - f32[0])
    ulp_close(F, expect, rel=1e-5, abs_=2e-5)


@pytest.mark.parametrize("side", [1.0, 3.0, 8.0])
def test_equilateral_triangle(orc, side):
    h = side * np.sqrt(3) / 2
    pos = np.array([[0, 0, 0], [side, 0, 0], [side / 2, h, 0]], np.float32)
    f = [[0, 0, 1]] * 3
    c = pos.astype(np.float64).mean(0)
    for i in range(3):
        F, idx, cnt = steer_case(orc, pos, f, i)
        assert cnt == 2
        away = unit(pos[i].astype(np.float64) - c)
        ulp_close(F, 4.0 * away, rel=1e-5, abs_=2e-5)


def test_clamp_case_exact(orc):
    pos = [[0, 0, 0], [0.5, 0, 0], [-8, 0, 0]]
    fwd = [[1, 0, 0], [-1, 0, 0], [1, 0, 0]]
    F, idx, cnt = steer_case(orc, pos, fwd, 0)
    assert cnt == 2 and list(idx[:2]) == [1, 2]
    assert F.tolist() == [-28.0, 0.0, 0.0]  # every term is exact in fp32
    out = orc.modify_one([0, 0, 0], [1, 0, 0], [0, 1, 0], [-1, 0, 0], 0.0, F, 1.0)
    # a = F' (mass 1), v = a*dt = -27 (clamp at maxSpeed 9) -> |v| = 9, heading flips to -x
    ulp_close(out["speed"], 9.0)
    ulp_close(out["fwd"], [-1, 0, 0])
    ulp_close(out["pos"], [-9, 0, 0])


def test_no_neighbours_zero_force(orc):
    F, idx, cnt = steer_case(orc, [[0, 0, 0], [50, 0, 0]], [[1, 0, 0], [0, 1, 0]], 0)
    assert cnt == 0 and F.tolist() == [0.0, 0.0, 0.0]


def test_coincident_separation_guard(orc):
    # a different agent at d2 == 0 is a neighbour, but its separation term is 0 (Q6)
    F, idx, cnt = steer_case(orc, [[1, 2, 3], [1, 2, 3]], [[1, 0, 0], [0, 1, 0]], 0)
    assert cnt == 1
    expect = 8.0 * unit(np.array([-1.0, 1.0, 0.0]))
    ulp_close(F, expect)


def test_modify_zero_force_keeps_velocity(orc):
    f = unit([1, 2, 2]).astype(np.float32)
    out = orc.modify_one([1, 1, 1], f, [0, 1, 0], [1, 0, 0], 3.0, [0, 0, 0], DT)
    ulp_close(out["speed"], 3.0)
    ulp_close(out["fwd"], f)
    ulp_close(out["pos"], np.array([1, 1, 1]) + f.astype(np.float64) * 3.0 * DT)


def test_modify_speed_clamp(orc):
    f = unit([0, 0, 1]).astype(np.float32)
    out = orc.modify_one([0, 0, 0], f, [0, 1, 0], [1, 0, 0], 9.0, [0, 0, 27.0], DT)
    ulp_close(out["speed"], 9.0)
    assert out["speed"] <= 9.0 * (1 + 4 * 2**-23)


def test_modify_wrap_exact(orc):
    out = orc.modify_one([50.5, 0, 0], [1, 0, 0], [0, 1, 0], [0, 0, -1], 0.0, [0, 0, 0], DT)
    assert out["pos"].tolist() == [-49.5, 0.0, 0.0]  # diametric opposite point (Q12)


def test_modify_dt_zero(orc):
    out = orc.modify_one([3, -4, 5], unit([1, 1, 0]), [0, 0, 1], [1, 0, 0], 2.0, [1, 2, 3], 0.0)
    assert out["pos"].tolist() == [3.0, -4.0, 5.0]


def test_modify_zero_speed_keeps_frame(orc):
    out = orc.modify_one([0, 0, 0], [1, 0, 0], [0, 1, 0], [0, 0, -1], 0.0, [0, 0, 0], DT)
    assert out["speed"] == 0.0
    assert out["fwd"].tolist() == [1, 0, 0] and out["up"].tolist() == [0, 1, 0]
    assert out["side"].tolist() == [0, 0, -1]


@pytest.mark.parametrize("seed", range(10))
def test_modify_invariants(orc, seed):
    rng = np.random.default_rng(seed)
    for _ in range(200):
        p = rng.uniform(-55, 55, 3)
        f = unit(rng.standard_normal(3))
        u = unit(np.cross(unit(rng.standard_normal(3)), f))
        s = np.cross(f, u)
        F = rng.standard_normal(3) * rng.uniform(0, 60)
        sp = rng.uniform(0, 9)
        o = orc.modify_one(p, f, u, s, sp, F, DT)
        assert o["speed"] <= 9.0 * (1 + 4 * 2**-23)
        assert np.linalg.norm(o["pos"].astype(np.float64)) <= 50.0 * (1 + 4 * 2**-23)
        if o["speed"] > 0:
            F3 = np.array([o["fwd"], o["up"], o["side"]], np.float64)
            np.testing.assert_allclose(F3 @ F3.T, np.eye(3), atol=1e-5)


def test_synchronous_update_two_agents(orc):
    """Jacobi semantics: agent 1 steers from agent 0's OLD state."""
    s = W.ball_flock(2, seed=1, radius=1.0)
    s["fwd"] = np.array([[1, 0, 0], [0, 1, 0]], np.float32)
    s["up"] = np.array([[0, 1, 0], [0, 0, 1]], np.float32)
    s["side"] = np.array([[0, 0, -1], [1, 0, 0]], np.float32)
    out, idx, cnt, F = orc.step(orc.State(s), DT)
    for i, j in ((0, 1), (1, 0)):
        o = s["pos"][j].astype(np.float64) - s["pos"][i].astype(np.float64)
        expect = -4.0 * unit(o) + 8.0 * unit(s["fwd"][j].astype(np.float64) - s["fwd"][i])
        ulp_close(F[i], expect, rel=1e-5, abs_=2e-5)


def test_step_sample_consistent(orc):
    s = orc.State(W.ball_flock(300, seed=4, radius=12.0))
    full = orc.step(s, DT)
    ag = np.array([0, 5, 123, 299])
    samp = orc.step_sample(s, ag, DT)
    for k in ("pos", "fwd", "up", "side", "speed"):
        assert np.array_equal(samp[0][k], full[0][k][ag])
    assert np.array_equal(samp[1], full[1][ag])


# ---------------- Appendix B init ----------------
def splitmix64_stream(seed):
    M = 2**64 - 1
    s = seed & M
    while True:
        s = (s + 0x9E3779B97F4A7C15) & M
        z = s
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M
        yield z ^ (z >> 31)


def test_splitmix64_test_vector():
    # published first output of SplitMix64 seeded with 0
    assert next(splitmix64_stream(0)) == 0xE220A8397B1DCDAF


def test_init_agent_zero_position(orc):
    seed = 1
    h = next(splitmix64_stream(0))  # splitmix64(i=0)
    g = splitmix64_stream(next(splitmix64_stream(seed ^ h)))
    while True:
        c = [np.float32(np.float32(np.float32(next(g) >> 40) * np.float32(2**-24)) * np.float32(2)) - np.float32(1)
             for _ in range(3)]
        x, y, z = c
        if (x * x + y * y) + z * z < np.float32(1):
            break
    s = orc.init(3, seed=seed)
    assert s["pos"][0].tolist() == [float(x * np.float32(20)), float(y * np.float32(20)), float(z * np.float32(20))]


@pytest.mark.parametrize("mode,R", [(0, 20.0), (1, 50.0)])
def test_init_invariants(orc, mode, R):
    p = orc.default_params(init_mode=mode)
    s = orc.init(20000, p, seed=2)
    r = np.linalg.norm(s["pos"].astype(np.float64), axis=1)
    assert r.max() <= R * (1 + 1e-6)
    # uniform in the ball: P(r < R q^(1/3)) = q
    for q in (0.1, 0.5, 0.9):
        assert abs((r < R * q ** (1 / 3)).mean() - q) < 0.02
    assert np.abs(s["pos"].mean(0)).max() < 0.03 * R
    np.testing.assert_allclose(np.linalg.norm(s["fwd"], axis=1), 1.0, atol=1e-6)
    F = np.stack([s["fwd"], s["up"], s["side"]], 1).astype(np.float64)
    G = np.einsum("nij,nkj->nik", F, F)
    np.testing.assert_allclose(G, np.broadcast_to(np.eye(3), G.shape), atol=2e-6)
    assert (s["speed"] == np.float32(np.float32(0.3) * np.float32(9.0))).all()
    # forwards uniform on the sphere: mean ~ 0
    assert np.abs(s["fwd"].mean(0)).max() < 0.03


def test_init_deterministic_and_seeded(orc):
    a = orc.init(100, seed=5)
    b = orc.init(100, seed=5)
    c = orc.init(100, seed=6)
    assert all(np.array_equal(a[k], b[k]) for k in a)
    assert not np.array_equal(a["pos"], c["pos"])
    # per-agent streams: the prefix of a larger flock is the smaller flock
    d = orc.init(300, seed=5)
    assert np.array_equal(d["pos"][:100], a["pos"])


def test_polarisation_rises(orc):
    """Qualitative emergent behaviour of flocking: neighbours align.

    Smoke check, not parity: the mean cosine between an agent's heading and its
    neighbours' headings starts near 0 (random init) and rises."""
    s = orc.init(400, seed=3)

    def local_alignment(st):
        idx, cnt = orc.search(st["pos"], 9.0)
        v = [np.mean(st["fwd"][idx[i, :cnt[i]]] @ st["fwd"][i]) for i in range(st.n) if cnt[i]]
        return float(np.mean(v))

    a0 = local_alignment(s)
    a1 = local_alignment(orc.run(s, DT, 300))
    assert abs(a0) < 0.05 and a1 > a0 + 0.1


# ---------------- local-space handedness (reading Q25) ----------------
# OpenSteer's LocalSpace is right-handed [ext]: regenerateOrthonormalBasisUF sets
# side = normalize(forward x up), then up = side x forward.  Two consequences
# fixed by the vector algebra alone, not by the oracle's code:
#   * up' = side x forward = (f x u) x f = u - (u . f) f (triple product): the new
#     up is the OLD up projected onto the plane normal to the new forward -- it
#     never flips (u' . u > 0 whenever u is not parallel to f);
#   * det[side, up, forward] = (f x u) . (u x f) / |f x u| < 0, i.e. -1.
# A swapped operand order in either cross product flips up' (first pin) or side
# (the det sign); orthonormality alone (test_modify_invariants) cannot tell.


def _det3(s, u, f):
    return float(np.dot(np.asarray(s, np.float64), np.cross(np.asarray(u, np.float64), np.asarray(f, np.float64))))


def test_local_space_closed_form(orc):
    """f = (0,0,1), u = (0,1,0), F = 0: forward stays, side = f x u = (-1,0,0),
    up = side x f = (0,1,0) -- exact (every product is 0 or +-1)."""
    o = orc.modify_one([0, 0, 0], [0, 0, 1], [0, 1, 0], [0, 0, 0], 1.0, [0, 0, 0], 0.1)
    assert o["fwd"].tolist() == [0, 0, 1]
    assert o["side"].tolist() == [-1, 0, 0]
    assert o["up"].tolist() == [0, 1, 0]
    assert _det3(o["side"], o["up"], o["fwd"]) == -1.0


def test_local_space_turn_closed_form(orc):
    """Turning in the horizontal plane keeps up = (0,1,0): f = (1,0,0), speed 1,
    F = (0,0,60) (clamped to 27), dt = 0.1 -> v = (1, 0, 2.7), f' = v / |v|;
    up' must be exactly perpendicular to the turn plane, (0,1,0), and side' =
    f' x up' = (-f'z, 0, f'x)."""
    o = orc.modify_one([0, 0, 0], [1, 0, 0], [0, 1, 0], [0, 0, -1], 1.0, [0, 0, 60], 0.1)
    f = np.asarray(o["fwd"], np.float64)
    ref = np.array([1.0, 0.0, 2.7]) / np.linalg.norm([1.0, 0.0, 2.7])
    np.testing.assert_allclose(f, ref, rtol=1e-6, atol=1e-7)
    np.testing.assert_allclose(o["up"], [0, 1, 0], atol=1e-7)
    np.testing.assert_allclose(o["side"], [-f[2], 0.0, f[0]], rtol=1e-6, atol=1e-7)
    assert _det3(o["side"], o["up"], o["fwd"]) < 0


@pytest.mark.parametrize("seed", range(5))
def test_local_space_up_is_projected_old_up(orc, seed):
    """Random frames and forces: up' = n^(u - (u . f') f') (triple-product
    identity) and det[s', u', f'] = -1."""
    rng = np.random.default_rng(100 + seed)
    for _ in range(200):
        f = unit(rng.standard_normal(3))
        u = unit(np.cross(unit(rng.standard_normal(3)), f))
        s = np.cross(f, u)
        F = rng.standard_normal(3) * rng.uniform(1, 60)
        o = orc.modify_one(rng.uniform(-20, 20, 3), f, u, s, rng.uniform(0.5, 9), F, DT)
        f1 = np.asarray(o["fwd"], np.float64)
        proj = unit(u - np.dot(u, f1) * f1)
        if np.linalg.norm(u - np.dot(u, f1) * f1) < 1e-3:
            continue  # new forward (nearly) parallel to the old up: reading Q13
        np.testing.assert_allclose(o["up"], proj, atol=2e-5)
        assert np.dot(o["up"], u) > 0
        assert abs(_det3(o["side"], o["up"], o["fwd"]) + 1.0) < 1e-5


@pytest.mark.parametrize("mode", [0, 1])
def test_init_local_space_handedness(orc, mode):
    """Appendix B: up0 = (0,1,0), side = n^(f x up0), up = side x f -- so up is
    the world y axis projected normal to the forward (u . y > 0) and
    det[side, up, fwd] = -1 for every agent."""
    s = orc.init(5000, orc.default_params(init_mode=mode), seed=7)
    f = s["fwd"].astype(np.float64)
    y = np.array([0.0, 1.0, 0.0])
    proj = y - (f @ y)[:, None] * f
    ok = np.linalg.norm(proj, axis=1) > 1e-3
    proj = proj[ok] / np.linalg.norm(proj[ok], axis=1)[:, None]
    np.testing.assert_allclose(s["up"][ok], proj, atol=2e-5)
    assert (s["up"][ok][:, 1] > 0).all()
    det = np.einsum("ij,ij->i", s["side"].astype(np.float64),
                    np.cross(s["up"].astype(np.float64), f))
    np.testing.assert_allclose(det[ok], -1.0, atol=1e-5)
