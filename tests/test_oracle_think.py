"""Pins for the think-frequency step (sec 5.3, Figs 5.6 / 6.3; Q15).

* k = 1 is exactly the plain step (every agent thinks);
* with k > 1, exactly the agents with (i + t) mod k == 0 think: their lists and
  steering equal the plain step's from the same state, the others keep their
  lists and use the stored vector -- with a zero store they coast, p' = p + v dt;
* over k consecutive steps every agent thinks exactly once.
"""
import numpy as np
import pytest

import workloads as W

DT = float(W.DT)


def fresh(orc, n):
    return np.full((n, 7), -1, np.int32), np.zeros(n, np.int32), np.zeros((n, 3), np.float32)


def test_k1_equals_plain_step(orc):
    s = orc.State(W.ball_flock(400, seed=2, radius=12.0))
    p = orc.default_params(think_every=1)
    idx, cnt, fs = fresh(orc, 400)
    o1, i1, c1, fs1, F1 = orc.step_think(s, DT, 5, fs, idx, cnt, p)
    o0, i0, c0, F0 = orc.step(s, DT)
    for k in o0:
        assert np.array_equal(o1[k], o0[k])
    assert np.array_equal(i1, i0) and np.array_equal(F1, F0) and np.array_equal(fs1, F0)


@pytest.mark.parametrize("k,t", [(3, 0), (3, 1), (10, 7)])
def test_only_thinkers_search(orc, k, t):
    n = 300
    s = orc.State(W.ball_flock(n, seed=k + t, radius=10.0))
    p = orc.default_params(think_every=k)
    idx, cnt, fs = fresh(orc, n)
    o, i2, c2, fs2, F = orc.step_think(s, DT, t, fs, idx, cnt, p)
    o0, i0, c0, F0 = orc.step(s, DT)
    think = (np.arange(n) + t) % k == 0
    assert np.array_equal(i2[think], i0[think]) and np.array_equal(F[think], F0[think])
    assert (i2[~think] == -1).all() and (c2[~think] == 0).all()
    assert (F[~think] == 0).all() and (fs2[~think] == 0).all()
    # zero stored force: non-thinkers coast in a straight line
    v = s["fwd"][~think].astype(np.float64) * s["speed"][~think, None]
    np.testing.assert_allclose(o["pos"][~think], s["pos"][~think] + v * DT, rtol=1e-5, atol=1e-5)
    for key in ("pos", "fwd", "speed"):
        assert np.array_equal(o[key][think], o0[key][think])


def test_every_agent_thinks_once_per_period(orc):
    n, k = 120, 4
    s = orc.State(W.ball_flock(n, seed=9, radius=8.0))
    p = orc.default_params(think_every=k)
    idx, cnt, fs = fresh(orc, n)
    thought = np.zeros(n, int)
    for t in range(k):
        before = fs.copy()
        s, idx, cnt, fs, F = orc.step_think(s, DT, t, fs, idx, cnt, p)
        thought += (np.any(fs != before, axis=1) | (cnt > 0)).astype(int) * ((np.arange(n) + t) % k == 0)
    assert (thought == 1).all()


@pytest.mark.parametrize("k,t", [(10, 11), (4, 2)])
def test_step_think_sample_matches_full(orc, k, t):
    """The sampled form used for full-size GPU checks (C4/C5 think 10) is
    step_think restricted to the sampled rows, with a nonzero stored force."""
    n = 400
    s = orc.State(W.ball_flock(n, seed=k * t, radius=10.0))
    p = orc.default_params(think_every=k)
    fs = W.random_forces(n, seed=3)
    idx, cnt, _ = fresh(orc, n)
    o, i2, c2, fs2, F = orc.step_think(s, DT, t, fs, idx, cnt, p)
    ag = np.array([0, 1, 2, 9, 10, 11, 57, 123, 398, 399])
    so, si, sc, sfs, sF = orc.step_think_sample(s, ag, DT, t, fs[ag], idx[ag], cnt[ag], p)
    for key in ("pos", "fwd", "up", "side", "speed"):
        assert np.array_equal(so[key], o[key][ag]), key
    assert np.array_equal(si, i2[ag]) and np.array_equal(sc, c2[ag])
    assert np.array_equal(sfs, fs2[ag]) and np.array_equal(sF, F[ag])
