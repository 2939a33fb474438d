"""Pins for the oracle's neighbour search (Listing 5.2; Listing 6.3).

Independent checks (none re-types the oracle's streaming algorithm):
  * brute force: sort ALL (d2, j) with numpy and take the first 7 with
    d2 < r2 (readings Q2-Q5), exhaustively on tiny flocks;
  * invariants: cnt <= 7, all d2 < r2, self excluded, keys ascending,
    cnt == min(7, #in radius), d2(i,j) bitwise == d2(j,i);
  * boundary: an agent exactly at r is excluded, nextafter(r, 0) included;
  * relabelling equivariance on tie-free inputs;
  * scipy cKDTree (fp64) on tie-free, boundary-free inputs;
  * the hand-worked golden fixture tests/golden/line_search.json.
"""
import json
import os

import numpy as np
import pytest

import workloads as W

R = np.float32(9.0)
R2 = np.float32(R * R)


def d2_row(pos, i):
    """fl(fl(fl(dx*dx) + fl(dy*dy)) + fl(dz*dz)) with d = p_i - p_j (Q3), numpy float32."""
    d = pos[i][None, :] - pos  # float32 elementwise, rounded per op
    xx = d[:, 0] * d[:, 0]
    yy = d[:, 1] * d[:, 1]
    zz = d[:, 2] * d[:, 2]
    return (xx + yy) + zz


def brute(pos, r2=R2):
    n = pos.shape[0]
    idx = np.full((n, 7), -1, np.int32)
    cnt = np.zeros(n, np.int32)
    for i in range(n):
        d2 = d2_row(pos, i)
        j = np.arange(n)
        ok = (d2 < r2) & (j != i)
        jj, dd = j[ok], d2[ok]
        order = np.lexsort((jj, dd))  # primary d2, secondary index
        take = jj[order][:7]
        idx[i, : take.size] = take
        cnt[i] = take.size
    return idx, cnt


def check_invariants(pos, idx, cnt, r2=R2):
    n = pos.shape[0]
    assert (cnt >= 0).all() and (cnt <= 7).all()
    for i in range(n):
        c = int(cnt[i])
        assert (idx[i, c:] == -1).all()
        nb = idx[i, :c]
        assert (nb != i).all(), "self must be excluded (P:523 global_index != my_index)"
        assert len(set(nb.tolist())) == c
        d2 = d2_row(pos, i)
        assert (d2[nb] < r2).all()
        keys = list(zip(d2[nb].tolist(), nb.tolist()))
        assert keys == sorted(keys) and len(set(keys)) == c
        inr = int(((d2 < r2) & (np.arange(n) != i)).sum())
        assert c == min(7, inr)


@pytest.mark.parametrize("seed", range(200))
def test_bruteforce_random_tiny(orc, seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 65))
    rad = float(rng.choice([4.0, 8.0, 15.0]))
    s = W.ball_flock(n, seed=seed, radius=rad)
    idx, cnt = orc.search(s["pos"], 9.0)
    bi, bc = brute(s["pos"])
    np.testing.assert_array_equal(idx, bi)
    np.testing.assert_array_equal(cnt, bc)
    check_invariants(s["pos"], idx, cnt)


@pytest.mark.parametrize("side,spacing", [(3, 1.0), (4, 1.0), (4, 2.0), (5, 3.0), (3, 4.5)])
def test_lattice_ties(orc, side, spacing):
    s = W.lattice_flock(side, spacing, seed=side)
    idx, cnt = orc.search(s["pos"], 9.0)
    bi, bc = brute(s["pos"])
    np.testing.assert_array_equal(idx, bi)
    np.testing.assert_array_equal(cnt, bc)
    check_invariants(s["pos"], idx, cnt)


@pytest.mark.parametrize("n,groups", [(2, 1), (9, 1), (20, 3), (40, 5)])
def test_coincident(orc, n, groups):
    s = W.coincident_flock(n, groups, seed=n)
    idx, cnt = orc.search(s["pos"], 9.0)
    bi, bc = brute(s["pos"])
    np.testing.assert_array_equal(idx, bi)
    # a different agent at d2 == 0 is a neighbour (Q6)
    same = np.all(s["pos"][:, None, :] == s["pos"][None, :, :], axis=2)
    for i in range(n):
        k = int(same[i].sum()) - 1
        assert cnt[i] >= min(7, k)


def test_radius_boundary(orc):
    s = W.radius_shell_flock(9.0)
    idx, cnt = orc.search(s["pos"], 9.0)
    nb = set(idx[0, : cnt[0]].tolist())
    pos = s["pos"]
    for j in range(1, pos.shape[0]):
        on_r = np.abs(pos[j]).max() == np.float32(9.0)
        assert (j in nb) == (not on_r), (j, pos[j])
    assert cnt[0] == 6


def test_d2_symmetric_bitwise():
    s = W.ball_flock(50, seed=3)
    p = s["pos"]
    M = np.stack([d2_row(p, i) for i in range(50)])
    assert np.array_equal(M.view(np.uint32), M.T.view(np.uint32))


@pytest.mark.parametrize("seed", range(5))
def test_relabel_equivariance(orc, seed):
    s = W.ball_flock(300, seed=seed, radius=15.0)
    p = s["pos"]
    perm = np.random.default_rng(seed + 100).permutation(300)
    inv = np.argsort(perm)
    i1, c1 = orc.search(p, 9.0)
    i2, c2 = orc.search(np.ascontiguousarray(p[perm]), 9.0)
    # agent k of the permuted flock is agent perm[k] of the original
    np.testing.assert_array_equal(c2, c1[perm])
    for k in range(300):
        got = [perm[j] for j in i2[k, : c2[k]]]
        # tie-free check: compare as sets (keys with equal d2 would reorder)
        assert set(got) == set(i1[perm[k], : c1[perm[k]]].tolist())


def test_ckdtree_fp64(orc):
    from scipy.spatial import cKDTree

    s = W.ball_flock(2000, seed=11, radius=20.0)
    p = s["pos"]
    idx, cnt = orc.search(p, 9.0)
    tree = cKDTree(p.astype(np.float64))
    dist, nb = tree.query(p.astype(np.float64), k=9, distance_upper_bound=9.0)
    checked = 0
    for i in range(2000):
        ok = np.isfinite(dist[i])
        dd, jj = dist[i][ok], nb[i][ok]
        keep = jj != i
        dd, jj = dd[keep], jj[keep]
        # skip rows where rounding could matter: near-ties at the 7/8 cut or near the radius
        if dd.size >= 8 and abs(dd[7] - dd[6]) < 1e-4:
            continue
        if dd.size and np.any(np.abs(dd - 9.0) < 1e-4):
            continue
        ref = jj[:7]
        assert set(ref.tolist()) == set(idx[i, : cnt[i]].tolist())
        checked += 1
    assert checked > 1900


def test_golden_line(orc):
    """Hand-worked example from Listing 5.2's rules (tests/golden/line_search.json)."""
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "line_search.json")))
    pos = np.array(g["positions"], np.float32)
    idx, cnt = orc.search(pos, g["radius"])
    for i, exp in enumerate(g["expected_neighbors"]):
        assert idx[i, : cnt[i]].tolist() == exp, (i, idx[i], exp)


def test_search_one_matches_all(orc):
    s = W.ball_flock(100, seed=5, radius=10.0)
    idx, cnt = orc.search(s["pos"], 9.0)
    for i in (0, 17, 99):
        i1, c1 = orc.search_one(s["pos"], i, 9.0)
        assert c1 == cnt[i] and (i1 == idx[i]).all()
