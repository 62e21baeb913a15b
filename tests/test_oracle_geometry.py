"""Pins for the oracle's box, keys, sort and neighbour search.

Independent references: numpy's stable argsort (library sort), scipy's cKDTree
(library neighbour search), lattice counting (closed form, golden 92)."""
import math

import numpy as np
import pytest
from scipy.spatial import cKDTree

import oracle
from paper_conf_sc_simsekpc24_b200 import ics


def test_box_open_and_periodic():
    w = ics.random_box(500, seed=1, periodic=False)
    s = w.state
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], w.params)
    assert np.array_equal(bmin, [s["x"].min(), s["y"].min(), s["z"].min()])
    assert np.array_equal(bmax, [s["x"].max(), s["y"].max(), s["z"].max()])
    p = ics.StepParams(periodic=(1, 0, 1))
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], p)
    assert bmin[0] == -0.5 and bmax[2] == 0.5 and bmin[1] == s["y"].min()
    with pytest.raises(ValueError):
        oracle.box(np.zeros(3), np.zeros(3), np.zeros(3), ics.StepParams(periodic=(0, 0, 0)))


def test_keys_quantise_and_clamp():
    bmin, bmax = np.array([-0.5] * 3), np.array([0.5] * 3)
    x = np.array([-0.5, 0.5, 0.0, -0.5 + 1.0 / 2 ** 21, 0.4999999999])
    zero = np.full(x.size, -0.5)
    k = oracle.keys(x, zero, zero, bmin, bmax)
    # x-only coordinates: key = morton(ix, 0, 0)
    ix = [0, 2 ** 21 - 1, 2 ** 20, 1, 2 ** 21 - 1]
    assert [int(v) for v in k] == [oracle.morton(i, 0, 0) for i in ix]
    # beyond the box (x == max after a periodic wrap rounding) clamps to the last cell
    k2 = oracle.keys(np.array([0.5, 0.7, -0.9]), np.zeros(3), np.zeros(3), bmin, bmax)
    assert int(k2[0]) == int(k2[1]) == oracle.morton(2 ** 21 - 1, 2 ** 20, 2 ** 20)
    assert int(k2[2]) == oracle.morton(0, 2 ** 20, 2 ** 20)


def test_sort_is_stable_sort_by_key():
    rng = np.random.default_rng(3)
    k = rng.integers(0, 50, 5000).astype(np.uint64)  # many ties
    perm = oracle.sort_order(k)
    assert np.array_equal(perm, np.argsort(k, kind="stable"))
    k = rng.integers(0, 2 ** 63 - 1, 10000, dtype=np.int64).astype(np.uint64)
    assert np.array_equal(oracle.sort_order(k), np.argsort(k, kind="stable"))


def _kdtree_sets(w):
    s = w.state
    L = 1.0
    pts = np.stack([s["x"], s["y"], s["z"]], axis=1) + 0.5
    pts = np.mod(pts, L)
    tree = cKDTree(pts, boxsize=L if all(w.params.periodic) else None)
    res = tree.query_ball_point(pts, r=2 * s["h"])
    return [sorted(set(r) - {i}) for i, r in enumerate(res)]


@pytest.mark.parametrize("periodic", [True, False])
def test_neighbors_match_kdtree(periodic):
    """Brute force == scipy cKDTree (minimum image for periodic boxes), away from
    pairs whose distance sits within 1e-9 of the 2h boundary (rounding differs)."""
    w = ics.random_box(3000, seed=11, periodic=periodic)
    s = w.state
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], w.params)
    nb = oracle.neighbors(s["x"], s["y"], s["z"], s["h"], bmin, bmax, w.params.periodic)
    ref = _kdtree_sets(w)
    for i in range(s["x"].size):
        got = nb.idx[nb.offsets[i]:nb.offsets[i + 1]].tolist()
        assert got == sorted(got)
        assert i not in got
        if got != ref[i]:
            diff = set(got) ^ set(ref[i])
            for j in diff:
                d = np.array([s["x"][i] - s["x"][j], s["y"][i] - s["y"][j], s["z"][i] - s["z"][j]])
                if periodic:
                    d -= np.round(d)
                assert abs(np.linalg.norm(d) - 2 * s["h"][i]) < 1e-9 * s["h"][i]


@pytest.mark.parametrize("nside", [8, 10, 16])
def test_lattice_neighbour_count(golden, nside):
    """Perfect periodic lattice with h0(ng0=100): 2h/a = (75/pi)^(1/3); the
    lattice vectors with |v|^2 < 8.29 are 6+12+8+6+24+24+12 = 92 (7 is not a sum
    of three squares)."""
    w = ics.sedov(nside)
    s = w.state
    a = 1.0 / nside
    assert 2 * s["h"][0] / a == pytest.approx((75 / math.pi) ** (1 / 3), rel=1e-14)
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], w.params)
    nb = oracle.neighbors(s["x"], s["y"], s["z"], s["h"], bmin, bmax, w.params.periodic)
    assert np.all(nb.nc == golden["lattice_nc"]["value"])


def test_neighbors_empty_and_single():
    p = ics.StepParams()
    nb = oracle.neighbors(np.zeros(1), np.zeros(1), np.zeros(1), np.full(1, 0.1),
                          np.array(p.box_min), np.array(p.box_max), p.periodic)
    assert nb.nc.tolist() == [0] and nb.offsets.tolist() == [0, 0]
    nb = oracle.neighbors(np.zeros(0), np.zeros(0), np.zeros(0), np.zeros(0),
                          np.array(p.box_min), np.array(p.box_max), p.periodic)
    assert nb.nc.size == 0


def test_minimum_image_across_the_boundary():
    """A pair straddling the periodic face at distance 0.02 is found; the same pair in
    an open box (raw distance 0.98) is not."""
    x = np.array([-0.49, 0.49])
    y = np.zeros(2)
    h = np.full(2, 0.02)
    per = ics.StepParams()
    nb = oracle.neighbors(x, y, y, h, np.array(per.box_min), np.array(per.box_max), (1, 1, 1))
    assert nb.nc.tolist() == [1, 1]
    nb = oracle.neighbors(x, y, y, h, np.array(per.box_min), np.array(per.box_max), (0, 1, 1))
    assert nb.nc.tolist() == [0, 0]


def test_gather_criterion_is_asymmetric():
    """j in N(i) iff r < 2 h_i: with h_i large and h_j small only i sees j."""
    x = np.array([0.0, 0.1])
    z = np.zeros(2)
    h = np.array([0.06, 0.04])
    p = ics.StepParams()
    nb = oracle.neighbors(x, z, z, h, np.array(p.box_min), np.array(p.box_max), (1, 1, 1))
    assert nb.nc.tolist() == [1, 0]
