"""Pins of the oracle's softened direct-sum gravity (reading 20)
against closed forms: the two-body force, Newton's third law (total momentum
change zero), the softened pair at r = 0, the interior field and the potential
energy of a uniform sphere, and the Evrard profile's enclosed mass law."""
import math

import numpy as np

import oracle
from paper_conf_sc_simsekpc24_b200 import ics


def test_two_body_closed_form():
    x = np.array([0.0, 0.3]); y = np.array([0.0, 0.4]); z = np.zeros(2)
    m = np.array([2.0, 5.0])
    g = oracle.gravity(x, y, z, m, G=1.5, eps=0.1)
    r2 = 0.25 + 0.01
    s = 1.5 / r2 ** 1.5
    assert abs(g["ax"][0] / (s * 5.0 * 0.3) - 1) < 1e-14 and abs(g["ay"][0] / (s * 5.0 * 0.4) - 1) < 1e-14
    assert abs(g["ax"][1] / (-s * 2.0 * 0.3) - 1) < 1e-14
    assert abs(g["phi"][0] / (-1.5 * 5.0 / math.sqrt(r2)) - 1) < 1e-14


def test_coincident_pair_is_finite_and_zero():
    g = oracle.gravity(np.zeros(2), np.zeros(2), np.zeros(2), np.ones(2), G=1.0, eps=0.05)
    assert np.all(g["ax"] == 0) and np.all(np.isfinite(g["phi"]))
    assert abs(g["phi"][0] + 1.0 / 0.05) < 1e-12


def test_third_law():
    rng = np.random.default_rng(1)
    n = 500
    x, y, z = rng.normal(size=(3, n))
    m = rng.uniform(0.5, 2.0, n)
    g = oracle.gravity(x, y, z, m, G=1.0, eps=0.02)
    for k, a in (("ax", 0), ("ay", 1), ("az", 2)):
        assert abs((m * g[k]).sum()) < 1e-13 * (m[:, None] * g["a_abs"]).sum()


def test_uniform_sphere_field_and_energy():
    # lattice points of a unit sphere, total mass 1: interior field -G M r / R^3,
    # potential energy -3/5 G M^2 / R (discreteness + softening: a few percent)
    g1 = np.arange(26) + 0.5
    X, Y, Z = np.meshgrid(g1, g1, g1, indexing="ij")
    X, Y, Z = (2 * X / 26 - 1).ravel(), (2 * Y / 26 - 1).ravel(), (2 * Z / 26 - 1).ravel()
    r = np.sqrt(X * X + Y * Y + Z * Z)
    k = r < 1.0
    X, Y, Z, r = X[k], Y[k], Z[k], r[k]
    m = np.full(X.size, 1.0 / X.size)
    g = oracle.gravity(X, Y, Z, m, G=1.0, eps=0.02)
    inner = (r > 0.2) & (r < 0.7)
    ar = (g["ax"] * X + g["ay"] * Y + g["az"] * Z)[inner] / r[inner]
    assert np.abs(ar / (-r[inner]) - 1.0).mean() < 0.03
    W = 0.5 * (m * g["phi"]).sum()
    assert abs(W / (-0.6) - 1.0) < 0.03


def test_evrard_enclosed_mass_profile():
    w = ics.evrard(30)
    r = np.sqrt(w.state["x"] ** 2 + w.state["y"] ** 2 + w.state["z"] ** 2)
    assert r.max() < 1.0
    for R in (0.3, 0.5, 0.8):
        frac = (r < R).mean()
        assert abs(frac - R ** 2) < 0.02, (R, frac)
