"""Pins of the oracle's velocity divergence / curl (IADVelocityDivCurl, P:180;
DESIGN.md reading 19) and of the Balsara AV switch, against closed forms: the
IAD gradient is exact for linear velocity fields, so for v = A x the tensor T
equals A^T (T_ab = dv_b/dx_a) at every target whose neighbours need no
periodic image; rigid rotation and pure expansion are special cases; the
switch is 1 for compression without vorticity, ~0 for rotation without
compression, and the viscosity with the switch at 1 (0) equals the plain
(no) viscosity bit for bit."""
import numpy as np

import oracle
from paper_conf_sc_simsekpc24_b200 import ics


def _setup(nside=12, A=None, seed=3):
    w = ics.turbulence(nside)
    s = {k: v.copy() for k, v in w.state.items()}
    P = w.params
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], P)
    nb = oracle.neighbors(s["x"], s["y"], s["z"], s["h"], bmin, bmax, P.periodic)
    if A is not None:
        X = np.stack([s["x"], s["y"], s["z"]])
        s["vx"], s["vy"], s["vz"] = A @ X
    rho = oracle.density(s["x"], s["y"], s["z"], s["h"], s["m"], bmin, bmax, P.periodic, nb, P)
    p, c = oracle.eos(rho, s["u"], P)
    Cm, _, _, sing = oracle.iad(s["x"], s["y"], s["z"], s["h"], s["m"], rho, bmin, bmax,
                                P.periodic, nb, P)
    assert not sing
    T, Tabs, dv, curl = oracle.divcurl(s["x"], s["y"], s["z"], s["vx"], s["vy"], s["vz"], s["h"],
                                       s["m"], rho, Cm, bmin, bmax, P.periodic, nb, P)
    # targets whose 2h sphere stays inside the box: v_j - v_i = A (x_j - x_i) exactly
    inner = np.all(np.abs(np.stack([s["x"], s["y"], s["z"]])) < 0.5 - 2.05 * s["h"], axis=0)
    return dict(s=s, P=P, bmin=bmin, bmax=bmax, nb=nb, rho=rho, p=p, c=c, C=Cm, T=T, Tabs=Tabs,
                divv=dv, curl=curl, inner=inner)


def test_linear_field_gradient_is_exact():
    A = np.array([[0.3, -1.1, 0.4], [0.7, -0.2, 1.3], [-0.5, 0.9, 0.6]])
    r = _setup(A=A)
    assert r["inner"].sum() > 100
    T = r["T"][r["inner"]].reshape(-1, 3, 3)
    assert np.abs(T - A.T[None]).max() < 1e-12 * np.abs(A).max()
    assert np.abs(r["divv"][r["inner"]] - np.trace(A)).max() < 1e-12
    curl = np.array([A[2, 1] - A[1, 2], A[0, 2] - A[2, 0], A[1, 0] - A[0, 1]])
    assert np.abs(r["curl"][r["inner"]] - curl[None]).max() < 1e-12


def test_rigid_rotation_and_expansion():
    Om = np.array([0.2, -0.5, 1.1])
    skew = np.array([[0, -Om[2], Om[1]], [Om[2], 0, -Om[0]], [-Om[1], Om[0], 0]])  # v = Om x x
    r = _setup(A=skew)
    k = r["inner"]
    assert np.abs(r["divv"][k]).max() < 1e-12
    assert np.abs(r["curl"][k] - 2 * Om[None]).max() < 1e-12
    r = _setup(A=np.eye(3))
    k = r["inner"]
    assert np.abs(r["divv"][k] - 3.0).max() < 1e-12 and np.abs(r["curl"][k]).max() < 1e-12


def test_balsara_limits():
    c, h = np.full(3, 1.0), np.full(3, 0.01)
    f = oracle.balsara(np.array([-2.0, 0.0, 1.0]), np.array([[0, 0, 0], [0, 3.0, 0], [1.0, 0, 0]]),
                       c, h)
    assert abs(f[0] - 2.0 / (2.0 + 1e-2)) < 1e-15      # compression, no vorticity: ~1
    assert f[1] == 0.0                                    # rotation only: 0
    assert abs(f[2] - 1.0 / (2.0 + 1e-2)) < 1e-15


def test_switch_at_one_and_zero_is_plain_and_no_viscosity():
    r = _setup()
    s, P = r["s"], r["P"]
    args = (s["x"], s["y"], s["z"], s["vx"], s["vy"], s["vz"], s["h"], s["m"], r["rho"], r["p"],
            r["c"], r["C"], r["bmin"], r["bmax"], P.periodic, r["nb"], P)
    plain = oracle.momentum_energy(*args)
    one = oracle.momentum_energy(*args, fav=np.ones(s["x"].size))
    for k in ("ax", "ay", "az", "du"):
        assert np.array_equal(plain[k], one[k])
    zero = oracle.momentum_energy(*args, fav=np.zeros(s["x"].size))
    import dataclasses
    P0 = dataclasses.replace(P, av_alpha=0.0, av_beta=0.0)
    noav = oracle.momentum_energy(*args[:-1], P0)
    for k in ("ax", "ay", "az", "du"):
        assert np.array_equal(zero[k], noav[k])
