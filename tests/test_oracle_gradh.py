"""Pins of the oracle's NormalizationGradh (reading 21) and of the
signal-velocity time step (reading 22), both optional parts of the step.

grad-h: dW/dh is checked against a central difference of the oracle's own W
(an independent route: W is pinned by quadrature elsewhere), and Omega against
a central difference of the density in h -- Omega_i = 1 + h_i/(3 rho_i)
d rho_i/d h_i is the definition, the analytic sum is what the oracle computes.
Omega = 1 must reproduce the plain step bit for bit, and the Omega-weighted
pressure terms must keep momentum and energy conserved for symmetric pairs.
vsig: closed forms on two particles and on a lattice at rest.
Volume elements (reading 23): kx = 1 on a perfect lattice, mass scaling, a
loose partition of unity, Omega_VE against a central difference of kx(h), and
conservation with the VE density."""
import math

import numpy as np
import pytest

import oracle
from paper_conf_sc_simsekpc24_b200 import ics
from paper_conf_sc_simsekpc24_b200.ics import K_SINC6, StepParams


@pytest.mark.parametrize("r,h", [(0.0, 1.0), (0.3, 0.7), (1.0, 1.0), (1.7, 1.0), (1.99, 1.0),
                                 (0.05, 0.02)])
def test_dWdh_is_the_h_derivative_of_W(r, h):
    d = 1e-6 * h
    fd = (oracle.W(r, h + d, K_SINC6) - oracle.W(r, h - d, K_SINC6)) / (2 * d)
    an = oracle.dWdh(r, h, K_SINC6)
    assert an == pytest.approx(fd, rel=1e-7, abs=1e-9 * K_SINC6 / h ** 4)


def test_dWdh_closed_forms_and_support():
    assert oracle.dWdh(0.0, 2.0, K_SINC6) == pytest.approx(-3 * K_SINC6 / 16.0, rel=1e-15)
    # r = h: x = pi/2, cos x = 0 -> +3 K S^6 / h^4 with S = 2/pi
    assert oracle.dWdh(1.0, 1.0, K_SINC6) == pytest.approx(3 * K_SINC6 * (2 / math.pi) ** 6,
                                                           rel=1e-14)
    assert oracle.dWdh(2.0, 1.0, K_SINC6) == 0.0 and oracle.dWdh(2.5, 1.0, K_SINC6) == 0.0


def _jittered(nside=10, seed=4):
    w = ics.turbulence(nside)
    s = w.state
    rng = np.random.default_rng(seed)
    s["h"] = s["h"] * rng.uniform(0.9, 1.1, s["x"].size)     # variable h
    s["m"] = s["m"] * rng.uniform(0.5, 1.5, s["x"].size)
    return w


def _rho(w, h):
    s, P = w.state, w.params
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], P)
    nb = oracle.neighbors(s["x"], s["y"], s["z"], h, bmin, bmax, P.periodic)
    return oracle.density(s["x"], s["y"], s["z"], h, s["m"], bmin, bmax, P.periodic, nb, P), nb


def test_omega_is_one_plus_h_over_3rho_drho_dh():
    """Central difference of rho_i(h_i) (each rho_i depends on h_i only; the
    neighbour lists are recomputed exactly at each h, W is C^5 at the support
    edge) against the analytic sum of m_j dW/dh."""
    w = _jittered()
    s, P = w.state, w.params
    h = s["h"]
    rho, nb = _rho(w, h)
    d = 1e-4
    rp, _ = _rho(w, h * (1 + d))
    rm, _ = _rho(w, h * (1 - d))
    drho_dh = (rp - rm) / (2 * d * h)
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], P)
    om, dsum, dabs = oracle.gradh(s["x"], s["y"], s["z"], h, s["m"], rho, bmin, bmax, P.periodic,
                                  nb, P)
    assert np.all(np.abs(dsum - drho_dh) <= 1e-6 * dabs)
    assert np.allclose(om, 1 + h / (3 * rho) * drho_dh, rtol=1e-6, atol=0)
    assert np.all(np.isfinite(om)) and np.all(om > 0)


def test_omega_uniform_on_a_perfect_lattice():
    w = ics.sedov(12)
    s, P = w.state, w.params
    rho, nb = _rho(w, s["h"])
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], P)
    om, dsum, dabs = oracle.gradh(s["x"], s["y"], s["z"], s["h"], s["m"], rho, bmin, bmax,
                                  P.periodic, nb, P)
    assert np.ptp(om) <= 1e-13 * abs(om[0])
    # the sum of m dW/dh is a derivative of a sum of positive terms that changes
    # sign across the support: it is much smaller than its term scale
    assert abs(dsum[0]) < dabs[0]


def _chain(w, omega_mode):
    s, P = w.state, w.params
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], P)
    nb = oracle.neighbors(s["x"], s["y"], s["z"], s["h"], bmin, bmax, P.periodic)
    rho = oracle.density(s["x"], s["y"], s["z"], s["h"], s["m"], bmin, bmax, P.periodic, nb, P)
    p, c = oracle.eos(rho, s["u"], P)
    Cm, _, _, sing = oracle.iad(s["x"], s["y"], s["z"], s["h"], s["m"], rho, bmin, bmax,
                                P.periodic, nb, P)
    assert not sing
    om = None
    if omega_mode == "ones":
        om = np.ones(rho.size)
    elif omega_mode == "gradh":
        om = oracle.gradh(s["x"], s["y"], s["z"], s["h"], s["m"], rho, bmin, bmax, P.periodic,
                          nb, P)[0]
    return oracle.momentum_energy(s["x"], s["y"], s["z"], s["vx"], s["vy"], s["vz"], s["h"],
                                  s["m"], rho, p, c, Cm, bmin, bmax, P.periodic, nb, P,
                                  omega=om), om


def test_omega_one_is_the_plain_step():
    w = _jittered()
    a, _ = _chain(w, None)
    b, _ = _chain(w, "ones")
    for k in ("ax", "ay", "az", "du"):
        assert np.array_equal(a[k], b[k])


def test_gradh_changes_the_pressure_terms_and_conserves():
    """Uniform h (symmetric pairs): sum m a = 0 and sum m (v.a + du) = 0 with the
    Omega-weighted pressure terms; and Omega != 1 does change the result."""
    w = ics.turbulence(10)
    s = w.state
    rng = np.random.default_rng(9)
    s["u"] = rng.uniform(0.5, 2.0, s["x"].size)
    w.params.eos = 0
    r, om = _chain(w, "gradh")
    r0, _ = _chain(w, None)
    assert np.max(np.abs(om - 1)) > 1e-3
    assert not np.allclose(r["ax"], r0["ax"], rtol=1e-6, atol=0)
    m = s["m"]
    scale = (m[:, None] * r["a_abs"]).sum(0)
    mom = np.array([(m * r["ax"]).sum(), (m * r["ay"]).sum(), (m * r["az"]).sum()])
    assert np.all(np.abs(mom) < 1e-14 * scale)
    power = (m * (s["vx"] * r["ax"] + s["vy"] * r["ay"] + s["vz"] * r["az"] + r["du"])).sum()
    pscale = (m * (np.abs(s["vx"]) * r["a_abs"][:, 0] + np.abs(s["vy"]) * r["a_abs"][:, 1]
                   + np.abs(s["vz"]) * r["a_abs"][:, 2] + r["du_abs"])).sum()
    assert abs(power) < 1e-14 * pscale


# ----------------------------------------------------------------- vsig
def _pair(v, c=(1.0, 2.0), h=1.0):
    x = np.array([0.0, 1.0])
    z = np.zeros(2)
    P = StepParams(box_min=(-10, -10, -10), box_max=(10, 10, 10), k_cour=0.2, dt_max_growth=1e9)
    bmin, bmax = np.array(P.box_min), np.array(P.box_max)
    nb = oracle.neighbors(x, z, z, np.full(2, h), bmin, bmax, P.periodic)
    vx = np.array([v, -v])
    return oracle.timestep_vsig(x, z, z, vx, z, z, np.full(2, h), np.array(c), bmin, bmax,
                                P.periodic, nb, 1.0, P)


def test_vsig_two_particles():
    # approaching head on at relative speed 2v: w = -2v, vsig = c_i + c_j + 6v
    dt, vs = _pair(0.5)
    assert vs == pytest.approx([1 + 2 + 3.0, 1 + 2 + 3.0], rel=1e-15)
    assert dt == pytest.approx(0.2 * 1.0 / 6.0, rel=1e-15)
    # receding: vsig = max(2 c_i, c_i + c_j)
    dt, vs = _pair(-0.5)
    assert vs.tolist() == [3.0, 4.0]
    assert dt == pytest.approx(0.2 / 4.0, rel=1e-15)


def test_vsig_lattice_at_rest_and_growth_cap():
    w = ics.sedov(8)
    s, P = w.state, w.params
    c = np.full(s["x"].size, 1.5)
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], P)
    nb = oracle.neighbors(s["x"], s["y"], s["z"], s["h"], bmin, bmax, P.periodic)
    dt, vs = oracle.timestep_vsig(s["x"], s["y"], s["z"], s["vx"], s["vy"], s["vz"], s["h"], c,
                                  bmin, bmax, P.periodic, nb, 1.0, P)
    assert np.all(vs == 3.0)
    assert dt == P.k_cour * (s["h"].min() / 3.0)
    dt2, _ = oracle.timestep_vsig(s["x"], s["y"], s["z"], s["vx"], s["vy"], s["vz"], s["h"], c,
                                  bmin, bmax, P.periodic, nb, 1e-9, P)
    assert dt2 == P.dt_max_growth * 1e-9


def test_step_with_gradh_and_vsig_runs_and_conserves_mass():
    w = ics.sedov(8)
    w.params.gradh = 1
    w.params.dt_vsig = 1
    st, o = oracle.step({k: v.copy() for k, v in w.state.items()}, w.params, w.params.dt_first,
                        True)
    assert "omega" in o and "vsig" in o
    assert np.all(np.isfinite(st["u"])) and st["m"].sum() == pytest.approx(w.state["m"].sum(),
                                                                           rel=1e-15)


# ----------------------------------------------------------------- volume elements
def _ve_parts(w):
    s, P = w.state, w.params
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], P)
    nb = oracle.neighbors(s["x"], s["y"], s["z"], s["h"], bmin, bmax, P.periodic)
    import dataclasses
    P2 = dataclasses.replace(P, ve=1, gradh=1)
    st, o = oracle.step({k: v.copy() for k, v in s.items()}, P2, P2.dt_first, True)
    return o, nb


def test_ve_lattice_normalisation_is_one():
    """Perfect lattice, uniform masses: X = m/rho0 is uniform, so the
    normalisation kx = sum_j X_j W_ij = X rho0 / m = 1 and rho = rho0."""
    o, _ = _ve_parts(ics.sedov(12))
    assert np.allclose(o["kx"], 1.0, rtol=1e-13, atol=0)
    assert np.allclose(o["rho"], o["rho0"], rtol=1e-13, atol=0)


def test_ve_mass_scaling_and_partition_of_unity():
    """Doubling every mass doubles rho0 and rho and leaves X, kx unchanged; on
    a disordered set kx stays a partition of unity to within the kernel's
    accuracy (a few %)."""
    w = _jittered()
    o1, _ = _ve_parts(w)
    w.state["m"] = 2.0 * w.state["m"]
    o2, _ = _ve_parts(w)
    assert np.allclose(o2["kx"], o1["kx"], rtol=1e-13, atol=0)
    assert np.allclose(o2["rho"], 2 * o1["rho"], rtol=1e-13, atol=0)
    # (h varies by +-10% and m by +-50% here: the sum is a loose partition of unity)
    assert np.all(np.abs(o1["kx"] - 1) < 0.3) and abs(np.mean(o1["kx"]) - 1) < 0.05
    assert np.std(o1["kx"]) > 1e-4


def test_ve_omega_is_the_h_derivative_of_kx():
    """Omega_VE = 1 + (h/(3 kx)) d kx/dh with X held fixed (central difference
    of the normalisation sum, lists recomputed at each h)."""
    w = _jittered(seed=8)
    s, P = w.state, w.params
    o, nb = _ve_parts(w)
    X, h = o["X"], o["pre"]["h"]
    pre = o["pre"]
    bmin, bmax = o["bmin"], o["bmax"]

    def kx_at(hh):
        nbh = oracle.neighbors(pre["x"], pre["y"], pre["z"], hh, bmin, bmax, P.periodic)
        return oracle.density(pre["x"], pre["y"], pre["z"], hh, X, bmin, bmax, P.periodic, nbh, P)
    d = 1e-4
    dk = (kx_at(h * (1 + d)) - kx_at(h * (1 - d))) / (2 * d * h)
    assert np.all(np.abs(o["dWdh_sum"] - dk) <= 1e-6 * o["dWdh_abs"])
    assert np.allclose(o["omega"], 1 + h / (3 * o["kx"]) * dk, rtol=1e-6, atol=0)


def test_ve_conserves_momentum_and_energy_uniform_h():
    import dataclasses
    w = ics.turbulence(10)
    s = w.state
    rng = np.random.default_rng(9)
    s["u"] = rng.uniform(0.5, 2.0, s["x"].size)
    w.params = dataclasses.replace(w.params, eos=0, ve=1, gradh=1)
    st, r = oracle.step({k: v.copy() for k, v in s.items()}, w.params, w.params.dt_first, True)
    pre = r["pre"]
    m = pre["m"]
    scale = (m[:, None] * r["a_abs"]).sum(0)
    mom = np.array([(m * r["ax"]).sum(), (m * r["ay"]).sum(), (m * r["az"]).sum()])
    assert np.all(np.abs(mom) < 1e-14 * scale)
    power = (m * (pre["vx"] * r["ax"] + pre["vy"] * r["ay"] + pre["vz"] * r["az"] + r["du"])).sum()
    pscale = (m * (np.abs(pre["vx"]) * r["a_abs"][:, 0] + np.abs(pre["vy"]) * r["a_abs"][:, 1]
                   + np.abs(pre["vz"]) * r["a_abs"][:, 2] + r["du_abs"])).sum()
    assert abs(power) < 1e-14 * pscale
