"""Pins for the oracle's density, EOS, IAD, momentum-energy, timestep and update
(SURVEY 8(c) steps 5-10 and its 'Pins' table).

Each test is chosen so that a plausible slip -- a dropped term, a sign, a
transposed index, a wrong mean -- fails it: golden lattice values, closed forms
for continuum gradients/divergences, exact conservation identities and the IAD
linear-exactness property."""
import math

import numpy as np
import pytest

import oracle
from paper_conf_sc_simsekpc24_b200 import ics
from paper_conf_sc_simsekpc24_b200.ics import K_SINC6, StepParams


def _prep(w):
    s = w.state
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], w.params)
    nb = oracle.neighbors(s["x"], s["y"], s["z"], s["h"], bmin, bmax, w.params.periodic)
    return s, bmin, bmax, nb


def _chain(w, s=None):
    s0, bmin, bmax, nb = _prep(w)
    s = s or s0
    P = w.params
    rho = oracle.density(s["x"], s["y"], s["z"], s["h"], s["m"], bmin, bmax, P.periodic, nb, P)
    p, c = oracle.eos(rho, s["u"], P)
    Cm, tau, tabs, sing = oracle.iad(s["x"], s["y"], s["z"], s["h"], s["m"], rho, bmin, bmax,
                                     P.periodic, nb, P)
    assert not sing
    acc = oracle.momentum_energy(s["x"], s["y"], s["z"], s["vx"], s["vy"], s["vz"], s["h"],
                                 s["m"], rho, p, c, Cm, bmin, bmax, P.periodic, nb, P)
    return dict(rho=rho, p=p, c=c, C=Cm, tau=tau, tau_abs=tabs, nb=nb, **acc)


# ----------------------------------------------------------------- density
def test_density_pair(golden):
    """Two particles, m = 1, h = 1, separation 1 (box large enough to be irrelevant)."""
    x = np.array([0.0, 1.0])
    z = np.zeros(2)
    h = np.ones(2)
    P = StepParams(box_min=(-10, -10, -10), box_max=(10, 10, 10))
    nb = oracle.neighbors(x, z, z, h, np.array(P.box_min), np.array(P.box_max), P.periodic)
    rho = oracle.density(x, z, z, h, np.ones(2), np.array(P.box_min), np.array(P.box_max),
                         P.periodic, nb, P)
    assert rho == pytest.approx([golden["rho_pair"]["value"]] * 2, rel=2e-15)
    assert golden["rho_pair"]["value"] == pytest.approx(K_SINC6 * (1 + (2 / math.pi) ** 6), rel=1e-15)


@pytest.mark.parametrize("nside", [10, 16])
def test_density_lattice(golden, nside):
    """Perfect lattice, exact K: rho = 0.99995886562268914 for every particle, any N."""
    w = ics.sedov(nside)
    r = _chain(w)
    assert np.allclose(r["rho"], golden["lattice_rho"]["value"], rtol=1e-14, atol=0)


def test_density_mass_scaling_and_self_term():
    """rho is linear in the masses; a lone particle has rho = m W(0,h) = m K/h^3."""
    w = ics.random_box(800, seed=4)
    s, bmin, bmax, nb = _prep(w)
    P = w.params
    r1 = oracle.density(s["x"], s["y"], s["z"], s["h"], s["m"], bmin, bmax, P.periodic, nb, P)
    r2 = oracle.density(s["x"], s["y"], s["z"], s["h"], 3 * s["m"], bmin, bmax, P.periodic, nb, P)
    assert np.allclose(r2, 3 * r1, rtol=1e-14)
    one = oracle.neighbors(np.zeros(1), np.zeros(1), np.zeros(1), np.full(1, 0.1), bmin, bmax, P.periodic)
    r = oracle.density(np.zeros(1), np.zeros(1), np.zeros(1), np.full(1, 0.1), np.full(1, 2.0),
                       bmin, bmax, P.periodic, one, P)
    assert r[0] == pytest.approx(2.0 * K_SINC6 / 0.1 ** 3, rel=1e-15)


# ----------------------------------------------------------------- EOS
def test_eos_closed_forms():
    rho = np.array([1.0, 2.0, 0.5])
    u = np.array([1.0, 3.0, 0.1])
    p, c = oracle.eos(rho, u, StepParams(eos=0, gamma=5 / 3))
    assert np.allclose(p, (2 / 3) * rho * u, rtol=1e-15)
    assert np.allclose(c, np.sqrt(10 / 9 * u), rtol=1e-15)
    p, c = oracle.eos(rho, u, StepParams(eos=1, cs0=2.0))
    assert np.allclose(p, 4 * rho, rtol=1e-15) and np.all(c == 2.0)
    # ideal gas: c^2 = gamma p / rho
    p, c = oracle.eos(rho, u, StepParams(eos=0, gamma=1.4))
    assert np.allclose(c * c, 1.4 * p / rho, rtol=1e-14)


# ----------------------------------------------------------------- IAD
def test_iad_lattice16(golden):
    w = ics.sedov(16)
    r = _chain(w)
    tau = r["tau"]
    assert np.allclose(tau[:, 0], golden["lattice16_tau11"]["value"], rtol=1e-13)
    assert np.allclose(tau[:, 3], tau[:, 0], rtol=1e-13) and np.allclose(tau[:, 5], tau[:, 0], rtol=1e-13)
    assert np.all(np.abs(tau[:, [1, 2, 4]]) < 1e-15 * tau[:, [0]])
    assert np.allclose(r["C"][:, 0], golden["lattice16_C11"]["value"], rtol=1e-13)


def test_iad_linear_exactness():
    """sum_j V_j (f_j - f_i) C_i Delta W_ij = g for linear f = g . x (jittered periodic
    lattice, f_j - f_i = g . Delta with the minimum image).  Pins C = tau^{-1}, the
    Delta sign and the pairing of tau with the same W and V as the gradient."""
    w = ics.turbulence(10)
    s, bmin, bmax, nb = _prep(w)
    r = _chain(w)
    g = np.array([0.3, -1.7, 0.9])
    V = s["m"] / r["rho"]
    err = 0.0
    for i in range(s["x"].size):
        js = nb.idx[nb.offsets[i]:nb.offsets[i + 1]]
        D = np.stack([s["x"][js] - s["x"][i], s["y"][js] - s["y"][i], s["z"][js] - s["z"][i]], 1)
        D -= np.round(D)  # minimum image in the unit box
        Wv = np.array([oracle.W(np.linalg.norm(d), s["h"][i], K_SINC6) for d in D])
        c = r["C"][i]
        Cm = np.array([[c[0], c[1], c[2]], [c[1], c[3], c[4]], [c[2], c[4], c[5]]])
        grad = ((V[js] * Wv * (D @ g))[:, None] * (D @ Cm.T)).sum(0)
        err = max(err, np.abs(grad - g).max() / np.abs(g).max())
    assert err < 1e-13


def test_iad_singular_detected():
    """A particle with a single neighbour has a rank-1 tau -> singular flag."""
    x = np.array([0.0, 0.05])
    z = np.zeros(2)
    h = np.full(2, 0.05)
    P = StepParams()
    nb = oracle.neighbors(x, z, z, h, np.array(P.box_min), np.array(P.box_max), P.periodic)
    _, _, _, sing = oracle.iad(x, z, z, h, np.ones(2), np.ones(2), np.array(P.box_min),
                               np.array(P.box_max), P.periodic, nb, P)
    assert sing


# ----------------------------------------------------------------- momentum / energy
def test_uniform_lattice_is_in_equilibrium():
    """Uniform lattice, uniform p, v = 0: a = du = 0 to roundoff of the term scale."""
    w = ics.sedov(12)
    w.state["u"][:] = 2.0
    r = _chain(w)
    for k, a in (("ax", 0), ("ay", 1), ("az", 2)):
        assert np.all(np.abs(r[k]) <= 1e-13 * r["a_abs"][:, a])
    assert np.all(np.abs(r["du"]) <= 1e-13 * r["du_abs"] + 1e-300)


def test_conservation_uniform_h():
    """Uniform h (symmetric pairs): sum m a = 0 and sum m (v.a + du) = 0 to roundoff."""
    w = ics.turbulence(10)
    s = w.state
    rng = np.random.default_rng(9)
    s["u"] = rng.uniform(0.5, 2.0, s["x"].size)
    w.params.eos = 0
    r = _chain(w)
    m = s["m"]
    scale = (m[:, None] * r["a_abs"]).sum(0)
    mom = np.array([(m * r["ax"]).sum(), (m * r["ay"]).sum(), (m * r["az"]).sum()])
    assert np.all(np.abs(mom) < 1e-14 * scale)
    power = (m * (s["vx"] * r["ax"] + s["vy"] * r["ay"] + s["vz"] * r["az"] + r["du"])).sum()
    pscale = (m * (np.abs(s["vx"]) * r["a_abs"][:, 0] + np.abs(s["vy"]) * r["a_abs"][:, 1]
                   + np.abs(s["vz"]) * r["a_abs"][:, 2] + r["du_abs"])).sum()
    assert abs(power) < 1e-14 * pscale


def _wave(nside, **kw):
    w = ics.sedov(nside)
    w.params.av_alpha = 0.0
    w.params.av_beta = 0.0
    for k, v in kw.items():
        w.state[k] = v(w.state)
    return w


def test_pressure_gradient_force():
    """u = 1 + eps sin(2 pi x), rho = 1, v = 0, gamma = 5/3:
    a_x -> -(1/rho) dp/dx = -(2/3) eps 2 pi cos(2 pi x); a_y = a_z = 0.
    The SPH estimate is the kernel-smoothed gradient: at k 2h ~ 0.9 the smoothing
    lowers it by ~2%, so agree to 4% (a dropped term or sign is off by >= 50%)."""
    eps = 0.01
    w = _wave(20, u=lambda s: 1 + eps * np.sin(2 * np.pi * s["x"]))
    r = _chain(w)
    s = w.state
    expect = -(2 / 3) * eps * 2 * np.pi * np.cos(2 * np.pi * s["x"]) * (r["rho"].mean() / r["rho"])
    assert np.abs(r["ax"] - expect).max() < 0.04 * np.abs(expect).max()
    assert np.abs(r["ay"]).max() < 1e-10 and np.abs(r["az"]).max() < 1e-10


def test_compression_heating():
    """v_x = v0 sin(2 pi x), uniform u: du/dt -> -(p/rho) div v = -(2/3) u v0 2 pi cos(2 pi x)."""
    v0 = 1e-3
    w = _wave(20, vx=lambda s: v0 * np.sin(2 * np.pi * s["x"]), u=lambda s: np.full(s["x"].size, 1.0))
    r = _chain(w)
    s = w.state
    p_over_rho = (2 / 3) * 1.0
    expect = -p_over_rho * v0 * 2 * np.pi * np.cos(2 * np.pi * s["x"])
    assert np.abs(r["du"] - expect).max() < 0.04 * np.abs(expect).max()


def test_viscosity_heats_and_decelerates_a_converging_flow():
    """Cold converging flow (u = 0, so p = c = 0 and only the beta mu^2 term acts;
    v = -0.1 r_hat inside r < 0.3): AV heats (du >= 0 everywhere, > 0 in total),
    removes kinetic energy (sum m v.a < 0) and conserves total energy exactly
    (sum m (v.a + du) = 0 with uniform h) -- the last pins the 1/2 in du."""
    w = ics.sedov(12)
    s = w.state
    rr = np.sqrt(s["x"] ** 2 + s["y"] ** 2 + s["z"] ** 2)
    for k in ("x", "y", "z"):
        s["v" + k] = -0.1 * s[k] / rr * (rr < 0.3)
    s["u"][:] = 0.0
    r = _chain(w)
    m = s["m"]
    assert np.all(r["du"] >= -1e-14 * r["du_abs"].max())  # sign noise only on ~1e-60 terms
    assert (m * r["du"]).sum() > 0
    kin = (m * (s["vx"] * r["ax"] + s["vy"] * r["ay"] + s["vz"] * r["az"])).sum()
    assert kin < 0
    assert abs(kin + (m * r["du"]).sum()) < 1e-13 * (m * r["du_abs"]).sum()


# ----------------------------------------------------------------- timestep / update
def test_timestep_sedov16(golden):
    w = ics.sedov(16)
    s = w.state
    _, c = oracle.eos(np.ones(s["x"].size), s["u"], w.params)
    dt = oracle.timestep(s["h"], c, w.params.dt_first, w.params)
    assert dt == golden["sedov16_dt0"]["value"] == 1.1 * 1e-6
    assert s["u"].max() == pytest.approx(golden["sedov16_u_max"]["value"], rel=1e-8)
    courant = 0.2 * s["h"][0] / math.sqrt(10 / 9 * s["u"].max())
    assert courant == pytest.approx(1.47e-3, rel=5e-3)  # SURVEY quotes 3 digits
    # Courant branch: a large dt_prev leaves the Courant limit
    dt2 = oracle.timestep(s["h"], c, 1.0, w.params)
    assert dt2 == 0.2 * float((s["h"] / c).min())


def test_update_free_streaming_and_h():
    """a = du = 0: x advances by v dt (wrapped), u unchanged; nc = 92 -> h' = 1.0083651 h;
    nc = ng0 -> h' = h exactly."""
    golden_ratio = 1.0083651
    n = 4
    st = {"x": np.array([0.1, 0.49, -0.49, 0.0]), "y": np.zeros(n), "z": np.zeros(n),
          "vx": np.array([1.0, 1.0, -1.0, 0.0]), "vy": np.zeros(n), "vz": np.zeros(n),
          "h": np.full(n, 0.01), "u": np.full(n, 3.0), "du_m1": np.zeros(n)}
    zero = {k: np.zeros(n) for k in ("ax", "ay", "az", "du")}
    nc = np.array([92, 100, 100, 0], dtype=np.int32)
    P = StepParams()
    x0 = st["x"].copy()
    oracle.update(st, zero, nc, 0.02, 0.02, True, np.array(P.box_min), np.array(P.box_max), P)
    assert st["x"][0] == x0[0] + 0.02
    assert st["x"][1] == pytest.approx(0.51 - 1.0, abs=1e-15)   # wrapped into [-0.5, 0.5)
    assert st["x"][2] == pytest.approx(-0.51 + 1.0, abs=1e-15)
    assert np.all(st["u"] == 3.0)
    assert st["h"][0] / 0.01 == pytest.approx(golden_ratio, abs=1e-7)
    assert st["h"][1] == 0.01 and st["h"][2] == 0.01
    assert st["h"][3] == pytest.approx(0.01 * 0.5 * (1 + 1023 * 100) ** 0.1, rel=1e-15)


def test_update_energy_integrator():
    """First step (du_m1 := du) is Euler: u += du dt.  Constant du over later steps:
    u advances by du dt exactly (AB2 of a constant); h clamps at h_cap."""
    n = 2
    st = {k: np.zeros(n) for k in ("x", "y", "z", "vx", "vy", "vz", "du_m1")}
    st["h"] = np.full(n, 0.2)
    st["u"] = np.full(n, 1.0)
    acc = {"ax": np.zeros(n), "ay": np.zeros(n), "az": np.zeros(n), "du": np.array([2.0, -1.0])}
    P = StepParams(h_cap=0.21)
    b0, b1 = np.array(P.box_min), np.array(P.box_max)
    oracle.update(st, acc, np.array([10, 10], dtype=np.int32), 0.01, 0.005, True, b0, b1, P)
    assert st["u"] == pytest.approx([1.02, 0.99], rel=1e-15)
    assert np.all(st["du_m1"] == acc["du"])
    assert np.all(st["h"] == 0.21)
    oracle.update(st, acc, np.array([100, 100], dtype=np.int32), 0.02, 0.01, False, b0, b1, P)
    assert st["u"] == pytest.approx([1.06, 0.97], rel=1e-14)


def test_leapfrog_constant_acceleration():
    """Constant a with constant dt: v (stored at half steps) gains a dt per step and
    x_n = x_0 + n dt v_{-1/2} + a dt^2 n (n+1)/2 (kick-drift leapfrog)."""
    n = 1
    st = {k: np.zeros(n) for k in ("x", "y", "z", "vx", "vy", "vz", "du_m1")}
    st["h"] = np.full(n, 0.01)
    st["u"] = np.ones(n)
    acc = {"ax": np.full(n, 0.5), "ay": np.zeros(n), "az": np.zeros(n), "du": np.zeros(n)}
    P = StepParams(periodic=(0, 0, 0), box_min=(-10, -10, -10), box_max=(10, 10, 10))
    dt = 0.125
    for k in range(1, 9):
        oracle.update(st, acc, np.array([100], dtype=np.int32), dt, dt, k == 1,
                      np.array(P.box_min), np.array(P.box_max), P)
        assert st["vx"][0] == pytest.approx(0.5 * dt * k, rel=1e-15)
        assert st["x"][0] == pytest.approx(0.5 * dt * dt * k * (k + 1) / 2, rel=1e-14)


# ----------------------------------------------------------------- variable h
def _mutual_lattice(nside=10, seed=31):
    """Perfect periodic lattice (a = 1/nside) with h jittered by +-1% around the
    ng0 = 100 value (2h/a = 2.87941), random u (ideal gas) and random v.  Then
    2h/a lies in [2.85, 2.91]: above the sqrt(8) shell and below the next one at
    3, so every particle has the same 92 neighbours at the same lattice offsets
    whatever its h -- every neighbour relation is mutual while h_i != h_j.  The
    exact pair antisymmetry of SURVEY 8(c) step 8 (A_ij = -B_ji, G_ij = -G_ji,
    Pi_ij = Pi_ji) then holds with VARIABLE h, which is what pins the j-side
    W(r, h_j), B = C_j Delta w_j and the symmetric means h-bar, c-bar, rho-bar."""
    w = ics.sedov(nside)
    s = w.state
    rng = np.random.default_rng(seed)
    n = s["x"].size
    s["h"] = s["h"] * (1.0 + rng.uniform(-0.01, 0.01, n))
    s["u"] = rng.uniform(0.5, 2.0, n)
    for k in ("vx", "vy", "vz"):
        s[k] = rng.uniform(-0.5, 0.5, n)
    w.params.eos = 0
    a = 1.0 / nside
    assert 2 * s["h"].min() / a > 2.85 > 8 ** 0.5 and 2 * s["h"].max() / a < 2.91 < 3.0
    return w


def test_mutual_lattice_is_mutual():
    w = _mutual_lattice()
    s, bmin, bmax, nb = _prep(w)
    assert np.all(nb.nc == 92)
    pairs = set()
    for i in range(s["x"].size):
        for j in nb.idx[nb.offsets[i]:nb.offsets[i + 1]]:
            pairs.add((i, int(j)))
    assert all((j, i) in pairs for (i, j) in pairs)
    assert np.ptp(s["h"]) > 0.01 * s["h"].mean()   # h really varies


def test_conservation_variable_h_mutual():
    """Variable h, every pair mutual: sum m a = 0 and sum m (v.a + du) = 0 to roundoff
    of the term scale.  Fails if the j-side kernel used h_i (w_j = W(r, h_i)), if B
    used C_i, or if a mean (h-bar, c-bar, rho-bar) were one-sided."""
    w = _mutual_lattice()
    s = w.state
    r = _chain(w)
    m = s["m"]
    scale = (m[:, None] * r["a_abs"]).sum(0)
    mom = np.array([(m * r["ax"]).sum(), (m * r["ay"]).sum(), (m * r["az"]).sum()])
    assert np.all(np.abs(mom) < 1e-14 * scale), mom / scale
    power = (m * (s["vx"] * r["ax"] + s["vy"] * r["ay"] + s["vz"] * r["az"] + r["du"])).sum()
    pscale = (m * (np.abs(s["vx"]) * r["a_abs"][:, 0] + np.abs(s["vy"]) * r["a_abs"][:, 1]
                   + np.abs(s["vz"]) * r["a_abs"][:, 2] + r["du_abs"])).sum()
    assert abs(power) < 1e-14 * pscale, power / pscale
    # the viscosity really acts (approaching pairs exist), so Pi is exercised
    assert np.abs(r["du"]).max() > 0


def _iad_gradient_error(w):
    s, bmin, bmax, nb = _prep(w)
    r = _chain(w)
    g = np.array([0.3, -1.7, 0.9])
    V = s["m"] / r["rho"]
    err = 0.0
    for i in range(s["x"].size):
        js = nb.idx[nb.offsets[i]:nb.offsets[i + 1]]
        D = np.stack([s["x"][js] - s["x"][i], s["y"][js] - s["y"][i], s["z"][js] - s["z"][i]], 1)
        D -= np.round(D)  # minimum image in the unit box
        # the gradient of f = g.x with the kernel of the TARGET's smoothing length
        Wv = np.array([oracle.W(np.linalg.norm(d), s["h"][i], K_SINC6) for d in D])
        c = r["C"][i]
        Cm = np.array([[c[0], c[1], c[2]], [c[1], c[3], c[4]], [c[2], c[4], c[5]]])
        grad = ((V[js] * Wv * (D @ g))[:, None] * (D @ Cm.T)).sum(0)
        err = max(err, np.abs(grad - g).max() / np.abs(g).max())
    return err


@pytest.mark.parametrize("kind", ["mutual_lattice", "jittered_varh"])
def test_iad_linear_exactness_variable_h(kind):
    """IAD linear exactness with variable h: C_i inverts tau_i built with W(r, h_i),
    so the gradient of a linear field taken with W(r, h_i) is exact.  A tau built
    with W(r, h_j) breaks it as soon as h varies (uniform-h sets cannot tell)."""
    if kind == "mutual_lattice":
        w = _mutual_lattice()
    else:
        w = ics.turbulence(10)
        rng = np.random.default_rng(5)
        w.state["h"] = w.state["h"] * (1.0 + rng.uniform(-0.1, 0.1, w.n))
    assert _iad_gradient_error(w) < 1e-13


def test_density_uses_own_h_only(golden):
    """Perfect 10^3 lattice at the ng0 = 100 h, one particle's h raised by 1%: every
    OTHER particle keeps the golden lattice density (its sum uses its own h_i, not
    the neighbour's), and the changed particle's density moves."""
    w = ics.sedov(10)
    s = w.state
    k = 437
    s["h"] = s["h"].copy()
    s["h"][k] *= 1.01
    r = _chain(w)
    others = np.arange(w.n) != k
    assert np.allclose(r["rho"][others], golden["lattice_rho"]["value"], rtol=1e-14, atol=0)
    assert abs(r["rho"][k] / golden["lattice_rho"]["value"] - 1) > 1e-6  # ~2e-5: a normalised estimate
