"""Pins for the oracle's kernel W and its scalar helpers (SURVEY 8(c) 'Pins': Kernel, AV, Morton).

Independent references: mpmath quadrature for the normalisation, scipy quadrature
of the oracle's W, closed forms, and golden values in tests/golden/pins.json."""
import math

import mpmath
import numpy as np
import pytest
from scipy import integrate

import oracle
from paper_conf_sc_simsekpc24_b200.ics import K_SINC6, StepParams

pytestmark = pytest.mark.filterwarnings("ignore::scipy.integrate.IntegrationWarning")


def test_K_is_the_exact_normalisation(golden):
    """K = 1/(4 pi int_0^2 S(pi v/2)^6 v^2 dv), evaluated here with mpmath at 30 digits."""
    mpmath.mp.dps = 30
    f = lambda v: (mpmath.sin(mpmath.pi * v / 2) / (mpmath.pi * v / 2)) ** 6 * v ** 2 if v != 0 else 0
    I = mpmath.quad(f, [0, 1, 2])
    K = 1 / (4 * mpmath.pi * I)
    assert abs(float(K) - golden["K_sinc6"]["value"]) < 1e-16
    assert abs(K_SINC6 - float(K)) < 1e-16
    # the SPHYNX fit is 1.29e-5 below (the alternative reading, not used)
    assert abs((float(K) - golden["K_sinc6_sphynx_fit"]["value"]) - 1.02e-5) < 1e-6


@pytest.mark.parametrize("h", [1.0, 0.37, 0.0071985])
def test_W_integrates_to_one(h):
    """int W d^3r = 4 pi int_0^{2h} r^2 W(r,h) dr = 1 (oracle's W under scipy quad)."""
    val, err = integrate.quad(lambda r: 4 * math.pi * r * r * oracle.W(r, h, K_SINC6), 0, 2 * h,
                              epsabs=1e-14, epsrel=1e-13, limit=200)
    assert abs(val - 1.0) < 1e-12


def test_W_micro_pins(golden):
    assert oracle.W(1.0, 1.0, K_SINC6) == pytest.approx(golden["W_1_1"]["value"], rel=2e-15)
    assert oracle.W(1.5, 1.0, K_SINC6) == pytest.approx(golden["W_1p5_1"]["value"], rel=2e-15)
    assert oracle.W(2.5, 1.0, K_SINC6) == golden["W_2p5_1"]["value"]


def test_W_closed_forms():
    h = 0.3
    # centre value K/h^3 and the closed form at r = h: K/h^3 (2/pi)^6
    assert oracle.W(0.0, h, K_SINC6) == pytest.approx(K_SINC6 / h ** 3, rel=1e-15)
    assert oracle.W(h, h, K_SINC6) == pytest.approx(K_SINC6 / h ** 3 * (2 / math.pi) ** 6, rel=1e-14)
    # support clamp: exactly zero at and beyond 2h although sinc has side lobes there
    assert oracle.W(2 * h, h, K_SINC6) == 0.0
    assert oracle.W(2.5 * h, h, K_SINC6) == 0.0
    assert math.sin(math.pi * 1.25) / (math.pi * 1.25) != 0.0
    # just inside the support the kernel vanishes like (2h - r)^6
    assert 0 < oracle.W(2 * h * (1 - 1e-3), h, K_SINC6) < 1e-15 / h ** 3
    # monotone decreasing on [0, 2h)
    r = np.linspace(0, 2 * h, 200, endpoint=False)
    w = np.array([oracle.W(v, h, K_SINC6) for v in r])
    assert np.all(np.diff(w) < 0)


def test_sinc():
    assert oracle.sinc(0.0) == 1.0
    for x in (1e-9, 0.3, 1.0, 2.5, math.pi):
        assert oracle.sinc(x) == pytest.approx(math.sin(x) / x, rel=1e-15, abs=1e-16)


def test_av_micro(golden):
    """d = x_i - x_j = -1, v_ij = +1 (approaching): rv = -1, mu = -1/1.01."""
    P = StepParams()
    rv, d2 = -1.0, 1.0
    mu = 1.0 * rv / (d2 + P.av_eps)
    assert mu == pytest.approx(golden["av_mu"]["value"], rel=1e-15)
    assert oracle.av_pi(rv, d2, 1.0, 1.0, 1.0, P) == pytest.approx(golden["av_pi"]["value"], rel=1e-15)
    # receding pairs and rv = 0 have no viscosity
    assert oracle.av_pi(+1.0, d2, 1.0, 1.0, 1.0, P) == 0.0
    assert oracle.av_pi(0.0, d2, 1.0, 1.0, 1.0, P) == 0.0
    # scaling: Pi is inversely proportional to rhobar
    assert oracle.av_pi(rv, d2, 1.0, 1.0, 2.0, P) == pytest.approx(golden["av_pi"]["value"] / 2, rel=1e-15)


def test_morton_micro(golden):
    for (ix, iy, iz), key in golden["morton"]["value"]:
        assert oracle.morton(ix, iy, iz) == key


def test_morton_is_bit_interleave():
    """Brute-force definition on random coordinates: bit b of ix lands at 3b+2, iy 3b+1, iz 3b."""
    rng = np.random.default_rng(5)
    for _ in range(200):
        ix, iy, iz = (int(v) for v in rng.integers(0, 2 ** 21, 3))
        s = "".join(f"{(ix >> b) & 1}{(iy >> b) & 1}{(iz >> b) & 1}" for b in range(20, -1, -1))
        assert oracle.morton(ix, iy, iz) == int(s, 2)
