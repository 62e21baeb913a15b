"""Pins of the oracle's turbulence driving (oracle.c "Turbulence
driving", reading 17) against things other than itself: a brute-force
enumeration of the mode set, the closed-form OU decay and its exact stationary
variance, the Helmholtz projection identities, and numpy's FFT of the driving
field sampled on a grid (which must return exactly the mode coefficients)."""
import itertools

import numpy as np

import oracle


def test_mode_set_is_the_half_space_shell():
    n3 = oracle.stir_modes()
    allv = [v for v in itertools.product(range(-3, 4), repeat=3) if 1 <= sum(c * c for c in v) <= 9]
    assert len(allv) == 122                       # 123 lattice points with |n| <= 3, minus 0
    got = {tuple(int(c) for c in v) for v in n3}
    assert len(got) == 61 == n3.shape[0]
    for v in allv:                                # exactly one of each +-n pair
        assert (v in got) != (tuple(-c for c in v) in got)
    assert [tuple(v) for v in n3] == sorted(got)  # lexicographic order


def test_ou_decay_closed_form_and_identity():
    rng = np.random.default_rng(5)
    A0 = rng.normal(size=(61, 6))
    A = A0.copy()
    dt, T = 0.013, 0.5
    for _ in range(7):
        A = oracle.stir_ou(A, np.zeros((61, 6)), dt, sigma=2.0, t_decay=T)
    np.testing.assert_allclose(A, A0 * np.exp(-7 * dt / T), rtol=1e-14)
    # dt = 0: f = 1, no noise enters
    B = oracle.stir_ou(A0, rng.normal(size=(61, 6)), 0.0, sigma=2.0, t_decay=T)
    assert np.array_equal(B, A0)


def test_ou_variance_is_exact_in_expectation():
    # From A = 0, Var(A_k) = sigma^2 (1 - f^(2k)); 120k independent chains.
    rng = np.random.default_rng(7)
    sigma, dt, T, k = 1.7, 0.1, 0.3, 5
    A = np.zeros((20000, 6))
    for _ in range(k):
        A = oracle.stir_ou(A, rng.normal(size=A.shape), dt, sigma, T)
    want = sigma ** 2 * (1.0 - np.exp(-2.0 * k * dt / T))
    assert abs(A.var() / want - 1.0) < 0.02


def _khat(L):
    k = 2 * np.pi * oracle.stir_modes() / np.asarray(L)[None, :]
    return k / np.linalg.norm(k, axis=1)[:, None]


def test_projection_identities():
    rng = np.random.default_rng(9)
    A = rng.normal(size=(61, 6))
    w = rng.uniform(0.2, 1.0, 61)
    L = [1.0, 1.3, 0.7]
    u = _khat(L)
    for zeta, check in ((1.0, "perp"), (0.0, "par")):
        B = oracle.stir_project(A, w, zeta, L).reshape(61, 3, 2)
        for part in range(2):
            v = B[:, :, part]
            if check == "perp":   # solenoidal: k . B = 0
                assert np.abs((u * v).sum(1)).max() < 1e-14 * np.abs(v).max()
            else:                 # compressive: B parallel to k
                assert np.abs(np.cross(u, v)).max() < 1e-14 * np.abs(v).max()
    # zeta = 1/2: (P_perp + P_par)/2 = I/2, so B = 2 w A / 2 = w A
    np.testing.assert_allclose(oracle.stir_project(A, w, 0.5, L), w[:, None] * A, rtol=1e-14, atol=1e-15)


def test_acceleration_field_fft_returns_the_mode_coefficients():
    N = 16
    lo = np.array([-0.5, -0.5, -0.5])
    L = np.array([1.0, 1.0, 1.0])
    rng = np.random.default_rng(11)
    B = rng.normal(size=(61, 6))
    g = (np.arange(N) / N)
    X, Y, Z = np.meshgrid(lo[0] + L[0] * g, lo[1] + L[1] * g, lo[2] + L[2] * g, indexing="ij")
    ax, ay, az = oracle.stir_accel(X.ravel(), Y.ravel(), Z.ravel(), lo, L, B)
    n3 = oracle.stir_modes()
    for c, a in enumerate((ax, ay, az)):
        F = np.fft.fftn(a.reshape(N, N, N)) / N ** 3
        want = np.zeros((N, N, N), complex)
        for m, (nx, ny, nz) in enumerate(n3):
            b = B[m, 2 * c] + 1j * B[m, 2 * c + 1]
            want[nx % N, ny % N, nz % N] += b / 2
            want[-nx % N, -ny % N, -nz % N] += np.conj(b) / 2
        assert np.abs(F - want).max() < 1e-13 * np.abs(B).max()


def test_solenoidal_field_is_divergence_free_spectrally():
    N = 16
    lo, L = np.zeros(3) - 0.5, np.ones(3)
    rng = np.random.default_rng(12)
    B = oracle.stir_project(rng.normal(size=(61, 6)), np.ones(61), 1.0, L)
    g = np.arange(N) / N - 0.5
    X, Y, Z = np.meshgrid(g, g, g, indexing="ij")
    a = oracle.stir_accel(X.ravel(), Y.ravel(), Z.ravel(), lo, L, B)
    F = [np.fft.fftn(c.reshape(N, N, N)) for c in a]
    k = np.fft.fftfreq(N, 1.0 / N)
    KX, KY, KZ = np.meshgrid(k, k, k, indexing="ij")
    div = KX * F[0] + KY * F[1] + KZ * F[2]
    assert np.abs(div).max() < 1e-10 * max(np.abs(f).max() for f in F)
