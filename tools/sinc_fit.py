"""Coefficients of the GPU's sinc polynomial (sph_internal.cuh: sinc_t).

S(t) = sin(sqrt t)/sqrt t on t in [0, pi^2] interpolated at the 11 Chebyshev
nodes by a degree-10 polynomial in t (40-digit mpmath), then the max abs error
of the fp64 Horner evaluation on a dense grid.  Prints coefficients, high degree
first.  (A design aid for the CUDA path; the oracle uses libm sin.)"""
import mpmath as mp
import numpy as np

mp.mp.dps = 40
T = mp.pi ** 2


def S(t):
    t = mp.mpf(t)
    if t == 0:
        return mp.mpf(1)
    r = mp.sqrt(t)
    return mp.sin(r) / r


def Ct(t):
    """cos(sqrt t): the grad-h kernel derivative (k_physics.cu gradh_body)."""
    return mp.cos(mp.sqrt(mp.mpf(t)))


def fit(deg, f=S):
    N = deg + 1
    nodes = [T / 2 * (1 + mp.cos(mp.pi * (2 * k + 1) / (2 * N))) for k in range(N)]
    A = mp.matrix([[x ** p for p in range(N)] for x in nodes])
    c = mp.lu_solve(A, mp.matrix([f(x) for x in nodes]))
    return [float(c[p]) for p in range(N)]


def report(coef, f):
    err = 0.0
    for t in np.linspace(0, float(T), 20001):
        s = coef[-1]
        for p in range(len(coef) - 2, -1, -1):
            s = s * t + coef[p]
        err = max(err, abs(s - float(f(t))))
    for p in range(len(coef) - 1, -1, -1):
        print(p, repr(coef[p]))
    print("max abs error", err)


if __name__ == "__main__":
    print("sin(x)/x, x^2 = t:")
    report(fit(10), S)
    print("cos(x), x^2 = t:")
    report(fit(11, Ct), Ct)
