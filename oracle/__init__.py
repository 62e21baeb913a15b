"""CPU oracle of one SPH step -- TEST INFRASTRUCTURE ONLY.

Only tests/, ``__graft_entry__.smoke()`` and bench.py's cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(paper_conf_sc_simsekpc24_b200, libsph) never does, and this package never
imports the product: the two meet only through the seeded input generators in
``paper_conf_sc_simsekpc24_b200.ics`` (inputs, no arithmetic of the method).

The arithmetic lives in ``oracle.c`` (plain C, fp64, -ffp-contract=off,
O(N^2) brute-force neighbours); this module is marshalling plus the step
composition in the order of SURVEY.md 8(c) "Algorithm, step by step" (box,
keys, sort, neighbours, density, EOS, IAD, momentum-energy, dt, update).

Parity unpinned (conventions only): Courant factor,
dt growth cap, dt_first, AV alpha/beta/eps, the h-update constants and the
first-step du_m1 := du.  Nothing in PAPER.md fixes them.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC", "-shared", "-std=c11"]


def build(force: bool = False) -> str:
    """Compile liboracle.so (gcc).  Part of __graft_entry__.build()."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", _LIB + ".tmp", "-lm"])
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


class _Params(C.Structure):
    _fields_ = [
        ("box_min", C.c_double * 3), ("box_max", C.c_double * 3), ("periodic", C.c_int32 * 3),
        ("eos", C.c_int32), ("gamma", C.c_double), ("cs0", C.c_double), ("K", C.c_double),
        ("ng0", C.c_double), ("k_cour", C.c_double), ("dt_max_growth", C.c_double),
        ("av_alpha", C.c_double), ("av_beta", C.c_double), ("av_eps", C.c_double),
        ("h_cap", C.c_double),
    ]


def params_struct(p) -> _Params:
    s = _Params()
    s.box_min[:] = list(p.box_min)
    s.box_max[:] = list(p.box_max)
    s.periodic[:] = [int(v) for v in p.periodic]
    for k in ("eos",):
        setattr(s, k, int(getattr(p, k)))
    for k in ("gamma", "cs0", "K", "ng0", "k_cour", "dt_max_growth", "av_alpha", "av_beta",
              "av_eps", "h_cap"):
        setattr(s, k, float(getattr(p, k)))
    return s


_lib = None
_D = C.POINTER(C.c_double)
_I64 = C.POINTER(C.c_int64)
_I32 = C.POINTER(C.c_int32)
_U64 = C.POINTER(C.c_uint64)


def _configure(L):
    if True:
        L.oracle_sinc.restype = C.c_double
        L.oracle_sinc.argtypes = [C.c_double]
        L.oracle_W.restype = C.c_double
        L.oracle_W.argtypes = [C.c_double, C.c_double, C.c_double]
        L.oracle_dWdh.restype = C.c_double
        L.oracle_dWdh.argtypes = [C.c_double, C.c_double, C.c_double]
        L.oracle_timestep_vsig.restype = C.c_double
        L.oracle_morton.restype = C.c_uint64
        L.oracle_morton.argtypes = [C.c_uint64] * 3
        L.oracle_av_pi.restype = C.c_double
        L.oracle_av_pi.argtypes = [C.c_double] * 5 + [C.POINTER(_Params)]
        L.oracle_timestep.restype = C.c_double
        L.oracle_ball.restype = C.c_int64
    return L


def lib():
    global _lib
    if _lib is None:
        _lib = _configure(C.CDLL(build()))
    return _lib


class use_library:
    """Context manager: run the oracle functions on another compiled copy of
    oracle.c (tests/test_oracle_mutants.py checks that deliberately broken copies
    fail the pins)."""

    def __init__(self, path: str):
        self.path = path

    def __enter__(self):
        global _lib
        self.prev = lib()
        _lib = _configure(C.CDLL(self.path))
        return _lib

    def __exit__(self, *exc):
        global _lib
        _lib = self.prev
        return False


def _p(a, t):
    return a.ctypes.data_as(t)


def _d(a):
    a = np.ascontiguousarray(a, dtype=np.float64)
    return a


# --------------------------------------------------------------------------
# Scalar helpers (pinned directly in tests/test_oracle_*.py)
# --------------------------------------------------------------------------
def sinc(x: float) -> float:
    return lib().oracle_sinc(float(x))


def W(r: float, h: float, K: float) -> float:
    return lib().oracle_W(float(r), float(h), float(K))


def dWdh(r: float, h: float, K: float) -> float:
    """dW/dh at fixed r (oracle.c oracle_dWdh, reading 21)."""
    return lib().oracle_dWdh(float(r), float(h), float(K))


def morton(ix: int, iy: int, iz: int) -> int:
    return int(lib().oracle_morton(ix, iy, iz))


def av_pi(rv, d2, hbar, cbar, rhobar, params) -> float:
    ps = params_struct(params)
    return lib().oracle_av_pi(rv, d2, hbar, cbar, rhobar, C.byref(ps))


# --------------------------------------------------------------------------
# Array steps
# --------------------------------------------------------------------------
def box(x, y, z, params):
    x, y, z = _d(x), _d(y), _d(z)
    bmin = np.zeros(3)
    bmax = np.zeros(3)
    ps = params_struct(params)
    rc = lib().oracle_box(C.c_int64(x.size), _p(x, _D), _p(y, _D), _p(z, _D), C.byref(ps),
                          _p(bmin, _D), _p(bmax, _D))
    if rc != 0:
        raise ValueError("degenerate open-axis box (max == min)")
    return bmin, bmax


def keys(x, y, z, bmin, bmax):
    x, y, z = _d(x), _d(y), _d(z)
    out = np.zeros(x.size, dtype=np.uint64)
    bmin, bmax = _d(bmin), _d(bmax)
    lib().oracle_keys(C.c_int64(x.size), _p(x, _D), _p(y, _D), _p(z, _D), _p(bmin, _D),
                      _p(bmax, _D), _p(out, _U64))
    return out


def sort_order(k):
    k = np.ascontiguousarray(k, dtype=np.uint64)
    perm = np.zeros(k.size, dtype=np.int64)
    lib().oracle_sort_order(C.c_int64(k.size), _p(k, _U64), _p(perm, _I64))
    return perm


@dataclass
class Neighbors:
    nc: np.ndarray        # int32 [n]
    offsets: np.ndarray   # int64 [n+1]
    idx: np.ndarray       # int64 [sum nc], ascending within each list


def neighbors(x, y, z, h, bmin, bmax, periodic) -> Neighbors:
    x, y, z, h = _d(x), _d(y), _d(z), _d(h)
    n = x.size
    bmin, bmax = _d(bmin), _d(bmax)
    per = np.ascontiguousarray(periodic, dtype=np.int32)
    nc = np.zeros(n, dtype=np.int32)
    L = lib()
    L.oracle_neighbor_counts(C.c_int64(n), _p(x, _D), _p(y, _D), _p(z, _D), _p(h, _D),
                             _p(bmin, _D), _p(bmax, _D), _p(per, _I32), _p(nc, _I32))
    off = np.zeros(n + 1, dtype=np.int64)
    off[1:] = np.cumsum(nc)
    idx = np.zeros(max(int(off[-1]), 1), dtype=np.int64)
    L.oracle_neighbor_lists(C.c_int64(n), _p(x, _D), _p(y, _D), _p(z, _D), _p(h, _D),
                            _p(bmin, _D), _p(bmax, _D), _p(per, _I32), _p(off, _I64),
                            _p(idx, _I64))
    return Neighbors(nc, off, idx[: int(off[-1])])


def ball(x, y, z, t, R, bmin, bmax, periodic):
    """Indices l (ascending) with minimum-image distance to particle t below R."""
    x, y, z = _d(x), _d(y), _d(z)
    per = np.ascontiguousarray(periodic, dtype=np.int32)
    bmin, bmax = _d(bmin), _d(bmax)
    cap = 1 << 16
    while True:
        out = np.zeros(cap, dtype=np.int64)
        c = lib().oracle_ball(C.c_int64(x.size), _p(x, _D), _p(y, _D), _p(z, _D), C.c_int64(t),
                              C.c_double(R), _p(bmin, _D), _p(bmax, _D), _p(per, _I32),
                              _p(out, _I64), C.c_int64(cap))
        if c <= cap:
            return out[:c]
        cap = int(c)


def density(x, y, z, h, m, bmin, bmax, periodic, nb: Neighbors, params):
    x, y, z, h, m = map(_d, (x, y, z, h, m))
    per = np.ascontiguousarray(periodic, dtype=np.int32)
    bmin, bmax = _d(bmin), _d(bmax)
    rho = np.zeros(x.size)
    ps = params_struct(params)
    idx = nb.idx if nb.idx.size else np.zeros(1, dtype=np.int64)
    lib().oracle_density(C.c_int64(x.size), _p(x, _D), _p(y, _D), _p(z, _D), _p(h, _D), _p(m, _D),
                         _p(bmin, _D), _p(bmax, _D), _p(per, _I32), _p(nb.offsets, _I64),
                         _p(idx, _I64), C.byref(ps), _p(rho, _D))
    return rho


def gradh(x, y, z, h, m, rho, bmin, bmax, periodic, nb: Neighbors, params):
    """NormalizationGradh (reading 21): returns (omega, dsum, dsum_abs) with
    dsum_i = sum_j m_j dW/dh(r_ij, h_i) (self term included)."""
    x, y, z, h, m, rho = map(_d, (x, y, z, h, m, rho))
    per = np.ascontiguousarray(periodic, dtype=np.int32)
    bmin, bmax = _d(bmin), _d(bmax)
    n = x.size
    om, ds, da = np.zeros(n), np.zeros(n), np.zeros(n)
    ps = params_struct(params)
    idx = nb.idx if nb.idx.size else np.zeros(1, dtype=np.int64)
    lib().oracle_gradh(C.c_int64(n), _p(x, _D), _p(y, _D), _p(z, _D), _p(h, _D), _p(m, _D),
                       _p(rho, _D), _p(bmin, _D), _p(bmax, _D), _p(per, _I32),
                       _p(nb.offsets, _I64), _p(idx, _I64), C.byref(ps), _p(om, _D), _p(ds, _D),
                       _p(da, _D))
    return om, ds, da


def eos(rho, u, params):
    rho, u = _d(rho), _d(u)
    p = np.zeros(rho.size)
    c = np.zeros(rho.size)
    ps = params_struct(params)
    lib().oracle_eos(C.c_int64(rho.size), _p(rho, _D), _p(u, _D), C.byref(ps), _p(p, _D),
                     _p(c, _D))
    return p, c


def iad(x, y, z, h, m, rho, bmin, bmax, periodic, nb: Neighbors, params):
    """Returns (C, tau, tau_abs, singular) with C, tau, tau_abs of shape [n, 6]."""
    x, y, z, h, m, rho = map(_d, (x, y, z, h, m, rho))
    per = np.ascontiguousarray(periodic, dtype=np.int32)
    bmin, bmax = _d(bmin), _d(bmax)
    n = x.size
    Cm = np.zeros((n, 6))
    tau = np.zeros((n, 6))
    tabs = np.zeros((n, 6))
    ps = params_struct(params)
    idx = nb.idx if nb.idx.size else np.zeros(1, dtype=np.int64)
    rc = lib().oracle_iad(C.c_int64(n), _p(x, _D), _p(y, _D), _p(z, _D), _p(h, _D), _p(m, _D),
                          _p(rho, _D), _p(bmin, _D), _p(bmax, _D), _p(per, _I32),
                          _p(nb.offsets, _I64), _p(idx, _I64), C.byref(ps), _p(Cm, _D),
                          _p(tau, _D), _p(tabs, _D))
    return Cm, tau, tabs, rc == 2


def divcurl(x, y, z, vx, vy, vz, h, m, rho, Cm, bmin, bmax, periodic, nb: Neighbors, params):
    """IAD velocity gradient T [n, 9] (T_ab = dv_b/dx_a), its scale T_abs, div v [n]
    and curl v [n, 3] (oracle.c oracle_divcurl)."""
    arrs = list(map(_d, (x, y, z, vx, vy, vz, h, m, rho)))
    Cm = np.ascontiguousarray(Cm, dtype=np.float64)
    per = np.ascontiguousarray(periodic, dtype=np.int32)
    bmin, bmax = _d(bmin), _d(bmax)
    n = arrs[0].size
    T, Tabs, curl = np.zeros((n, 9)), np.zeros((n, 9)), np.zeros((n, 3))
    dv = np.zeros(n)
    ps = params_struct(params)
    idx = nb.idx if nb.idx.size else np.zeros(1, dtype=np.int64)
    lib().oracle_divcurl(C.c_int64(n), *[_p(a, _D) for a in arrs], _p(Cm, _D), _p(bmin, _D),
                         _p(bmax, _D), _p(per, _I32), _p(nb.offsets, _I64), _p(idx, _I64),
                         C.byref(ps), _p(T, _D), _p(Tabs, _D), _p(dv, _D), _p(curl, _D))
    return T, Tabs, dv, curl


def balsara(divv, curl, c, h):
    """Balsara switch f = |div| / (|div| + |curl| + 1e-4 c/h)."""
    divv, c, h = _d(divv), _d(c), _d(h)
    curl = np.ascontiguousarray(curl, dtype=np.float64)
    f = np.zeros(divv.size)
    lib().oracle_balsara(C.c_int64(divv.size), _p(divv, _D), _p(curl, _D), _p(c, _D), _p(h, _D),
                         _p(f, _D))
    return f


def momentum_energy(x, y, z, vx, vy, vz, h, m, rho, p, c, Cm, bmin, bmax, periodic,
                    nb: Neighbors, params, fav=None, omega=None):
    """Returns dict(ax, ay, az, du, a_abs [n,3], du_abs).  ``fav``: per-particle AV
    switch factors (None = 1, the plain Monaghan viscosity).  ``omega``: grad-h
    factors (None = the plain p/rho^2, reading 21)."""
    arrs = list(map(_d, (x, y, z, vx, vy, vz, h, m, rho, p, c)))
    Cm = np.ascontiguousarray(Cm, dtype=np.float64)
    per = np.ascontiguousarray(periodic, dtype=np.int32)
    bmin, bmax = _d(bmin), _d(bmax)
    n = arrs[0].size
    ax, ay, az, du, dabs = (np.zeros(n) for _ in range(5))
    aabs = np.zeros((n, 3))
    ps = params_struct(params)
    idx = nb.idx if nb.idx.size else np.zeros(1, dtype=np.int64)
    fv = None if fav is None else _d(fav)
    ov = None if omega is None else _d(omega)
    lib().oracle_momentum_energy(C.c_int64(n), *[_p(a, _D) for a in arrs], _p(Cm, _D),
                                 _p(bmin, _D), _p(bmax, _D), _p(per, _I32), _p(nb.offsets, _I64),
                                 _p(idx, _I64), C.byref(ps), None if fv is None else _p(fv, _D),
                                 None if ov is None else _p(ov, _D),
                                 _p(ax, _D), _p(ay, _D), _p(az, _D),
                                 _p(du, _D), _p(aabs, _D), _p(dabs, _D))
    return {"ax": ax, "ay": ay, "az": az, "du": du, "a_abs": aabs, "du_abs": dabs}


def timestep(h, c, dt_prev, params) -> float:
    h, c = _d(h), _d(c)
    ps = params_struct(params)
    L = lib()
    L.oracle_timestep.argtypes = [C.c_int64, _D, _D, C.c_double, C.POINTER(_Params)]
    return float(L.oracle_timestep(C.c_int64(h.size), _p(h, _D), _p(c, _D), C.c_double(dt_prev),
                                   C.byref(ps)))


def timestep_vsig(x, y, z, vx, vy, vz, h, c, bmin, bmax, periodic, nb: Neighbors, dt_prev,
                  params):
    """Signal-velocity time step (reading 22).  Returns (dt, vsig [n])."""
    arrs = list(map(_d, (x, y, z, vx, vy, vz, h, c)))
    per = np.ascontiguousarray(periodic, dtype=np.int32)
    bmin, bmax = _d(bmin), _d(bmax)
    vs = np.zeros(arrs[0].size)
    ps = params_struct(params)
    idx = nb.idx if nb.idx.size else np.zeros(1, dtype=np.int64)
    dt = lib().oracle_timestep_vsig(C.c_int64(vs.size), *[_p(a, _D) for a in arrs], _p(bmin, _D),
                                    _p(bmax, _D), _p(per, _I32), _p(nb.offsets, _I64),
                                    _p(idx, _I64), C.c_double(dt_prev), C.byref(ps), _p(vs, _D))
    return float(dt), vs


def update(state, acc, nc, dt, dt_m1, first_step, bmin, bmax, params):
    """In-place update of state arrays (x, y, z, vx, vy, vz, h, u, du_m1)."""
    ps = params_struct(params)
    bmin, bmax = _d(bmin), _d(bmax)
    s = {k: state[k] for k in ("x", "y", "z", "vx", "vy", "vz", "h", "u", "du_m1")}
    for k in s:
        assert s[k].dtype == np.float64 and s[k].flags.c_contiguous
    nc = np.ascontiguousarray(nc, dtype=np.int32)
    a = [_d(acc[k]) for k in ("ax", "ay", "az", "du")]
    lib().oracle_update(C.c_int64(s["x"].size), *[_p(s[k], _D) for k in
                        ("x", "y", "z", "vx", "vy", "vz", "h", "u", "du_m1")],
                        *[_p(v, _D) for v in a], _p(nc, _I32), C.c_double(dt),
                        C.c_double(dt_m1), C.c_int(1 if first_step else 0), _p(bmin, _D),
                        _p(bmax, _D), C.byref(ps))


# --------------------------------------------------------------------------
# Whole step (in order)
# --------------------------------------------------------------------------
STATE_KEYS = ("x", "y", "z", "vx", "vy", "vz", "h", "m", "u", "du_m1", "id")


# --------------------------------------------------------------------------
# Turbulence driving (oracle.c "Turbulence driving")
STIR_NMODES = 61


def stir_modes() -> np.ndarray:
    n3 = np.zeros((STIR_NMODES, 3), np.int32)
    m = lib().oracle_stir_modes(_p(n3, _I32))
    return n3[:m]


def stir_ou(A, xi, dt: float, sigma: float, t_decay: float) -> np.ndarray:
    """A <- f A + sigma sqrt(1-f^2) xi, f = exp(-dt/t_decay) (returns a new array)."""
    A = np.array(A, dtype=np.float64, copy=True)
    xi = _d(xi)
    lib().oracle_stir_ou(C.c_int(A.shape[0]), _p(A, _D), _p(xi, _D), C.c_double(dt),
                         C.c_double(sigma), C.c_double(t_decay))
    return A


def stir_project(A, w, zeta: float, L) -> np.ndarray:
    """B = 2 w (zeta A_perp + (1-zeta) A_par), per mode and real/imaginary part."""
    n3 = stir_modes()
    A, w = _d(A), _d(w)
    B = np.zeros_like(A)
    Lv = _d(np.asarray(L, dtype=np.float64))
    lib().oracle_stir_project(C.c_int(A.shape[0]), _p(n3, _I32), _p(Lv, _D), _p(A, _D), _p(w, _D),
                              C.c_double(zeta), _p(B, _D))
    return B


def stir_accel(x, y, z, lo, L, B):
    """sum_m Re(B_m exp(i k_m.(x - lo))) per particle -> (ax, ay, az)."""
    n3 = stir_modes()
    x, y, z, B = _d(x), _d(y), _d(z), _d(B)
    lo, L = _d(np.asarray(lo, np.float64)), _d(np.asarray(L, np.float64))
    ax, ay, az = (np.zeros(x.size) for _ in range(3))
    lib().oracle_stir_accel(C.c_int64(x.size), _p(x, _D), _p(y, _D), _p(z, _D), _p(lo, _D), _p(L, _D),
                            C.c_int(B.shape[0]), _p(n3, _I32), _p(B, _D), _p(ax, _D), _p(ay, _D),
                            _p(az, _D))
    return ax, ay, az


def stir_apply(stir: dict, x, y, z, dt_prev: float, bmin, bmax, acc: dict):
    """Phase STIR: advances stir["A"] with noise row stir["step"], adds the driving
    acceleration to acc["ax"/"ay"/"az"] in place; returns B."""
    xi = stir["noise"][stir["step"]]
    stir["A"] = stir_ou(stir["A"], xi, dt_prev, stir["sigma"], stir["t_decay"])
    L = [bmax[a] - bmin[a] for a in range(3)]
    B = stir_project(stir["A"], stir["w"], stir["zeta"], L)
    sx, sy, sz = stir_accel(x, y, z, bmin, L, B)
    # tolerance scale of the driven sums: sum_m |Re B| + |Im B| per component
    scale = np.abs(B).reshape(-1, 3, 2).sum(axis=(0, 2))
    acc["a_abs"] = acc["a_abs"] + scale[None, :]
    acc["ax"] = acc["ax"] + sx
    acc["ay"] = acc["ay"] + sy
    acc["az"] = acc["az"] + sz
    stir["step"] += 1
    return B


def gravity(x, y, z, m, G: float, eps: float):
    """Direct-sum softened gravity: dict(ax, ay, az, phi, a_abs [n, 3])."""
    x, y, z, m = map(_d, (x, y, z, m))
    n = x.size
    ax, ay, az, phi = (np.zeros(n) for _ in range(4))
    aabs = np.zeros((n, 3))
    lib().oracle_gravity(C.c_int64(n), _p(x, _D), _p(y, _D), _p(z, _D), _p(m, _D), C.c_double(G),
                         C.c_double(eps), _p(ax, _D), _p(ay, _D), _p(az, _D), _p(phi, _D),
                         _p(aabs, _D))
    return {"ax": ax, "ay": ay, "az": az, "phi": phi, "a_abs": aabs}


def _physics(st: dict, params, bmin, bmax, nb: Neighbors):
    """The neighbour sums of one step on a sorted particle set with its lists, in
    the order of SURVEY 8(c) steps 5-8 (+ the opt-in 8(f)-1 functions): density,
    [volume elements], [grad-h], EOS, IAD, [div/curl, Balsara switch],
    momentum-energy.  Returns every quantity by name."""
    rho = density(st["x"], st["y"], st["z"], st["h"], st["m"], bmin, bmax, params.periodic, nb,
                  params)
    omega = None
    out = {}
    if getattr(params, "ve", 0):
        # generalized volume elements (reading 23): X = m / rho0, the
        # normalisation kx = (K/h^3)[X_i + sum_j X_j S^6] (the density sum with X
        # in place of m), rho = kx m / X; grad-h with X and kx
        rho0 = rho
        X = st["m"] / rho0
        kx = density(st["x"], st["y"], st["z"], st["h"], X, bmin, bmax, params.periodic, nb, params)
        rho = kx * st["m"] / X
        out.update({"rho0": rho0, "X": X, "kx": kx})
        if getattr(params, "gradh", 0):
            omega, dWsum, dWabs = gradh(st["x"], st["y"], st["z"], st["h"], X, kx, bmin, bmax,
                                        params.periodic, nb, params)
    elif getattr(params, "gradh", 0):
        omega, dWsum, dWabs = gradh(st["x"], st["y"], st["z"], st["h"], st["m"], rho, bmin, bmax,
                                    params.periodic, nb, params)
    if omega is not None:
        out.update({"omega": omega, "dWdh_sum": dWsum, "dWdh_abs": dWabs})
    p, c = eos(rho, st["u"], params)
    Cm, tau, tabs, singular = iad(st["x"], st["y"], st["z"], st["h"], st["m"], rho, bmin, bmax,
                                  params.periodic, nb, params)
    if singular:
        raise ArithmeticError("IAD matrix singular")
    fav = None
    if getattr(params, "divcurl", 0) or getattr(params, "av_switch", 0):
        T, Tabs, dvv, curl = divcurl(st["x"], st["y"], st["z"], st["vx"], st["vy"], st["vz"],
                                     st["h"], st["m"], rho, Cm, bmin, bmax, params.periodic, nb,
                                     params)
        out.update({"T": T, "T_abs": Tabs, "divv": dvv, "curl": curl})
        if getattr(params, "av_switch", 0):
            fav = balsara(dvv, curl, c, st["h"])
            out["bal"] = fav
    acc = momentum_energy(st["x"], st["y"], st["z"], st["vx"], st["vy"], st["vz"], st["h"],
                          st["m"], rho, p, c, Cm, bmin, bmax, params.periodic, nb, params, fav,
                          omega)
    out.update({"rho": rho, "p": p, "c": c, "C": Cm, "tau": tau, "tau_abs": tabs, **acc})
    return out


def step(state: dict, params, dt_prev: float, first_step: bool, ngmax: int | None = None,
         stir: dict | None = None):
    """One full oracle step.  Returns (new_state, out) where new_state is in this
    step's sorted (Morton) order after the update, and ``out`` holds every
    intermediate of the step in the same order (keys, perm, nb, rho, p, c, C,
    accelerations, dt, box).  ``stir`` (optional, updated in place): driving state
    {A, w, noise, step, sigma, t_decay, zeta}; STIR runs after momentum-energy."""
    bmin, bmax = box(state["x"], state["y"], state["z"], params)
    k = keys(state["x"], state["y"], state["z"], bmin, bmax)
    perm = sort_order(k)
    st = {f: np.ascontiguousarray(state[f][perm]) for f in STATE_KEYS}
    ks = k[perm]
    nb = neighbors(st["x"], st["y"], st["z"], st["h"], bmin, bmax, params.periodic)
    if ngmax is not None and nb.nc.size and int(nb.nc.max()) > ngmax:
        raise OverflowError(f"neighbour count {int(nb.nc.max())} exceeds capacity {ngmax}")
    acc = _physics(st, params, bmin, bmax, nb)
    c = acc["c"]
    if getattr(params, "gravity", 0):
        gr = gravity(st["x"], st["y"], st["z"], st["m"], params.grav_G, params.grav_eps)
        for k in ("ax", "ay", "az"):
            acc[k] = acc[k] + gr[k]
        acc["a_abs"] = acc["a_abs"] + gr["a_abs"]
        acc["phi"] = gr["phi"]
    if stir is not None:
        acc["stir_B"] = stir_apply(stir, st["x"], st["y"], st["z"], dt_prev, bmin, bmax, acc)
    if getattr(params, "dt_vsig", 0):
        dt, acc["vsig"] = timestep_vsig(st["x"], st["y"], st["z"], st["vx"], st["vy"], st["vz"],
                                        st["h"], c, bmin, bmax, params.periodic, nb, dt_prev, params)
    else:
        dt = timestep(st["h"], c, dt_prev, params)
    out = {"bmin": bmin, "bmax": bmax, "keys": ks, "perm": perm, "nb": nb, "dt": dt,
           "pre": {f: st[f].copy() for f in STATE_KEYS}, **acc}
    update(st, acc, nb.nc, dt, dt_prev, first_step, bmin, bmax, params)
    return st, out


def sample_step(state: dict, params, dt_prev: float, first_step: bool, targets, margin=1e-6,
                dt: float | None = None):
    """One step evaluated at a few sampled particles of a large input.

    The full-size parts that are cheap stay exact and global: box, keys, stable
    sort (O(N log N)) and dt (O(N), needs only c(u) -- exact for both EOS).  The
    neighbour sums at a target t depend on particles a few kernel radii away:
    a_t needs C_j, Omega_j, f_j (j in N(t)); C_j needs rho_k (k in N(j)); rho_k
    needs the positions in N(k) -- three radii.  With volume elements rho_k needs
    X_l = m_l/rho0_l (l in N(k)), so four.  Every value at t is therefore a
    function of the particles within R = 2 h_t + 2 max h (ball 1) + 2 max h (ball
    2) [+ ...] of t only (the radius grown hop by hop, so a few large smoothing
    lengths far away do not inflate every ball).  We take that
    ball S (ascending order, so the summation order is unchanged), run the same
    plain functions (``_physics``) on S, and keep the values at t.  This is the
    same definition restricted to a set that provably contains t's whole
    dependency cone -- no approximation.

    The signal-velocity time step (cfg.dt_vsig) is a global minimum over every
    particle's neighbour list, which the sampled mode cannot form: there the
    caller passes ``dt`` (the GPU's) for the update, and ``out["vsig"]`` gives
    the exact v_sig of each target (the test checks dt against them).

    ``targets`` are positions in this step's sorted order.  Returns (order, out)
    with ``order`` = sorted ids (full) and ``out[name][k]`` the value at targets[k].
    """
    if getattr(params, "gravity", 0):
        raise NotImplementedError("sample_step: gravity is long-range (no finite dependency ball)")
    vsig_mode = bool(getattr(params, "dt_vsig", 0))
    if vsig_mode and dt is None:
        raise ValueError("sample_step with dt_vsig needs the caller's dt (global minimum)")
    bmin, bmax = box(state["x"], state["y"], state["z"], params)
    k = keys(state["x"], state["y"], state["z"], bmin, bmax)
    perm = sort_order(k)
    st = {f: np.ascontiguousarray(state[f][perm]) for f in STATE_KEYS}
    if not vsig_mode:
        p_all, c_all = eos(np.ones(st["x"].size), st["u"], params)  # c does not depend on rho
        dt = timestep(st["h"], c_all, dt_prev, params)
    hops = 4 if getattr(params, "ve", 0) else 3
    names = ["nc", "rho", "p", "c", "ax", "ay", "az", "du", "du_abs", "x", "y", "z", "vx", "vy",
             "vz", "u", "h"]
    extra = [nm for nm, on in (("omega", getattr(params, "gradh", 0)),
                               ("kx", getattr(params, "ve", 0)),
                               ("divv", getattr(params, "divcurl", 0) or getattr(params, "av_switch", 0)),
                               ("bal", getattr(params, "av_switch", 0)),
                               ("vsig", vsig_mode)) if on]
    out = {nm: np.zeros(len(targets)) for nm in names + extra}
    out["C"] = np.zeros((len(targets), 6))
    out["a_abs"] = np.zeros((len(targets), 3))
    out["nbrs"] = []
    out["ball_sizes"] = []
    for q, t in enumerate(targets):
        # dependency radius, hop by hop: N(t) lies within 2 h_t; the lists of the
        # particles within R lie within R + 2 max h of them (max over that ball)
        R = 2.0 * float(st["h"][t]) * (1.0 + margin)
        for _ in range(hops - 1):
            S = ball(st["x"], st["y"], st["z"], int(t), R, bmin, bmax, params.periodic)
            R = (R + 2.0 * float(st["h"][S].max())) * (1.0 + margin)
        S = ball(st["x"], st["y"], st["z"], int(t), R, bmin, bmax, params.periodic)
        sub = {f: np.ascontiguousarray(st[f][S]) for f in STATE_KEYS}
        loc = int(np.searchsorted(S, t))
        nb = neighbors(sub["x"], sub["y"], sub["z"], sub["h"], bmin, bmax, params.periodic)
        acc = _physics(sub, params, bmin, bmax, nb)
        if vsig_mode:
            _, vs = timestep_vsig(sub["x"], sub["y"], sub["z"], sub["vx"], sub["vy"], sub["vz"],
                                  sub["h"], acc["c"], bmin, bmax, params.periodic, nb, dt_prev,
                                  params)
            out["vsig"][q] = vs[loc]
        one = {f: np.ascontiguousarray(sub[f][loc:loc + 1]) for f in STATE_KEYS}
        acc1 = {kk: acc[kk][loc:loc + 1] for kk in ("ax", "ay", "az", "du")}
        nc1 = nb.nc[loc:loc + 1].copy()
        out["nbrs"].append(S[nb.idx[nb.offsets[loc]:nb.offsets[loc + 1]]])
        out["ball_sizes"].append(S.size)
        if "dWdh_abs" in acc:
            out.setdefault("dWdh_abs", np.zeros(len(targets)))[q] = acc["dWdh_abs"][loc]
        out["nc"][q] = nc1[0]
        for kk in ("rho", "p", "c", "ax", "ay", "az", "du", "du_abs"):
            out[kk][q] = acc[kk][loc]
        for kk in extra:
            if kk != "vsig":
                out[kk][q] = acc[kk][loc]
        out["C"][q] = acc["C"][loc]
        out["a_abs"][q] = acc["a_abs"][loc]
        update(one, acc1, nc1, dt, dt_prev, first_step, bmin, bmax, params)
        for f in ("x", "y", "z", "vx", "vy", "vz", "u", "h"):
            out[f][q] = one[f][0]
    return st["id"], {"dt": dt, "bmin": bmin, "bmax": bmax, "keys": k[perm], **out}
