"""Seeded synthetic initial conditions and workload presets.

This module is the ONE piece shared by the CUDA path and the CPU oracle
("Inputs").  It draws positions, velocities, energies and
smoothing lengths and states the step parameters; it holds none of the SPH
step's arithmetic (no kernel, neighbour, density, force or update code).

Workloads (BASELINE.json configs; recipes in SURVEY.md 8(d) "Configs as
concrete synthetic inputs"):

* ``sedov(nside)``       Sedov blast: periodic unit cube, cell-centred lattice,
                          Gaussian energy spike (configs[0], configs[1]).
* ``turbulence(nside)``  Subsonic turbulence: jittered lattice, isothermal,
                          seeded solenoidal velocity field with v_rms = 0.3
                          (configs[2], configs[4]; the paper's workload, P:108,
                          Table I).
* ``noh(nside)``         Noh implosion: open box, v = -r_hat (configs[3]).

The paper prints no SPH constants; the parameter values here are the readings
of SURVEY.md 8(c) "Parameter table" and are listed in DESIGN.md section 3.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field, asdict

import numpy as np

# Exact normalisation of the n = 6 sinc kernel, 1/(4 pi int_0^2 S(pi v/2)^6 v^2 dv)
# (SURVEY 8(c) parameter table; pinned by quadrature in tests/test_oracle_kernel.py).
K_SINC6 = 0.79044958943230290

FIELDS = ("x", "y", "z", "vx", "vy", "vz", "h", "m", "u", "du_m1")


@dataclass
class StepParams:
    """Step parameters shared by both sides as *inputs* (sph_config / oracle_params)."""

    box_min: tuple = (-0.5, -0.5, -0.5)
    box_max: tuple = (0.5, 0.5, 0.5)
    periodic: tuple = (1, 1, 1)
    eos: int = 0            # 0 ideal gas, 1 isothermal
    gamma: float = 5.0 / 3.0
    cs0: float = 1.0
    K: float = K_SINC6
    ng0: float = 100.0
    ngmax: int = 150        # neighbour-list capacity (never a truncation)
    k_cour: float = 0.2
    dt_max_growth: float = 1.1
    dt_first: float = 1e-6
    av_alpha: float = 1.0
    av_beta: float = 2.0
    av_eps: float = 0.01
    h_cap: float = 0.25
    divcurl: int = 0        # 1: IADVelocityDivCurl also computes div v, curl v
    av_switch: int = 0      # 1: Balsara switch on the AV (implies divcurl)
    gravity: int = 0        # 1: self-gravity (GRAVITY phase, open boxes)
    grav_G: float = 1.0
    grav_eps: float = 0.01  # Plummer softening length
    grav_theta: float = 0.5  # tree opening angle (0 = direct summation)
    grav_level: int = 6     # leaf level of the gravity octree
    grav_fp64: int = 0      # 1: fp64 multipole / direct terms also for theta > 0
    gradh: int = 0          # 1: NormalizationGradh, p/(Omega rho^2) in momentum (reading 21)
    dt_vsig: int = 0        # 1: signal-velocity time step (reading 22)
    ve: int = 0             # 1: generalized volume elements X = m/rho0 (reading 23)

    def as_dict(self):
        return asdict(self)


@dataclass
class Workload:
    name: str
    state: dict             # numpy arrays: FIELDS + "id" (int64)
    params: StepParams
    meta: dict = field(default_factory=dict)

    @property
    def n(self) -> int:
        return int(self.state["x"].shape[0])


def _lattice(nside: int):
    """Cell-centred lattice x = -0.5 + (i + 1/2)/nside, ids in generation order."""
    a = 1.0 / nside
    g = -0.5 + (np.arange(nside, dtype=np.float64) + 0.5) * a
    X, Y, Z = np.meshgrid(g, g, g, indexing="ij")
    return X.ravel().copy(), Y.ravel().copy(), Z.ravel().copy(), a


def h_initial(n: int, ng0: float, volume: float = 1.0) -> float:
    """h0 = 1/2 (3 ng0 V / (4 pi N))^(1/3): a 2h sphere holds ng0 particles on average."""
    return 0.5 * (3.0 * ng0 * volume / (4.0 * math.pi * n)) ** (1.0 / 3.0)


def _state(x, y, z, vx, vy, vz, h, m, u):
    n = x.shape[0]
    return {
        "x": x, "y": y, "z": z, "vx": vx, "vy": vy, "vz": vz,
        "h": np.full(n, h) if np.isscalar(h) else h,
        "m": np.full(n, m) if np.isscalar(m) else m,
        "u": u, "du_m1": np.zeros(n), "id": np.arange(n, dtype=np.int64),
    }


def sedov(nside: int, energy: float = 1.0, width: float = 0.1, u_floor: float = 1e-8) -> Workload:
    """Sedov blast on a periodic cell-centred lattice.

    u = E/(pi^(3/2) w^3) exp(-r^2/w^2) + u_floor, m = 1/N (rho0 = 1), v = 0.
    """
    x, y, z, a = _lattice(nside)
    n = x.shape[0]
    r2 = x * x + y * y + z * z
    u = energy / (math.pi ** 1.5 * width ** 3) * np.exp(-r2 / width ** 2) + u_floor
    zeros = np.zeros(n)
    p = StepParams(eos=0, gamma=5.0 / 3.0, dt_first=1e-6, h_cap=0.25)
    st = _state(x, y, z, zeros.copy(), zeros.copy(), zeros.copy(), h_initial(n, p.ng0), 1.0 / n, u)
    return Workload(f"sedov{nside}", st, p, {"nside": nside, "lattice_a": a})


def noh(nside: int, u0: float = 1e-20) -> Workload:
    """Noh implosion: open box, lattice, v = -r_hat, rho0 = 1."""
    x, y, z, a = _lattice(nside)
    n = x.shape[0]
    r = np.sqrt(x * x + y * y + z * z)
    inv = np.where(r > 0, 1.0 / np.where(r > 0, r, 1.0), 0.0)
    p = StepParams(periodic=(0, 0, 0), eos=0, gamma=5.0 / 3.0, dt_first=1e-4, h_cap=1e300)
    st = _state(x, y, z, -x * inv, -y * inv, -z * inv, h_initial(n, p.ng0), 1.0 / n, np.full(n, u0))
    return Workload(f"noh{nside}", st, p, {"nside": nside, "lattice_a": a})


def evrard(nside: int, radius: float = 1.0, mass: float = 1.0, u_frac: float = 0.05,
           eps: float = 0.01) -> Workload:
    """Evrard collapse (the paper's gravity workload):
    a gas sphere of radius R and mass M with rho = M / (2 pi R^2 r), at rest,
    u = 0.05 G M / R, gamma 5/3, open box.  Particles: the lattice points of the
    unit sphere (nside per diameter), stretched radially r = R r_u^(3/2) so that
    M(<r) = M (r/R)^2; h from the local density (ng0 neighbours)."""
    x, y, z, a = _lattice(nside)
    x, y, z = 2 * x, 2 * y, 2 * z                       # lattice on [-1, 1]^3
    ru = np.sqrt(x * x + y * y + z * z)
    keep = ru < 1.0
    x, y, z, ru = x[keep], y[keep], z[keep], ru[keep]
    s = radius * np.sqrt(ru)                            # r / r_u = R r_u^(1/2)
    x, y, z = x * s, y * s, z * s
    r = ru * s
    n = x.size
    m = mass / n
    rho = mass / (2.0 * math.pi * radius ** 2 * np.maximum(r, 1e-3 * radius))
    # octree leaf level: ~4 particles per leaf on average (measured best)
    level = int(min(8, max(3, round(math.log(max(n, 8) / 4.0, 8)))))
    p = StepParams(box_min=(-1.0, -1.0, -1.0), box_max=(1.0, 1.0, 1.0), periodic=(0, 0, 0), eos=0,
                   gamma=5.0 / 3.0, dt_first=1e-4, h_cap=1e300, gravity=1, grav_eps=eps,
                   grav_level=level)
    h = 0.5 * (3.0 * p.ng0 * m / (4.0 * math.pi * rho)) ** (1.0 / 3.0)
    u = np.full(n, u_frac * p.grav_G * mass / radius)
    zeros = np.zeros(n)
    st = _state(x, y, z, zeros.copy(), zeros.copy(), zeros.copy(), h, m, u)
    return Workload(f"evrard{nside}", st, p, {"nside": nside, "n": n})


def _solenoidal_modes(seed: int, nmax: float = 3.0):
    """The 61 wave-vector pairs 1 <= |n| <= 3 (one of each +-n), random amplitude
    vectors projected perpendicular to n with |n|^-2 weights, random phases."""
    rng = np.random.default_rng(seed)
    ns = []
    r = int(math.floor(nmax))
    for i in range(-r, r + 1):
        for j in range(-r, r + 1):
            for k in range(-r, r + 1):
                q = i * i + j * j + k * k
                if q == 0 or q > nmax * nmax:
                    continue
                if i > 0 or (i == 0 and j > 0) or (i == 0 and j == 0 and k > 0):
                    ns.append((i, j, k))
    ns = np.array(ns, dtype=np.float64)
    amps = rng.standard_normal((len(ns), 3))
    nhat = ns / np.linalg.norm(ns, axis=1, keepdims=True)
    amps -= (amps * nhat).sum(axis=1, keepdims=True) * nhat
    amps *= (np.linalg.norm(ns, axis=1) ** -2.0)[:, None]
    phases = rng.uniform(0.0, 2.0 * math.pi, len(ns))
    return ns, amps, phases


def turbulence(nside: int, v_rms: float = 0.3, jitter: float = 0.25, seed_pos: int = 1,
               seed_vel: int = 2, chunk: int = 1 << 19) -> Workload:
    """Subsonic turbulence: periodic unit cube, lattice with
    uniform jitter +-jitter*a (seed 1), isothermal c0 = 1, seeded solenoidal field
    (seed 2) scaled to mass-weighted v_rms."""
    x, y, z, a = _lattice(nside)
    n = x.shape[0]
    rng = np.random.default_rng(seed_pos)
    for c in (x, y, z):
        c += rng.uniform(-jitter * a, jitter * a, n)
    ns, amps, phases = _solenoidal_modes(seed_vel)
    v = np.zeros((3, n))
    k = 2.0 * math.pi * ns
    for s in range(0, n, chunk):
        e = min(n, s + chunk)
        arg = np.outer(k[:, 0], x[s:e]) + np.outer(k[:, 1], y[s:e]) + np.outer(k[:, 2], z[s:e])
        arg += phases[:, None]
        cs = np.cos(arg)
        v[:, s:e] = amps.T @ cs
    rms = math.sqrt(float((v * v).sum(axis=0).mean()))
    v *= v_rms / rms
    p = StepParams(eos=1, cs0=1.0, dt_first=1e-4, h_cap=0.25)
    st = _state(x, y, z, v[0].copy(), v[1].copy(), v[2].copy(), h_initial(n, p.ng0), 1.0 / n,
                np.full(n, 1.5))
    return Workload(f"turbulence{nside}", st, p, {"nside": nside, "lattice_a": a})


def turbulence_part(nside: int, rank: int, world: int, v_rms: float = 0.3, jitter: float = 0.25,
                    seed_pos: int = 1, seed_vel: int = 2, chunk: int = 1 << 19) -> Workload:
    """Particles [rank N/world, (rank+1) N/world) of ``turbulence(nside)``, drawn
    without generating the rest (multi-GPU runs): the jitter stream is advanced
    to the slice (PCG64 draws one 64-bit word per double) and the velocity field
    is a function of position.  The velocities come back unnormalised: the
    scale to v_rms needs the mean square over ALL particles, so every rank
    reports its slice's sum (meta["vsq_sum"]), the caller all-reduces it and
    applies ``normalise_velocity``.  Positions and ids equal the full
    generator's; velocities agree to rounding of the normalisation."""
    n = nside ** 3
    lo, hi = rank * n // world, (rank + 1) * n // world
    a = 1.0 / nside
    idx = np.arange(lo, hi, dtype=np.int64)
    g = -0.5 + (np.arange(nside, dtype=np.float64) + 0.5) * a
    ix, iy, iz = idx // (nside * nside), (idx // nside) % nside, idx % nside
    pos = [g[ix].copy(), g[iy].copy(), g[iz].copy()]
    for axis in range(3):
        bg = np.random.PCG64(seed_pos)
        bg.advance(axis * n + lo)
        pos[axis] += np.random.Generator(bg).uniform(-jitter * a, jitter * a, hi - lo)
    ns, amps, phases = _solenoidal_modes(seed_vel)
    k = 2.0 * math.pi * ns

    def field(xx, yy, zz):
        arg = np.outer(k[:, 0], xx) + np.outer(k[:, 1], yy) + np.outer(k[:, 2], zz)
        arg += phases[:, None]
        return amps.T @ np.cos(arg)

    v = np.zeros((3, hi - lo))
    for s in range(0, hi - lo, chunk):
        e = min(hi - lo, s + chunk)
        v[:, s:e] = field(pos[0][s:e], pos[1][s:e], pos[2][s:e])
    # the full generator normalises by the rms over ALL jittered particles; the
    # partial one needs that global number: every rank computes it from its own
    # slice, and the caller (decomposed run) combines them (`vrms_partial`).
    p = StepParams(eos=1, cs0=1.0, dt_first=1e-4, h_cap=0.25)
    st = _state(pos[0], pos[1], pos[2], v[0].copy(), v[1].copy(), v[2].copy(), h_initial(n, p.ng0),
                1.0 / n, np.full(hi - lo, 1.5))
    st["id"] = idx.copy()
    return Workload(f"turbulence{nside}[{rank}/{world}]", st, p,
                    {"nside": nside, "lattice_a": a, "vsq_sum": float((v * v).sum()), "n_total": n,
                     "v_rms": v_rms})


def normalise_velocity(w: Workload, vsq_sum_total: float):
    """Scale a ``turbulence_part`` slice with the global mean square velocity."""
    n = w.meta["n_total"]
    f = w.meta["v_rms"] / math.sqrt(vsq_sum_total / n)
    for k in ("vx", "vy", "vz"):
        w.state[k] = w.state[k] * f


def random_box(n: int, seed: int = 0, periodic: bool = True, h: float | None = None,
               v_scale: float = 0.1) -> Workload:
    """Uniform random particles (edge-case tests: ragged sizes, empty cells, ties)."""
    rng = np.random.default_rng(seed)
    x, y, z = (rng.uniform(-0.5, 0.5, n) for _ in range(3))
    vx, vy, vz = (rng.normal(0.0, v_scale, n) for _ in range(3))
    u = rng.uniform(0.5, 1.5, n)
    # Poisson positions: nc spreads far wider than on a lattice (max ~ 1.7 x mean)
    p = StepParams(periodic=(1, 1, 1) if periodic else (0, 0, 0), eos=0, dt_first=1e-4, ngmax=256,
                   h_cap=0.25 if periodic else 1e300)
    hh = h if h is not None else h_initial(n, p.ng0)
    hv = hh * rng.uniform(0.9, 1.1, n)
    if periodic:
        hv = np.minimum(hv, p.h_cap)
    st = _state(x, y, z, vx, vy, vz, hv, rng.uniform(0.5, 1.5, n) / n, u)
    return Workload(f"random{n}", st, p, {"seed": seed})


PRESETS = {
    "sedov16": lambda: sedov(16),
    "sedov100": lambda: sedov(100),
    "turbulence200": lambda: turbulence(200),
    "noh300": lambda: noh(300),
}


# ---------------------------------------------------------------------------
# Turbulence-driving inputs.  Conventions of the input, not the
# method: a parabolic spectral shape over |n| peaking at |n| = 2 (zero at 1 and
# 3, after Federrath et al.'s stirring), seeded Gaussian OU noise, and the OU
# parameters of a Mach ~0.3 box (sigma, t_decay ~ a large-eddy turnover / 6).
@dataclass
class StirInputs:
    sigma: float
    t_decay: float
    zeta: float
    w: np.ndarray       # [61] per-mode weights
    noise: np.ndarray   # [nsteps, 61, 6] standard normal draws


def stir_inputs(n3, nsteps: int, seed: int = 4, sigma: float = 0.05, t_decay: float = 0.5,
                zeta: float = 1.0) -> StirInputs:
    """Driving inputs for the mode set n3 [61, 3] (from sph.stir_modes() or
    oracle.stir_modes(): both enumerate the same fixed set)."""
    kn = np.sqrt((np.asarray(n3, dtype=np.float64) ** 2).sum(axis=1))
    w = np.maximum(0.0, 1.0 - (kn - 2.0) ** 2)
    rng = np.random.default_rng(seed)
    noise = rng.standard_normal((nsteps, len(kn), 6))
    return StirInputs(sigma, t_decay, zeta, w, noise)
