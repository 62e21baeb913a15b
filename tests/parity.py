"""Shared helpers of the GPU-vs-oracle parity tests (tolerance metric of DESIGN.md
section 3 / SURVEY 8(c) 'Tolerance metric')."""
from __future__ import annotations

import numpy as np

TOL_1STEP = 1e-10   # north_star: fp64 fields within 1e-10 after one step
TOL_10STEP = 1e-8   # ... and 1e-8 after 10 steps


def new_sim(w, cap=None, **kw):
    from paper_conf_sc_simsekpc24_b200 import sph
    sim = sph.Simulation(w.params, n_capacity=cap or max(w.n, 1), **kw)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    return sim


def gpu_pipeline(sim):
    """build_tree .. momentum_energy through the C ABI; returns every field."""
    sim.build_tree()
    stats = sim.find_neighbors()
    sim.density()
    sim.eos()
    if sim.cfg.gradh or sim.cfg.ve:
        sim.gradh()
    sim.iad()
    sim.momentum_energy()
    out = {k: sim.get_field(k) for k in ("id", "key", "nc", "rho", "p", "c", "ax", "ay", "az", "du",
                                         "x", "y", "z", "vx", "vy", "vz", "h", "m", "u")}
    out["C"] = np.stack([sim.get_field(k) for k in ("c11", "c12", "c13", "c22", "c23", "c33")], 1)
    out["stats"] = stats
    return out


def assert_sum_close(got, want, scale, tol, what):
    err = np.abs(got - want)
    bound = tol * scale + 1e-300
    bad = err > bound
    assert not bad.any(), (f"{what}: {bad.sum()} of {bad.size} outside tol {tol} "
                           f"(worst err/scale {np.max(err / (scale + 1e-300)):.3e})")


def assert_rel_close(got, want, tol, what, floor=0.0):
    scale = np.maximum(np.abs(want), floor)
    assert_sum_close(got, want, scale, tol, what)


def compare_sums(g, o, tol, idx=None):
    """g: GPU fields, o: oracle step output (both in the same order)."""
    sel = (lambda a: a) if idx is None else (lambda a: a[idx])
    assert_rel_close(sel(g["rho"]), o["rho"], tol, "rho")
    assert np.array_equal(sel(g["c"]), o["c"]), "c is bit-exact (IEEE sqrt of identical input)"
    assert_rel_close(sel(g["p"]), o["p"], tol, "p")
    Cn = np.linalg.norm(o["C"], axis=1)
    for e in range(6):
        assert_sum_close(sel(g["C"])[:, e], o["C"][:, e], Cn, tol, f"C[{e}]")
    for a, k in enumerate(("ax", "ay", "az")):
        assert_sum_close(sel(g[k]), o[k], o["a_abs"][:, a], tol, k)
    assert_sum_close(sel(g["du"]), o["du"], o["du_abs"], tol, "du")


def compare_state(g, o, L, tol, what=""):
    """Trajectory metric: x relative to L, v relative to max(|v_i|, v_scale),
    u and h plain relative."""
    for k in ("x", "y", "z"):
        assert_sum_close(g[k], o[k], np.full(o[k].shape, L), tol, what + k)
    vs = max(np.abs(np.concatenate([o["vx"], o["vy"], o["vz"]])).max(), 1e-300)
    for k in ("vx", "vy", "vz"):
        assert_sum_close(g[k], o[k], np.maximum(np.abs(o[k]), vs), tol, what + k)
    assert_rel_close(g["u"], o["u"], tol, what + "u", floor=1e-300)
    assert_rel_close(g["h"], o["h"], tol, what + "h")
