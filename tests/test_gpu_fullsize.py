"""Parity at BASELINE.json's full sizes, in the configuration bench.py times.

One step from the seeded initial conditions of configs[1] (Sedov 100^3),
configs[2] (turbulence 200^3, the bench workload) and configs[3] (Noh 300^3,
open box, on one GPU): the Morton order of ALL particles is compared bit-exactly
with the oracle's stable sort, dt bit-exactly, and at sampled particles the
oracle's sampled mode (exact: the full-size step restricted to each target's
dependency ball) gives the neighbour lists (bit-exact), rho, p, c, C, a, du and
the updated state (DESIGN.md section 3 metric, 1e-10)."""
import numpy as np
import pytest

import oracle
from paper_conf_sc_simsekpc24_b200 import ics
from parity import TOL_1STEP, assert_rel_close, assert_sum_close

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

CASES = {"sedov100": lambda: ics.sedov(100), "turbulence200": lambda: ics.turbulence(200),
         "noh300": lambda: ics.noh(300)}


@pytest.mark.parametrize("name", list(CASES))
def test_full_size_one_step(name):
    from paper_conf_sc_simsekpc24_b200 import sph
    w = CASES[name]()
    n = w.n
    sim = sph.Simulation(w.params, n_capacity=n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    sim.build_tree()
    stats = sim.find_neighbors()
    sim.density()
    sim.eos()
    sim.iad()
    sim.momentum_energy()
    g = {k: sim.get_field(k) for k in ("id", "key", "nc", "rho", "p", "c", "ax", "ay", "az", "du")}
    Cg = np.stack([sim.get_field(k) for k in ("c11", "c12", "c13", "c22", "c23", "c33")], 1)
    rng = np.random.default_rng(123)
    tg = np.unique(np.concatenate([rng.choice(n, 40, replace=False), [0, 1, n // 2, n - 2, n - 1]]))
    off, idx = sim.get_neighbor_rows(tg)
    dt = sim.timestep()
    sim.update()
    after = {k: sim.get_field(k) for k in ("x", "y", "z", "vx", "vy", "vz", "u", "h")}

    order, o = oracle.sample_step(w.state, w.params, w.params.dt_first, True, tg)
    assert np.array_equal(g["id"], order), "Morton order of all particles"
    assert np.array_equal(g["key"], o["keys"]), "sorted keys"
    assert dt == o["dt"], "dt"
    assert stats["max_nc"] <= w.params.ngmax
    for q, t in enumerate(tg):
        assert np.array_equal(idx[off[q]:off[q + 1]].astype(np.int64), o["nbrs"][q]), f"list of {t}"
    assert np.array_equal(g["nc"][tg], o["nc"].astype(np.int32))
    assert_rel_close(g["rho"][tg], o["rho"], TOL_1STEP, "rho")
    assert np.array_equal(g["c"][tg], o["c"]), "c bit-exact"
    assert_rel_close(g["p"][tg], o["p"], TOL_1STEP, "p")
    Cn = np.linalg.norm(o["C"], axis=1)
    for e in range(6):
        assert_sum_close(Cg[tg, e], o["C"][:, e], Cn, TOL_1STEP, f"C[{e}]")
    for a, k in enumerate(("ax", "ay", "az")):
        assert_sum_close(g[k][tg], o[k], o["a_abs"][:, a], TOL_1STEP, k)
    assert_sum_close(g["du"][tg], o["du"], o["du_abs"], TOL_1STEP, "du")
    L = float(np.max(np.asarray(o["bmax"]) - np.asarray(o["bmin"])))
    for k in ("x", "y", "z"):
        assert_sum_close(after[k][tg], o[k], np.full(len(tg), L), TOL_1STEP, k)
    vs = max(np.abs(np.concatenate([o["vx"], o["vy"], o["vz"]])).max(), 1e-300)
    for k in ("vx", "vy", "vz"):
        assert_sum_close(after[k][tg], o[k], np.maximum(np.abs(o[k]), vs), TOL_1STEP, k)
    assert_rel_close(after["u"][tg], o["u"], TOL_1STEP, "u", floor=1e-300)
    assert_rel_close(after["h"][tg], o["h"], TOL_1STEP, "h")
