"""Parity on EVOLVED states at full size (SURVEY 8(c) "For N >= 100^3, parity is
always '1 step from the GPU state' at steps {0, 1, 10, 50, 99}"; VERDICT r1
missing #3 and #8).

* configs[1], Sedov 100^3 run for 100 steps on the GPU.  After 1, 10, 50 and 99
  steps the GPU's own state is handed to the oracle's sampled mode and the next
  GPU step is compared with it at 64 targets, half of them in the shock shell
  (the densest particles: strongly variable h, approaching pairs, AV on):
  Morton order of all particles and dt bit-exact, neighbour lists bit-exact,
  fields within 1e-10 on the DESIGN.md section 3 metric.
* configs[2], turbulence 200^3 with the paper's function set (grad-h,
  div/curl + Balsara switch, signal-velocity dt; with and without volume
  elements), one step, against the sampled oracle (grad-h / VE / v_sig now
  covered by oracle.sample_step)."""
import dataclasses

import numpy as np
import pytest

import oracle
from paper_conf_sc_simsekpc24_b200 import ics
from parity import TOL_1STEP, assert_rel_close, assert_sum_close

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


def _gpu_staged_step(sim, tg_ids_fn, extra=()):
    """One step through the staged C ABI calls; returns GPU fields (current order),
    the targets (positions in the new order), their lists, dt and the updated state."""
    sim.build_tree()
    stats = sim.find_neighbors()
    sim.density()
    sim.eos()
    if sim.cfg.gradh or sim.cfg.ve:
        sim.gradh()
    sim.iad()
    sim.momentum_energy()
    g = {k: sim.get_field(k) for k in ("id", "key", "nc", "rho", "p", "c", "ax", "ay", "az", "du", *extra)}
    g["C"] = np.stack([sim.get_field(k) for k in ("c11", "c12", "c13", "c22", "c23", "c33")], 1)
    pos = np.empty(g["id"].size, dtype=np.int64)
    pos[g["id"]] = np.arange(g["id"].size)
    tg = np.unique(pos[np.asarray(tg_ids_fn(g), dtype=np.int64)])
    off, idx = sim.get_neighbor_rows(tg)
    dt = sim.timestep()
    sim.update()
    after = {k: sim.get_field(k) for k in ("x", "y", "z", "vx", "vy", "vz", "u", "h")}
    return g, tg, off, idx, dt, after, stats


def _compare(g, tg, off, idx, after, o, order):
    assert np.array_equal(g["id"], order), "Morton order of all particles"
    assert np.array_equal(g["key"], o["keys"]), "sorted keys"
    for q, t in enumerate(tg):
        assert np.array_equal(idx[off[q]:off[q + 1]].astype(np.int64), o["nbrs"][q]), f"list of {t}"
    assert np.array_equal(g["nc"][tg], o["nc"].astype(np.int32))
    assert_rel_close(g["rho"][tg], o["rho"], TOL_1STEP, "rho")
    assert np.array_equal(g["c"][tg], o["c"]), "c bit-exact"
    assert_rel_close(g["p"][tg], o["p"], TOL_1STEP, "p")
    Cn = np.linalg.norm(o["C"], axis=1)
    for e in range(6):
        assert_sum_close(g["C"][tg, e], o["C"][:, e], Cn, TOL_1STEP, f"C[{e}]")
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


def test_sedov100_evolved_states():
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.sedov(100)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    rng = np.random.default_rng(99)
    checkpoints = (1, 10, 50, 99)
    steps = 0
    report = []
    for cp in checkpoints:
        while steps < cp:
            sim.step()
            steps += 1
        st = sim.get_state()
        t, dt_prev, first = sim.get_time()
        rho_prev = sim.get_field("rho")            # last step's density, same order as st
        shell = st["id"][np.argsort(rho_prev)[-4000:]]  # the densest particles: the shock shell
        pick = lambda g: np.concatenate([rng.choice(shell, 32, replace=False),
                                         rng.choice(st["id"], 32, replace=False)])
        g, tg, off, idx, dt, after, stats = _gpu_staged_step(sim, pick)
        steps += 1
        order, o = oracle.sample_step(st, w.params, dt_prev, first, tg)
        assert dt == o["dt"], ("dt", cp)
        _compare(g, tg, off, idx, after, o, order)
        h = st["h"]
        report.append((cp, t, float(h.max() / h.min()), float(rho_prev.max()), int(stats["max_nc"])))
    sim.finalize()
    # the states really are evolved: h varies, a shock of compression > 2 exists
    last = report[-1]
    assert last[2] > 1.5 and last[3] > 2.0, report


@pytest.mark.parametrize("ve", [0, 1], ids=["gradh_balsara_vsig", "ve_gradh_balsara_vsig"])
def test_turbulence200_paper_function_set(ve):
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.turbulence(200)
    w.params = dataclasses.replace(w.params, gradh=1, av_switch=1, dt_vsig=1, ve=ve)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    rng = np.random.default_rng(7 + ve)
    chosen = {}

    def pick(g):
        # 40 random targets + the particle that sets the signal-velocity dt
        vs = g["vsig"]
        h = sim.get_field("h")
        chosen["argmin"] = int(g["id"][np.argmin(h / vs)])
        return np.concatenate([rng.choice(g["id"], 40, replace=False), [chosen["argmin"]]])

    g, tg, off, idx, dt, after, stats = _gpu_staged_step(sim, pick, extra=("vsig", "omega", "bal"))
    sim.finalize()
    order, o = oracle.sample_step(w.state, w.params, w.params.dt_first, True, tg, dt=dt)
    _compare(g, tg, off, idx, after, o, order)
    # grad-h factor, Balsara switch, signal velocity at the targets
    hh = w.state["h"][order][tg]
    rho_for_omega = o["kx"] if ve else o["rho"]
    assert_sum_close(g["omega"][tg], o["omega"], hh / (3 * rho_for_omega) * o["dWdh_abs"], TOL_1STEP, "omega")
    assert np.abs(g["bal"][tg] - o["bal"]).max() < 1e-9   # f in [0, 1], as tests/test_gpu_divcurl.py
    assert np.all(np.abs(g["vsig"][tg] - o["vsig"]) <= 1e-13 * o["vsig"])
    # dt: no target allows a larger step, and the arg-min target reproduces it
    C = w.params.k_cour
    assert np.all(dt <= C * hh / o["vsig"] * (1 + 1e-13))
    q = int(np.where(order[tg] == chosen["argmin"])[0][0])
    expect = min(C * hh[q] / o["vsig"][q], w.params.dt_max_growth * w.params.dt_first)
    assert dt == pytest.approx(expect, rel=1e-13)
