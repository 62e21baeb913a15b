"""Physics of the GPU step over many steps (SURVEY 8(c) pins "Sedov", "Noh" and
'Integrator'): the Sedov blast radius follows the similarity solution
R(t) = xi0 (E t^2 / rho0)^(1/5), xi0 = 1.1517 for gamma = 5/3, and the total
energy sum m (v^2/2 + u) follows the ORACLE's measured curve (the scheme drifts
+5-7% through the shock, reading 16, so SURVEY's heuristic 1e-3 gate
is replaced by agreement with the oracle's own trajectory)."""
import numpy as np
import pytest

from paper_conf_sc_simsekpc24_b200 import ics

pytestmark = pytest.mark.gpu


def _energy(st):
    return float((st["m"] * (0.5 * (st["vx"] ** 2 + st["vy"] ** 2 + st["vz"] ** 2) + st["u"])).sum())


def _gpu_sedov(nside, steps):
    """GPU Sedov nside^3 for `steps` sph_step calls: (t, energies per step, state, rho)."""
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.sedov(nside)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    Es = [_energy(w.state)]
    t = 0.0
    for _ in range(steps):
        t = sim.step()["t"]
        Es.append(_energy(sim.get_state()))
    st = sim.get_state()
    rho = sim.get_field("rho")  # density of the last step's (pre-update) positions, same order
    sim.finalize()
    return t, Es, st, rho


def _golden_drift(nside):
    import json, os
    return json.load(open(os.path.join(os.path.dirname(__file__), "golden", f"sedov{nside}_drift.json")))


@pytest.mark.parametrize("nside", [16, 32])
def test_sedov_drift_matches_oracle(nside):
    """The scheme of the readings (no grad-h terms with variable h, a sound-speed
    Courant step) does not conserve energy through a strong shock: the ORACLE
    gains 5.39% (16^3) and 6.85% (32^3) of total energy by t = 0.05
    (tests/golden/sedov{16,32}_drift.json, written by tools/golden_sedov_drift.py
    from the oracle alone; reading 16).  The GPU trajectory has the same
    step count, t_end to 1e-9, and the oracle's energy curve to 1e-6."""
    ref = _golden_drift(nside)
    t, Es, st, rho = _gpu_sedov(nside, ref["steps"])
    assert abs(t / ref["t_end"] - 1) < 1e-9, (t, ref["t_end"])
    assert abs(Es[0] / ref["E0"] - 1) < 1e-15
    drift = Es[-1] / Es[0] - 1
    assert abs(drift - ref["drift"]) < 1e-6, (drift, ref["drift"])
    for a, b in zip(Es[::10], ref["E_every_10"]):
        assert abs(a / b - 1) < 1e-6


def test_sedov_blast_radius(golden):
    """Sedov 40^3 to t = 0.05: the shock sits at the similarity radius
    R(t) = xi0 (E t^2 / rho0)^(1/5), xi0 = 1.1517 (gamma = 5/3), within 12%, and
    the shell is compressed.  (Its energy is the oracle's, checked at 16^3 and
    32^3 in test_sedov_drift_matches_oracle; the oracle is too slow at 40^3.)"""
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.sedov(40)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    t, steps = 0.0, 0
    while t < 0.05 and steps < 2000:
        t = sim.step()["t"]
        steps += 1
    st = sim.get_state()
    rho = sim.get_field("rho")
    sim.finalize()
    r = np.sqrt(st["x"] ** 2 + st["y"] ** 2 + st["z"] ** 2)
    # shock position: the radius of the density peak, averaged over the shell of
    # the 200 densest particles
    top = np.argsort(rho)[-200:]
    R_num = float(np.median(r[top]))
    xi0 = golden["sedov_xi0_gamma53"]["value"]
    R_th = xi0 * (1.0 * t * t / 1.0) ** 0.2
    assert abs(R_num - R_th) / R_th < 0.12, (R_num, R_th, t)
    # strong-shock compression: the peak density is well above ambient
    assert rho[top].mean() > 2.0


def test_sedov_radius_converges_at_100():
    """Sedov 100^3 (configs[1]'s workload) to t = 0.05: the shock radius is within
    3% of the similarity solution (40^3: -2.3%, 100^3: -1.7%, 200^3: -0.6%,
    profiles/r02_sedov_convergence.json) and the shell compression exceeds 3
    (strong-shock limit 4)."""
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.sedov(100)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    t, steps = 0.0, 0
    while t < 0.05 and steps < 2000:
        t = sim.step()["t"]
        steps += 1
    st = sim.get_state()
    rho = sim.get_field("rho")
    sim.finalize()
    r = np.sqrt(st["x"] ** 2 + st["y"] ** 2 + st["z"] ** 2)
    top = np.argsort(rho)[-int(0.003 * w.n):]
    R_th = 1.1517 * (t * t) ** 0.2
    assert abs(float(np.median(r[top])) - R_th) / R_th < 0.03
    assert rho[top].mean() > 3.0


def test_noh_implosion_jumps():
    """Noh (SURVEY 8(c) pin 'Noh'; config 4's workload, 80^3 lattice, open box):
    at t = 0.3 the pre-shock gas follows rho = (1 + t/r)^2 with v_r = -1, the
    shocked gas is at rest with u = 1/2 (gamma = 5/3), and the shock sits at
    r = t/3.  Run with the signal-velocity time step (reading 22): the cold
    inflow has c ~ 0, so the sound-speed criterion alone would not resolve it.
    SPH smooths the jump, so the post-shock density (64 exactly) is only
    required to exceed 0.6 of it and the shock radius to be within 30%."""
    import dataclasses
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.noh(80)
    w.params = dataclasses.replace(w.params, dt_vsig=1, ngmax=400)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    t, steps = 0.0, 0
    while t < 0.3 and steps < 3000:
        t = sim.step()["t"]
        steps += 1
    st = sim.get_state()
    rho = sim.get_field("rho")
    r = np.sqrt(st["x"] ** 2 + st["y"] ** 2 + st["z"] ** 2)
    vr = (st["vx"] * st["x"] + st["vy"] * st["y"] + st["vz"] * st["z"]) / np.maximum(r, 1e-12)
    sim.finalize()
    # undisturbed inflow: outside the shock (+ a smoothing length) and inside
    # r < 0.5 - t (the cube's faces have reached r = 0.2 along the axes)
    pre = (r > 0.145) & (r < 0.175)
    ratio = rho[pre] / (1 + t / r[pre]) ** 2
    assert abs(np.median(ratio) - 1) < 0.03 and abs(np.mean(ratio) - 1) < 0.06
    assert np.abs(np.median(vr[pre]) + 1) < 0.03
    post = (r > 0.05) & (r < 0.09)
    assert abs(np.median(st["u"][post]) - 0.5) < 0.1
    assert np.median(np.abs(vr[post])) < 0.05
    assert np.median(rho[post]) > 0.6 * 64
    # shock radius: where the median u of thin shells crosses 1/4
    edges = np.linspace(0.02, 0.3, 57)
    mids = 0.5 * (edges[1:] + edges[:-1])
    umed = np.array([np.median(st["u"][(r >= a) & (r < b)]) for a, b in zip(edges[:-1], edges[1:])])
    Rs = mids[np.argmax(umed < 0.25)]
    assert abs(Rs - t / 3) / (t / 3) < 0.3, (Rs, t, steps)
