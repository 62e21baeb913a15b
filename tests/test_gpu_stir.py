"""GPU parity of the turbulence driving: libsph's STIR phase
(OU update on the device, driving acceleration by per-axis complex powers) vs
the oracle (libm exp/cos/sin of the plain definition) on the same seeded inputs,
over several steps of the full pipeline; plus the noise-table capacity error."""
import numpy as np
import pytest

import oracle
from paper_conf_sc_simsekpc24_b200 import ics

pytestmark = pytest.mark.gpu


def _setup(nside, nsteps, stir_steps=None):
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.turbulence(nside)
    si = ics.stir_inputs(oracle.stir_modes(), nsteps)
    sim = sph.Simulation(w.params, n_capacity=w.n, stir_steps=stir_steps or nsteps)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    sim.stir_init(si.sigma, si.t_decay, si.zeta, si.w, si.noise)
    stir = {"A": np.zeros((61, 6)), "w": si.w, "noise": si.noise, "step": 0, "sigma": si.sigma,
            "t_decay": si.t_decay, "zeta": si.zeta}
    return w, sim, stir


def test_mode_sets_agree():
    from paper_conf_sc_simsekpc24_b200 import sph
    assert np.array_equal(sph.stir_modes(), oracle.stir_modes())


def test_stir_parity_over_steps():
    from parity import TOL_1STEP, TOL_10STEP, compare_state, compare_sums, gpu_pipeline
    w, sim, stir = _setup(16, 4)
    s = {k: v.copy() for k, v in w.state.items()}
    dt = w.params.dt_first
    for k in range(4):
        s_new, o = oracle.step(s, w.params, dt, k == 0, stir=stir)
        g = gpu_pipeline(sim)       # build_tree .. momentum_energy
        sim.stir()
        for f in ("ax", "ay", "az"):
            g[f] = sim.get_field(f)
        assert np.array_equal(g["id"], o["pre"]["id"])
        tol = TOL_1STEP if k == 0 else TOL_10STEP
        compare_sums(g, o, tol)
        A, n = sim.stir_state()
        assert n == k + 1
        # OU state: scale metric (the device fuses f*A + g*xi into one FMA)
        np.testing.assert_allclose(A, stir["A"], rtol=0, atol=1e-13 * np.abs(stir["A"]).max())
        assert sim.timestep() == pytest.approx(o["dt"], rel=1e-12)
        sim.update()
        s, dt = s_new, o["dt"]
    compare_state(sim.get_state(), s, 1.0, TOL_10STEP, "4 driven steps: ")


def test_driving_changes_the_flow_and_step_includes_stir():
    from paper_conf_sc_simsekpc24_b200 import sph
    w, sim, stir = _setup(12, 3)
    info = sim.step()                # sph_step runs STIR when enabled
    assert info["phase_ms"]["stir"] > 0
    A, n = sim.stir_state()
    assert n == 1 and np.abs(A).max() > 0


def test_noise_table_exhaustion_is_a_capacity_error():
    from paper_conf_sc_simsekpc24_b200 import sph
    w, sim, stir = _setup(8, 2, stir_steps=2)
    sim.step()
    sim.step()
    with pytest.raises(sph.SphError) as e:
        sim.step()
    assert e.value.name == "ERR_CAPACITY"


def test_step_graph_recaptured_when_driving_starts(monkeypatch):
    """sph_step's CUDA graph holds the kernel arguments of its capture: turning
    the driving on after two graph steps (new phase, new arguments) must give a
    new capture, and the run equals the eager one bit for bit."""
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.turbulence(12)
    si = ics.stir_inputs(oracle.stir_modes(), 4)
    out = {}
    for env in ("1", "0"):
        monkeypatch.setenv("SPH_NO_GRAPH", env)
        sim = sph.Simulation(w.params, n_capacity=w.n, stir_steps=4)
        sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
        sim.set_time(0.0, w.params.dt_first, True)
        infos = [sim.step(), sim.step()]
        sim.stir_init(si.sigma, si.t_decay, si.zeta, si.w, si.noise)
        infos += [sim.step() for _ in range(3)]
        out[env] = (sim.get_state(), infos)
        sim.finalize()
    (a, ia), (b, ib) = out["1"], out["0"]
    for k in a:
        assert np.array_equal(a[k], b[k]), k
    assert all(x["graph"] for x in ib) and not any(x["graph"] for x in ia)
    assert all(x["phase_ms"]["stir"] > 0 for x in ib[2:]) and ib[1]["phase_ms"]["stir"] == 0
