"""Pins for the composed oracle step (SURVEY 8(c) steps 1-10 in order) and for its
sampled mode (the full-size parity reference)."""
import numpy as np
import pytest

import oracle
from paper_conf_sc_simsekpc24_b200 import ics


def test_sedov16_one_step_invariants(golden):
    w = ics.sedov(16)
    s = {k: v.copy() for k, v in w.state.items()}
    st, out = oracle.step(s, w.params, w.params.dt_first, True)
    # order is the stable Morton order of the input; ids are a permutation
    assert np.array_equal(np.sort(st["id"]), np.arange(w.n))
    assert np.all(out["keys"][1:] >= out["keys"][:-1])
    assert out["dt"] == golden["sedov16_dt0"]["value"]
    assert np.all(out["nb"].nc == golden["lattice_nc"]["value"])
    m = st["m"]
    # mass is carried, never created
    assert m.sum() == pytest.approx(1.0, rel=1e-14)
    # symmetric pairs (uniform h): momentum is conserved by the step's forces
    scale = (m[:, None] * out["a_abs"]).sum(0)
    for k, a in (("ax", 0), ("ay", 1), ("az", 2)):
        assert abs((m * out[k]).sum()) < 1e-14 * scale[a]
    # the blast centre heats nothing yet (v = 0) but accelerates outward
    r = np.sqrt(out["pre"]["x"] ** 2 + out["pre"]["y"] ** 2 + out["pre"]["z"] ** 2)
    radial = (out["ax"] * out["pre"]["x"] + out["ay"] * out["pre"]["y"] + out["az"] * out["pre"]["z"])
    inner = (r > 0.03) & (r < 0.15)
    assert np.all(radial[inner] > 0)
    # h unchanged at nc = ng0 - 8 -> ratio 1.0083651
    assert np.allclose(st["h"] / out["pre"]["h"], golden["lattice_h_ratio_nc92"]["value"], atol=1e-7)


def test_ten_steps_energy_drift():
    """Total energy E = sum m (v^2/2 + u) over 10 Sedov 16^3 steps: drift tiny
    (dt ~ 1e-6 so the integrator error is O(dt^2 |du|))."""
    w = ics.sedov(16)
    s = {k: v.copy() for k, v in w.state.items()}
    E0 = (s["m"] * (0.5 * (s["vx"] ** 2 + s["vy"] ** 2 + s["vz"] ** 2) + s["u"])).sum()
    dt = w.params.dt_first
    for k in range(10):
        s, out = oracle.step(s, w.params, dt, k == 0)
        dt = out["dt"]
    E1 = (s["m"] * (0.5 * (s["vx"] ** 2 + s["vy"] ** 2 + s["vz"] ** 2) + s["u"])).sum()
    assert abs(E1 - E0) / E0 < 1e-6


def test_sample_step_equals_full_step():
    """The sampled mode (ball of radius 6 h_max around each target) reproduces the full
    O(N^2) step at the targets to the last bit of the sums it shares (same order)."""
    w = ics.random_box(2500, seed=21)
    w.params.eos = 0
    s = {k: v.copy() for k, v in w.state.items()}
    st, out = oracle.step({k: v.copy() for k, v in s.items()}, w.params, 1e-4, True)
    tg = np.array([0, 17, 1234, 2499])
    order, smp = oracle.sample_step(s, w.params, 1e-4, True, tg)
    assert np.array_equal(order, out["pre"]["id"])
    assert smp["dt"] == out["dt"]
    for q, t in enumerate(tg):
        nb = out["nb"]
        assert np.array_equal(smp["nbrs"][q], nb.idx[nb.offsets[t]:nb.offsets[t + 1]])
        assert smp["rho"][q] == out["rho"][t]
        assert np.array_equal(smp["C"][q], out["C"][t])
        for k in ("ax", "ay", "az", "du"):
            assert smp[k][q] == out[k][t]
        for k in ("x", "y", "z", "vx", "vy", "vz", "u", "h"):
            assert smp[k][q] == st[k][t]


@pytest.mark.parametrize("fset", ["gradh_vsig_balsara", "ve_gradh_vsig_balsara"])
def test_sample_step_equals_full_step_paper_functions(fset):
    """The sampled mode for the paper's function set (grad-h,
    volume elements, div/curl + Balsara, signal-velocity dt; 4-radius ball with
    volume elements) reproduces the full step at the targets bit for bit.  With
    dt_vsig the global dt is the caller's (here the full step's)."""
    w = ics.random_box(2500, seed=23)
    w.params.eos = 0
    w.params.gradh = 1
    w.params.dt_vsig = 1
    w.params.av_switch = 1
    w.params.ve = 1 if fset.startswith("ve") else 0
    s = {k: v.copy() for k, v in w.state.items()}
    st, out = oracle.step({k: v.copy() for k, v in s.items()}, w.params, 1e-4, True)
    tg = np.array([3, 888, 2100])
    with pytest.raises(ValueError):
        oracle.sample_step(s, w.params, 1e-4, True, tg)
    order, smp = oracle.sample_step(s, w.params, 1e-4, True, tg, dt=out["dt"])
    assert np.array_equal(order, out["pre"]["id"])
    for q, t in enumerate(tg):
        nb = out["nb"]
        assert np.array_equal(smp["nbrs"][q], nb.idx[nb.offsets[t]:nb.offsets[t + 1]])
        for k in ("rho", "p", "omega", "divv", "bal", "vsig", "ax", "ay", "az", "du"):
            assert smp[k][q] == out[k][t], k
        if w.params.ve:
            assert smp["kx"][q] == out["kx"][t]
        assert np.array_equal(smp["C"][q], out["C"][t])
        for k in ("x", "y", "z", "vx", "vy", "vz", "u", "h"):
            assert smp[k][q] == st[k][t]
    # the ball really needed more than one radius (dependency cone)
    assert min(smp["ball_sizes"]) > 3 * out["nb"].nc.max()


def test_step_keeps_gradh_and_divcurl_outputs_together():
    """oracle.step with grad-h AND div/curl returns omega and div v side by side
    (round-1 helper bug: the div/curl dict replaced the grad-h one)."""
    w = ics.random_box(600, seed=2)
    w.params.eos = 0
    w.params.gradh = 1
    w.params.divcurl = 1
    _, out = oracle.step({k: v.copy() for k, v in w.state.items()}, w.params, 1e-4, True)
    for k in ("omega", "dWdh_sum", "divv", "curl", "T"):
        assert k in out and out[k].shape[0] == w.n


def test_open_box_noh_step():
    """Noh (open box): box is the bounding box; converging flow is heated by AV."""
    w = ics.noh(12)
    s = {k: v.copy() for k, v in w.state.items()}
    st, out = oracle.step(s, w.params, w.params.dt_first, True)
    assert np.array_equal(out["bmin"], [w.state[k].min() for k in ("x", "y", "z")])
    assert (st["m"] * out["du"]).sum() > 0


def test_sample_step_lattice100(golden):
    """Sampled mode at 10^6 particles: IAD on the perfect 100^3 lattice gives
    C11 = 1/tau11 with tau11 = 3.5371030264962991e-5 and nc = 92 everywhere."""
    w = ics.sedov(100)
    order, smp = oracle.sample_step(w.state, w.params, w.params.dt_first, True, [0, 123457])
    assert np.all(smp["nc"] == golden["lattice_nc"]["value"])
    assert np.allclose(smp["C"][:, 0], 1.0 / golden["lattice100_tau11"]["value"], rtol=1e-12)
    assert np.allclose(smp["rho"], golden["lattice_rho"]["value"], rtol=1e-14)
    assert smp["dt"] == pytest.approx(1.1e-6, rel=1e-15)


def test_turbulence_slices_equal_the_full_generator():
    """The multi-GPU IC slices reproduce the single-GPU input (positions, ids
    exactly; velocities to the rounding of the global normalisation)."""
    full = ics.turbulence(12)
    parts = [ics.turbulence_part(12, r, 3) for r in range(3)]
    vsq = sum(p.meta["vsq_sum"] for p in parts)
    for p in parts:
        ics.normalise_velocity(p, vsq)
    cat = {k: np.concatenate([p.state[k] for p in parts]) for k in full.state}
    for k in ("x", "y", "z", "h", "m", "u", "id"):
        assert np.array_equal(cat[k], full.state[k]), k
    for k in ("vx", "vy", "vz"):
        assert np.allclose(cat[k], full.state[k], rtol=1e-14, atol=1e-16), k


def test_sedov16_energy_drift_measured():
    """DESIGN.md reading 16, measured: the oracle's own Sedov 16^3 run to t = 0.05
    gains ~5.4% total energy (variable h without grad-h terms, a sound-speed
    Courant step through a strong shock).  Recomputed here and pinned to the
    committed measurement (tests/golden/sedov16_drift.json, written by
    tools/golden_sedov_drift.py); the GPU run is held to the same drift in
    tests/test_gpu_physics.py."""
    import json
    import os
    import sys
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
    import golden_sedov_drift as g
    ref = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "sedov16_drift.json")))
    r = g.run()
    assert r["steps"] == ref["steps"] and r["t_end"] == ref["t_end"]
    assert r["drift"] == pytest.approx(ref["drift"], rel=1e-12, abs=1e-15)
    assert 0.03 < r["drift"] < 0.08
    # the drift builds up through the run (the shock), it is not a first-step jump
    E = np.array(r["E_every_10"])
    assert abs(E[1] / E[0] - 1) < 1e-3 < abs(E[-1] / E[0] - 1)
