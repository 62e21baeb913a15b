"""Per-function frequency tuning harness (Figs. 2, 6-8).
On hosts that forbid clock changes (this pool) the search must refuse cleanly,
leave the clocks at default and still measure every function under DVFS."""
import os

import numpy as np
import pytest

from paper_conf_sc_simsekpc24_b200 import ics

pytestmark = pytest.mark.gpu


def _sim():
    from parity import new_sim
    sim = new_sim(ics.turbulence(24))
    sim.step()
    sim.build_tree()
    sim.find_neighbors(stats=False)
    sim.density()
    sim.eos()
    sim.iad()
    sim.momentum_energy()
    return sim


def test_supported_clocks_and_pick():
    from paper_conf_sc_simsekpc24_b200 import tuning
    sim = _sim()
    sup = sim.supported_clocks()
    assert len(sup) > 1 and sup == sorted(sup, reverse=True) and sup[0] >= 1000
    pick = tuning.pick_clocks(sup, 4)
    assert pick[0] == sup[0] and len(pick) <= 4 and min(pick) >= 0.5 * sup[0]
    sim.finalize()


@pytest.mark.skipif(os.environ.get("SPH_ALLOW_CLOCK_CONTROL") == "1", reason="host permits clock control")
def test_search_refuses_cleanly_and_measures_dvfs():
    from paper_conf_sc_simsekpc24_b200 import sph, tuning
    sim = _sim()
    res = tuning.frequency_search(sim, phases=("density", "momentum_energy"), nclocks=2,
                                  min_seconds=0.2)
    assert res["clock_control"] == "refused"
    assert "ERR_NO_PERMISSION" in res["why"]
    for ph in ("density", "momentum_energy"):
        assert res["dvfs"][ph]["ms"] > 0 and res["dvfs"][ph]["reps"] >= 3
    pol = tuning.compare_policies(sim, {"density": 1000}, static_clocks=(1965,), seconds=0.2)
    assert pol["clock_control"] == "refused" and pol["dvfs"]["ms_per_step"] > 0
    sim.finalize()


def test_repeat_phase_leaves_the_pipeline_state_unchanged():
    """sph_repeat_phase (the KernelTuner-style isolated repetition) must not change
    what the next phases read: SORT keeps SPH_F_ORDER, EOS after GRADH keeps
    p/(Omega rho^2), IAD / MOMENTUM_ENERGY give the same fields; DENSITY after the
    volume-element GRADH is refused (it would overwrite the normalised rho)."""
    import dataclasses
    from paper_conf_sc_simsekpc24_b200 import ics, sph
    from parity import new_sim
    w = ics.turbulence(16)
    w.params = dataclasses.replace(w.params, gradh=1)
    sim = new_sim(w)
    sim.build_tree()
    order = sim.get_field("order").copy()
    sim.repeat_phase("sort", 3)
    assert np.array_equal(sim.get_field("order"), order)
    sim.find_neighbors()
    sim.density()
    sim.eos()
    sim.gradh()
    sim.iad()
    sim.momentum_energy()
    ref = {k: sim.get_field(k).copy() for k in ("ax", "ay", "az", "du", "rho", "c11")}
    for ph in ("eos", "gradh", "iad", "momentum_energy"):
        sim.repeat_phase(ph, 2)
    sim.momentum_energy()
    for k, v in ref.items():
        assert np.array_equal(sim.get_field(k), v), k
    sim.finalize()
    w2 = ics.turbulence(16)
    w2.params = dataclasses.replace(w2.params, gradh=1, ve=1)
    sim2 = new_sim(w2)
    sim2.build_tree()
    sim2.find_neighbors()
    sim2.density()
    sim2.eos()
    sim2.gradh()
    with pytest.raises(sph.SphError):
        sim2.repeat_phase("density", 2)
    sim2.finalize()
