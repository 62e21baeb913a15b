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
