"""DVFS trace (Fig. 9): the NVML sampling thread of
sph_trace_start records the SM clock, power and energy counter while the device
runs the step, each sample tagged with the phase the stream is executing."""
import numpy as np
import pytest

from paper_conf_sc_simsekpc24_b200 import ics

pytestmark = pytest.mark.gpu


def test_trace_tags_phases_and_samples_nvml():
    from paper_conf_sc_simsekpc24_b200 import sph
    from parity import new_sim
    w = ics.turbulence(64)
    sim = new_sim(w)
    sim.step()  # warm-up
    import time
    sim.trace_start(period_ms=0.2, capacity=200_000)
    t0 = time.perf_counter()
    steps = 0
    while time.perf_counter() - t0 < 1.0:  # NVML queries take ms: sample ~1 s of steps
        sim.step()
        steps += 1
    tr = sim.trace_stop(capacity=200_000)
    sim.finalize()
    assert tr.size > 20, (tr.size, steps)
    assert np.all(np.diff(tr["t_ms"]) >= 0)
    assert np.all((tr["phase"] >= -1) & (tr["phase"] < sph.NPHASES))
    seen = {sph.PHASES[p] for p in np.unique(tr["phase"]) if p >= 0}
    # the two longest phases (~70% of the step) are caught
    assert {"neighbors", "momentum_energy"} <= seen, (seen, np.median(tr["query_us"]))
    assert np.all(tr["sm_mhz"] > 0) and np.all(tr["power_mw"] > 0)
    assert np.all(np.diff(tr["energy_mj"].astype(np.int64)) >= 0)


def test_trace_state_errors():
    from paper_conf_sc_simsekpc24_b200 import sph
    from parity import new_sim
    sim = new_sim(ics.turbulence(8))
    with pytest.raises(sph.SphError) as e:
        sim.trace_stop(capacity=1)
    assert e.value.name == "ERR_STATE"
    with pytest.raises(sph.SphError) as e:
        sim.trace_start(period_ms=0.0)
    assert e.value.name == "ERR_ARG"
    sim.trace_start(period_ms=1.0, capacity=4)
    with pytest.raises(sph.SphError) as e:
        sim.trace_start(period_ms=1.0, capacity=4)
    assert e.value.name == "ERR_STATE"
    sim.step()
    tr = sim.trace_stop(capacity=4)
    assert tr.size <= 4
    sim.finalize()
