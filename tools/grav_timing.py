"""Gravity phase time of Evrard ~1M at leaf levels 5-7 (A/B helper: one line)."""
import dataclasses
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_sc_simsekpc24_b200 import ics, sph  # noqa: E402

out = {}
w0 = ics.evrard(124)
for level in (5, 6, 7):
    w = dataclasses.replace(w0)
    w.params = dataclasses.replace(w0.params, grav_level=level)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0, w.params.dt_first, True)
    g = []
    for s in range(6):
        info = sim.step()
        if s >= 2:
            g.append(info["phase_ms"]["gravity"])
    out[level] = round(float(np.median(g)), 3)
    sim.finalize()
print(sys.argv[1] if len(sys.argv) > 1 else "base", "gravity ms by leaf level", out)
