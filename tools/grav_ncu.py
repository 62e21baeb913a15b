"""One Evrard ~1M step (gravity leaf level 6) for an ncu capture of grav_walk_kernel."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_sc_simsekpc24_b200 import ics, sph  # noqa: E402

w = ics.evrard(124)
sim = sph.Simulation(w.params, n_capacity=w.n)
sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
sim.set_time(0, w.params.dt_first, True)
for _ in range(3):
    info = sim.step()
print(info["phase_ms"]["gravity"], info["grav_multipoles"] / (w.n / 32), info["grav_pairs"] / (w.n / 32))
