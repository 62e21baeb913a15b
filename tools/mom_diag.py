"""Times MOMENTUM_ENERGY alone (sph_repeat_phase on valid inputs of the first
turbulence 200^3 step) for whatever libsph build is in place -- with
SPH_NVCC_EXTRA=-DSPH_MOM_DIAG=1 (gathers only) / 2 (arithmetic only, broadcast
records) it gives the two ceilings of the kernel."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_simsekpc24_b200 import ics, sph  # noqa: E402

w = ics.turbulence(int(sys.argv[1]) if len(sys.argv) > 1 else 200)
sim = sph.Simulation(w.params, n_capacity=w.n)
sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
sim.set_time(0.0, w.params.dt_first, True)
sim.build_tree()
sim.find_neighbors()
sim.density()
sim.eos()
sim.iad()
sim.momentum_energy()
sim.repeat_phase("momentum_energy", 3)
ms, _ = sim.repeat_phase("momentum_energy", 20)
print(f"{os.environ.get('SPH_NVCC_EXTRA', '') or 'base'}: momentum_energy {ms:.3f} ms")
