"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck,
SURVEY.md section 5): every libsph kernel family runs at least once on 16^3-ish
inputs -- keys, onesweep sort + permute, cells, the warp-cooperative neighbour
search (periodic, open, several groups), density, EOS, grad-h / volume
elements, IAD (+ div/curl), momentum-energy (+ Balsara, v_sig), timestep,
update, stirring, Barnes-Hut gravity, the decomposition plumbing and the
repeat / trace / accounting paths."""
import dataclasses
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_simsekpc24_b200 import decomp, ics, sph  # noqa: E402


def run(w, steps=2, **kw):
    sim = sph.Simulation(w.params, n_capacity=w.n, **kw)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    for _ in range(steps):
        sim.step()
    return sim


sim = run(ics.turbulence(16))
sim.build_tree()
sim.find_neighbors()
sim.get_neighbors()
sim.finalize()
run(ics.sedov(16)).finalize()
w = ics.noh(14)
w.params = dataclasses.replace(w.params, dt_vsig=1, ngmax=400)
run(w).finalize()
w = ics.random_box(5000, seed=3)
w.params = dataclasses.replace(w.params, gradh=1, av_switch=1, dt_vsig=1, ve=1)
run(w).finalize()
w = ics.turbulence(16)
w.params = dataclasses.replace(w.params, gradh=1)
sim = run(w, accounting=sph.ACCOUNTING_PHASE)
for ph in ("keys", "sort", "neighbors", "density", "iad", "momentum_energy"):
    sim.build_tree(); sim.find_neighbors(); sim.density(); sim.eos(); sim.gradh(); sim.iad(); sim.momentum_energy()
    sim.repeat_phase(ph, 2)
sim.energy_report()
sim.finalize()
w = ics.turbulence(16)
si = ics.stir_inputs(sph.stir_modes(), 8)
sim = sph.Simulation(w.params, n_capacity=w.n, stir_steps=8)
sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
sim.set_time(0.0, w.params.dt_first, True)
sim.stir_init(si.sigma, si.t_decay, si.zeta, si.w, si.noise)
sim.step()
sim.finalize()
w = ics.evrard(12)
run(w, steps=1).finalize()
w = ics.evrard(12)
w.params = dataclasses.replace(w.params, grav_fp64=1)   # fp64 gravity terms
run(w, steps=1).finalize()
# search: coarse grid (multi-chunk streams, "full" periodic axes) and the
# merged-run path of the run table
run(ics.turbulence(12), steps=2, max_cell_level=2).finalize()
os.environ["SPH_NBR_MERGE_RUNS"] = "0"
run(ics.random_box(3000, seed=5, periodic=False), steps=2).finalize()
del os.environ["SPH_NBR_MERGE_RUNS"]
w = ics.sedov(14)
w.params = dataclasses.replace(w.params, av_switch=1)
ds = decomp.DistributedSim(w.params, w.state, n_capacity=w.n, device=0, force_exchange=True)
for _ in range(2):
    ds.step()
print("sanitize workload done")
