"""Probe: cost of the decomposed step (decomp.py) at world = 1 against the plain
sph_step on the same workload, with a synchronising section timer."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import time

import numpy as np
import torch

from paper_conf_sc_simsekpc24_b200 import decomp, ics, sph

nside = int(sys.argv[1]) if len(sys.argv) > 1 else 200
w = ics.turbulence(nside)
ds = decomp.DistributedSim(w.params, w.state, n_capacity=int(1.2 * w.n), device=0, force_exchange=True)
for _ in range(3):
    ds.step()
torch.cuda.synchronize()
t0 = time.perf_counter()
K = 5
for _ in range(K):
    ds.step()
torch.cuda.synchronize()
print(f"decomposed world=1 (plumbing forced on): {1e3 * (time.perf_counter() - t0) / K:.2f} ms/step")
ds.profile = {}
for _ in range(K):
    ds.step()
print({k: round(1e3 * v / K, 2) for k, v in ds.profile.items()})
sim = ds.sim
sim.set_particles({k: v.contiguous() for k, v in ds.local.items()})
for _ in range(3):
    sim.step()
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(K):
    sim.step()
torch.cuda.synchronize()
print(f"plain sph_step: {1e3 * (time.perf_counter() - t0) / K:.2f} ms/step")
