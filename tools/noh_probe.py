"""Probe: Noh implosion on the GPU (SURVEY 8(c) pin 'Noh': shock speed 1/3,
post-shock rho = 64 rho0 in 3D for gamma = 5/3, u = 1/2; pre-shock
rho = rho0 (1 + t/r)^2).  Prints the radial profile at t_end."""
import dataclasses
import sys
import time

import numpy as np

from paper_conf_sc_simsekpc24_b200 import ics, sph

nside = int(sys.argv[1]) if len(sys.argv) > 1 else 80
t_end = float(sys.argv[2]) if len(sys.argv) > 2 else 0.3
vsig = int(sys.argv[3]) if len(sys.argv) > 3 else 1
w = ics.noh(nside)
w.params = dataclasses.replace(w.params, dt_vsig=vsig, ngmax=400)
sim = sph.Simulation(w.params, n_capacity=w.n)
sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
sim.set_time(0.0, w.params.dt_first, True)
t, steps, t0 = 0.0, 0, time.time()
while t < t_end and steps < 5000:
    info = sim.step()
    t = info["t"]
    steps += 1
st = sim.get_state()
rho = sim.get_field("rho")
r = np.sqrt(st["x"] ** 2 + st["y"] ** 2 + st["z"] ** 2)
print(f"nside {nside} steps {steps} t {t:.4f} wall {time.time() - t0:.1f}s max_nc {info['max_nc']}")
edges = np.linspace(0, 0.4, 21)
for a, b in zip(edges[:-1], edges[1:]):
    m = (r >= a) & (r < b)
    if m.sum():
        rr = 0.5 * (a + b)
        pre = (1 + t / rr) ** 2
        vr = -(st["vx"][m] * st["x"][m] + st["vy"][m] * st["y"][m] + st["vz"][m] * st["z"][m]) / np.maximum(r[m], 1e-12)
        print(f"r {rr:.3f} n {m.sum():6d} rho {np.median(rho[m]):8.3f} pre-shock {pre:7.3f} "
              f"u {np.median(st['u'][m]):.4f} v_in {np.median(vr):.3f}")
