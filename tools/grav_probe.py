import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
"""Probe of the gravity phase: Barnes-Hut accuracy vs the oracle direct sum at a
few (level, theta), and the step time of Evrard at ~1M and ~8M particles."""
import dataclasses, time, json
import numpy as np, torch
import oracle
from paper_conf_sc_simsekpc24_b200 import ics, sph
out = {}
for nside, level, theta in ((24, 5, 0.5),):
    w = ics.evrard(nside); w.params = dataclasses.replace(w.params, grav_theta=theta, grav_level=level)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()}); sim.set_time(0, w.params.dt_first, True)
    sim.build_tree(); sim.find_neighbors(stats=False); sim.density(); sim.eos(); sim.iad(); sim.momentum_energy()
    b = {k: sim.get_field(k) for k in ("ax","ay","az")}; sim.gravity(); a = {k: sim.get_field(k) - b[k] for k in b}
    g = {k: sim.get_field(k) for k in ("x","y","z","m")}
    o = oracle.gravity(g["x"], g["y"], g["z"], g["m"], 1.0, w.params.grav_eps)
    A = np.stack([a["ax"], a["ay"], a["az"]], 1); B = np.stack([o["ax"], o["ay"], o["az"]], 1)
    err = np.linalg.norm(A - B, axis=1) / np.linalg.norm(B, axis=1)
    out[f"n{w.n}_L{level}_th{theta}"] = {"rms": float(np.sqrt(np.mean(err**2))), "p99": float(np.percentile(err, 99)), "max": float(err.max())}
    sim.finalize()
print(json.dumps(out))
# timing at ~1M and ~8M
for nside, level in ((124, 5), (124, 6), (124, 7)):
    w = ics.evrard(nside)
    w.params = dataclasses.replace(w.params, grav_level=level)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()}); sim.set_time(0, w.params.dt_first, True)
    for _ in range(3): info = sim.step()
    torch.cuda.synchronize(); t0 = time.perf_counter()
    for _ in range(5): info = sim.step()
    torch.cuda.synchronize(); dt = (time.perf_counter() - t0) / 5
    print(json.dumps({"evrard_n": w.n, "level": level, "ms_per_step": dt * 1e3, "phase_ms": info["phase_ms"], "mean_nc": info["mean_nc"], "max_nc": info["max_nc"],
                      "per_warp": {k: info[k] / (w.n / 32) for k in ("grav_multipoles", "grav_pairs", "grav_pops")}}))
    sim.finalize()
