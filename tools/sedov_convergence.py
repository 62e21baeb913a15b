"""Sedov blast wave at 40^3, 100^3 and 200^3 on the GPU to t = 0.05: shock radius
(median radius of the densest 0.3% of the particles) against the similarity
solution R(t) = xi0 (E t^2 / rho0)^(1/5), xi0 = 1.1517 (gamma = 5/3, E = rho0 =
1), and the peak compression, as the resolution grows (SURVEY 8(c) 'Sedov')."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_sc_simsekpc24_b200 import ics, sph  # noqa: E402

XI0 = 1.1517
out = []
for nside in [int(a) for a in (sys.argv[1:] or ["40", "100", "200"])]:
    w = ics.sedov(nside)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    t, steps, t0 = 0.0, 0, time.perf_counter()
    while t < 0.05 and steps < 20000:
        t = sim.step()["t"]
        steps += 1
    wall = time.perf_counter() - t0
    st = sim.get_state()
    rho = sim.get_field("rho")
    sim.finalize()
    r = np.sqrt(st["x"] ** 2 + st["y"] ** 2 + st["z"] ** 2)
    top = np.argsort(rho)[-max(200, int(0.003 * w.n)):]
    R_num = float(np.median(r[top]))
    R_th = XI0 * (t * t) ** 0.2
    out.append({"nside": nside, "n": int(w.n), "t": t, "steps": steps, "wall_s": round(wall, 1),
                "R_num": R_num, "R_similarity": R_th, "rel_err": (R_num - R_th) / R_th,
                "rho_peak_mean_top": float(rho[top].mean()), "rho_max": float(rho.max()),
                "strong_shock_limit": 4.0})
    print(json.dumps(out[-1]), flush=True)
