"""Writes tests/golden/sedov{N}_drift.json (N = argv[1], default 16): the
ORACLE's total-energy drift over a Sedov N^3 run to t >= 0.05 (reading 16).  Calls only oracle/ and the
input generator (no CUDA path).  Re-run after any change to the oracle's
arithmetic; tests/test_oracle_step.py recomputes it and must agree."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from paper_conf_sc_simsekpc24_b200 import ics  # noqa: E402

T_END = 0.05


def energy(s):
    return float((s["m"] * (0.5 * (s["vx"] ** 2 + s["vy"] ** 2 + s["vz"] ** 2) + s["u"])).sum())


def run(nside=16):
    w = ics.sedov(nside)
    s = {k: v.copy() for k, v in w.state.items()}
    E0 = energy(s)
    dt, t, k = w.params.dt_first, 0.0, 0
    Es = [E0]
    while t < T_END:
        s, out = oracle.step(s, w.params, dt, k == 0)
        dt = out["dt"]
        t += dt
        k += 1
        Es.append(energy(s))
    return {"steps": k, "t_end": t, "E0": E0, "E_end": Es[-1], "drift": Es[-1] / E0 - 1.0,
            "E_every_10": Es[::10]}


if __name__ == "__main__":
    nside = int(sys.argv[1]) if len(sys.argv) > 1 else 16
    r = run(nside)
    r["what"] = (f"oracle total energy sum m (v^2/2 + u), Sedov {nside}^3 (ics.sedov), stepped until "
                 "t >= 0.05; DESIGN.md reading 16")
    r["script"] = f"tools/golden_sedov_drift.py {nside}"
    path = os.path.join(ROOT, "tests", "golden", f"sedov{nside}_drift.json")
    with open(path, "w") as f:
        json.dump(r, f, indent=1)
    print(json.dumps({k: r[k] for k in ("steps", "t_end", "drift")}))
