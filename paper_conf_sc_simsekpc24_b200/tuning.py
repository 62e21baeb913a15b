"""Per-function GPU frequency tuning.

The paper tunes the SM clock of every SPH-EXA function separately: an isolated,
KernelTuner-style brute-force search over the supported clocks picks, per
function, the clock with the best energy-delay product (Fig. 2); the
whole simulation is then run with that clock set before each function
("ManDyn") and compared with statically locked clocks and with
the driver's DVFS (Figs. 6-8), normalised to the maximum clock
(P:178).  This module is that harness over libsph:

* ``phase_profile``   -- one function re-run back to back on the same inputs
  (``sph_repeat_phase``) for >= min_seconds, so that the NVML energy counter
  (which advances every ~100 ms on a B200, reading 12) resolves it:
  ms, J, W and EDP = J * s per call;
* ``frequency_search`` -- ``phase_profile`` of every function at each of
  ``nclocks`` supported clocks from the maximum down to ~half of it (the B200
  analog of the paper's 1410 -> 1005 MHz on A100), locking the clock with
  ``sph_set_clock_policy(STATIC)``; returns the table and the best-EDP clock per
  function;
* ``compare_policies`` -- whole steps under DVFS, static clocks and the
  per-function (ManDyn) policy: time, energy and EDP per step.

Locking clocks needs root and an explicit ``SPH_ALLOW_CLOCK_CONTROL=1`` (shared
hosts, like this project's B200 pool, forbid clock changes).  When the library
refuses, every function reports ``{"clock_control": "refused", "why": ...}`` and
still measures the DVFS arm, which is what the bench records.
"""
from __future__ import annotations

import json
import math
import time

from . import sph

REPEATABLE = ("keys", "sort", "cells", "neighbors", "density", "eos", "iad", "momentum_energy",
              "timestep")


def phase_profile(sim, phases=REPEATABLE, min_seconds: float = 1.0) -> dict:
    """{phase: {ms, J, W, EDP_Js}} per call, each phase repeated for >= min_seconds."""
    out = {}
    for ph in phases:
        ms1, _ = sim.repeat_phase(ph, 3)
        reps = max(3, int(math.ceil(min_seconds * 1e3 / max(ms1, 1e-3))))
        ms, J = sim.repeat_phase(ph, reps)
        row = {"ms": ms, "reps": reps}
        if J is not None:
            row.update({"J": J, "W": J / (ms * 1e-3), "EDP_Js": J * ms * 1e-3})
        out[ph] = row
    return out


def pick_clocks(supported, nclocks: int, low_frac: float = 0.5):
    """nclocks supported clocks from the maximum down to ~low_frac of it."""
    sup = sorted(supported, reverse=True)
    top = sup[0]
    cand = [f for f in sup if f >= low_frac * top]
    if nclocks >= len(cand):
        return cand
    step = (len(cand) - 1) / max(nclocks - 1, 1)
    return sorted({cand[int(round(k * step))] for k in range(nclocks)}, reverse=True)


def frequency_search(sim, phases=REPEATABLE, nclocks: int = 8, min_seconds: float = 1.0) -> dict:
    """Brute-force per-function clock search (Fig. 2 analog)."""
    try:
        clocks = pick_clocks(sim.supported_clocks(), nclocks)
    except sph.SphError as e:
        return {"clock_control": "unavailable", "why": str(e),
                "dvfs": phase_profile(sim, phases, min_seconds)}
    table = {}
    try:
        for f in clocks:
            sim.set_clock_policy(sph.CLOCK_STATIC, [f] + [0] * (sph.NPHASES - 1))
            table[f] = phase_profile(sim, phases, min_seconds)
    except sph.SphError as e:
        return {"clock_control": "refused", "why": str(e), "clocks": clocks,
                "dvfs": phase_profile(sim, phases, min_seconds)}
    finally:
        sim.set_clock_policy(sph.CLOCK_DEFAULT)
    best = {}
    for ph in phases:
        rows = [(table[f][ph].get("EDP_Js", float("inf")), f) for f in clocks]
        best[ph] = min(rows)[1]
    return {"clock_control": "ok", "clocks": clocks, "table": {str(f): v for f, v in table.items()},
            "best_mhz": best}


def _run_steps(sim, seconds: float):
    import torch
    e0 = sim.energy_counter_mj()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    steps = 0
    while time.perf_counter() - t0 < seconds or steps < 3:
        sim.step()
        steps += 1
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    e1 = sim.energy_counter_mj()
    J = (e1 - e0) * 1e-3 / steps if e0 is not None and e1 is not None else None
    ms = dt * 1e3 / steps
    return {"steps": steps, "ms_per_step": ms, "J_per_step": J,
            "EDP_Js": None if J is None else J * ms * 1e-3}


def compare_policies(sim, best_mhz: dict | None, static_clocks=(), seconds: float = 3.0) -> dict:
    """DVFS vs static clocks vs per-function ManDyn, whole steps (Figs. 6-8 analog),
    normalised to the first static clock (the maximum) when it could be set."""
    res = {"dvfs": _run_steps(sim, seconds)}
    try:
        for f in static_clocks:
            sim.set_clock_policy(sph.CLOCK_STATIC, [f] + [0] * (sph.NPHASES - 1))
            res[f"static_{f}"] = _run_steps(sim, seconds)
        if best_mhz:
            mhz = [int(best_mhz.get(p, 0)) for p in sph.PHASES]
            sim.set_clock_policy(sph.CLOCK_PER_PHASE, mhz)
            res["mandyn"] = _run_steps(sim, seconds)
    except sph.SphError as e:
        res["clock_control"] = "refused"
        res["why"] = str(e)
    finally:
        sim.set_clock_policy(sph.CLOCK_DEFAULT)
    if static_clocks and f"static_{static_clocks[0]}" in res:
        ref = res[f"static_{static_clocks[0]}"]
        for k, v in res.items():
            if isinstance(v, dict) and v.get("J_per_step") and ref.get("J_per_step"):
                v["rel_time"] = v["ms_per_step"] / ref["ms_per_step"]
                v["rel_energy"] = v["J_per_step"] / ref["J_per_step"]
                v["rel_EDP"] = v["EDP_Js"] / ref["EDP_Js"]
    return res


def main(argv=None):
    import argparse

    import numpy as np

    from . import ics
    ap = argparse.ArgumentParser(description=__doc__.split("\n\n")[0])
    ap.add_argument("--nside", type=int, default=100, help="turbulence nside^3 particles")
    ap.add_argument("--nclocks", type=int, default=8)
    ap.add_argument("--min-seconds", type=float, default=1.0)
    ap.add_argument("--policy-seconds", type=float, default=3.0)
    args = ap.parse_args(argv)
    w = ics.turbulence(args.nside)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    for _ in range(3):
        sim.step()
    sim.build_tree()
    sim.find_neighbors(stats=False)
    sim.density()
    sim.eos()
    sim.iad()
    sim.momentum_energy()
    sim.timestep()  # every repeatable function's inputs are now in place
    search = frequency_search(sim, nclocks=args.nclocks, min_seconds=args.min_seconds)
    clocks = search.get("clocks", [])
    statics = tuple(clocks[:1] + clocks[-1:]) if search.get("clock_control") == "ok" else ()
    policies = compare_policies(sim, search.get("best_mhz"), statics, args.policy_seconds)
    print(json.dumps({"workload": f"turbulence{args.nside}", "search": search, "policies": policies}))
    sim.finalize()


if __name__ == "__main__":
    main()
