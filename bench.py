#!/usr/bin/env python
"""Benchmark of the SPH time step (libsph) -- the driver's contract.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload turbulence200]
    python bench.py --impl reference ...      # the CPU oracle arm

A *step* is one full pass of the hot path (sph_step: keys, sort, cells,
neighbours, density, EOS, IAD, momentum-energy, dt, update) over the particle
state, which stays resident in HBM.  Metric (BASELINE.json): particle-updates/s
per SPH step.  Default workload: subsonic turbulence 200^3 (8M particles per
GPU; BASELINE.json configs[2], the north star's headline target).  Inputs are
~1 GB of particle state plus ~3 GB of neighbour lists per GPU, far larger than
the 126 MB L2, so no flush is needed between steps.

The JSON line carries: value (device-timed, CUDA events on libsph's stream,
max over ranks), e2e (the same metric through the C ABI with the state copied
from pinned host buffers in and back out every step), roofline (dominant
kernel: momentum-energy, FP64 pipe), energy (per-phase J/step from NVML in a
separate accounted pass), cpu_baseline (the oracle on a bounded sample),
clocks (nvidia-smi sampled during the timed region) and gpu_launches.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "particle-updates/s per SPH step"
UNIT = "particle-updates/s"

# Algorithmic FP64 flops per neighbour pair: SURVEY.md 8(d)'s counts (density
# 44, IAD 60, momentum-energy 171 incl. the artificial viscosity), the figures
# the roofline fractions are quoted against.  The DP
# instructions the kernels actually execute are counted by ncu
# (profiles/r02_dp_counts.json, 2 x DFMA + DMUL + DADD per pair) and reported
# beside them.
FLOPS_PER_PAIR = {"density": 44, "iad": 60, "momentum_energy": 171}
# FP64 peak: 148 SMs x 64 FP64 FMA/clk x 2 flop x 1.965 GHz, DERIVED from the
# guide's SM count and max SM clock (B200_PROFILING.md; MEASURED_PEAKS.json has
# no FP64 figure).  A DFMA microbenchmark on this B200 measured 34.1 TF/s
# (tools/probe_fp64.cu, profiles/r01_probe_fp64.json).
FP64_PEAK_TFLOPS = 148 * 64 * 2 * 1.965e9 / 1e12
FP64_PEAK_MEASURED_TFLOPS = 34.082
# Algorithmic HBM bytes per particle of the momentum-energy launch (i-side fields
# once, neighbour list once, outputs once): 19 doubles + nc + 4 B per neighbour + 4 doubles.
MOM_BYTES_PER_PARTICLE = 19 * 8 + 4 + 4 * 8   # + 4 * nc

# Per-phase algorithmic cost (DESIGN.md section 6 / SURVEY 8(d)): HBM bytes per
# particle (fields read and written once), + bytes per neighbour pair (the list
# entry), FP64 flops per pair, and the roofline that binds the phase.
PHASE_COST = {
    "keys": (40, 0, 0, "hbm"),
    "sort": (8 + 92 + 8 + 224, 0, 0, "hbm"),   # histogram, 4 radix passes (top digits), run fixup, permutation
    "cells": (8, 0, 0, "hbm"),
    "neighbors": (52, 4, 0, "issue"),          # pos4/x/y/z/h in, nc out, list out
    "density": (48, 4, FLOPS_PER_PAIR["density"], "fp64"),
    "eos": (112, 0, 0, "hbm"),               # rho is L2-resident after DENSITY: frac_hbm can exceed 1
    "gradh": (56, 4, 60, "fp64"),
    "iad": (96, 4, FLOPS_PER_PAIR["iad"], "fp64"),
    "momentum_energy": (MOM_BYTES_PER_PARTICLE, 4, FLOPS_PER_PAIR["momentum_energy"], "fp64"),
    "timestep": (0, 0, 0, "latency"),
    "update": (180, 0, 0, "hbm"),
}


def hbm_peak_gbs():
    """The driver-measured copy bandwidth (MEASURED_PEAKS.json), else the
    profiling guide's fallback."""
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return float(json.load(f)["hbm_gbs"]), "MEASURED_PEAKS.json hbm_gbs"
    except Exception:
        return 6540.8, "fallback (earlier measured copy bandwidth)"


def idle_power(sim, seconds=2.0):
    """Board power with the context alive and nothing running: NVML energy
    counter delta over `seconds` (P:73's whole-board energy includes it)."""
    e0 = sim.energy_counter_mj()
    if e0 is None:
        return None
    time.sleep(seconds)
    e1 = sim.energy_counter_mj()
    return (e1 - e0) * 1e-3 / seconds


def phase_table(phase_ms, pairs, n, energy, p_idle):
    """SURVEY 8(d)'s per-phase record: ms, algorithmic GB/s and TF/s with their
    roofline fractions, the binding bound, and (from the repeat-phase energy)
    J, J above idle and EDP = J x s."""
    peak, _ = hbm_peak_gbs()
    out = {}
    for name, ms in phase_ms.items():
        if ms <= 0 or name not in PHASE_COST:
            continue
        b_part, b_pair, f_pair, bound = PHASE_COST[name]
        t = ms * 1e-3
        gbs = (b_part * n + b_pair * pairs) / t / 1e9
        tfs = f_pair * pairs / t / 1e12
        row = {"ms": ms, "GBps": gbs, "frac_hbm": gbs / peak, "DP_TFLOPs": tfs,
               "frac_fp64": tfs / FP64_PEAK_TFLOPS, "bound": bound}
        e = (energy or {}).get("phases", {}).get(name)
        if e and e.get("J") is not None:
            row["J"] = e["J"]
            row["EDP_Js"] = e["J"] * e["ms"] * 1e-3
            if p_idle is not None:
                row["J_above_idle"] = e["J"] - p_idle * e["ms"] * 1e-3
        out[name] = row
    return out


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="turbulence200")
    ap.add_argument("--impl", default="libsph", choices=["libsph", "reference"])
    # (the pipelined e2e loop's fill -- the first input copy -- and drain -- the
    # last read-back -- are inside its timed region: 40 steps amortise them)
    ap.add_argument("--e2e-steps", type=int, default=40)
    ap.add_argument("--energy-seconds", type=float, default=10.0,
                    help="length of each energy window (the NVML counter ticks every ~100 ms / "
                         "~99 J on a B200: >= 10 s keeps a window within ~1%%); 0 = no energy")
    ap.add_argument("--energy-repeats", type=int, default=3,
                    help="whole-step energy windows (median and CV)")
    ap.add_argument("--timing-repeats", type=int, default=3,
                    help="extra blocks of --steps timed steps after the contract's block (median, CV)")
    ap.add_argument("--av-switch", action="store_true",
                    help="IADVelocityDivCurl div/curl + Balsara AV switch (SURVEY 8(f)-1)")
    ap.add_argument("--gradh", action="store_true",
                    help="NormalizationGradh phase, p/(Omega rho^2) in momentum (SURVEY 8(f)-1)")
    ap.add_argument("--ve", action="store_true",
                    help="generalized volume elements X = m/rho0 in XMass/NormalizationGradh (SURVEY 8(f)-1)")
    ap.add_argument("--dt-vsig", action="store_true",
                    help="signal-velocity time step (SURVEY 8(f)-1)")
    ap.add_argument("--stir", action="store_true",
                    help="turbulence driving (OU stirring, SURVEY 8(f)-3) inside every step")
    ap.add_argument("--trace-seconds", type=float, default=1.5,
                    help="seconds of steps under the NVML DVFS trace (Fig. 9); 0 = off")
    ap.add_argument("--cpu-sample", type=int, default=0, help="oracle targets (0 = auto)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--force-decomp", action="store_true",
                    help="N = 1: run the decomposed (N > 1) path on a one-rank NCCL group with every "
                         "collective issued (checks that path on one GPU; not a headline number)")
    ap.add_argument("--out", default=None)
    return ap.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def make_workload(name: str, rank: int):
    from paper_conf_sc_simsekpc24_b200 import ics
    if name.startswith("turbulence"):
        return ics.turbulence(int(name[len("turbulence"):]))
    import dataclasses
    # ngmax is a capacity (never a truncation): the shocked Sedov / Noh states of
    # a long run exceed the 150 of the turbulence preset
    if name.startswith("sedov"):
        w = ics.sedov(int(name[len("sedov"):]))
        w.params = dataclasses.replace(w.params, ngmax=256)
        return w
    if name.startswith("noh"):
        w = ics.noh(int(name[len("noh"):]))
        w.params = dataclasses.replace(w.params, ngmax=256)
        return w
    if name.startswith("evrard"):   # with self-gravity (Barnes-Hut, theta 0.5)
        return ics.evrard(int(name[len("evrard"):]))
    raise SystemExit(f"unknown workload {name}")


class ClockSampler:
    """SM clock, power and clock-event (throttle) reasons sampled every ~10 ms by
    an NVML thread during the timed region (nvidia-smi -lms 100 as fallback)."""

    REASONS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown"}

    def __init__(self, gpu_index: int, period_s: float = 0.01):
        self.gpu = gpu_index
        self.period = period_s
        self.samples = []
        self.p = None
        self.th = None

    def _nvml_loop(self, N, h):
        import time as _t
        while not self.stop:
            try:
                sm = N.nvmlDeviceGetClockInfo(h, N.NVML_CLOCK_SM)
                mx = N.nvmlDeviceGetMaxClockInfo(h, N.NVML_CLOCK_SM)
                pw = N.nvmlDeviceGetPowerUsage(h) / 1e3
                try:
                    rs = N.nvmlDeviceGetCurrentClocksEventReasons(h)
                except AttributeError:
                    rs = N.nvmlDeviceGetCurrentClocksThrottleReasons(h)
                self.samples.append((sm, mx, pw, rs))
            except Exception:
                pass
            _t.sleep(self.period)

    def __enter__(self):
        self.stop = False
        try:
            import threading
            import pynvml as N
            N.nvmlInit()
            h = None
            try:  # the CUDA device's own board (CUDA and NVML may enumerate differently)
                import torch
                pr = torch.cuda.get_device_properties(self.gpu)
                bus = f"{pr.pci_domain_id:08x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
                h = N.nvmlDeviceGetHandleByPciBusId(bus)
            except Exception:
                h = None
            if h is None:
                h = N.nvmlDeviceGetHandleByIndex(self.gpu)
            self.th = threading.Thread(target=self._nvml_loop, args=(N, h), daemon=True)
            self.th.start()
        except Exception:
            self.th = None
            try:
                self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), "--query-gpu=clocks.sm,clocks.max.sm,"
                                           "power.draw,clocks_event_reasons.active", "--format=csv,noheader,nounits",
                                           "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            except OSError:
                self.p = None
        time.sleep(0.05)
        return self

    def __exit__(self, *a):
        self.stop = True
        if self.th:
            self.th.join(timeout=2)
        if self.p:
            time.sleep(0.25)
            self.p.terminate()
            out, _ = self.p.communicate(timeout=10)
            for l in out.splitlines():
                f = [x.strip() for x in l.split(",")]
                try:
                    self.samples.append((float(f[0]), float(f[1]), float(f[2]), int(f[3], 16)))
                except (ValueError, IndexError):
                    pass

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        reasons = set()
        counts = {}
        for _, _, _, rs in self.samples:
            for bit, name in self.REASONS.items():
                if rs & bit:
                    reasons.add(name)
                    counts[name] = counts.get(name, 0) + 1
        return {"sm_mhz": statistics.median(x[0] for x in self.samples),
                "sm_max_mhz": max(x[1] for x in self.samples), "reasons": sorted(reasons),
                "reason_samples": counts,
                "power_w_median": statistics.median(x[2] for x in self.samples), "samples": len(self.samples),
                "source": "NVML thread, ~10 ms period" if self.th else "nvidia-smi -lms 100"}


def cpu_baseline(w, n_targets: int, seed: int = 3, keep: dict | None = None, dt_override=None):
    """The oracle as it stands on a bounded sample: one step at n_targets random
    particles of the same workload (sampled mode: exact global sort/dt, each
    target's dependency ball brute-forced).  Returns (targets/s, seconds, threads)."""
    import numpy as np
    import oracle
    rng = np.random.default_rng(seed)
    tg = np.sort(rng.choice(w.n, size=n_targets, replace=False))
    t0 = time.perf_counter()
    res = oracle.sample_step({k: v for k, v in w.state.items()}, w.params, w.params.dt_first, True, tg,
                             dt=dt_override) if dt_override is not None else \
        oracle.sample_step({k: v for k, v in w.state.items()}, w.params, w.params.dt_first, True, tg)
    dt = time.perf_counter() - t0
    threads = int(os.environ.get("OMP_NUM_THREADS", os.cpu_count() or 1))
    if keep is not None:
        keep.update({"targets": tg, "order": res[0], "out": res[1]})
    return n_targets / dt, dt, threads


def gpu_first_step(sim, w):
    """The staged first step of the workload's initial state on `sim` (for the
    per-run parity block); returns the GPU fields in the step's sorted order."""
    import numpy as np
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    sim.build_tree()
    sim.find_neighbors(stats=False)
    sim.density()
    sim.eos()
    if sim.cfg.gradh or sim.cfg.ve:
        sim.gradh()
    sim.iad()
    sim.momentum_energy()
    g = {k: sim.get_field(k) for k in ("id", "rho", "p", "c", "ax", "ay", "az", "du")}
    g["C"] = np.stack([sim.get_field(k) for k in ("c11", "c12", "c13", "c22", "c23", "c33")], 1)
    g["sim"] = sim
    g["dt"] = sim.timestep()
    return g


def parity_block(sim, g, ref):
    """SURVEY 8(d)'s per-run parity record: the bench workload's first step on
    the GPU against the oracle's sampled mode at the cpu_baseline targets (the
    same oracle run): Morton order of all particles, neighbour lists, dt, and
    the largest error of each field in the DESIGN.md section 3 metric."""
    import numpy as np
    tg, o = ref["targets"], ref["out"]
    off, idx = sim.get_neighbor_rows(tg)
    nbr_exact = all(np.array_equal(idx[off[q]:off[q + 1]].astype(np.int64), o["nbrs"][q]) for q in range(len(tg)))
    sim.update()
    after = {k: sim.get_field(k) for k in ("x", "y", "z", "vx", "vy", "vz", "u", "h")}
    err = {}

    def rel(a, b, scale):
        return float(np.max(np.abs(a - b) / np.maximum(scale, 1e-300)))
    err["rho"] = rel(g["rho"][tg], o["rho"], np.abs(o["rho"]))
    err["p"] = rel(g["p"][tg], o["p"], np.abs(o["p"]))
    err["c"] = rel(g["c"][tg], o["c"], np.abs(o["c"]))
    Cn = np.linalg.norm(o["C"], axis=1)
    err["C"] = max(rel(g["C"][tg, e], o["C"][:, e], Cn) for e in range(6))
    for a, k in enumerate(("ax", "ay", "az")):
        err[k] = rel(g[k][tg], o[k], o["a_abs"][:, a])
    err["du"] = rel(g["du"][tg], o["du"], o["du_abs"])
    L = float(np.max(np.asarray(o["bmax"]) - np.asarray(o["bmin"])))
    err["x"] = max(rel(after[k][tg], o[k], np.full(len(tg), L)) for k in ("x", "y", "z"))
    vs = max(np.abs(np.concatenate([o["vx"], o["vy"], o["vz"]])).max(), 1e-300)
    err["v"] = max(rel(after[k][tg], o[k], np.maximum(np.abs(o[k]), vs)) for k in ("vx", "vy", "vz"))
    err["u"] = rel(after["u"][tg], o["u"], np.abs(o["u"]))
    err["h"] = rel(after["h"][tg], o["h"], np.abs(o["h"]))
    return {"targets": int(len(tg)), "order_exact": bool(np.array_equal(g["id"], ref["order"])),
            "nbr_exact": bool(nbr_exact), "dt_exact": bool(g["dt"] == o["dt"]),
            "max_err_by_field": err, "tolerance": 1e-10,
            "pass": bool(nbr_exact and np.array_equal(g["id"], ref["order"]) and max(err.values()) <= 1e-10),
            "what": "first step of the bench workload, GPU vs oracle.sample_step at the cpu_baseline targets"}


def _cv(xs):
    return statistics.pstdev(xs) / statistics.mean(xs) if len(xs) > 1 and statistics.mean(xs) else 0.0


def cpu_physics_only(w, m: int = 32768):
    """SURVEY 8(d)'s fair per-kernel CPU baseline: the oracle's physics only
    (density, EOS, IAD, momentum-energy), GIVEN the neighbour lists, per
    particle -- on the first m particles of the workload in Morton order (a
    compact block; lists from the oracle's brute force, not timed)."""
    import numpy as np
    import oracle
    s = w.state
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], w.params)
    k = oracle.keys(s["x"], s["y"], s["z"], bmin, bmax)
    sel = oracle.sort_order(k)[:min(m, w.n)]
    st = {f: np.ascontiguousarray(s[f][sel]) for f in oracle.STATE_KEYS}
    nb = oracle.neighbors(st["x"], st["y"], st["z"], st["h"], bmin, bmax, w.params.periodic)
    P = w.params
    t0 = time.perf_counter()
    rho = oracle.density(st["x"], st["y"], st["z"], st["h"], st["m"], bmin, bmax, P.periodic, nb, P)
    p, c = oracle.eos(rho, st["u"], P)
    Cm, _, _, _ = oracle.iad(st["x"], st["y"], st["z"], st["h"], st["m"], rho, bmin, bmax, P.periodic, nb, P)
    oracle.momentum_energy(st["x"], st["y"], st["z"], st["vx"], st["vy"], st["vz"], st["h"], st["m"], rho, p, c,
                           Cm, bmin, bmax, P.periodic, nb, P)
    dt = time.perf_counter() - t0
    return {"s_per_particle": dt / sel.size, "particle_updates_per_s": sel.size / dt, "particles": int(sel.size),
            "mean_nc": float(nb.nc.mean()), "seconds": dt,
            "what": "oracle density+EOS+IAD+momentum-energy given the neighbour lists (C, OpenMP over targets)"}


def measure_energy(sim, sph, n, args, gpu_index, ms_off):
    """Per-step and per-phase energy at default DVFS clocks.

    * Whole step, in situ: `energy_repeats` windows of >= `energy_seconds` of
      back-to-back steps with PHASE accounting on (no phase-edge syncs: a host
      thread integrates the NVML instant power per device-tagged phase).  Per
      window: J/step from the NVML total-energy counter, the sampled integral of
      P dt (the accounting's self-check: counter vs integral), the sum of the
      per-phase joules, and the accounting's time overhead vs OFF.  The instant
      power refreshes every ~100 ms on a B200, so in-situ per-phase joules are
      TIME-APPORTIONED (each phase's device time at the power around it).
    * Per phase, isolated: the KernelTuner-style repetition of P:81-87 -- each
      repeatable phase re-run on the same inputs for >= `energy_seconds`
      (sph_repeat_phase; counter delta / reps), with the SM clock sampled
      meanwhile (Fig. 9's DVFS clock).  UPDATE (not repeatable: it advances the
      state) takes time x the step's average power.
    """
    import torch
    torch.cuda.synchronize()
    if sim.energy_counter_mj() is None:
        return {"available": False, "why": "NVML energy counter unavailable"}
    T = args.energy_seconds
    windows = []
    insitu = None
    for r in range(max(args.energy_repeats, 1)):
        sim.set_accounting(sph.ACCOUNTING_PHASE)
        sim.energy_reset()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with ClockSampler(gpu_index) as clk:
            t0 = time.perf_counter()
            ev0.record(sim.stream)
            k = 0
            while time.perf_counter() - t0 < T:
                sim.step()
                k += 1
            ev1.record(sim.stream)
            torch.cuda.synchronize()
        tot = sim.energy_totals()
        rows = sim.energy_report()
        sim.set_accounting(sph.ACCOUNTING_OFF)
        ms = ev0.elapsed_time(ev1) / k
        cj = tot["counter_joules"]
        ph = {x["name"]: x["joules"] / k for x in rows if x["calls"] and x["joules"] is not None}
        windows.append({"steps": k, "seconds": tot["wall_seconds"], "ms_per_step": ms,
                        "J_per_step_counter": cj / k if cj is not None else None,
                        "J_per_step_sampled": tot["sampled_joules"] / k,
                        "counter_over_sampled": (cj / tot["sampled_joules"]) if cj and tot["sampled_joules"] else None,
                        "phase_J_sum_over_step": (sum(ph.values()) / (cj / k)) if cj else None,
                        "between_phases_J_per_step": tot["between_joules"] / k,
                        "overhead_pct_vs_off": 100.0 * (ms / ms_off - 1.0),
                        "clocks": clk.summary()})
        if r == 0:
            insitu = ph
    step_J = [w["J_per_step_counter"] for w in windows if w["J_per_step_counter"] is not None]
    step_ms = [w["ms_per_step"] for w in windows]
    J = statistics.median(step_J)
    out = {"available": True,
           "counter": "nvmlDeviceGetTotalEnergyConsumption (mJ, ~100 ms / ~99 J update)",
           "power_sensor": "NVML_FI_DEV_POWER_INSTANT, refreshed ~every 100 ms (profiles/r02_probe_nvml_instant.json)",
           "clock_policy": ("default DVFS: SM clock locking is implemented (sph_set_clock_policy) but "
                            "not exercised -- this shared host forbids clock changes"),
           "step": {"windows": windows, "J_median": J, "J_cv": _cv(step_J), "ms_median": statistics.median(step_ms),
                    "W": J / (statistics.median(step_ms) * 1e-3)},
           "uJ_per_particle_update": J / n * 1e6,
           "in_situ_phase_J_per_step": {"kind": "time-apportioned (PHASE accounting, sampled P dt per device-tagged phase)",
                                        "J": insitu},
           "phases": {}}
    # one more step, stopped before the update so every repeatable phase has its inputs
    sim.build_tree()
    sim.find_neighbors(stats=False)
    sim.density()
    sim.eos()
    if sim.cfg.gradh or sim.cfg.ve:
        sim.gradh()
    sim.iad()
    sim.momentum_energy()
    sim.timestep()
    # (with volume elements DENSITY would overwrite the normalised rho and GRADH
    # rewrites rho from itself: neither is repeatable after the step's GRADH)
    for ph in ("keys", "sort", "cells", "neighbors") + (() if sim.cfg.ve else ("density",)) + ("eos",) + (
            ("gradh",) if sim.cfg.gradh and not sim.cfg.ve else ()) + ("iad", "momentum_energy", "timestep"):
        ms1, _ = sim.repeat_phase(ph, 3)
        reps = int(min(2000000, max(5, 1e3 * T / max(ms1, 1e-4))))
        with ClockSampler(gpu_index) as c2:
            ms, Jp = sim.repeat_phase(ph, reps)
        out["phases"][ph] = {"ms": ms, "J": Jp, "W": (Jp / (ms * 1e-3)) if Jp else None, "reps": reps,
                             "window_s": ms * reps * 1e-3, "sm_mhz": c2.summary().get("sm_mhz")}
    sim.update()
    ms_upd = sim.step()["phase_ms"]["update"]
    W = out["step"]["W"]
    out["phases"]["update"] = {"ms": ms_upd, "J": ms_upd * 1e-3 * W, "W": W,
                               "reps": 0, "note": "not repeatable; step-average power x time"}
    out["repeat_phase_J_sum_over_step"] = sum(p["J"] or 0.0 for p in out["phases"].values()) / J
    return out


def dvfs_trace(sim, sph, seconds):
    """Fig. 9 analog: SM clock and board power the driver picks while
    each phase runs, from sph_trace_start's NVML sampling thread over ~`seconds`
    of back-to-back steps at default (DVFS) clocks.  Samples are tagged with the
    phase the device is executing (a device-written marker, not host timing)."""
    import time
    import numpy as np
    try:
        sim.trace_start(period_ms=1.0, capacity=1 << 18)
    except sph.SphError as e:
        return {"available": False, "why": str(e)}
    t0 = time.perf_counter()
    steps = 0
    while time.perf_counter() - t0 < seconds:
        sim.step()
        steps += 1
    tr = sim.trace_stop(capacity=1 << 18)
    out = {"available": True, "steps": steps, "samples": int(tr.size),
           "query_ms_median": float(np.median(tr["query_us"])) / 1e3 if tr.size else None,
           "phases": {}}
    for p, name in enumerate(sph.PHASES):
        sel = tr[tr["phase"] == p]
        if sel.size:
            out["phases"][name] = {"samples": int(sel.size),
                                   "sm_mhz_median": float(np.median(sel["sm_mhz"])),
                                   "power_w_mean": float(sel["power_mw"].mean()) / 1e3}
    gap = tr[tr["phase"] < 0]
    if gap.size:
        out["between_phases"] = {"samples": int(gap.size), "sm_mhz_median": float(np.median(gap["sm_mhz"]))}
    return out


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle timed on this host's cores (rank 0 only)."""
    if rank != 0:
        return
    w = make_workload(args.workload, rank)
    k = args.cpu_sample or 48
    vals = []
    for s in range(args.warmup + args.steps):
        v, sec, threads = cpu_baseline(w, k, seed=100 + s)
        if s >= args.warmup:
            vals.append((v, sec))
    tot_t = sum(s for _, s in vals)
    value = k * len(vals) / tot_t
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": 0, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * tot_t / len(vals), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": args.workload, "n_particles": w.n, "parallelism": "cpu-openmp"},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle",
                             "sample": f"{k} random targets per step of {args.workload} (oracle sampled mode)"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_decomposed(args, rank, world, local, forced=False):
    """N > 1: SFC domain decomposition with halo exchange over NCCL (decomp.py),
    weak scaling: turbulence with ~8M particles per GPU in one periodic box
    (nside = round(200 N^(1/3)): 252^3, 317^3, 400^3 at N = 2, 4, 8 -- SURVEY
    8(d) config 5).  Each rank draws its slice of the initial conditions."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_simsekpc24_b200 import decomp, ics, sph

    base = int(args.workload[len("turbulence"):]) if args.workload.startswith("turbulence") else 200
    nside = int(round(base * world ** (1.0 / 3.0)))
    w = ics.turbulence_part(nside, rank, world)
    vsq = torch.tensor([w.meta["vsq_sum"]], dtype=torch.float64, device="cuda")
    dist.all_reduce(vsq)
    ics.normalise_velocity(w, float(vsq.item()))
    n_total = nside ** 3
    cap = int(1.4 * n_total / world) + 1024
    ds = decomp.DistributedSim(w.params, w.state, n_capacity=cap, device=local,
                               force_exchange=forced, comm_always=forced)
    del w
    stream = ds.sim.stream  # every event on the stream the step's kernels run on

    def barrier():
        dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        ds.step()
    barrier()
    l0 = sph.kernel_launches()
    ds.sim.energy_reset()
    e_start = ds.sim.energy_counter_mj()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        barrier()
        ev0.record(stream)
        for _ in range(args.steps):
            ds.step()
        ev1.record(stream)
        barrier()
    e_end = ds.sim.energy_counter_mj()
    ms = torch.tensor([ev0.elapsed_time(ev1)], device="cuda")
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    ms_max = float(ms.item())
    rows = ds.sim.energy_report()
    phase_ms = {r["name"]: 1e3 * r["seconds"] / args.steps for r in rows}
    joules = torch.tensor([(e_end - e_start) * 1e-3 if e_start is not None and e_end is not None else 0.0],
                          device="cuda", dtype=torch.float64)
    dist.all_reduce(joules)
    ghosts = torch.tensor([ds.stats["n_ghost"], ds.stats["n_local"]], device="cuda", dtype=torch.float64)
    dist.all_reduce(ghosts)
    launches = sph.kernel_launches() - l0
    # roofline of the dominant kernel on rank 0 (its momentum-energy phase time,
    # interior + boundary launches, over its own targets' pairs of the last step)
    roofline = None
    if rank == 0:
        import numpy as np
        nc = ds.sim.get_field("nc")
        pairs0 = float(np.minimum(nc, ds.sim.cfg.ngmax).sum())
        mom_s = phase_ms.get("momentum_energy", 0.0) * 1e-3
        if mom_s > 0 and pairs0 > 0:
            ach = FLOPS_PER_PAIR["momentum_energy"] * pairs0 / mom_s / 1e12
            roofline = {"bound": "alu", "achieved": ach, "peak": FP64_PEAK_TFLOPS, "unit": "TFLOP/s",
                        "frac": ach / FP64_PEAK_TFLOPS, "traffic": None, "kernel": "momentum_energy_kernel",
                        "flops_per_pair": FLOPS_PER_PAIR["momentum_energy"], "scope": "rank 0",
                        "peak_source": "derived: 148 SM x 64 DFMA/clk x 2 x 1.965 GHz",
                        "frac_of_measured_peak": ach / FP64_PEAK_MEASURED_TFLOPS}
    # e2e: each rank's particles copied in from pinned host memory and back out
    # (into pinned buffers of the rank's capacity: the local count varies) every step
    loc = ds.local
    nloc = next(iter(loc.values())).shape[0]
    pinned = {k: torch.empty((cap,), dtype=v.dtype).pin_memory() for k, v in loc.items()}
    for k, v in loc.items():
        pinned[k][:nloc].copy_(v)
    del loc
    h2d = d2h = 0
    barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(max(args.e2e_steps, 1)):
        with torch.cuda.stream(stream):  # the copies in the step's stream order
            ds.local = {k: v[:nloc].to("cuda", non_blocking=True) for k, v in pinned.items()}
        h2d = sum(v[:nloc].numel() * v.element_size() for v in pinned.values())
        ds.step()
        with torch.cuda.stream(stream):
            loc = ds.local
            nloc = next(iter(loc.values())).shape[0]
            for k, v in loc.items():
                pinned[k][:nloc].copy_(v, non_blocking=True)
        stream.synchronize()
        d2h = sum(v[:nloc].numel() * v.element_size() for v in pinned.values())
    e1.record(stream)
    barrier()
    ems = torch.tensor([e0.elapsed_time(e1)], device="cuda")
    dist.all_reduce(ems, op=dist.ReduceOp.MAX)
    if rank == 0:
        value = n_total * args.steps / (ms_max * 1e-3)
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": f"turbulence{nside}", "n_particles_total": n_total,
                           "n_particles_per_gpu": n_total / world,
                           "parallelism": (f"SFC domain decomposition over {world} GPUs, halo exchange ({dist.get_backend().upper()})"
                                           + (" -- forced at N = 1: every collective issued on a one-rank group" if forced else "")),
                           "ghost_fraction": float(ghosts[0] / ghosts[1]),
                           "l2": "inputs >> 126 MB L2; no flush"},
                "phase_ms_rank0": phase_ms, "roofline": roofline,
                "e2e": {"value": n_total * max(args.e2e_steps, 1) / (float(ems.item()) * 1e-3), "unit": UNIT,
                        "h2d_bytes_per_step": h2d * world, "d2h_bytes_per_step": d2h * world,
                        "path": "rank-local state from pinned host -> DistributedSim.step -> host"},
                "energy": {"J_per_step_all_gpus": float(joules.item()) / args.steps,
                           "uJ_per_particle_update": float(joules.item()) / args.steps / n_total * 1e6},
                "cpu_baseline": None, "clocks": clk.summary(), "gpu_launches": launches}
        print(json.dumps(line), flush=True)
    dist.destroy_process_group()


def main():
    args = parse()
    rank, world, local = dist_env()
    if args.impl == "reference":
        return run_reference(args, rank, world)

    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_sc_simsekpc24_b200 import sph

    if world == 1 and args.force_decomp:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29511")
        os.environ.setdefault("RANK", "0")
        os.environ.setdefault("WORLD_SIZE", "1")
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", init_method="env://", device_id=torch.device("cuda", local))
        return run_decomposed(args, rank, world, local, forced=True)
    if world > 1:
        # SPH_DIST_BACKEND=gloo lets several ranks share one GPU (tests); NCCL otherwise
        backend = os.environ.get("SPH_DIST_BACKEND", "nccl")
        local = local % torch.cuda.device_count()
        torch.cuda.set_device(local)
        if backend == "nccl":
            dist.init_process_group("nccl", init_method="env://", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend, init_method="env://")
        return run_decomposed(args, rank, world, local)
    torch.cuda.set_device(local)
    w = make_workload(args.workload, rank)
    n = w.n
    if args.av_switch or args.gradh or args.dt_vsig or args.ve:
        import dataclasses
        w.params = dataclasses.replace(w.params, av_switch=int(args.av_switch), ve=int(args.ve),
                                       gradh=int(args.gradh), dt_vsig=int(args.dt_vsig))
    stir_steps = 8192 if args.stir else 0
    sim = sph.Simulation(w.params, n_capacity=n, device=local, stir_steps=stir_steps)
    stream = sim.stream
    if args.stir:
        from paper_conf_sc_simsekpc24_b200 import ics
        si = ics.stir_inputs(sph.stir_modes(), stir_steps)
        sim.stir_init(si.sigma, si.t_decay, si.zeta, si.w, si.noise)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    host_state = {k: np.ascontiguousarray(v) for k, v in w.state.items()}
    sim.set_particles(host_state)
    sim.set_time(0.0, w.params.dt_first, True)

    infos = []
    for _ in range(args.warmup):
        sim.step()
    barrier()
    launches0 = sph.kernel_launches()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    mom_ms = []
    with ClockSampler(local) as clk:
        barrier()
        ev0.record(stream)
        for _ in range(args.steps):
            info = sim.step()
            infos.append(info)
            mom_ms.append(info["phase_ms"]["momentum_energy"])
        ev1.record(stream)
        barrier()
    launches = sph.kernel_launches() - launches0
    ms = ev0.elapsed_time(ev1)
    # >= 3 repeats, median and CV (extra blocks of K steps, after
    # the contract's timed block, which alone gives `value`)
    rep_ms = [ms / args.steps]
    for _ in range(max(args.timing_repeats, 0)):
        r0, r1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        barrier()
        r0.record(stream)
        for _ in range(args.steps):
            sim.step()
        r1.record(stream)
        barrier()
        rep_ms.append(r0.elapsed_time(r1) / args.steps)
    repeats = {"blocks": len(rep_ms), "steps_per_block": args.steps, "ms_per_step": rep_ms,
               "median": statistics.median(rep_ms), "cv": _cv(rep_ms)}
    ms_t = torch.tensor([ms], device="cuda")
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms_max = float(ms_t.item())
    value = n * world * args.steps / (ms_max * 1e-3)
    phase_ms = {p: statistics.mean(i["phase_ms"][p] for i in infos) for p in sph.PHASES}
    mean_nc = statistics.mean(i["mean_nc"] for i in infos)

    # --- roofline of the dominant kernel (momentum-energy; FP64 pipe) ---
    pairs = mean_nc * n
    mom_s = statistics.mean(mom_ms) * 1e-3
    achieved = FLOPS_PER_PAIR["momentum_energy"] * pairs / mom_s / 1e12
    traffic = None
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            traffic = json.load(f)["momentum_energy_kernel"]["dram_bytes_per_launch"]
    except (OSError, KeyError, ValueError):
        pass
    dp = {}
    try:
        with open(os.path.join(ROOT, "profiles", "r02_dp_counts.json")) as f:
            dp = json.load(f)["kernels"]
    except (OSError, KeyError, ValueError):
        pass

    def counted(kernel, t):
        c = dp.get(kernel)
        if not c:
            return None
        fl = c["dp_flops_per_pair"] * pairs / t / 1e12
        return {"dp_flops_per_pair": c["dp_flops_per_pair"], "tflops": fl, "frac": fl / FP64_PEAK_TFLOPS,
                "source": "ncu sm__sass_thread_inst_executed_op_{dfma,dmul,dadd}_pred_on (profiles/r02_dp_counts.json)"}

    roofline = {"bound": "alu", "achieved": achieved, "peak": FP64_PEAK_TFLOPS, "unit": "TFLOP/s",
                "frac": achieved / FP64_PEAK_TFLOPS, "traffic": traffic,
                "traffic_unit": "DRAM bytes per launch (ncu --set full, profiles/ncu_traffic.json)",
                "algorithmic_bytes_per_launch": (MOM_BYTES_PER_PARTICLE + 4 * mean_nc) * n,
                "kernel": "momentum_energy_kernel",
                "flops_per_pair": FLOPS_PER_PAIR["momentum_energy"],
                "flops_source": "SURVEY.md 8(d) algorithmic count (171 per pair incl. the AV)",
                "peak_source": "derived: 148 SM x 64 DFMA/clk x 2 x 1.965 GHz (guide's unit counts and max clock)",
                "peak_measured_dfma_probe": FP64_PEAK_MEASURED_TFLOPS,
                "frac_of_measured_peak": achieved / FP64_PEAK_MEASURED_TFLOPS,
                "counted": counted("momentum_energy_kernel", mom_s),
                "hbm_GBps_algorithmic": (MOM_BYTES_PER_PARTICLE + 4 * mean_nc) * n / mom_s / 1e9,
                "share_of_step": statistics.mean(mom_ms) / (ms_max / args.steps)}
    other = {}
    for p, kname in (("density", "density_kernel"), ("iad", "iad_kernel")):
        t = phase_ms[p] * 1e-3
        other[p] = {"flops_per_pair": FLOPS_PER_PAIR[p], "tflops": FLOPS_PER_PAIR[p] * pairs / t / 1e12,
                    "frac_fp64": FLOPS_PER_PAIR[p] * pairs / t / 1e12 / FP64_PEAK_TFLOPS,
                    "counted": counted(kname, t)}

    # --- e2e: same metric through the C ABI with host buffers ---
    # Every step copies its input state in from pinned host memory
    # (sph_set_particles) and reads the updated state back (sph_get_field x 11).
    # Two contexts alternate: step s+1's input is copied from pinned host
    # memory (H2D) on a copy stream into a device staging buffer while step s
    # computes and step s-1's read-back (D2H, sph_get_field async) runs on the
    # other context's stream; sph_set_particles then moves the staged input in
    # on that context's stream (device to device).  Both copy directions and the
    # compute overlap (what a production loop with asynchronous I/O does; 704 MB
    # each way per step at 8M, the host link does ~78 GB/s both ways together,
    # tools/link_probe.py).  With the H2D on the context's own stream it queued
    # behind that stream's D2H (~26.6 ms of serial copies per 24.4 ms step).
    # The sequential variant (copy in, step, copy out, no overlap) is reported
    # beside it.
    e2e = None
    if args.e2e_steps > 0:
        pinned = {k: torch.from_numpy(v).pin_memory() for k, v in sim.get_state().items()}
        h2d = sum(v.numel() * v.element_size() for v in pinned.values())
        d2h = h2d
        NCTX = 2
        sims = [sim] + [sph.Simulation(w.params, n_capacity=n, device=local) for _ in range(NCTX - 1)]
        copy_stream = torch.cuda.Stream(device=local)
        stage = [{k: torch.empty(v.shape, dtype=v.dtype, device=f"cuda:{local}") for k, v in pinned.items()}
                 for _ in sims]
        staged = [torch.cuda.Event() for _ in sims]  # stage[c] consumed by context c
        t_now, dtp, first = sim.get_time()
        for sm in sims:
            sm.set_time(t_now, dtp, first)
        outs = [{k: torch.empty_like(v).pin_memory() for k, v in pinned.items()} for _ in sims]

        def timed(fn):
            barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(sims[0].stream)
            for sm in sims:
                sm.stream.wait_event(e0)
            fn()
            for sm in sims[1:]:
                ev = torch.cuda.Event()
                ev.record(sm.stream)
                sims[0].stream.wait_event(ev)
            e1.record(sims[0].stream)
            barrier()
            t = torch.tensor([e0.elapsed_time(e1)], device="cuda")
            if world > 1:
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
            return float(t.item())

        def load(c):
            """H2D of the input into stage[c] on the copy stream, then into context c."""
            copy_stream.wait_event(staged[c])
            with torch.cuda.stream(copy_stream):
                for k, v in pinned.items():
                    stage[c][k].copy_(v, non_blocking=True)
                sims[c].set_particles(stage[c])  # its stream waits for the copy stream
            staged[c].record(sims[c].stream)

        def pipelined():
            K = args.e2e_steps
            load(0)
            for s_ in range(K):
                cur = sims[s_ % NCTX]
                if s_ + 1 < K:
                    load((s_ + 1) % NCTX)             # step s+1's input
                cur.step()                             # host waits for this step only
                for k, v in outs[s_ % NCTX].items():
                    cur.get_field(k, out=v, async_=True)  # read-back overlaps the next step
            for sm in sims:
                sm.sync()

        def sequential():
            for _ in range(args.e2e_steps):
                sim.set_particles(pinned)
                sim.step()
                for k, v in outs[0].items():
                    sim.get_field(k, out=v)

        pipelined()  # untimed: each context's first steps capture its step graphs
        ms_pipe = timed(pipelined)
        ms_seq = timed(sequential)
        for sm in sims[1:]:
            sm.finalize()
        e2e = {"value": n * world * args.e2e_steps / (ms_pipe * 1e-3), "unit": UNIT,
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
               "path": ("two libsph contexts alternating: step s+1's input H2D from pinned host (copy stream, "
                        "then sph_set_particles device-to-device) and step s-1's sph_get_field x11 (pinned host, "
                        "SPH_MEM_HOST_ASYNC) overlap sph_step of step s"),
               "sequential": {"value": n * world * args.e2e_steps / (ms_seq * 1e-3),
                              "path": "sph_set_particles(pinned host) + sph_step + sph_get_field x11 (host), no overlap"}}

    p_idle = idle_power(sim) if args.energy_seconds > 0 else None
    energy = measure_energy(sim, sph, n, args, local, ms_max / args.steps) if args.energy_seconds > 0 else None
    if energy is not None and p_idle is not None:
        energy["idle_W"] = p_idle
    accounting = None
    if energy and energy.get("available"):
        ws = energy["step"]["windows"]
        accounting = {"mode": "phase (in situ, no phase-edge syncs; sampled instant power per device-tagged phase)",
                      "overhead_pct": statistics.median(w["overhead_pct_vs_off"] for w in ws),
                      "counter_over_sampled": [w["counter_over_sampled"] for w in ws],
                      "phase_J_sum_over_step": [w["phase_J_sum_over_step"] for w in ws]}
    trace = dvfs_trace(sim, sph, args.trace_seconds) if args.trace_seconds > 0 else None

    cpu = None
    parity = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline and w.params.gravity:
        cpu = {"unavailable": "gravity is long-range: the sampled oracle has no finite dependency ball",
               "physics_only": cpu_physics_only(w)}
    elif rank == 0 and world == 1 and not args.no_cpu_baseline:
        k = args.cpu_sample or 240  # ~10 s of oracle work on the host cores
        ref = {}
        gfirst = gpu_first_step(sim, w)
        v, sec, threads = cpu_baseline(w, k, keep=ref, dt_override=gfirst["dt"] if w.params.dt_vsig else None)
        phys = cpu_physics_only(w)
        cpu = {"value": v, "unit": UNIT, "cores": threads, "kind": "oracle",
               "sample": f"{k} random targets of {args.workload}, one step (oracle sampled mode), {sec:.1f} s",
               "physics_only": phys}
        try:
            parity = parity_block(sim, gfirst, ref)
        except Exception as e:  # reported, never hidden
            parity = {"error": repr(e)}

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": args.workload + ("+stir" if args.stir else "")
                           + ("+balsara" if args.av_switch else "")
                           + ("+gradh" if args.gradh else "") + ("+vsig" if args.dt_vsig else "")
                           + ("+ve" if args.ve else ""),
                           "n_particles_per_gpu": n,
                           "n_particles_total": n * world,
                           "parallelism": "single GPU" if world == 1 else
                           f"{world} independent replicas (SFC decomposition not yet built)",
                           "l2": "inputs (~1 GB state + ~3 GB lists) >> 126 MB L2; no flush",
                           "mean_nc": mean_nc,
                           "cell_level": infos[-1]["cell_level"],
                           "search_candidates_per_target": infos[-1]["search_candidates"] / n,
                           "search_passes_per_warp": infos[-1]["search_passes"] / (n / 32)},
                "phase_ms": phase_ms, "fp64_other": other, "roofline": roofline, "e2e": e2e,
                "phases": phase_table(phase_ms, pairs, n, energy, p_idle),
                "repeats": repeats, "parity": parity, "energy": energy, "accounting": accounting, "dvfs_trace": trace, "cpu_baseline": cpu, "clocks": clk.summary(),
                "gpu_launches": launches}
        s = json.dumps(line)
        print(s, flush=True)
        if args.out:
            with open(args.out, "w") as f:
                f.write(s + "\n")
    sim.finalize()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
