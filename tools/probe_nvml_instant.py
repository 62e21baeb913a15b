"""Probe of the B200's NVML power sensors (reading 12, a11 accounting):
how fast NVML_FI_DEV_POWER_INSTANT (field 186) can be read, how often it
changes, and whether its time integral matches the total-energy counter
(nvmlDeviceGetTotalEnergyConsumption, ~100 ms / ~99 J quanta) over a ~12 s load
that alternates SPH steps with idle gaps.  Writes gpurun_out/probe_nvml_instant.json."""
import json
import os
import subprocess
import sys
import time

import pynvml as N

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LOAD = r'''
import sys, time, numpy as np
sys.path.insert(0, %r)
from paper_conf_sc_simsekpc24_b200 import ics, sph
w = ics.turbulence(160)
sim = sph.Simulation(w.params, n_capacity=w.n)
sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
sim.set_time(0.0, w.params.dt_first, True)
print("ready", flush=True)
for burst in range(4):
    t0 = time.time()
    while time.time() - t0 < 2.0:
        sim.step()
    time.sleep(1.0)
print("done", flush=True)
''' % ROOT


def main():
    N.nvmlInit()
    h = N.nvmlDeviceGetHandleByIndex(0)
    p = subprocess.Popen([sys.executable, "-c", LOAD], stdout=subprocess.PIPE, text=True)
    assert p.stdout.readline().strip() == "ready"
    samples = []
    t_end = time.time() + 13.0
    lat = []
    while time.time() < t_end and p.poll() is None:
        t0 = time.perf_counter()
        fv = N.nvmlDeviceGetFieldValues(h, [N.NVML_FI_DEV_POWER_INSTANT])[0]
        t1 = time.perf_counter()
        e = N.nvmlDeviceGetTotalEnergyConsumption(h)
        t2 = time.perf_counter()
        pw = fv.value.uiVal if fv.nvmlReturn == 0 else -1
        samples.append((t1, pw, e))
        lat.append((t1 - t0, t2 - t1))
    p.wait()
    # instant power update period: times between changes of the value
    ch = [samples[i][0] for i in range(1, len(samples)) if samples[i][1] != samples[i - 1][1]]
    dts = [b - a for a, b in zip(ch, ch[1:])]
    ech = [i for i in range(1, len(samples)) if samples[i][2] != samples[i - 1][2]]
    # integral of instant power between the first and last energy-counter change
    i0, i1 = ech[0], ech[-1]
    integ = sum(samples[i][1] * 1e-3 * (samples[i + 1][0] - samples[i][0]) for i in range(i0, i1))
    cnt = (samples[i1][2] - samples[i0][2]) * 1e-3
    lat_f = sorted(a for a, b in lat)
    lat_e = sorted(b for a, b in lat)
    res = {
        "samples": len(samples),
        "field186_ok": samples[0][1] >= 0,
        "read_latency_ms_instant_median": 1e3 * lat_f[len(lat_f) // 2],
        "read_latency_ms_energy_median": 1e3 * lat_e[len(lat_e) // 2],
        "instant_changes": len(ch),
        "instant_update_period_ms_median": 1e3 * sorted(dts)[len(dts) // 2] if dts else None,
        "energy_counter_changes": len(ech),
        "energy_counter_J": cnt,
        "instant_power_integral_J": integ,
        "ratio_counter_over_integral": cnt / integ if integ else None,
        "power_W_min_max": [min(s[1] for s in samples) * 1e-3, max(s[1] for s in samples) * 1e-3],
        "trace_head": [(round(s[0] - samples[0][0], 4), s[1], s[2]) for s in samples[:: max(1, len(samples) // 400)]],
    }
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    json.dump(res, open(os.path.join(ROOT, "gpurun_out", "probe_nvml_instant.json"), "w"), indent=1)
    print(json.dumps({k: v for k, v in res.items() if k != "trace_head"}))


if __name__ == "__main__":
    main()
