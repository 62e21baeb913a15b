"""Probe the NVML energy counter of GPU 0 under load: update period, quantum,
agreement with integrated power, and whether locked clocks would be permitted
(read-only checks; never changes a clock).  Writes one JSON line."""
import json
import threading
import time

import pynvml
import torch

pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(0)
stop = False


def load():
    a = torch.randn(8192, 8192, device="cuda", dtype=torch.bfloat16)
    while not stop:
        for _ in range(20):
            a @ a
        torch.cuda.synchronize()


th = threading.Thread(target=load)
th.start()
time.sleep(1.0)
samples = []
t_end = time.perf_counter() + 3.0
while time.perf_counter() < t_end:
    samples.append((time.perf_counter(), pynvml.nvmlDeviceGetTotalEnergyConsumption(h),
                    pynvml.nvmlDeviceGetPowerUsage(h)))
stop = True
th.join()
changes = [(t, e) for (t, e, _), (_, ep, _) in zip(samples[1:], samples[:-1]) if e != ep]
dts = [b[0] - a[0] for a, b in zip(changes[:-1], changes[1:])]
des = [b[1] - a[1] for a, b in zip(changes[:-1], changes[1:])]
e_delta = (samples[-1][1] - samples[0][1]) * 1e-3
p_int = sum((b[0] - a[0]) * a[2] * 1e-3 for a, b in zip(samples[:-1], samples[1:]))
out = {"samples": len(samples), "changes": len(changes),
       "update_period_ms_median": 1e3 * sorted(dts)[len(dts) // 2] if dts else None,
       "update_period_ms_min": 1e3 * min(dts) if dts else None,
       "delta_mJ_median": sorted(des)[len(des) // 2] if des else None,
       "counter_J": e_delta, "power_integral_J": p_int,
       "ratio": e_delta / p_int if p_int else None}
try:
    r = pynvml.nvmlDeviceGetAPIRestriction(h, pynvml.NVML_RESTRICTED_API_SET_APPLICATION_CLOCKS)
    out["app_clock_restricted"] = int(r)
except pynvml.NVMLError as e:
    out["app_clock_restricted"] = str(e)
out["sm_clock_mhz"] = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
print(json.dumps(out))
