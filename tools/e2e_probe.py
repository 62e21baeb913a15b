"""Phase times of sph_step while the pipelined e2e copies run (bench.py's e2e
loop), against the same steps without copies: do the host-link transfers slow
the step's kernels (L2 pollution by the DMA traffic)?"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_sc_simsekpc24_b200 import ics, sph  # noqa: E402

w = ics.turbulence(200)
n = w.n
sims = [sph.Simulation(w.params, n_capacity=n) for _ in range(2)]
for sm in sims:
    sm.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sm.set_time(0.0, w.params.dt_first, True)
    for _ in range(3):
        sm.step()
pinned = {k: torch.from_numpy(v).pin_memory() for k, v in sims[0].get_state().items()}
outs = [{k: torch.empty_like(v).pin_memory() for k, v in pinned.items()} for _ in sims]
copy_stream = torch.cuda.Stream()
stage = [{k: torch.empty(v.shape, dtype=v.dtype, device="cuda") for k, v in pinned.items()} for _ in sims]
staged = [torch.cuda.Event() for _ in sims]


def load(c):
    copy_stream.wait_event(staged[c])
    with torch.cuda.stream(copy_stream):
        for k, v in pinned.items():
            stage[c][k].copy_(v, non_blocking=True)
        sims[c].set_particles(stage[c])
    staged[c].record(sims[c].stream)


def phases(infos):
    keys = infos[0]["phase_ms"].keys()
    return {k: round(float(np.median([i["phase_ms"][k] for i in infos])), 3) for k in keys
            if infos[0]["phase_ms"][k] > 0.05}


# with copies (pipelined as in bench.py)
import time
K = 10
infos = []
marks = []
torch.cuda.synchronize()
t0 = time.perf_counter()
load(0)
for s in range(K):
    cur = sims[s % 2]
    ta = time.perf_counter()
    if s + 1 < K:
        load((s + 1) % 2)
    tb = time.perf_counter()
    infos.append(cur.step())
    tc = time.perf_counter()
    for k, v in outs[s % 2].items():
        cur.get_field(k, out=v, async_=True)
    td = time.perf_counter()
    marks.append((round(1e3 * (tb - ta), 2), round(1e3 * (tc - tb), 2), round(1e3 * (td - tc), 2)))
for sm in sims:
    sm.sync()
total = 1e3 * (time.perf_counter() - t0) / K
with_copies = phases(infos)
print("ms per iteration", round(total, 2), "[load, step, readback enqueue] ms:", marks)
# without copies
infos = [sims[0].step() for _ in range(K)]
without = phases(infos)
print(json.dumps({"with_copies": with_copies, "without": without}))
