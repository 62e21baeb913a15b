"""Runs the decomposed step on WORLD ranks sharing one GPU (gloo) and compares
with the single-rank run (for torchrun debugging of tests/test_gpu_decomp.py)."""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
from paper_conf_sc_simsekpc24_b200 import decomp, ics, sph  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "turbulence16"
dist.init_process_group("gloo")
rank, world = dist.get_rank(), dist.get_world_size()
import test_gpu_decomp as T  # noqa: E402
w = T._make(name)
mine = {k: np.ascontiguousarray(v[rank::world]) for k, v in w.state.items()}
ds = decomp.DistributedSim(w.params, mine, n_capacity=w.n, device=0)
dts = []
for s in range(3):
    dts.append(ds.step())
    print(f"rank {rank} step {s} dt {dts[-1]!r} stats {ds.stats}", flush=True)
st = ds.gather_state()
if rank == 0:
    dts1, st1 = T._single(name)
    ok = dts == dts1 and all(np.array_equal(st[k], st1[k]) for k in ("id", "x", "vx", "u", "h"))
    print("IDENTICAL" if ok else f"DIFFERENT {dts} {dts1}", flush=True)
dist.destroy_process_group()
