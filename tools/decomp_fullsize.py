"""SURVEY 8(d) config 4 at full size on ONE GPU: Noh implosion 300^3 (open box,
27M particles) decomposed over W ranks that share cuda:0 (gloo collectives),
K steps, then compared bit for bit with the single-rank run of the same initial
conditions (sorted by id).  Also a periodic turbulence case.  The ranks share one
GPU, so the timings say nothing about scaling; they show the decomposed step and
its halo / migration plumbing running at the configuration's size.

usage: python tools/decomp_fullsize.py [--workload noh300] [--world 2] [--steps 3]
"""
import argparse
import json
import os
import socket
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
FIELDS = ("id", "x", "y", "z", "vx", "vy", "vz", "h", "u", "du_m1")


def _make(name, rank=0, world=1, vsq=None):
    """The whole initial state (rank 0 of 1) or rank's slice of it.  Turbulence
    slices come from ics.turbulence_part (no rank generates the whole box) and
    every run normalises with the same given sum of v^2, so the slices are
    bit-identical to the single run's particles."""
    import dataclasses
    from paper_conf_sc_simsekpc24_b200 import ics
    if name.startswith("noh"):
        w = ics.noh(int(name[3:]))
        w.params = dataclasses.replace(w.params, ngmax=256)  # capacity for the shocked shell
        if world > 1:
            w.state = {k: np.ascontiguousarray(v[rank::world]) for k, v in w.state.items()}
    else:
        w = ics.turbulence_part(int(name[len("turbulence"):]), rank, world)
        ics.normalise_velocity(w, vsq)
    return w


def _vsq(name):
    from paper_conf_sc_simsekpc24_b200 import ics
    if name.startswith("noh"):
        return None
    return ics.turbulence_part(int(name[len("turbulence"):]), 0, 1).meta["vsq_sum"]


def _worker(rank, world, port, name, steps, out, vsq):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_sc_simsekpc24_b200 import decomp
    w = _make(name, rank, world, vsq)
    n = w.meta.get("n_total", w.n * world)
    cap = int(1.4 * n / world) + 4096
    ds = decomp.DistributedSim(w.params, w.state, n_capacity=cap, device=0)
    del w
    ms = []
    dts = []
    for _ in range(steps):
        dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        dts.append(ds.step())
        torch.cuda.synchronize()
        ms.append(1e3 * (time.perf_counter() - t0))
    # every rank writes its own particles (an all-gather of the whole state to
    # every rank does not fit when 8 ranks share one GPU); the parent merges
    with torch.cuda.stream(ds.sim.stream):
        loc = {k: v.cpu().numpy() for k, v in ds.local.items()}
    np.savez(f"{out}.{rank}.npz", **{k: loc[k] for k in FIELDS}, dts=np.array(dts), ms=np.array(ms),
             n_ghost=ds.stats["n_ghost"], n_local=ds.stats["n_local"])
    dist.barrier()
    dist.destroy_process_group()


def _single(name, steps, vsq):
    import torch
    from paper_conf_sc_simsekpc24_b200 import sph
    w = _make(name, 0, 1, vsq)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    dts, ms = [], []
    for _ in range(steps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        dts.append(sim.step()["dt"])
        torch.cuda.synchronize()
        ms.append(1e3 * (time.perf_counter() - t0))
    st = sim.get_state()
    sim.finalize()
    o = np.argsort(st["id"])
    return dts, ms, {k: st[k][o] for k in FIELDS}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="noh300")
    ap.add_argument("--world", type=int, default=2)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--out", default="gpurun_out/decomp_fullsize.json")
    a = ap.parse_args()
    import torch.multiprocessing as mp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    vsq = _vsq(a.workload)
    tmp = f"/tmp/decomp_fullsize_{os.getpid()}"
    ctx = mp.get_context("spawn")
    t0 = time.perf_counter()
    procs = [ctx.Process(target=_worker, args=(r, a.world, port, a.workload, a.steps, tmp, vsq)) for r in range(a.world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join()
    bad = [p.exitcode for p in procs if p.exitcode]
    if bad:
        raise SystemExit(f"rank exit codes {bad}")
    t_dec = time.perf_counter() - t0
    parts = [dict(np.load(f"{tmp}.{r}.npz")) for r in range(a.world)]
    for r in range(a.world):
        os.remove(f"{tmp}.{r}.npz")
    d = {k: np.concatenate([p[k] for p in parts]) for k in FIELDS}
    o = np.argsort(d["id"])
    d = {k: v[o] for k, v in d.items()}
    d.update({k: parts[0][k] for k in ("dts", "ms", "n_ghost", "n_local")})
    del parts
    dts1, ms1, st1 = _single(a.workload, a.steps, vsq)
    same = {k: bool(np.array_equal(d[k], st1[k])) for k in FIELDS}
    rec = {"workload": a.workload, "n": int(st1["id"].size), "world": a.world, "steps": a.steps,
           "backend": "gloo (all ranks on cuda:0)",
           "dt_decomposed": d["dts"].tolist(), "dt_single": dts1, "dt_equal": d["dts"].tolist() == dts1,
           "bit_identical": same, "all_bit_identical": all(same.values()),
           "rank0_ghosts": int(d["n_ghost"]), "rank0_local": int(d["n_local"]),
           "ms_per_step_decomposed_wall": d["ms"].tolist(), "ms_per_step_single_wall": ms1,
           "decomposed_run_wall_s": t_dec}
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(rec, f, indent=1)
    print(json.dumps(rec))
    if not rec["all_bit_identical"] or not rec["dt_equal"]:
        raise SystemExit(1)


if __name__ == "__main__":
    main()
