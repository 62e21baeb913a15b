"""Host logic of the multi-GPU decomposition (paper_conf_sc_simsekpc24_b200.decomp)
on CPU with the gloo backend, world size 2 -- partition, migration, ghost
selection and the halo all-to-all -- checked against brute force."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_sc_simsekpc24_b200 import decomp, ics


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, fn, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        q.put((rank, fn(rank, world)))
    except Exception as e:  # surfaced in the parent
        q.put((rank, e))
    finally:
        dist.destroy_process_group()


def run_world(fn, world=2):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, fn, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    for r, v in res.items():
        if isinstance(v, Exception):
            raise v
    return [res[r] for r in range(world)]


def _workload():
    return ics.random_box(4000, seed=31, periodic=True)


def _keys(w):
    s = w.state
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], w.params)
    return oracle.keys(s["x"], s["y"], s["z"], bmin, bmax)


def _partition_fn(rank, world):
    w = _workload()
    k = _keys(w)
    mine = np.arange(w.n)[rank::world]          # arbitrary initial distribution
    comm = decomp.Comm()
    kt = torch.from_numpy(k[mine].astype(np.int64))
    splits = decomp.sfc_splits(kt, comm)
    own = decomp.owners(kt, splits)
    st = {f: torch.from_numpy(np.ascontiguousarray(w.state[f][mine])) for f in decomp.STATE + ("id",)}
    rows = decomp.pack(st)
    got = decomp.unpack(torch.cat(comm.alltoallv([rows[own == r] for r in range(world)]), 0))
    return splits.numpy(), got["id"].numpy()


def test_partition_and_migration():
    (s0, ids0), (s1, ids1) = run_world(_partition_fn)
    assert np.array_equal(s0, s1), "every rank computes the same split points"
    w = _workload()
    k = _keys(w)
    # ownership is a contiguous key range, complete and disjoint
    assert len(set(ids0) & set(ids1)) == 0 and len(ids0) + len(ids1) == w.n
    b = (k >> np.uint64(63 - decomp.HIST_BITS)).astype(np.int64)
    assert np.all(b[ids0] < s0[1]) and np.all(b[ids1] >= s0[1])
    # balanced to within one histogram bin's worth of particles
    assert abs(len(ids0) - len(ids1)) < 0.05 * w.n


def _ghost_fn(rank, world):
    w = _workload()
    k = _keys(w)
    comm = decomp.Comm()
    kt = torch.from_numpy(k.astype(np.int64))
    splits = decomp.sfc_splits(kt[rank::world], comm)
    own = decomp.owners(kt, splits).numpy()
    mine = np.nonzero(own == rank)[0]
    x = torch.from_numpy(np.stack([w.state[a][mine] for a in ("x", "y", "z")], 1))
    boxes = decomp.domain_boxes(x, comm)
    radius = 2.0 * float(w.state["h"].max()) * (1 + 1e-9)
    box_len = [b - a for a, b in zip(w.params.box_min, w.params.box_max)]
    masks = decomp.ghost_masks(x, boxes, rank, radius, box_len, w.params.periodic)
    st = {f: torch.from_numpy(np.ascontiguousarray(w.state[f][mine])) for f in decomp.STATE + ("id",)}
    rows = decomp.pack(st)
    recv = comm.alltoallv([rows[m] for m in masks])
    ghosts = np.concatenate([decomp.unpack(r)["id"].numpy() for r in recv])
    return mine, ghosts


def test_ghosts_cover_every_neighbour():
    """Locals + ghosts of each rank contain every brute-force neighbour of its
    locals (the halo is conservative), and no rank receives its own particles."""
    res = run_world(_ghost_fn)
    w = _workload()
    s = w.state
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], w.params)
    nb = oracle.neighbors(s["x"], s["y"], s["z"], s["h"], bmin, bmax, w.params.periodic)
    for mine, ghosts in res:
        held = set(mine.tolist()) | set(ghosts.tolist())
        assert not set(ghosts.tolist()) & set(mine.tolist())
        need = set(nb.idx[np.concatenate([np.arange(nb.offsets[i], nb.offsets[i + 1]) for i in mine])].tolist())
        assert need <= held


def test_positions_of_and_pack_roundtrip():
    ids = torch.tensor([7, 3, 11, 5, 1 | decomp.GHOST_BIT], dtype=torch.int64)
    q = torch.tensor([11, 1 | decomp.GHOST_BIT, 7], dtype=torch.int64)
    assert decomp.positions_of(ids, q).tolist() == [2, 4, 0]
    st = {f: torch.arange(5, dtype=torch.float64) * (c + 1) for c, f in enumerate(decomp.STATE)}
    st["id"] = ids
    back = decomp.unpack(decomp.pack(st))
    for f in decomp.STATE + ("id",):
        assert torch.equal(back[f], st[f])


def test_box_distance_minimum_image():
    x = torch.tensor([[0.49, 0.0, 0.0], [-0.3, 0.0, 0.0]], dtype=torch.float64)
    lo = torch.tensor([-0.5, -0.1, -0.1], dtype=torch.float64)
    hi = torch.tensor([-0.45, 0.1, 0.1], dtype=torch.float64)
    d = decomp.box_distance(x, lo, hi, [1.0, 1.0, 1.0], (1, 1, 1))
    assert d[0].item() == pytest.approx(0.01, abs=1e-12)   # through the periodic face
    assert d[1].item() == pytest.approx(0.15, abs=1e-12)
    d = decomp.box_distance(x, lo, hi, [1.0, 1.0, 1.0], (0, 1, 1))
    assert d[0].item() == pytest.approx(0.94, abs=1e-12)
