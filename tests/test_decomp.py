"""Host side of the multi-GPU decomposition on CPU with the gloo backend at world
sizes 2, 4 and 8: decomp.Comm's collectives (MAX/SUM all-reduce, all-to-all with
host counts) driving the selection logic of tests/decomp_reference.py (global
box, SFC split points, owners, cell-stencil ghosts) -- checked against the
one-rank box and brute-force neighbours, periodic and open boxes."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import decomp_reference as ref
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


def _workload(case="periodic"):
    if case == "periodic":
        return ics.random_box(4000, seed=31, periodic=True)
    w = ics.noh(16)  # open box (bounding box per step)
    return w


def _route_fn(rank, world, case):
    """One rank of the decomposition's selection logic (tests/decomp_reference.py)
    driven through decomp.Comm's real collectives: global box (MAX), key
    histogram (SUM), migration and ghost rows (all-to-all with host counts)."""
    w = _workload(case)
    s = w.state
    comm = decomp.Comm()
    mine = np.arange(w.n)[rank::world]          # arbitrary initial distribution
    red = torch.from_numpy(ref.red7(s["x"][mine], s["y"][mine], s["z"][mine], s["h"][mine]))
    comm.all_reduce_(red, dist.ReduceOp.MAX)
    lo, hi = ref.key_box(red.numpy(), w.params)
    keys_all = oracle.keys(s["x"], s["y"], s["z"], lo, hi)
    k = keys_all[mine]
    hist = torch.from_numpy(np.bincount((k >> np.uint64(63 - ref.HIST_BITS)).astype(np.int64),
                                        minlength=1 << ref.HIST_BITS).astype(np.int64))
    comm.all_reduce_(hist, dist.ReduceOp.SUM)
    splits = ref.splits_from_hist(hist.numpy(), world)
    own = ref.owners(k, splits)
    st = {f: torch.from_numpy(np.ascontiguousarray(s[f][mine])) for f in decomp.STATE + ("id",)}
    rows = decomp.pack(st)

    def exchange(sel_rows, dest_lists):
        send_c = [len(d) for d in dest_lists]
        sc = torch.tensor(send_c, dtype=torch.int64)
        rc = torch.empty_like(sc)
        comm.all_to_all(rc, sc, [1] * world, [1] * world)
        send = torch.cat([sel_rows[d] for d in dest_lists], 0) if sum(send_c) else torch.zeros((0, decomp.ROW), dtype=torch.float64)
        recv = torch.empty((int(rc.sum()), decomp.ROW), dtype=torch.float64)
        comm.all_to_all(recv, send, rc.tolist(), send_c)
        return decomp.unpack(recv)

    mig = exchange(rows, [torch.from_numpy(np.nonzero((own == r) & (r != rank))[0]) for r in range(world)])
    keep = own == rank
    loc = {f: torch.cat([st[f][torch.from_numpy(keep)], mig[f]]) for f in st}
    ids = loc["id"].numpy()
    # ghosts by cells of the new locals (keys from the same global box)
    kl = keys_all[ids]
    gm = ref.ghost_masks_cells(kl, lo, hi, float(red[6]), w.params.periodic, splits, rank, world)
    lrows = decomp.pack(loc)
    g = exchange(lrows, [torch.from_numpy(np.nonzero((gm >> np.uint64(r)) & np.uint64(1))[0]) for r in range(world)])
    return splits, red.numpy(), ids, g["id"].numpy()


@pytest.mark.parametrize("case,world", [("periodic", 2), ("periodic", 4), ("open", 4), ("periodic", 8)])
def test_route_partition_and_halo_coverage(case, world):
    """Every rank computes the same global box and split points; ownership is
    complete, disjoint and a contiguous key range per rank, balanced to within a
    histogram bin; locals + ghosts of each rank hold every brute-force neighbour
    of its locals (the cell-stencil halo is conservative), and no rank receives
    its own particles as ghosts."""
    import functools
    res = run_world(functools.partial(_route_fn, case=case), world=world)
    w = _workload(case)
    s = w.state
    for r in range(1, world):
        assert np.array_equal(res[r][0], res[0][0]) and np.array_equal(res[r][1], res[0][1])
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], w.params)
    lo, hi = ref.key_box(res[0][1], w.params)
    assert np.array_equal(lo, bmin) and np.array_equal(hi, bmax), "the global box is the one-rank box"
    keys = oracle.keys(s["x"], s["y"], s["z"], bmin, bmax)
    bins = (keys >> np.uint64(63 - ref.HIST_BITS)).astype(np.int64)
    splits = res[0][0]
    all_ids = np.concatenate([r[2] for r in res])
    assert np.array_equal(np.sort(all_ids), np.arange(w.n)), "ownership complete and disjoint"
    for r, (_, _, ids, _) in enumerate(res):
        assert np.all((bins[ids] >= splits[r]) & (bins[ids] < splits[r + 1]))
        assert abs(len(ids) - w.n / world) < 0.05 * w.n
    nb = oracle.neighbors(s["x"], s["y"], s["z"], s["h"], bmin, bmax, w.params.periodic)
    for r, (_, _, ids, ghosts) in enumerate(res):
        held = set(ids.tolist()) | set(ghosts.tolist())
        assert not set(ghosts.tolist()) & set(ids.tolist())
        need = set(nb.idx[np.concatenate([np.arange(nb.offsets[i], nb.offsets[i + 1]) for i in ids])].tolist())
        assert need <= held, f"rank {r} misses {len(need - held)} neighbours"
        assert len(ghosts) < 0.9 * w.n  # not everything


def test_splits_reference_edge_cases():
    assert ref.splits_from_hist(np.zeros(8, np.int64), 3).tolist() == [0, 8, 8, 8]
    h = np.zeros(8, np.int64)
    h[5] = 10
    assert ref.splits_from_hist(h, 2).tolist() == [0, 5, 8]
    assert ref.splits_from_hist(np.ones(8, np.int64), 4).tolist() == [0, 2, 4, 6, 8]


def test_pack_roundtrip():
    ids = torch.tensor([7, 3, 11, 5, 1 | decomp.GHOST_BIT], dtype=torch.int64)
    st = {f: torch.arange(5, dtype=torch.float64) * (c + 1) for c, f in enumerate(decomp.STATE)}
    st["id"] = ids
    back = decomp.unpack(decomp.pack(st))
    for f in decomp.STATE + ("id",):
        assert torch.equal(back[f], st[f])


def test_box_distance_minimum_image():
    x = torch.tensor([[0.49, 0.0, 0.0], [-0.3, 0.0, 0.0]], dtype=torch.float64)
    lo = torch.tensor([-0.5, -0.1, -0.1], dtype=torch.float64)
    hi = torch.tensor([-0.45, 0.1, 0.1], dtype=torch.float64)
    d = ref.box_distance(x, lo, hi, [1.0, 1.0, 1.0], (1, 1, 1))
    assert d[0].item() == pytest.approx(0.01, abs=1e-12)   # through the periodic face
    assert d[1].item() == pytest.approx(0.15, abs=1e-12)
    d = ref.box_distance(x, lo, hi, [1.0, 1.0, 1.0], (0, 1, 1))
    assert d[0].item() == pytest.approx(0.94, abs=1e-12)
