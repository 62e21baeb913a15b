"""Multi-GPU decomposition end to end on ONE GPU: two ranks (gloo for the
collectives, both processes on cuda:0) run the decomposed step; for a periodic
box the result must be bit-identical to the single-rank run (same neighbour sets,
same summation order, owners' values over the ghosts)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_simsekpc24_b200 import ics

pytestmark = pytest.mark.gpu

STEPS = 3


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _sedov_balsara():
    import dataclasses
    w = ics.sedov(14)
    w.params = dataclasses.replace(w.params, av_switch=1)  # halo of the Balsara factors too
    return w


def _random_gradh_vsig():
    import dataclasses
    w = ics.random_box(6000, seed=5)
    w.params = dataclasses.replace(w.params, gradh=1, dt_vsig=1)  # halo of Omega
    return w


def _random_ve():
    import dataclasses
    w = ics.random_box(6000, seed=5)
    w.params = dataclasses.replace(w.params, ve=1, gradh=1)  # halo of the normalised rho and Omega
    return w


def _noh():
    import dataclasses
    w = ics.noh(14)  # open box: the global key box of sph_set_key_box
    w.params = dataclasses.replace(w.params, dt_vsig=1, ngmax=400)
    return w


def _make(name):
    return {"turbulence16": lambda: ics.turbulence(16), "random": lambda: ics.random_box(6000, seed=5),
            "noh14_open": _noh,
            "sedov14": lambda: ics.sedov(14), "sedov14_balsara": _sedov_balsara,
            "random_gradh_vsig": _random_gradh_vsig, "random_ve": _random_ve}[name]()


def _worker(rank, world, port, name, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_simsekpc24_b200 import decomp
        w = _make(name)
        mine = {k: np.ascontiguousarray(v[rank::world]) for k, v in w.state.items()}
        ds = decomp.DistributedSim(w.params, mine, n_capacity=w.n, device=0)
        dts = [ds.step() for _ in range(STEPS)]
        st = ds.gather_state()
        q.put((rank, (dts, st, ds.stats)))
    except Exception as e:
        import traceback
        q.put((rank, RuntimeError(traceback.format_exc())))
    finally:
        dist.destroy_process_group()


def _single(name):
    from paper_conf_sc_simsekpc24_b200 import sph
    w = _make(name)
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    dts = [sim.step()["dt"] for _ in range(STEPS)]
    st = sim.get_state()
    o = np.argsort(st["id"])
    return dts, {k: v[o] for k, v in st.items()}


@pytest.mark.parametrize("name", ["turbulence16", "random", "sedov14", "sedov14_balsara",
                                  "random_gradh_vsig", "random_ve", "noh14_open"])
def test_two_ranks_bit_identical_to_one(name):
    _ranks_bit_identical(name, 2)


@pytest.mark.parametrize("name,world", [("turbulence16", 4), ("noh14_open", 4), ("random", 8)])
def test_more_ranks_bit_identical_to_one(name, world):
    """The 4- and 8-rank paths (split points, 64-bit ghost masks, halo lists over
    several peers): still bit-identical to one rank (all ranks on one GPU, gloo)."""
    _ranks_bit_identical(name, world)


def _ranks_bit_identical(name, world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=900) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    for v in res.values():
        if isinstance(v, Exception):
            raise v
    dts1, st1 = _single(name)
    for r in range(world):
        dts2, st2, stats = res[r]
        assert dts2 == dts1, "dt is the same global minimum"
        assert stats["n_ghost"] > 0
        for k in ("id", "x", "y", "z", "vx", "vy", "vz", "h", "u", "du_m1"):
            assert np.array_equal(st2[k], st1[k]), f"{name}: {k} differs from the single-rank run"


def test_one_rank_decomposed_equals_plain():
    from paper_conf_sc_simsekpc24_b200 import decomp
    w = _make("turbulence16")
    ds = decomp.DistributedSim(w.params, w.state, n_capacity=w.n, device=0)
    dts = [ds.step() for _ in range(STEPS)]
    st = ds.gather_state()
    dts1, st1 = _single("turbulence16")
    assert dts == dts1
    for k in ("x", "vx", "u", "h"):
        assert np.array_equal(st[k], st1[k])


def test_one_rank_forced_plumbing_equals_plain():
    """The whole exchange path (compact, keys, partition, ghost selection, maps,
    halo gathers/scatters) run on one rank moves nothing and changes nothing."""
    from paper_conf_sc_simsekpc24_b200 import decomp
    w = _make("sedov14_balsara")
    ds = decomp.DistributedSim(w.params, w.state, n_capacity=w.n, device=0, force_exchange=True)
    dts = [ds.step() for _ in range(STEPS)]
    st = ds.gather_state()
    dts1, st1 = _single("sedov14_balsara")
    assert dts == dts1
    for k in ("x", "vx", "u", "h"):
        assert np.array_equal(st[k], st1[k])


def test_device_plumbing_matches_host_logic():
    """sph_select_ghosts == decomp.ghost_masks; compact / pack / append /
    gather / scatter move exactly the selected particles."""
    import decomp_reference as ref
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.random_box(5000, seed=11)
    sim = sph.Simulation(w.params, n_capacity=2 * w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    dev = torch.device("cuda", 0)
    with torch.cuda.stream(sim.stream):
        x = torch.stack([torch.as_tensor(w.state[k], device=dev) for k in ("x", "y", "z")], 1)
        boxes = torch.tensor([[[-0.5, -0.5, -0.5], [0.0, 0.5, 0.5]], [[0.0, -0.5, -0.5], [0.5, 0.5, 0.5]],
                              [[0.1, 0.1, 0.1], [0.2, 0.2, 0.3]],
                              [[float("inf")] * 3, [-float("inf")] * 3]], dtype=torch.float64, device=dev)
        box_len = [1.0, 1.0, 1.0]
        want = ref.ghost_masks_boxes(x, boxes, 0, 0.07, box_len, w.params.periodic)
        got = sim.select_ghosts(boxes.reshape(4, 6).cpu().numpy(), 0, 0.07)
        for r in range(4):
            assert torch.equal(((got >> r) & 1).bool(), want[r]), r
        # pack -> append round trip, then compact back
        idx = torch.nonzero(want[1]).flatten()
        rows = sim.pack_rows(idx, sph.GHOST_BIT)
        sim.append_rows(rows)
        st = sim.get_state()
        n0 = w.n
        assert np.array_equal(st["x"][n0:], w.state["x"][idx.cpu().numpy()])
        assert np.all(st["id"][n0:] == (w.state["id"][idx.cpu().numpy()] | sph.GHOST_BIT))
        keep = torch.zeros(sim.n, dtype=torch.bool, device=dev)
        keep[::3] = True
        n = sim.compact(keep=keep, drop_ghosts=True)
        sel = np.arange(n0 + idx.numel())[::3]
        sel = sel[sel < n0]
        assert n == sel.size
        st2 = sim.get_state()
        for k in ("x", "vz", "u", "id"):
            assert np.array_equal(st2[k], w.state[k][sel]), k
        g = sim.gather_field("h", torch.tensor([2, 0, 1], device=dev))
        assert g.cpu().tolist() == st2["h"][[2, 0, 1]].tolist()
    sim.finalize()


def test_device_plumbing_edge_cases():
    """Empty compaction, append past the capacity (SPH_ERR_CAPACITY, state
    unchanged), too many ranks for the ghost mask (SPH_ERR_ARG), empty packs."""
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.random_box(500, seed=3)
    sim = sph.Simulation(w.params, n_capacity=600)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    dev = torch.device("cuda", 0)
    with torch.cuda.stream(sim.stream):
        rows = sim.pack_rows(torch.arange(200, device=dev))
        with pytest.raises(sph.SphError) as e:
            sim.append_rows(rows)                 # 500 + 200 > 600
        assert "CAPACITY" in str(e.value)
        assert sim.n == 500
        sim.append_rows(rows[:100])
        assert sim.n == 600
        assert sim.pack_rows(torch.zeros(0, dtype=torch.int64, device=dev)).shape == (0, sph.ROW_DOUBLES)
        with pytest.raises(sph.SphError):
            sim.select_ghosts(np.zeros((65, 6)), 0, 0.1)
        assert sim.compact(keep=torch.zeros(600, dtype=torch.bool, device=dev)) == 0
        assert sim.n == 0
        sim.append_rows(rows[:10])
        st = sim.get_state()
        assert np.array_equal(st["x"], w.state["x"][:10])
    sim.finalize()


@pytest.mark.parametrize("case", ["periodic", "open"])
def test_device_routing_matches_reference(case):
    """libsph's device routing (sph_decomp_reduce / sph_key_histogram /
    sph_decomp_owners / sph_decomp_ghosts / sph_decomp_pack / sph_decomp_drop /
    sph_decomp_map) equals tests/decomp_reference.py element by element: one
    context holding every particle plays rank 1 of 4."""
    import decomp_reference as ref
    import oracle
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.random_box(7000, seed=13, periodic=True) if case == "periodic" else ics.noh(18)
    s = w.state
    sim = sph.Simulation(w.params, n_capacity=w.n)
    sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
    sim.set_time(0.0, w.params.dt_first, True)
    world, rank = 4, 1
    with torch.cuda.stream(sim.stream):
        red = sim.decomp_reduce()
        want_red = ref.red7(s["x"], s["y"], s["z"], s["h"])
        assert np.array_equal(red.cpu().numpy(), want_red)
        sim.set_key_box(red)
        sim.compute_keys()
        keys = sim.get_field("key")
        lo, hi = ref.key_box(want_red, w.params)
        assert np.array_equal(keys, oracle.keys(s["x"], s["y"], s["z"], lo, hi))
        hist = sim.key_histogram(ref.HIST_BITS)
        want_hist = np.bincount((keys >> np.uint64(63 - ref.HIST_BITS)).astype(np.int64), minlength=1 << ref.HIST_BITS)
        assert np.array_equal(hist.cpu().numpy(), want_hist)
        mig, cnt = sim.decomp_owners(hist, ref.HIST_BITS, rank, world)
        splits = ref.splits_from_hist(want_hist, world)
        own = ref.owners(keys, splits)
        want_mig = np.where(own == rank, 0, 1 << own).astype(np.int64)
        assert np.array_equal(mig.cpu().numpy(), want_mig)
        assert cnt.cpu().tolist() == [int((own == r).sum()) for r in range(world)]
        # grouped pack: by destination rank, particle order within one
        total = int((want_mig != 0).sum())
        rows, pos = sim.decomp_pack(mig, world, total)
        order = np.concatenate([np.nonzero(own == r)[0] for r in range(world) if r != rank])
        assert np.array_equal(pos.cpu().numpy(), order)
        assert np.array_equal(rows[:, 0].cpu().numpy(), s["x"][order])
        # keep rank 1's particles; ghosts of them by cells
        sim.decomp_drop(mig, int((own == rank).sum()))
        kept = np.nonzero(own == rank)[0]
        st = sim.get_state()
        assert np.array_equal(st["id"], s["id"][kept])
        sim.compute_keys()
        gm, gc = sim.decomp_ghosts(ref.HIST_BITS, rank, world)
        want_gm = ref.ghost_masks_cells(keys[kept], lo, hi, want_red[6], w.params.periodic, splits, rank, world)
        assert np.array_equal(gm.cpu().numpy().view(np.uint64), want_gm)
        assert gc.cpu().tolist() == [int(((want_gm >> np.uint64(r)) & np.uint64(1)).sum()) for r in range(world)]
        assert gc.cpu().numpy().sum() > 0
        # positions through the sort
        sim.build_tree()
        perm = sim.get_field("order").astype(np.int64)
        pre = torch.tensor([0, 5, len(kept) - 1], dtype=torch.int64, device="cuda")
        post = sim.decomp_map(pre).cpu().numpy()
        inv = np.empty_like(perm)
        inv[perm] = np.arange(perm.size)
        assert np.array_equal(post, inv[[0, 5, len(kept) - 1]])
        assert np.array_equal(sim.decomp_map(None, first=2, m=3).cpu().numpy(), inv[2:5])
    sim.finalize()


def test_split_parts_state_machine_and_identity():
    """sph_set_part on one rank: INTERIOR leaves the stage, BOUNDARY advances it;
    the split calls give the unsplit fields bit for bit; GHOSTS is EOS-only;
    split calls are refused with grad-h."""
    from paper_conf_sc_simsekpc24_b200 import sph
    from parity import gpu_pipeline, new_sim
    w = ics.turbulence(16)
    a = new_sim(w)
    ga = gpu_pipeline(a)
    b = new_sim(w)
    b.build_tree()
    b.find_neighbors()
    b.density()
    b.eos()
    b.set_part(sph.PART_INTERIOR)
    b.iad()
    with pytest.raises(sph.SphError):
        b.momentum_energy()                 # the boundary IAD half is pending
    b.set_part(sph.PART_GHOSTS)
    b.eos()
    with pytest.raises(sph.SphError):
        b.iad()                              # GHOSTS is for EOS only
    b.set_part(sph.PART_BOUNDARY)
    b.iad()
    b.set_part(sph.PART_INTERIOR)
    b.momentum_energy()
    b.set_part(sph.PART_BOUNDARY)
    b.momentum_energy()
    b.set_part(sph.PART_ALL)
    for k in ("rho", "c11", "c23", "ax", "ay", "az", "du"):
        assert np.array_equal(b.get_field(k), a.get_field(k)), k
    assert b.timestep() == a.timestep()
    a.finalize()
    b.finalize()
    import dataclasses
    w.params = dataclasses.replace(w.params, gradh=1)
    c = new_sim(w)
    with pytest.raises(sph.SphError):
        c.set_part(sph.PART_INTERIOR)
    c.finalize()
