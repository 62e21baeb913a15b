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


def _make(name):
    return {"turbulence16": lambda: ics.turbulence(16), "random": lambda: ics.random_box(6000, seed=5),
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
                                  "random_gradh_vsig", "random_ve"])
def test_two_ranks_bit_identical_to_one(name):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, name, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    for v in res.values():
        if isinstance(v, Exception):
            raise v
    dts1, st1 = _single(name)
    for r in (0, 1):
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
    from paper_conf_sc_simsekpc24_b200 import decomp, sph
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
        want = decomp.ghost_masks(x, boxes, 0, 0.07, box_len, w.params.periodic)
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
