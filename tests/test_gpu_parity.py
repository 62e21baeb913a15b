"""GPU (libsph through the C ABI) vs the CPU oracle on identical seeded inputs.

Bars (BASELINE.json north_star): Morton order and neighbour lists bit-exact;
fp64 fields within 1e-10 after one step and 1e-8 after ten, in the metric of
DESIGN.md section 3 (|err| <= tol * sum_j |term_j| for the neighbour sums)."""
import hashlib

import numpy as np
import pytest

import oracle
from paper_conf_sc_simsekpc24_b200 import ics
from parity import (TOL_1STEP, TOL_10STEP, compare_state, compare_sums, gpu_pipeline, new_sim)

pytestmark = pytest.mark.gpu


def _workloads():
    w_open = ics.random_box(3001, seed=7, periodic=False)
    w_rand = ics.random_box(5003, seed=8, periodic=True)   # ragged: not a multiple of any tile
    w_turb = ics.turbulence(20)
    w_sedov = ics.sedov(16)
    w_noh = ics.noh(14)
    return {"sedov16": w_sedov, "turbulence20": w_turb, "random_periodic": w_rand,
            "random_open": w_open, "noh14": w_noh}


WORKLOADS = _workloads()


@pytest.fixture(scope="module", params=list(WORKLOADS))
def case(request):
    w = WORKLOADS[request.param]
    st, o = oracle.step({k: v.copy() for k, v in w.state.items()}, w.params, w.params.dt_first, True)
    sim = new_sim(w)
    g = gpu_pipeline(sim)
    return request.param, w, sim, g, st, o


def test_morton_order_bit_exact(case):
    name, w, sim, g, st, o = case
    assert np.array_equal(g["key"], o["keys"]), "sorted Morton keys"
    assert np.array_equal(g["id"], o["pre"]["id"]), "Morton order (id sequence)"
    for k in ("x", "y", "z", "h", "m", "u"):
        assert np.array_equal(g[k], o["pre"][k]), f"permuted {k}"


def test_neighbour_lists_bit_exact(case):
    name, w, sim, g, st, o = case
    nb = o["nb"]
    assert np.array_equal(g["nc"], nb.nc)
    off, idx = sim.get_neighbors()
    assert np.array_equal(off, nb.offsets)
    assert np.array_equal(idx.astype(np.int64), nb.idx)
    s = g["stats"]
    assert s["max_nc"] == nb.nc.max() and s["min_nc"] == nb.nc.min() and s["total"] == nb.nc.sum()


def test_neighbour_sums_within_tolerance(case):
    name, w, sim, g, st, o = case
    compare_sums(g, o, TOL_1STEP)


def test_step_parity_one_step(case):
    name, w, sim, g, st, o = case
    dt = sim.timestep()
    assert dt == o["dt"], "dt is bit-exact (min of IEEE h/c, same operations)"
    sim.update()
    t, dtp, first = sim.get_time()
    assert t == dt and dtp == dt and not first
    gs = sim.get_state()
    assert np.array_equal(gs["id"], st["id"])
    L = float(np.max(np.array(o["bmax"]) - np.array(o["bmin"])))
    compare_state(gs, st, L, TOL_1STEP)


def test_ten_steps_sedov16():
    w = ics.sedov(16)
    s = {k: v.copy() for k, v in w.state.items()}
    dt = w.params.dt_first
    sim = new_sim(w)
    for k in range(10):
        s, out = oracle.step(s, w.params, dt, k == 0)
        dt = out["dt"]
        info = sim.step()
        assert info["dt"] == pytest.approx(dt, rel=1e-12)
    gs = sim.get_state()
    assert np.array_equal(gs["id"], s["id"])
    compare_state(gs, s, 1.0, TOL_10STEP, "10 steps: ")


def test_ten_steps_turbulence():
    w = ics.turbulence(14)
    s = {k: v.copy() for k, v in w.state.items()}
    dt = w.params.dt_first
    sim = new_sim(w)
    for k in range(10):
        s, out = oracle.step(s, w.params, dt, k == 0)
        dt = out["dt"]
        sim.step()
    gs = sim.get_state()
    assert np.array_equal(gs["id"], s["id"])
    compare_state(gs, s, 1.0, TOL_10STEP, "10 steps: ")


def test_deterministic_bitwise():
    w = ics.turbulence(16)
    hashes = set()
    for _ in range(3):
        sim = new_sim(w)
        for _ in range(2):
            sim.step()
        h = hashlib.sha256()
        for k, v in sim.get_state().items():
            h.update(v.tobytes())
        hashes.add(h.hexdigest())
        sim.finalize()
    assert len(hashes) == 1


def test_step_graph_matches_eager(monkeypatch):
    """sph_step replays a captured CUDA graph (one per buffer parity and sort
    pass count); SPH_NO_GRAPH=1 runs the same phases eagerly.  Both give the
    same state bit for bit, the same times and neighbour statistics, and the
    graph path still reports per-phase times and kernel launches."""
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.turbulence(16)
    out = {}
    for env in ("1", "0"):
        monkeypatch.setenv("SPH_NO_GRAPH", env)
        sim = new_sim(w)
        l0 = sph.kernel_launches()
        infos = [sim.step() for _ in range(5)]
        launches = sph.kernel_launches() - l0
        st = sim.get_state()
        out[env] = (st, sim.get_time(), infos, launches)
        sim.finalize()
    (a, ta, ia, la), (b, tb, ib, lb) = out["1"], out["0"]
    for k in a:
        assert np.array_equal(a[k], b[k]), k
    assert ta == tb
    for x, y in zip(ia, ib):
        assert x["dt"] == y["dt"] and x["max_nc"] == y["max_nc"] and x["mean_nc"] == y["mean_nc"]
        assert y["phase_ms"]["neighbors"] > 0 and y["phase_ms"]["momentum_energy"] > 0
    assert la == lb > 0
    assert all(x["graph"] for x in ib) and not any(x["graph"] for x in ia)


def test_empty_input():
    w = ics.sedov(4)
    from paper_conf_sc_simsekpc24_b200 import sph
    sim = sph.Simulation(w.params, n_capacity=64)
    sim.set_particles({k: v[:0] for k, v in w.state.items()})
    sim.set_time(0.0, 1e-3, True)
    info = sim.step()
    assert info["dt"] == pytest.approx(1.1e-3, rel=1e-15)


def test_lone_particle_is_singular():
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.random_box(1, seed=3)
    sim = new_sim(w, cap=16)
    with pytest.raises(sph.SphError) as e:
        sim.step()
    assert e.value.name == "ERR_SINGULAR"


@pytest.mark.parametrize("wname,level", [("turbulence20", 2), ("turbulence20", 3), ("random_open", 3),
                                         ("noh14", 3)])
def test_neighbour_lists_coarse_grid(wname, level):
    """A coarse cell grid (max_cell_level 2-3: 2-4 cells per axis) gives warps
    thousands of candidates: more than the search's per-warp scratch holds in one
    segment (nrows_ld chunks of 32 candidates), so the lists are expanded segment by
    segment (lanes at different list positions), and at level 2 the periodic axes
    are "full" (minimum image per candidate).  Lists stay bit-exact vs brute force."""
    w = WORKLOADS[wname]
    o = oracle.step({k: v.copy() for k, v in w.state.items()}, w.params, w.params.dt_first, True)[1]
    sim = new_sim(w, max_cell_level=level)
    sim.build_tree()
    stats = sim.find_neighbors()
    nb = o["nb"]
    assert np.array_equal(sim.get_field("nc"), nb.nc)
    off, idx = sim.get_neighbors()
    assert np.array_equal(off, nb.offsets)
    assert np.array_equal(idx.astype(np.int64), nb.idx)
    # at level 2 (every axis "full") the candidate streams exceed one segment
    nrows_ld = (w.params.ngmax + 8) // 8 * 8
    if level == 2:
        assert stats["candidates"] / max(stats["passes"], 1) > nrows_ld * 32
    sim.finalize()


@pytest.mark.parametrize("wname", ["turbulence20", "random_open", "sedov16"])
def test_neighbour_lists_merged_runs(wname, monkeypatch):
    """The search's run table overflow path: with SPH_NBR_MERGE_RUNS=0 every
    cell's needed children are merged into one run (more candidates, the same
    decisions), as happens when a group's runs exceed the table.  Lists stay
    bit-exact and the candidate count does not drop."""
    w = WORKLOADS[wname]
    o = oracle.step({k: v.copy() for k, v in w.state.items()}, w.params, w.params.dt_first, True)[1]
    cand = {}
    for env in (None, "0"):
        if env is None:
            monkeypatch.delenv("SPH_NBR_MERGE_RUNS", raising=False)
        else:
            monkeypatch.setenv("SPH_NBR_MERGE_RUNS", env)
        sim = new_sim(w)
        sim.build_tree()
        stats = sim.find_neighbors()
        cand[env] = stats["candidates"]
        off, idx = sim.get_neighbors()
        assert np.array_equal(off, o["nb"].offsets)
        assert np.array_equal(idx.astype(np.int64), o["nb"].idx)
        sim.finalize()
    assert cand["0"] >= cand[None]


def test_capacity_error_reports_needed_size():
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.sedov(10)
    w.params.ngmax = 50
    sim = new_sim(w)
    sim.build_tree()
    with pytest.raises(sph.SphError) as e:
        sim.find_neighbors()
    assert e.value.name == "ERR_CAPACITY" and "92" in str(e.value)


def test_degenerate_open_box():
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.random_box(100, seed=3, periodic=False)
    w.state["z"][:] = 0.25
    sim = new_sim(w)
    sim.build_tree()
    with pytest.raises(sph.SphError) as e:
        sim.find_neighbors()
    assert e.value.name == "ERR_BOX"


def test_stage_machine():
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.sedov(8)
    sim = new_sim(w)
    with pytest.raises(sph.SphError) as e:
        sim.density()
    assert e.value.name == "ERR_STATE"
    sim.build_tree()
    with pytest.raises(sph.SphError):
        sim.iad()
    with pytest.raises(sph.SphError) as e:
        sim.set_particles({k: v[: 10 ** 6] for k, v in ics.sedov(12).state.items()})
    assert e.value.name == "ERR_CAPACITY"


def test_host_and_device_inputs_agree():
    import torch
    w = ics.turbulence(12)
    a = new_sim(w)
    a.step()
    b = new_sim(w)
    dev = {k: torch.from_numpy(np.ascontiguousarray(v)).cuda() for k, v in w.state.items()}
    b.set_particles(dev)
    b.set_time(0.0, w.params.dt_first, True)
    b.step()
    for k in ("x", "vx", "u", "h"):
        assert np.array_equal(a.get_field(k), b.get_field(k))


@pytest.mark.parametrize("spread", [1e-4, 3e-3])
def test_sort_fixup_and_fallback_bit_exact(spread):
    """The production sort runs the LSD passes over the top key digits only and
    then stable-sorts the runs of equal top digits by the full key (k_sort.cu).
    Clustered particles (all within `spread` of a point, with exact duplicate
    positions: ties keep the input order) make long runs: the fixup's result,
    and the all-8-pass fallback the next build takes after a long run, both equal
    the oracle's stable sort bit for bit."""
    from paper_conf_sc_simsekpc24_b200 import sph
    w = ics.random_box(6000, seed=17, periodic=True)
    rng = np.random.default_rng(5)
    for k in ("x", "y", "z"):
        w.state[k] = 0.1 + rng.uniform(0, spread, w.n)
    dup = np.arange(0, w.n - 1, 7)
    for k in ("x", "y", "z"):
        w.state[k][dup] = w.state[k][dup + 1]   # exact duplicate positions: equal keys
    w.state["h"][:] = 1e-5
    sim = sph.Simulation(w.params, n_capacity=w.n)
    s = {k: np.ascontiguousarray(v) for k, v in w.state.items()}
    sim.set_particles(s)
    sim.set_time(0.0, w.params.dt_first, True)
    bmin, bmax = oracle.box(s["x"], s["y"], s["z"], w.params)
    want = s["id"][oracle.sort_order(oracle.keys(s["x"], s["y"], s["z"], bmin, bmax))]
    for rep in range(3):   # fixup, then (after the long runs) the full-pass fallback
        sim.build_tree()
        assert np.array_equal(sim.get_field("id"), want), rep
        sim.find_neighbors()  # its scalar sync updates the sort policy
        sim.set_particles(s)  # same input again
    sim.finalize()
