"""Multi-GPU SPH step: space-filling-curve domain decomposition with halo
exchange ("domain decomposition, halo exchanges",
P:216 DomainDecompAndSync, P:220 the end-of-step collective for dt).

One process per GPU.  Every rank owns a contiguous range of the 63-bit Morton
curve; the split points come from a global histogram of the top key bits
(all-reduce).  Each step:

  1. keys of the local particles (libsph sph_build_tree), migration of the
     particles whose key left the rank's range (all-to-all);
  2. ghosts: every local particle within 2 h_max (minimum image) of another
     rank's domain box is sent to it (all-to-all) with SPH_GHOST_BIT in its id;
  3. the full hot path in libsph on locals + ghosts, with two halo refreshes of
     the owners' values over the ghosts: rho after DENSITY (then EOS derives
     p, c, V) and C after IAD (H2, H3 of SURVEY 8(e));
  4. dt = global min over ranks (all-reduce), update; the ghosts are dropped
     (sph_compact) at the start of the next step.
The particles stay in libsph; only emigrants, ghosts and halo values move.

The held set is sorted in the global Morton order and every target's
neighbours are the same particles as in a single-GPU run, so for a periodic box
the result is bit-identical to the one-GPU step (tests/test_gpu_decomp.py).

The data-path collectives are torch.distributed calls on device tensors (NCCL
over NVLink on GPUs; gloo on host tensors in the CPU tests).  All arithmetic of
the method stays in libsph; this module moves particles and values between
ranks and selects which to move (plumbing).
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

GHOST_BIT = 1 << 62
STATE = ("x", "y", "z", "vx", "vy", "vz", "h", "m", "u", "du_m1")
HIST_BITS = 15  # SFC partition granularity: 2^15 bins of the top key bits


# ----------------------------------------------------------------------------- comm
class Comm:
    """Collectives over the default process group; host tensors for gloo."""

    def __init__(self):
        self.rank = dist.get_rank() if dist.is_initialized() else 0
        self.world = dist.get_world_size() if dist.is_initialized() else 1
        self.host = (dist.get_backend() == "gloo") if dist.is_initialized() else True

    def _to(self, t):
        return t.cpu() if self.host else t

    def all_reduce(self, t, op):
        if self.world == 1:
            return t
        x = self._to(t.clone())
        dist.all_reduce(x, op=op)
        return x.to(t.device)

    def all_gather(self, t):
        if self.world == 1:
            return [t]
        x = self._to(t.contiguous())
        out = [torch.empty_like(x) for _ in range(self.world)]
        dist.all_gather(out, x)
        return [o.to(t.device) for o in out]

    def alltoallv(self, parts):
        """parts[r]: tensor [n_r, ...] for rank r -> list of received [m_s, ...]."""
        if self.world == 1:
            return [parts[0]]
        dev = parts[0].device
        tail = tuple(parts[0].shape[1:])
        width = int(np.prod(tail)) if tail else 1
        cdev = torch.device("cpu") if self.host else dev
        counts = torch.tensor([p.shape[0] for p in parts], dtype=torch.int64, device=cdev)
        rc = torch.empty_like(counts)
        dist.all_to_all_single(rc, counts)
        counts, rc = counts.cpu(), rc.cpu()
        send = self._to(torch.cat([p.reshape(-1, width) for p in parts], 0).reshape(-1))
        recv = torch.empty(int(rc.sum()) * width, dtype=send.dtype, device=send.device)
        dist.all_to_all_single(recv, send, [int(c) * width for c in rc],
                               [int(c) * width for c in counts])
        recv = recv.to(dev).reshape((-1,) + tail)
        return list(torch.split(recv, [int(c) for c in rc], 0))


# ----------------------------------------------------------------------------- partition
def sfc_splits(keys, comm: Comm, bits: int = HIST_BITS):
    """Split bins of the global key histogram: rank r owns bins [s[r], s[r+1])."""
    nb = 1 << bits
    b = (keys >> (63 - bits)).to(torch.int64)
    hist = torch.bincount(b, minlength=nb).to(torch.int64)
    hist = comm.all_reduce(hist, dist.ReduceOp.SUM if comm.world > 1 else None)
    cum = torch.cumsum(hist, 0)
    total = int(cum[-1])
    targets = torch.tensor([total * r // comm.world for r in range(1, comm.world)], dtype=torch.int64,
                           device=cum.device)
    inner = torch.searchsorted(cum, targets, right=True)  # first bin past each quota
    s = torch.cat([torch.zeros(1, dtype=torch.int64, device=cum.device), inner,
                   torch.full((1,), nb, dtype=torch.int64, device=cum.device)])
    return s


def owners(keys, splits, bits: int = HIST_BITS):
    b = (keys >> (63 - bits)).to(torch.int64)
    return torch.searchsorted(splits, b, right=True) - 1


def domain_boxes(x, comm: Comm):
    """[world, 2, 3] bounding boxes (min, max) of every rank's particles."""
    if x.shape[0]:
        lo, hi = x.min(0).values, x.max(0).values
    else:
        lo = torch.full((3,), float("inf"), dtype=x.dtype, device=x.device)
        hi = torch.full((3,), -float("inf"), dtype=x.dtype, device=x.device)
    return torch.stack(comm.all_gather(torch.stack([lo, hi])))


def box_distance(x, lo, hi, box_len, periodic):
    """Minimum-image distance of points x [n,3] to the axis-aligned box [lo, hi]."""
    d2 = torch.zeros(x.shape[0], dtype=x.dtype, device=x.device)
    for a in range(3):
        if periodic[a]:
            best = None
            for k in (-1.0, 0.0, 1.0):
                xa = x[:, a] + k * box_len[a]
                da = torch.clamp(torch.maximum(lo[a] - xa, xa - hi[a]), min=0.0)
                best = da if best is None else torch.minimum(best, da)
        else:
            best = torch.clamp(torch.maximum(lo[a] - x[:, a], x[:, a] - hi[a]), min=0.0)
        d2 = d2 + best * best
    return torch.sqrt(d2)


def ghost_masks(x, boxes, rank, radius, box_len, periodic):
    """masks[r]: local particles within `radius` of rank r's domain box (r != rank)."""
    out = []
    for r in range(boxes.shape[0]):
        if r == rank or not torch.isfinite(boxes[r]).all():
            out.append(torch.zeros(x.shape[0], dtype=torch.bool, device=x.device))
            continue
        out.append(box_distance(x, boxes[r, 0], boxes[r, 1], box_len, periodic) < radius)
    return out


# ----------------------------------------------------------------------------- rows
def pack(state, idx=None):
    """Particles as rows [n, 11] of float64 (id bit-cast into the last column)."""
    cols = [state[k] if idx is None else state[k][idx] for k in STATE]
    ids = state["id"] if idx is None else state["id"][idx]
    return torch.cat([torch.stack(cols, 1), ids.view(torch.float64).unsqueeze(1)], 1)


def unpack(rows):
    st = {k: rows[:, c].contiguous() for c, k in enumerate(STATE)}
    st["id"] = rows[:, len(STATE)].contiguous().view(torch.int64)
    return st


def positions_of(ids_current, query):
    """Positions in the current order of the particles with ids `query`."""
    order = torch.argsort(ids_current)
    srt = ids_current[order]
    p = torch.searchsorted(srt, query)
    assert bool((srt[p.clamp(max=srt.numel() - 1)] == query).all()), "halo id not found"
    return order[p]


# ----------------------------------------------------------------------------- stepping
class DistributedSim:
    """One rank of the decomposed simulation.  `state` holds this rank's share of
    the particles.  The particles stay resident in libsph between steps; only
    emigrants, ghosts and halo values travel, packed and unpacked by libsph's
    device plumbing (sph_compact / sph_pack_rows / sph_append_rows /
    sph_select_ghosts / sph_gather_field / sph_scatter_field).  All torch work
    runs on the libsph stream, so the two never need cross-stream ordering."""

    def __init__(self, params, state, n_capacity: int, device: int = 0, force_exchange: bool = False,
                 **kw):
        from . import sph
        if getattr(params, "gravity", 0):
            # self-gravity is long-range: a 2 h_max halo cannot supply it (a global
            # tree or multipole exchange would be needed)
            raise NotImplementedError("DistributedSim: self-gravity is not decomposed")
        self.sph = sph
        # force_exchange: run the partition / migration / ghost / halo plumbing even
        # on one rank (it then moves nothing) -- measures its cost (tools/decomp_probe.py)
        self.xchg = force_exchange
        self.params = params
        self.comm = Comm()
        self.dev = torch.device("cuda", device)
        self.sim = sph.Simulation(params, n_capacity=n_capacity, device=device, **kw)
        self.box_len = [float(b - a) for a, b in zip(params.box_min, params.box_max)]
        self.t, self.dt_prev, self.first = 0.0, float(params.dt_first), True
        self.stats = {}
        self.profile = None  # dict name -> seconds when set (synchronising section timer)
        self._t_last = None
        self.local = {k: torch.as_tensor(np.ascontiguousarray(v)) for k, v in state.items()}

    # the local (owned) particles: uploading replaces the held set
    @property
    def local(self):
        st = self._held_state()
        keep = (st["id"] & GHOST_BIT) == 0
        return {k: v[keep].contiguous() for k, v in st.items()}

    @local.setter
    def local(self, st):
        # the caller may have produced st on its own stream (e.g. async H2D copies)
        self.sim.stream.wait_stream(torch.cuda.current_stream(self.dev))
        with torch.cuda.stream(self.sim.stream):
            self.sim.set_particles({k: st[k].to(self.dev).contiguous() for k in STATE + ("id",)})
        self.sim.set_time(self.t, self.dt_prev, self.first)
        self.has_ghosts = False

    def _mark(self, name):
        if self.profile is None:
            return
        import time
        torch.cuda.synchronize(self.dev)
        now = time.perf_counter()
        if self._t_last is not None and name:
            self.profile[name] = self.profile.get(name, 0.0) + now - self._t_last
        self._t_last = now

    def _field(self, name, dtype=torch.float64):
        out = torch.empty(self.sim.n, dtype=dtype, device=self.dev)
        self.sim.get_field(name, out=out)
        return out

    def _held_state(self):
        st = {k: self._field(k) for k in STATE}
        st["id"] = self._field("id", torch.int64)
        return st

    def step(self):
        caller = torch.cuda.current_stream(self.dev)
        self.sim.stream.wait_stream(caller)
        with torch.cuda.stream(self.sim.stream):
            dt = self._step()
        caller.wait_stream(self.sim.stream)  # the caller's later work (events, copies) follows the step
        return dt

    def _exchange_rows(self, idx, dest, or_id=0):
        """Rows of the particles idx (current order) to ranks dest; returns the
        received rows (cat, in source-rank order) and the per-source counts."""
        world = self.comm.world
        order = torch.argsort(dest, stable=True)
        idx = idx[order]
        counts = torch.bincount(dest, minlength=world).cpu().tolist()
        rows = self.sim.pack_rows(idx, or_id)
        recv = self.comm.alltoallv(list(torch.split(rows, counts, 0)))
        return torch.cat(recv, 0), [int(r.shape[0]) for r in recv], idx, counts

    def _step(self):
        comm, sim = self.comm, self.sim
        world, rank = comm.world, comm.rank
        xchg = world > 1 or self.xchg
        self._mark(None)
        if xchg:
            # 1. drop last step's ghosts; keys in the current order; SFC partition
            if self.has_ghosts:
                sim.compact(drop_ghosts=True)
            sim.compute_keys()
            keys = self._field("key", torch.int64)
            splits = sfc_splits(keys, comm)
            own = owners(keys, splits)
            self._mark("keys_partition")
            # migration: particles whose key left this rank's range
            emig = own != rank
            eidx = torch.nonzero(emig).flatten()
            rows, _, _, _ = self._exchange_rows(eidx, own[eidx])
            sim.compact(keep=~emig)
            sim.append_rows(rows)
            self._mark("migrate")
            # 2. ghosts within 2 h_max of every other rank's domain box
            x = torch.stack([self._field("x"), self._field("y"), self._field("z")], 1)
            hl = self._field("h")
            hmax = comm.all_reduce(hl.max().reshape(1) if hl.numel() else
                                   torch.zeros(1, dtype=torch.float64, device=self.dev),
                                   dist.ReduceOp.MAX if world > 1 else None)
            boxes = domain_boxes(x, comm)
            radius = float(2.0 * hmax.item()) * (1.0 + 1e-9)
            mask = sim.select_ghosts(boxes.reshape(world, 6).cpu().numpy(), rank, radius)
            gidx, gdest = [], []
            for r in range(world):
                if r == rank:
                    continue
                ir = torch.nonzero((mask >> r) & 1).flatten()
                gidx.append(ir)
                gdest.append(torch.full_like(ir, r))
            e = torch.zeros(0, dtype=torch.int64, device=self.dev)
            gidx, gdest = torch.cat(gidx + [e]), torch.cat(gdest + [e])
            grows, gcounts, sent_idx, scounts = self._exchange_rows(gidx, gdest, GHOST_BIT)
            n_loc = sim.n
            sim.append_rows(grows)
            self.has_ghosts = True
            self.stats = {"n_local": n_loc, "n_ghost": int(sum(gcounts))}
            self._mark("ghosts")
        # 3. the hot path with the halo refreshes
        sim.build_tree()
        if xchg:
            order = self._field("order", torch.int32).to(torch.int64)
            inv = torch.empty_like(order)
            inv[order] = torch.arange(order.numel(), device=self.dev)
            self._src = torch.split(inv[sent_idx], scounts, 0)              # mine others hold
            self._dst = inv[n_loc:n_loc + sum(gcounts)]                      # theirs I hold
            self._mark("tree_maps")
        sim.find_neighbors(stats=False)
        sim.density()
        self._halo(["rho"])
        sim.eos()
        if getattr(self.params, "gradh", 0) or getattr(self.params, "ve", 0):
            sim.gradh()  # owners' normalised rho (volume elements) and Omega over the ghosts
            self._halo((["rho"] if getattr(self.params, "ve", 0) else [])
                       + (["omega"] if getattr(self.params, "gradh", 0) else []))
        sim.iad()
        # H3: the owners' C (and Balsara factors when the AV switch is on)
        h3 = ["c11", "c12", "c13", "c22", "c23", "c33"]
        if getattr(self.params, "av_switch", 0):
            h3.append("bal")
        self._halo(h3)
        sim.momentum_energy()
        if sim.stir_enabled:  # driving: every rank holds the same OU state and noise
            sim.stir()
        self._mark("physics_halos")
        # 4. global dt, update (ghosts are dropped at the next step)
        if xchg:
            mhc = torch.tensor([sim.get_local_min_hc()], dtype=torch.float64, device=self.dev)
            mhc = comm.all_reduce(mhc, dist.ReduceOp.MIN if world > 1 else None)
            sim.set_global_min_hc(float(mhc.item()))
        dt = sim.timestep()
        sim.update()
        self.t, self.dt_prev, self.first = self.t + dt, dt, False
        self._mark("dt_update")
        return dt

    def _halo(self, names):
        if not (self.comm.world > 1 or self.xchg):
            return
        sim = self.sim
        parts = [torch.stack([sim.gather_field(k, p) for k in names], 1) for p in self._src]
        recv = torch.cat(self.comm.alltoallv(parts), 0)
        for c, k in enumerate(names):
            sim.scatter_field(k, self._dst, recv[:, c].contiguous())

    def gather_state(self):
        """All particles on every rank, sorted by id (host numpy) -- for tests."""
        with torch.cuda.stream(self.sim.stream):
            return self._gather_state()

    def _gather_state(self):
        rows = pack(self.local)
        n = torch.tensor([rows.shape[0]], dtype=torch.int64, device=self.dev)
        ns = [int(v.item()) for v in self.comm.all_gather(n)]
        m = max(ns)
        pad = torch.zeros((m, rows.shape[1]), dtype=rows.dtype, device=self.dev)
        pad[:rows.shape[0]] = rows
        allr = torch.cat([a[:k] for a, k in zip(self.comm.all_gather(pad), ns)], 0)
        st = unpack(allr)
        order = torch.argsort(st["id"])
        return {k: v[order].cpu().numpy() for k, v in st.items()}
