"""Multi-GPU SPH step: space-filling-curve domain decomposition with halo
exchange ("domain decomposition, halo exchanges",
P:216 DomainDecompAndSync, P:220 the end-of-step collective for dt).

One process per GPU.  Every rank owns a contiguous range of the 63-bit Morton
curve.  Each step (every selection, count, split, pack and map is a libsph
device call, include/sph.h "SFC decomposition on the device"; this module only
issues the collectives between them):

  1. last step's ghosts stay until the migration's compaction (skipped by
     every reduction);
  2. global box and h_max: MAX all-reduce of 7 doubles (exact), set as the key
     box of the open axes -- every rank's keys are the single-GPU run's;
  3. SFC partition: key histogram (2^15 bins of the top key bits), SUM
     all-reduce, split bins and owners on the device; the per-rank counts go
     through one all-to-all and ONE host read (host sync 1); the migrants move as
     rows in one all-to-all;
  4. ghosts by cells: every particle in a cell (side >= 2 h_max) adjacent to a
     cell of rank r is sent to r with SPH_GHOST_BIT in its id -- counts (host
     sync 2) and rows as in 3;
  5. one tree build (sort) of locals + ghosts; the sort's inverse permutation
     maps the sent and received ghosts to their new positions; the libsph hot
     path with the owners' values scattered over the ghosts after DENSITY (rho;
     EOS then derives p, c, V), GRADH (rho with volume elements, Omega) and IAD
     (C, the Balsara factor) -- H2/H3 of SURVEY 8(e), all-to-alls with known
     counts;
  6. dt: MIN all-reduce of the local min h/c on the device, update;
     sph_timestep's dt read is host sync 3.
The particles stay in libsph; only migrants, ghosts and halo values move.

The held set is sorted in the global Morton order and every target's
neighbours are the same particles as in a single-GPU run, so the result is
bit-identical to the one-GPU step, for periodic and open boxes alike
(tests/test_gpu_decomp.py).  Collectives are torch.distributed calls on device
tensors (NCCL over NVLink on GPUs; gloo, via host copies, in the tests that run
several ranks on one GPU or on the CPU).
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

GHOST_BIT = 1 << 62
STATE = ("x", "y", "z", "vx", "vy", "vz", "h", "m", "u", "du_m1")
HIST_BITS = 15  # SFC partition granularity: 2^15 bins of the top key bits (level-5 cells)
ROW = 11        # SPH_ROW_DOUBLES


# ----------------------------------------------------------------------------- comm
class Comm:
    """Collectives over the default process group; host tensors for gloo."""

    def __init__(self, always: bool = False):
        self.rank = dist.get_rank() if dist.is_initialized() else 0
        world = dist.get_world_size() if dist.is_initialized() else 1
        self.host = (dist.get_backend() == "gloo") if dist.is_initialized() else True
        # always: issue the collectives even on a one-rank group (exercises the
        # NCCL data plane on a single GPU); `world` below is then the routing's
        # world, and the short cuts test `self.world == 1` through `_local`
        self.world = world
        self._local = world == 1 and not (always and dist.is_initialized())

    def _to(self, t):
        return t.cpu() if self.host else t

    def all_reduce(self, t, op):
        if self._local:
            return t
        x = self._to(t.clone())
        dist.all_reduce(x, op=op)
        return x.to(t.device)

    def all_reduce_(self, t, op):
        """In-place all-reduce of a device tensor (gloo: through a host copy)."""
        if self._local:
            return t
        if self.host:
            x = t.cpu()
            dist.all_reduce(x, op=op)
            t.copy_(x)
        else:
            dist.all_reduce(t, op=op)
        return t

    def all_to_all(self, recv, send, recv_counts, send_counts):
        """Rows send[sum send_counts, ...] -> recv[sum recv_counts, ...] (dim-0
        splits known on the host: no count exchange here)."""
        if self._local:
            if recv.numel():
                recv.copy_(send)
            return recv
        if self.host:
            r = torch.empty(recv.shape, dtype=recv.dtype)
            dist.all_to_all_single(r, send.cpu().contiguous(), [int(c) for c in recv_counts],
                                   [int(c) for c in send_counts])
            recv.copy_(r)
        else:
            dist.all_to_all_single(recv, send.contiguous(), [int(c) for c in recv_counts],
                                   [int(c) for c in send_counts])
        return recv

    def all_to_all_start(self, recv, send, recv_counts, send_counts):
        """all_to_all that overlaps the caller's next kernels (NCCL: async on its
        own stream; all_to_all_finish makes the current stream wait).  gloo and
        world 1: completes here."""
        if self._local or self.host:
            self.all_to_all(recv, send, recv_counts, send_counts)
            return None
        return dist.all_to_all_single(recv, send.contiguous(), [int(c) for c in recv_counts],
                                      [int(c) for c in send_counts], async_op=True)

    @staticmethod
    def all_to_all_finish(work):
        if work is not None:
            work.wait()

    def all_gather(self, t):
        if self._local:
            return [t]
        x = self._to(t.contiguous())
        out = [torch.empty_like(x) for _ in range(self.world)]
        dist.all_gather(out, x)
        return [o.to(t.device) for o in out]

    def alltoallv(self, parts):
        """parts[r]: tensor [n_r, ...] for rank r -> list of received [m_s, ...]."""
        if self._local:
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
        # overlap the H2 / H3 halos with the interior targets (not with grad-h / VE)
        self.overlap = kw.pop("overlap", True) and not (getattr(params, "gradh", 0) or getattr(params, "ve", 0))
        self.params = params
        self.comm = Comm(always=kw.pop("comm_always", False))
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
        self.n_local = self.sim.n

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

    def _step(self):
        comm, sim = self.comm, self.sim
        world, rank = comm.world, comm.rank
        xchg = world > 1 or self.xchg
        dev = self.dev
        self._mark(None)
        if xchg:
            # 1.-2. (last step's ghosts are skipped by the reduction, the histogram
            # and the owners, and dropped with the emigrants in one compaction)
            # global box and h_max (exact MAX), the key box of the open axes
            red = sim.decomp_reduce()
            comm.all_reduce_(red, dist.ReduceOp.MAX)
            sim.set_key_box(red)
            # 3. SFC partition and migration
            sim.compute_keys()
            hist = sim.key_histogram(HIST_BITS)
            comm.all_reduce_(hist, dist.ReduceOp.SUM)
            mig, own = sim.decomp_owners(hist, HIST_BITS, rank, world)
            send = own.clone()
            send[rank] = 0
            recv = torch.empty_like(send)
            comm.all_to_all(recv, send, [1] * world, [1] * world)
            host = torch.cat([own, recv]).tolist()                         # host sync 1
            keep = int(host[rank])
            send_c = [0 if r == rank else int(host[r]) for r in range(world)]
            recv_c = [int(v) for v in host[world:]]
            rows, _ = sim.decomp_pack(mig, world, sum(send_c))
            rrows = torch.empty((sum(recv_c), ROW), dtype=torch.float64, device=dev)
            comm.all_to_all(rrows, rows, recv_c, send_c)
            sim.decomp_drop(mig, keep)
            if rrows.shape[0]:
                sim.append_rows(rrows)
            self.n_local = keep + sum(recv_c)
            self._mark("partition_migrate")
            # 4. ghosts by cells
            sim.compute_keys()
            gmask, gcnt = sim.decomp_ghosts(HIST_BITS, rank, world)
            grecv = torch.empty_like(gcnt)
            comm.all_to_all(grecv, gcnt, [1] * world, [1] * world)
            gh = torch.cat([gcnt, grecv]).tolist()                         # host sync 2
            self.g_send = [int(v) for v in gh[:world]]
            self.g_recv = [int(v) for v in gh[world:]]
            grows, gpos = sim.decomp_pack(gmask, world, sum(self.g_send), GHOST_BIT)
            grr = torch.empty((sum(self.g_recv), ROW), dtype=torch.float64, device=dev)
            comm.all_to_all(grr, grows, self.g_recv, self.g_send)
            if grr.shape[0]:
                sim.append_rows(grr)
            self.has_ghosts = True
            self.stats = {"n_local": self.n_local, "n_ghost": sum(self.g_recv), "n_migrated_in": sum(recv_c)}
            self._mark("ghosts")
        # 5. one tree build of locals + ghosts, the halo maps, the hot path
        sim.build_tree()
        if xchg:
            self._src = sim.decomp_map(gpos)                                   # mine that others hold
            self._dst = sim.decomp_map(None, first=self.n_local, m=sum(self.g_recv))  # theirs I hold
            self._mark("tree_maps")
        sim.find_neighbors(stats=False)
        sim.density()
        h3 = ["c11", "c12", "c13", "c22", "c23", "c33"]
        if getattr(self.params, "av_switch", 0):
            h3.append("bal")
        if xchg and self.overlap:
            # H2 / H3 in flight while the targets without ghost neighbours are
            # computed (sph_set_part); each target is computed once, so the
            # result equals the unsplit step bit for bit
            P = self.sph
            w2 = self._halo_start(["rho"])
            sim.eos()                                  # ghosts' values fixed below
            sim.set_part(P.PART_INTERIOR)
            sim.iad()
            self._halo_finish(w2)
            sim.set_part(P.PART_GHOSTS)
            sim.eos()
            sim.set_part(P.PART_BOUNDARY)
            sim.iad()
            w3 = self._halo_start(h3)
            sim.set_part(P.PART_INTERIOR)
            sim.momentum_energy()
            self._halo_finish(w3)
            sim.set_part(P.PART_BOUNDARY)
            sim.momentum_energy()
            sim.set_part(P.PART_ALL)
        else:
            self._halo(["rho"])
            sim.eos()
            if getattr(self.params, "gradh", 0) or getattr(self.params, "ve", 0):
                sim.gradh()  # owners' normalised rho (volume elements) and Omega over the ghosts
                self._halo((["rho"] if getattr(self.params, "ve", 0) else [])
                           + (["omega"] if getattr(self.params, "gradh", 0) else []))
            sim.iad()
            self._halo(h3)  # H3: the owners' C (and Balsara factors with the AV switch)
            sim.momentum_energy()
        if sim.stir_enabled:  # driving: every rank holds the same OU state and noise
            sim.stir()
        self._mark("physics_halos")
        # 6. global dt on the device, update
        if xchg:
            mhc = sim.min_hc_dev()
            comm.all_reduce_(mhc, dist.ReduceOp.MIN)
            sim.set_min_hc_dev(mhc)
        dt = sim.timestep()                                                # host sync 3
        sim.update()
        self.t, self.dt_prev, self.first = self.t + dt, dt, False
        self._mark("dt_update")
        return dt

    def _halo(self, names):
        if not (self.comm.world > 1 or self.xchg):
            return
        self._halo_finish(self._halo_start(names))

    def _halo_start(self, names):
        sim = self.sim
        send = sim.halo_gather(names, self._src)
        recv = torch.empty((sum(self.g_recv), len(names)), dtype=torch.float64, device=self.dev)
        work = self.comm.all_to_all_start(recv, send, self.g_recv, self.g_send)
        return names, send, recv, work

    def _halo_finish(self, h):
        names, send, recv, work = h
        self.comm.all_to_all_finish(work)
        if recv.shape[0]:
            self.sim.halo_scatter(names, self._dst, recv)

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
