"""Thin ctypes binding of libsph (include/sph.h): argument marshalling only.

Every step of the SPH path runs in libsph's CUDA kernels.  PyTorch provides the
device arena (one uint8 tensor), the CUDA stream and, for multi-GPU runs, the
process group.  There is no CPU fallback: if libsph.so cannot be loaded, or no
CUDA device is present, constructing a :class:`Simulation` raises.

Names follow the C ABI: ``Simulation.build_tree`` calls ``sph_build_tree`` etc.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

from . import _build

SPH_OK = 0
STATUS = {0: "OK", 1: "ERR_ARG", 2: "ERR_STATE", 3: "ERR_CUDA", 4: "ERR_NCCL", 5: "ERR_NVML",
          6: "ERR_NO_PERMISSION", 7: "ERR_NOT_SUPPORTED", 8: "ERR_CAPACITY", 9: "ERR_HCAP",
          10: "ERR_SINGULAR", 11: "ERR_BOX"}
PHASES = ("keys", "sort", "cells", "neighbors", "density", "eos", "iad", "momentum_energy",
          "timestep", "update", "stir", "gravity", "gradh")
STIR_NMODES = 61
NPHASES = len(PHASES)
FIELDS = ("x", "y", "z", "vx", "vy", "vz", "h", "m", "u", "du_m1", "id", "key", "nc", "rho", "p",
          "c", "c11", "c12", "c13", "c22", "c23", "c33", "ax", "ay", "az", "du", "divv", "curlx",
          "curly", "curlz", "bal", "phi", "omega", "vsig", "order")
FIELD_ID = {name: k for k, name in enumerate(FIELDS)}
FIELD_DTYPE = {"id": np.int64, "key": np.uint64, "nc": np.int32, "order": np.int32}
ROW_DOUBLES = 11  # SPH_ROW_DOUBLES: x y z vx vy vz h m u du_m1 id(bits)
MEM_HOST, MEM_DEVICE, MEM_HOST_ASYNC = 0, 1, 2
PART_ALL, PART_INTERIOR, PART_BOUNDARY, PART_GHOSTS = 0, 1, 2, 3
ACCOUNTING_OFF, ACCOUNTING_PHASE = 0, 1
CLOCK_DEFAULT, CLOCK_STATIC, CLOCK_PER_PHASE = 0, 1, 2


class SphError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"{STATUS.get(code, code)}: {msg}")
        self.code = code
        self.name = STATUS.get(code, str(code))


class Config(C.Structure):
    _fields_ = [
        ("n_capacity", C.c_int64), ("box_min", C.c_double * 3), ("box_max", C.c_double * 3),
        ("periodic", C.c_int32 * 3), ("eos", C.c_int32), ("gamma", C.c_double),
        ("cs0", C.c_double), ("K", C.c_double), ("ng0", C.c_double), ("ngmax", C.c_int32),
        ("max_cell_level", C.c_int32), ("h_cap", C.c_double), ("k_cour", C.c_double),
        ("dt_max_growth", C.c_double), ("dt_first", C.c_double), ("av_alpha", C.c_double),
        ("av_beta", C.c_double), ("av_eps", C.c_double), ("device", C.c_int32),
        ("accounting", C.c_int32), ("rank", C.c_int32), ("nranks", C.c_int32),
        ("stir_steps", C.c_int32), ("divcurl", C.c_int32), ("av_switch", C.c_int32),
        ("gravity", C.c_int32), ("grav_level", C.c_int32), ("grav_G", C.c_double),
        ("grav_eps", C.c_double), ("grav_theta", C.c_double), ("gradh", C.c_int32),
        ("dt_vsig", C.c_int32), ("ve", C.c_int32), ("grav_fp64", C.c_int32), ("reserved", C.c_int32 * 4),
    ]


class NbrStats(C.Structure):
    _fields_ = [("min_nc", C.c_int32), ("max_nc", C.c_int32), ("mean_nc", C.c_double),
                ("total", C.c_int64), ("candidates", C.c_int64), ("passes", C.c_int64)]


class StepInfo(C.Structure):
    _fields_ = [("t", C.c_double), ("dt", C.c_double), ("nbr", NbrStats),
                ("cell_level", C.c_int32), ("graph", C.c_int32),
                ("phase_ms", C.c_double * NPHASES), ("grav_multipoles", C.c_int64),
                ("grav_pairs", C.c_int64), ("grav_pops", C.c_int64)]


class EnergyRow(C.Structure):
    _fields_ = [("phase", C.c_int32), ("name", C.c_char * 32), ("calls", C.c_int64),
                ("seconds", C.c_double), ("joules", C.c_double), ("mean_sm_mhz", C.c_double),
                ("locked_mhz", C.c_uint32), ("available", C.c_int32)]


class EnergyWindow(C.Structure):
    _fields_ = [("wall_seconds", C.c_double), ("sampled_seconds", C.c_double),
                ("sampled_joules", C.c_double), ("between_joules", C.c_double),
                ("counter_joules", C.c_double), ("samples", C.c_int64)]


class StirParams(C.Structure):
    _fields_ = [("sigma", C.c_double), ("t_decay", C.c_double), ("sol_weight", C.c_double)]


class TraceSample(C.Structure):
    _fields_ = [("t_ms", C.c_double), ("phase", C.c_int32), ("sm_mhz", C.c_uint32),
                ("power_mw", C.c_uint32), ("query_us", C.c_uint32), ("energy_mj", C.c_uint64)]


# Every symbol include/sph.h declares (checked by tests/test_abi.py).
EXPORTS = ("sph_config_default", "sph_workspace_size", "sph_init", "sph_finalize",
           "sph_last_error", "sph_phase_name", "sph_set_particles", "sph_set_time",
           "sph_get_time", "sph_get_n", "sph_get_field", "sph_build_tree", "sph_find_neighbors",
           "sph_get_neighbors", "sph_density", "sph_eos", "sph_iad", "sph_momentum_energy",
           "sph_timestep", "sph_update", "sph_step", "sph_set_clock_policy",
           "sph_energy_report", "sph_energy_reset", "sph_energy_counter_mj", "sph_energy_totals", "sph_repeat_phase",
           "sph_set_accounting", "sph_kernel_launches", "sph_set_field",
           "sph_get_local_min_hc", "sph_set_global_min_hc", "sph_get_neighbor_rows",
           "sph_trace_start", "sph_trace_stop", "sph_stir_modes", "sph_stir_init", "sph_stir",
           "sph_stir_get_state", "sph_supported_clocks", "sph_gravity", "sph_gradh",
           "sph_compute_keys", "sph_compact", "sph_pack_rows", "sph_append_rows",
           "sph_select_ghosts", "sph_gather_field", "sph_scatter_field",
           "sph_decomp_reduce", "sph_set_key_box", "sph_key_histogram", "sph_decomp_owners",
           "sph_decomp_ghosts", "sph_decomp_pack", "sph_decomp_drop", "sph_decomp_map",
           "sph_halo_gather", "sph_halo_scatter", "sph_min_hc_dev", "sph_set_min_hc_dev", "sph_sync",
           "sph_set_part")
GHOST_BIT = 1 << 62

_lib = None


def load(build_if_missing: bool = True):
    """Loads libsph.so (building it in-tree first when missing/stale and nvcc exists)."""
    global _lib
    if _lib is not None:
        return _lib
    path = _build.LIB
    if build_if_missing and (not os.path.exists(path) or _build.stale()):
        if os.path.exists(_build.NVCC):
            _build.build()
    if not os.path.exists(path):
        raise RuntimeError(f"libsph.so not found at {path}; run __graft_entry__.build()")
    L = C.CDLL(path)
    P, I, I64, D, V = C.c_void_p, C.c_int, C.c_int64, C.c_double, C.c_void_p
    L.sph_last_error.restype = C.c_char_p
    L.sph_last_error.argtypes = [P]
    L.sph_phase_name.restype = C.c_char_p
    L.sph_phase_name.argtypes = [I]
    L.sph_config_default.argtypes = [C.POINTER(Config)]
    L.sph_workspace_size.argtypes = [C.POINTER(Config), C.POINTER(C.c_size_t)]
    L.sph_init.argtypes = [C.POINTER(Config), V, C.c_size_t, V, C.POINTER(P)]
    L.sph_finalize.argtypes = [P]
    L.sph_finalize.restype = None
    L.sph_set_particles.argtypes = [P, I64] + [V] * 11 + [I]
    L.sph_set_time.argtypes = [P, D, D, I]
    L.sph_get_time.argtypes = [P, C.POINTER(D), C.POINTER(D), C.POINTER(I)]
    L.sph_get_n.argtypes = [P, C.POINTER(I64)]
    L.sph_get_field.argtypes = [P, I, V, I]
    for f in ("sph_build_tree", "sph_density", "sph_eos", "sph_iad", "sph_momentum_energy",
              "sph_update", "sph_energy_reset"):
        getattr(L, f).argtypes = [P]
    L.sph_find_neighbors.argtypes = [P, C.POINTER(NbrStats)]
    L.sph_get_neighbors.argtypes = [P, V, V, I64]
    L.sph_timestep.argtypes = [P, C.POINTER(D)]
    L.sph_step.argtypes = [P, C.POINTER(StepInfo)]
    L.sph_set_clock_policy.argtypes = [P, I, C.POINTER(C.c_uint32)]
    L.sph_energy_report.argtypes = [P, C.POINTER(EnergyRow), I, C.POINTER(I)]
    L.sph_energy_counter_mj.argtypes = [P, C.POINTER(C.c_uint64)]
    L.sph_energy_totals.argtypes = [P, C.POINTER(EnergyWindow)]
    L.sph_repeat_phase.argtypes = [P, I, I, C.POINTER(D), C.POINTER(D)]
    L.sph_set_accounting.argtypes = [P, I]
    L.sph_set_field.argtypes = [P, I, V, I]
    L.sph_get_neighbor_rows.argtypes = [P, V, I64, V, V, I64]
    L.sph_get_local_min_hc.argtypes = [P, C.POINTER(D)]
    L.sph_set_global_min_hc.argtypes = [P, D]
    L.sph_kernel_launches.argtypes = [C.POINTER(I64)]
    L.sph_stir_modes.argtypes = [V, I]
    L.sph_stir_init.argtypes = [P, C.POINTER(StirParams), V, V, V, I64, I]
    L.sph_stir.argtypes = [P]
    L.sph_gravity.argtypes = [P]
    L.sph_gradh.argtypes = [P]
    L.sph_compute_keys.argtypes = [P]
    L.sph_compact.argtypes = [P, V, I, C.POINTER(I64)]
    L.sph_pack_rows.argtypes = [P, V, I64, C.c_uint64, V]
    L.sph_append_rows.argtypes = [P, V, I64]
    L.sph_select_ghosts.argtypes = [P, V, I, I, D, V]
    L.sph_gather_field.argtypes = [P, I, V, I64, V]
    L.sph_scatter_field.argtypes = [P, I, V, I64, V]
    L.sph_stir_get_state.argtypes = [P, V, C.POINTER(I64)]
    L.sph_decomp_reduce.argtypes = [P, V]
    L.sph_set_key_box.argtypes = [P, V]
    L.sph_key_histogram.argtypes = [P, I, V]
    L.sph_decomp_owners.argtypes = [P, V, I, I, I, V, V]
    L.sph_decomp_ghosts.argtypes = [P, I, I, I, V, V]
    L.sph_decomp_pack.argtypes = [P, V, I, C.c_uint64, V, V]
    L.sph_decomp_drop.argtypes = [P, V, I64]
    L.sph_decomp_map.argtypes = [P, V, I64, I64, V]
    L.sph_halo_gather.argtypes = [P, V, I, V, I64, V]
    L.sph_halo_scatter.argtypes = [P, V, I, V, I64, V]
    L.sph_min_hc_dev.argtypes = [P, V]
    L.sph_set_min_hc_dev.argtypes = [P, V]
    L.sph_sync.argtypes = [P]
    L.sph_set_part.argtypes = [P, I]
    L.sph_supported_clocks.argtypes = [P, V, I, C.POINTER(I)]
    L.sph_trace_start.argtypes = [P, D, I64]
    L.sph_trace_stop.argtypes = [P, V, I64, C.POINTER(I64)]
    _lib = L
    return L


def kernel_launches() -> int:
    """libsph kernels launched so far by this process (sph_kernel_launches)."""
    v = C.c_int64()
    _check(load().sph_kernel_launches(C.byref(v)), None)
    return int(v.value)


def config_from_params(params, n_capacity: int, device: int = 0, accounting: int = 0,
                       max_cell_level: int = 8, stir_steps: int = 0) -> Config:
    """sph_config from the StepParams preset of paper_conf_sc_simsekpc24_b200.ics."""
    L = load()
    c = Config()
    _check(L.sph_config_default(C.byref(c)), None)
    c.n_capacity = int(n_capacity)
    c.box_min[:] = [float(v) for v in params.box_min]
    c.box_max[:] = [float(v) for v in params.box_max]
    c.periodic[:] = [int(v) for v in params.periodic]
    c.eos = int(params.eos)
    for k in ("gamma", "cs0", "K", "ng0", "h_cap", "k_cour", "dt_max_growth", "dt_first",
              "av_alpha", "av_beta", "av_eps"):
        setattr(c, k, float(getattr(params, k)))
    c.ngmax = int(params.ngmax)
    c.max_cell_level = int(max_cell_level)
    c.device = int(device)
    c.accounting = int(accounting)
    c.stir_steps = int(stir_steps)
    c.divcurl = int(getattr(params, "divcurl", 0))
    c.av_switch = int(getattr(params, "av_switch", 0))
    c.gravity = int(getattr(params, "gravity", 0))
    c.gradh = int(getattr(params, "gradh", 0))
    c.dt_vsig = int(getattr(params, "dt_vsig", 0))
    c.ve = int(getattr(params, "ve", 0))
    if c.gravity:
        c.grav_level = int(params.grav_level)
        c.grav_G = float(params.grav_G)
        c.grav_eps = float(params.grav_eps)
        c.grav_theta = float(params.grav_theta)
        c.grav_fp64 = int(getattr(params, "grav_fp64", 0))
    return c


def stir_modes() -> np.ndarray:
    """sph_stir_modes: the fixed driving mode set, int32 [61, 3] (host only)."""
    n3 = np.zeros((STIR_NMODES, 3), np.int32)
    m = load().sph_stir_modes(C.c_void_p(n3.ctypes.data), STIR_NMODES)
    if m < 0:
        raise SphError(-m, "sph_stir_modes")
    return n3[:m]


def _check(rc, ctx):
    if rc != SPH_OK:
        L = load()
        msg = L.sph_last_error(ctx)
        raise SphError(rc, msg.decode() if msg else "")


def _ptr(a):
    """Pointer + memory kind of a numpy array (host) or torch tensor (host/device)."""
    if a is None:
        return None, MEM_HOST
    if isinstance(a, np.ndarray):
        assert a.flags.c_contiguous
        return a.ctypes.data, MEM_HOST
    import torch
    assert isinstance(a, torch.Tensor) and a.is_contiguous()
    return a.data_ptr(), (MEM_DEVICE if a.is_cuda else MEM_HOST)


class Simulation:
    """One libsph context on one CUDA device (arena + stream owned by torch)."""

    def __init__(self, params, n_capacity: int, device: int = 0, accounting: int = ACCOUNTING_OFF,
                 stream=None, max_cell_level: int = 8, stir_steps: int = 0):
        import torch
        if not torch.cuda.is_available():
            raise RuntimeError("libsph needs a CUDA device (no CPU fallback)")
        self.L = load()
        self.torch = torch
        self.device = torch.device("cuda", device)
        self.cfg = config_from_params(params, n_capacity, device, accounting, max_cell_level, stir_steps)
        nbytes = C.c_size_t(0)
        _check(self.L.sph_workspace_size(C.byref(self.cfg), C.byref(nbytes)), None)
        self.arena_bytes = int(nbytes.value)
        self.arena = torch.empty(self.arena_bytes + 256, dtype=torch.uint8, device=self.device)
        base = self.arena.data_ptr()
        self._base = (base + 255) // 256 * 256
        self.stream = stream if stream is not None else torch.cuda.Stream(device=self.device)
        self.ctx = C.c_void_p()
        _check(self.L.sph_init(C.byref(self.cfg), C.c_void_p(self._base), C.c_size_t(self.arena_bytes),
                               C.c_void_p(self.stream.cuda_stream), C.byref(self.ctx)), None)
        self.n = 0
        self.stir_enabled = False

    # ---------------------------------------------------------------- lifetime
    def finalize(self):
        if self.ctx:
            self.L.sph_finalize(self.ctx)
            self.ctx = C.c_void_p()

    def __del__(self):
        try:
            self.finalize()
        except Exception:
            pass

    def _ok(self, rc):
        _check(rc, self.ctx)

    # ---------------------------------------------------------------- I/O
    def set_particles(self, state: dict):
        """state: x y z vx vy vz h m u [du_m1] [id] as numpy (host) or torch (cuda) arrays."""
        n = int(len(state["x"]))
        ptrs = []
        mem = None
        for k in ("x", "y", "z", "vx", "vy", "vz", "h", "m", "u", "du_m1", "id"):
            a = state.get(k)
            if isinstance(a, np.ndarray):
                want = np.int64 if k == "id" else np.float64
                if a.dtype != want or not a.flags.c_contiguous:
                    a = np.ascontiguousarray(a, dtype=want)
                    state = dict(state)
                    state[k] = a
            p, m = _ptr(a)
            if a is not None:
                if mem is None:
                    mem = m
                elif mem != m:
                    raise ValueError("all arrays must live in the same memory kind")
            ptrs.append(C.c_void_p(p) if p is not None else None)
        self._keep = state  # host buffers must outlive the async copies
        if mem == MEM_DEVICE:  # inputs produced on torch's stream: order libsph's copy after them
            self.stream.wait_stream(self.torch.cuda.current_stream(self.device))
        self._ok(self.L.sph_set_particles(self.ctx, n, *ptrs, mem if mem is not None else MEM_HOST))
        self.n = n

    def set_time(self, t: float, dt_prev: float, first_step: bool):
        self._ok(self.L.sph_set_time(self.ctx, t, dt_prev, 1 if first_step else 0))

    def get_time(self):
        t, d, f = C.c_double(), C.c_double(), C.c_int()
        self._ok(self.L.sph_get_time(self.ctx, C.byref(t), C.byref(d), C.byref(f)))
        return t.value, d.value, bool(f.value)

    def get_field(self, name: str, out=None, async_: bool = False):
        """Field `name` (current order) into `out` (numpy / torch host or cuda).
        async_: a pinned host `out` is filled asynchronously (valid after sync())."""
        dt = FIELD_DTYPE.get(name, np.float64)
        if out is None:
            out = np.empty(self.n, dtype=dt)
        p, mem = _ptr(out)
        if mem == MEM_DEVICE:  # the destination may be memory torch's stream still uses
            self.stream.wait_stream(self.torch.cuda.current_stream(self.device))
        elif async_:
            mem = MEM_HOST_ASYNC
        self._ok(self.L.sph_get_field(self.ctx, FIELD_ID[name], C.c_void_p(p), mem))
        return out

    def sync(self):
        self._ok(self.L.sph_sync(self.ctx))

    def set_field(self, name: str, src):
        """Overwrite RHO or C11..C33 (n values, current order) -- multi-GPU halo."""
        p, mem = _ptr(src)
        if mem == MEM_DEVICE:
            self.stream.wait_stream(self.torch.cuda.current_stream(self.device))
        self._keep_field = src
        self._ok(self.L.sph_set_field(self.ctx, FIELD_ID[name], C.c_void_p(p), mem))

    # ------------------------------------------------ decomposition plumbing (8(e))
    # Device tensors in/out; callers run their torch work on self.stream (the
    # libsph stream) so that no cross-stream ordering is needed.
    def compute_keys(self):
        self._ok(self.L.sph_compute_keys(self.ctx))

    def compact(self, keep=None, drop_ghosts: bool = False) -> int:
        """Stable compaction (keep: cuda uint8/bool tensor [n] or None)."""
        n = C.c_int64()
        kp = None if keep is None else C.c_void_p(keep.to(self.torch.uint8).contiguous().data_ptr())
        self._keep_field = keep
        self._ok(self.L.sph_compact(self.ctx, kp, 1 if drop_ghosts else 0, C.byref(n)))
        self.n = int(n.value)
        return self.n

    def pack_rows(self, idx, or_id: int = 0):
        """Rows [m, ROW_DOUBLES] (cuda float64) of the particles at idx (cuda int64)."""
        idx = idx.to(self.torch.int64).contiguous()
        out = self.torch.empty((idx.numel(), ROW_DOUBLES), dtype=self.torch.float64, device=self.device)
        self._ok(self.L.sph_pack_rows(self.ctx, C.c_void_p(idx.data_ptr()), idx.numel(),
                                      C.c_uint64(or_id), C.c_void_p(out.data_ptr())))
        self._keep_field = (idx, out)
        return out

    def append_rows(self, rows):
        rows = rows.contiguous()
        self._keep_field = rows
        self._ok(self.L.sph_append_rows(self.ctx, C.c_void_p(rows.data_ptr()), rows.shape[0]))
        self.n += int(rows.shape[0])

    def select_ghosts(self, boxes, self_rank: int, radius: float):
        """int64 cuda tensor [n]: bit r set iff the particle is within radius of rank r's box."""
        b = np.ascontiguousarray(boxes, dtype=np.float64).reshape(-1, 6)
        mask = self.torch.empty(self.n, dtype=self.torch.int64, device=self.device)
        self._ok(self.L.sph_select_ghosts(self.ctx, C.c_void_p(b.ctypes.data), b.shape[0], int(self_rank),
                                          float(radius), C.c_void_p(mask.data_ptr())))
        return mask

    def gather_field(self, name: str, idx):
        idx = idx.to(self.torch.int64).contiguous()
        out = self.torch.empty(idx.numel(), dtype=self.torch.float64, device=self.device)
        self._ok(self.L.sph_gather_field(self.ctx, FIELD_ID[name], C.c_void_p(idx.data_ptr()), idx.numel(),
                                         C.c_void_p(out.data_ptr())))
        self._keep_field = idx
        return out

    def scatter_field(self, name: str, idx, src):
        idx = idx.to(self.torch.int64).contiguous()
        src = src.to(self.torch.float64).contiguous()
        self._keep_field = (idx, src)
        self._ok(self.L.sph_scatter_field(self.ctx, FIELD_ID[name], C.c_void_p(idx.data_ptr()), idx.numel(),
                                          C.c_void_p(src.data_ptr())))

    # ------------------------------------------ SFC decomposition on the device (8(e))
    # All tensors are cuda tensors on self.device; callers run under
    # torch.cuda.stream(self.stream).  Nothing here synchronises.
    def _t(self, a):
        self._keep_field = a
        return C.c_void_p(a.data_ptr()) if a is not None else None

    def decomp_reduce(self):
        """float64 [7]: (-min x, -min y, -min z, max x, max y, max z, max h) of the non-ghosts."""
        red = self.torch.empty(7, dtype=self.torch.float64, device=self.device)
        self._ok(self.L.sph_decomp_reduce(self.ctx, self._t(red)))
        return red

    def set_key_box(self, red):
        self._keep_box = red
        self._ok(self.L.sph_set_key_box(self.ctx, None if red is None else C.c_void_p(red.data_ptr())))

    def key_histogram(self, bits: int):
        hist = self.torch.empty(1 << bits, dtype=self.torch.int64, device=self.device)
        self._ok(self.L.sph_key_histogram(self.ctx, int(bits), self._t(hist)))
        return hist

    def decomp_owners(self, hist, bits: int, rank: int, world: int):
        """(migration mask int64 [n] = 1 << owner or 0, counts int64 [world])."""
        mask = self.torch.empty(max(self.n, 1), dtype=self.torch.int64, device=self.device)
        counts = self.torch.empty(world, dtype=self.torch.int64, device=self.device)
        self._keep_hist = hist
        self._ok(self.L.sph_decomp_owners(self.ctx, C.c_void_p(hist.data_ptr()), int(bits), int(rank), int(world),
                                          C.c_void_p(mask.data_ptr()), C.c_void_p(counts.data_ptr())))
        return mask[:self.n], counts

    def decomp_ghosts(self, bits: int, rank: int, world: int):
        """(ghost mask int64 [n], counts int64 [world])."""
        mask = self.torch.empty(max(self.n, 1), dtype=self.torch.int64, device=self.device)
        counts = self.torch.empty(world, dtype=self.torch.int64, device=self.device)
        self._ok(self.L.sph_decomp_ghosts(self.ctx, int(bits), int(rank), int(world), C.c_void_p(mask.data_ptr()),
                                          C.c_void_p(counts.data_ptr())))
        return mask[:self.n], counts

    def decomp_pack(self, mask, world: int, total: int, or_id: int = 0):
        """(rows [total, ROW_DOUBLES], pos int64 [total]) grouped by destination rank."""
        rows = self.torch.empty((max(total, 1), ROW_DOUBLES), dtype=self.torch.float64, device=self.device)
        pos = self.torch.empty(max(total, 1), dtype=self.torch.int64, device=self.device)
        self._keep_mask = mask
        self._ok(self.L.sph_decomp_pack(self.ctx, C.c_void_p(mask.data_ptr()), int(world), C.c_uint64(or_id),
                                        C.c_void_p(rows.data_ptr()), C.c_void_p(pos.data_ptr())))
        return rows[:total], pos[:total]

    def decomp_drop(self, mask, n_expected: int):
        """Keep mask == 0 (mask None: drop the ghosts); the new n is n_expected (no sync)."""
        self._keep_mask = mask
        self._ok(self.L.sph_decomp_drop(self.ctx, None if mask is None else C.c_void_p(mask.data_ptr()),
                                        int(n_expected)))
        self.n = int(n_expected)

    def decomp_map(self, pre=None, first: int = 0, m: int | None = None):
        """Post-sort positions of pre-sort positions (pre, or first + arange(m))."""
        m = int(pre.numel()) if pre is not None else int(m)
        post = self.torch.empty(max(m, 1), dtype=self.torch.int64, device=self.device)
        self._keep_pre = pre
        self._ok(self.L.sph_decomp_map(self.ctx, None if pre is None else C.c_void_p(pre.data_ptr()), int(first), m,
                                       C.c_void_p(post.data_ptr())))
        return post[:m]

    def halo_gather(self, names, idx):
        f = (C.c_int32 * len(names))(*[FIELD_ID[k] for k in names])
        out = self.torch.empty((max(idx.numel(), 1), len(names)), dtype=self.torch.float64, device=self.device)
        self._keep_idx = idx
        self._ok(self.L.sph_halo_gather(self.ctx, f, len(names), C.c_void_p(idx.data_ptr()), idx.numel(),
                                        C.c_void_p(out.data_ptr())))
        return out[:idx.numel()]

    def halo_scatter(self, names, idx, src):
        f = (C.c_int32 * len(names))(*[FIELD_ID[k] for k in names])
        src = src.contiguous()
        self._keep_src = (idx, src)
        self._ok(self.L.sph_halo_scatter(self.ctx, f, len(names), C.c_void_p(idx.data_ptr()), idx.numel(),
                                         C.c_void_p(src.data_ptr())))

    def set_part(self, part: int):
        """sph_set_part: PART_ALL / PART_INTERIOR / PART_BOUNDARY / PART_GHOSTS."""
        self._ok(self.L.sph_set_part(self.ctx, int(part)))

    def min_hc_dev(self):
        out = self.torch.empty(1, dtype=self.torch.float64, device=self.device)
        self._ok(self.L.sph_min_hc_dev(self.ctx, C.c_void_p(out.data_ptr())))
        return out

    def set_min_hc_dev(self, v):
        self._keep_mhc = v
        self._ok(self.L.sph_set_min_hc_dev(self.ctx, C.c_void_p(v.data_ptr())))

    def get_local_min_hc(self) -> float:
        v = C.c_double()
        self._ok(self.L.sph_get_local_min_hc(self.ctx, C.byref(v)))
        return v.value

    def set_global_min_hc(self, v: float):
        self._ok(self.L.sph_set_global_min_hc(self.ctx, float(v)))

    def get_state(self):
        return {k: self.get_field(k) for k in ("x", "y", "z", "vx", "vy", "vz", "h", "m", "u",
                                               "du_m1", "id")}

    # ---------------------------------------------------------------- hot path
    def build_tree(self):
        self._ok(self.L.sph_build_tree(self.ctx))

    def find_neighbors(self, stats: bool = True):
        s = NbrStats()
        self._ok(self.L.sph_find_neighbors(self.ctx, C.byref(s) if stats else None))
        return {"min_nc": s.min_nc, "max_nc": s.max_nc, "mean_nc": s.mean_nc, "total": s.total,
                "candidates": s.candidates, "passes": s.passes}

    def get_neighbors(self):
        off = np.zeros(self.n + 1, dtype=np.int64)
        nc = self.get_field("nc")
        total = int(np.minimum(nc, self.cfg.ngmax).sum())
        idx = np.zeros(max(total, 1), dtype=np.int32)
        self._ok(self.L.sph_get_neighbors(self.ctx, C.c_void_p(off.ctypes.data),
                                          C.c_void_p(idx.ctypes.data), total))
        return off, idx[:total]

    def get_neighbor_rows(self, targets):
        """Neighbour lists of the given current-order indices only."""
        t = np.ascontiguousarray(targets, dtype=np.int64)
        off = np.zeros(t.size + 1, dtype=np.int64)
        cap = int(t.size * self.cfg.ngmax)
        idx = np.zeros(max(cap, 1), dtype=np.int32)
        self._ok(self.L.sph_get_neighbor_rows(self.ctx, C.c_void_p(t.ctypes.data), t.size,
                                              C.c_void_p(off.ctypes.data), C.c_void_p(idx.ctypes.data), cap))
        return off, idx[:off[-1]]

    def density(self):
        self._ok(self.L.sph_density(self.ctx))

    def eos(self):
        self._ok(self.L.sph_eos(self.ctx))

    def iad(self):
        self._ok(self.L.sph_iad(self.ctx))

    def momentum_energy(self):
        self._ok(self.L.sph_momentum_energy(self.ctx))

    def timestep(self) -> float:
        d = C.c_double()
        self._ok(self.L.sph_timestep(self.ctx, C.byref(d)))
        return d.value

    def update(self):
        self._ok(self.L.sph_update(self.ctx))

    def step(self):
        info = StepInfo()
        self._ok(self.L.sph_step(self.ctx, C.byref(info)))
        return {"t": info.t, "dt": info.dt, "min_nc": info.nbr.min_nc, "max_nc": info.nbr.max_nc,
                "mean_nc": info.nbr.mean_nc, "cell_level": info.cell_level,
                "search_candidates": info.nbr.candidates, "search_passes": info.nbr.passes,
                "phase_ms": {PHASES[p]: info.phase_ms[p] for p in range(NPHASES)},
                "grav_multipoles": info.grav_multipoles, "grav_pairs": info.grav_pairs,
                "grav_pops": info.grav_pops, "graph": bool(info.graph)}

    # ---------------------------------------------------------------- energy / clocks
    def set_clock_policy(self, mode: int, mhz=None):
        arr = (C.c_uint32 * NPHASES)(*([0] * NPHASES if mhz is None else [int(v) for v in mhz]))
        self._ok(self.L.sph_set_clock_policy(self.ctx, mode, arr))

    def supported_clocks(self):
        """sph_supported_clocks: SM clocks (MHz, descending) the device supports."""
        buf = (C.c_uint32 * 512)()
        n = C.c_int()
        self._ok(self.L.sph_supported_clocks(self.ctx, C.cast(buf, C.c_void_p), 512, C.byref(n)))
        return [int(buf[k]) for k in range(n.value)]

    def energy_report(self):
        rows = (EnergyRow * NPHASES)()
        n = C.c_int()
        self._ok(self.L.sph_energy_report(self.ctx, rows, NPHASES, C.byref(n)))
        return [{"phase": r.phase, "name": r.name.decode(), "calls": r.calls, "seconds": r.seconds,
                 "joules": r.joules if r.available else None, "mean_sm_mhz": r.mean_sm_mhz,
                 "locked_mhz": r.locked_mhz} for r in rows[: n.value]]

    def energy_reset(self):
        self._ok(self.L.sph_energy_reset(self.ctx))

    def energy_totals(self):
        """sph_energy_totals: the accounting window since energy_reset -- sampled
        joules (PHASE accounting) vs the NVML counter delta (None if unreadable)."""
        t = EnergyWindow()
        self._ok(self.L.sph_energy_totals(self.ctx, C.byref(t)))
        return {"wall_seconds": t.wall_seconds, "sampled_seconds": t.sampled_seconds,
                "sampled_joules": t.sampled_joules, "between_joules": t.between_joules,
                "counter_joules": t.counter_joules if t.counter_joules >= 0 else None,
                "samples": int(t.samples)}

    def energy_counter_mj(self):
        v = C.c_uint64()
        rc = self.L.sph_energy_counter_mj(self.ctx, C.byref(v))
        return int(v.value) if rc == SPH_OK else None

    def set_accounting(self, mode: int):
        self._ok(self.L.sph_set_accounting(self.ctx, mode))

    def repeat_phase(self, phase: str, reps: int):
        ms, j = C.c_double(), C.c_double()
        self._ok(self.L.sph_repeat_phase(self.ctx, PHASES.index(phase), reps, C.byref(ms), C.byref(j)))
        return ms.value, (j.value if j.value >= 0 else None)

    def trace_start(self, period_ms: float = 1.0, capacity: int = 1 << 20):
        """sph_trace_start: NVML DVFS sampling thread (Fig. 9)."""
        self._ok(self.L.sph_trace_start(self.ctx, float(period_ms), int(capacity)))

    def trace_stop(self, capacity: int = 1 << 20):
        """sph_trace_stop: the samples as a numpy structured array (t_ms, phase,
        sm_mhz, power_mw, energy_mj)."""
        buf = (TraceSample * capacity)()
        n = C.c_int64()
        self._ok(self.L.sph_trace_stop(self.ctx, C.cast(buf, C.c_void_p), capacity, C.byref(n)))
        m = min(int(n.value), capacity)
        a = np.ctypeslib.as_array(buf)[:m].copy()
        return a

    # ---------------------------------------------------------------- driving
    def stir_init(self, sigma: float, t_decay: float, sol_weight: float, w, noise, A0=None):
        """sph_stir_init: weights w[61], noise[nsteps, 61, 6], optional A0[61, 6]."""
        prm = StirParams(float(sigma), float(t_decay), float(sol_weight))
        w = np.ascontiguousarray(w, np.float64)
        noise = np.ascontiguousarray(noise, np.float64)
        a0 = None if A0 is None else np.ascontiguousarray(A0, np.float64)
        assert w.shape == (STIR_NMODES,) and noise.shape[1:] == (STIR_NMODES, 6)
        self._ok(self.L.sph_stir_init(self.ctx, C.byref(prm), C.c_void_p(w.ctypes.data),
                                      None if a0 is None else C.c_void_p(a0.ctypes.data),
                                      C.c_void_p(noise.ctypes.data), noise.shape[0], MEM_HOST))
        self.stir_enabled = True

    def stir(self):
        self._ok(self.L.sph_stir(self.ctx))

    def gravity(self):
        """sph_gravity: phase GRAVITY (cfg.gravity)."""
        self._ok(self.L.sph_gravity(self.ctx))

    def gradh(self):
        """sph_gradh: phase GRADH, NormalizationGradh (cfg.gradh)."""
        self._ok(self.L.sph_gradh(self.ctx))

    def stir_state(self):
        """(A[61, 6], number of STIR phases run)."""
        A = np.zeros((STIR_NMODES, 6))
        n = C.c_int64()
        self._ok(self.L.sph_stir_get_state(self.ctx, C.c_void_p(A.ctypes.data), C.byref(n)))
        return A, int(n.value)
