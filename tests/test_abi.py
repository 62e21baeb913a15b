"""CPU-side checks of the C ABI: libsph.so builds, loads without a GPU and exports
every function include/sph.h declares; pure host entry points behave."""
import ctypes as C
import os
import re

import pytest

from paper_conf_sc_simsekpc24_b200 import sph

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "sph.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(sph_[a-z_0-9]+)\s*\(", src)))


def test_header_and_binding_agree():
    assert sorted(sph.EXPORTS) == _declared()


def test_library_exports_every_symbol():
    L = sph.load()
    for name in _declared():
        assert hasattr(L, name), name


def test_config_default_and_workspace():
    L = sph.load()
    cfg = sph.Config()
    assert L.sph_config_default(C.byref(cfg)) == 0
    assert cfg.ngmax == 150 and cfg.K == pytest.approx(0.7904495894323029, rel=1e-16)
    assert tuple(cfg.periodic) == (1, 1, 1) and cfg.nranks == 1
    nbytes = C.c_size_t()
    cfg.n_capacity = 8_000_000
    assert L.sph_workspace_size(C.byref(cfg), C.byref(nbytes)) == 0
    # SoA fields + neighbour lists [ngmax][cap] dominate: ~8 GB at 8M particles
    assert 6e9 < nbytes.value < 12e9
    cfg.n_capacity = 0
    assert L.sph_workspace_size(C.byref(cfg), C.byref(nbytes)) == 1  # SPH_ERR_ARG
    assert b"n_capacity" in L.sph_last_error(None)


def test_phase_names():
    L = sph.load()
    assert [L.sph_phase_name(p).decode() for p in range(sph.NPHASES)] == list(sph.PHASES)
    assert L.sph_phase_name(99) == b"unknown"


def test_init_rejects_bad_arena_without_touching_cuda():
    L = sph.load()
    cfg = sph.Config()
    L.sph_config_default(C.byref(cfg))
    ctx = C.c_void_p()
    assert L.sph_init(C.byref(cfg), None, 0, None, C.byref(ctx)) == 1
    assert b"arena" in L.sph_last_error(None)
    cfg.nranks = 2
    assert L.sph_init(C.byref(cfg), None, 0, None, C.byref(ctx)) == 7  # NOT_SUPPORTED


def test_null_context_calls_fail_cleanly():
    L = sph.load()
    assert L.sph_build_tree(None) == 1
    assert L.sph_step(None, None) == 1
    L.sph_finalize(None)


def test_trace_entry_points_reject_null_context():
    L = sph.load()
    n = C.c_int64()
    assert L.sph_trace_start(None, C.c_double(1.0), C.c_int64(10)) == 1  # SPH_ERR_ARG
    assert L.sph_trace_stop(None, None, C.c_int64(0), C.byref(n)) == 1
