"""Mutation check of the oracle's pins (VERDICT r1 'Next round' item 1): each
mutant below is oracle.c with one plausible slip -- a one-sided mean, the wrong
smoothing length or matrix on the j side, a sign, a dropped 1/2 -- compiled into
a temporary library.  The pins named next to it must FAIL on the mutant (and
pass on the real oracle, which the ordinary test run shows).  This is what makes
the variable-h parts of momentum-energy (oracle.c, step 8) and IAD (step 7)
pinned rather than merely self-consistent."""
import json
import os
import subprocess

import pytest

import oracle
import test_oracle_physics as phys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "oracle.c")

# (name, original text, mutated text, occurrence to replace (1-based), killer pins)
MUTANTS = [
    ("momentum w_j with h_i", "double wj = oracle_W(r, h[j], P->K);", "double wj = oracle_W(r, h[i], P->K);", 1,
     ["test_conservation_variable_h_mutual"]),
    ("momentum h-bar one-sided", "double hbar = (h[i] + h[j]) / 2.0;", "double hbar = (h[i] + h[i]) / 2.0;", 1,
     ["test_conservation_variable_h_mutual"]),
    ("momentum c-bar one-sided", "double cbar = (c[i] + c[j]) / 2.0;", "double cbar = (c[i] + c[i]) / 2.0;", 1,
     ["test_conservation_variable_h_mutual"]),
    ("momentum rho-bar one-sided", "double rhobar = (rho[i] + rho[j]) / 2.0;",
     "double rhobar = (rho[i] + rho[i]) / 2.0;", 1, ["test_conservation_variable_h_mutual"]),
    ("momentum B with C_i", "sym_mul(C + 6 * j, D, CjD);", "sym_mul(C + 6 * i, D, CjD);", 1,
     ["test_conservation_variable_h_mutual", "test_conservation_uniform_h"]),
    ("momentum G = (A - B)/2", "G[a] = (A[a] + B[a]) / 2.0;", "G[a] = (A[a] - B[a]) / 2.0;", 1,
     ["test_conservation_variable_h_mutual"]),
    ("energy without the 1/2 on Pi", "e2 = 0.5 * Pi * vG;", "e2 = Pi * vG;", 1,
     ["test_conservation_variable_h_mutual", "test_viscosity_heats_and_decelerates_a_converging_flow"]),
    ("momentum p_j/rho_j^2 -> p_i/rho_i^2", ": p[j] / (rho[j] * rho[j]);", ": p[i] / (rho[i] * rho[i]);", 1,
     ["test_conservation_variable_h_mutual", "test_pressure_gradient_force"]),
    ("IAD tau with W(r, h_j)", "double vw = (m[j] / rho[j]) * oracle_W(r, h[i], P->K);",
     "double vw = (m[j] / rho[j]) * oracle_W(r, h[j], P->K);", 1, ["test_iad_linear_exactness_variable_h"]),
    ("IAD tau with V_i", "double vw = (m[j] / rho[j]) * oracle_W(r, h[i], P->K);",
     "double vw = (m[i] / rho[i]) * oracle_W(r, h[i], P->K);", 1, ["test_iad_linear_exactness_variable_h"]),
    ("density with h_j", "sum += m[j] * pow(oracle_sinc(M_PI * r / (2.0 * h[i])), 6.0);",
     "sum += m[j] * pow(oracle_sinc(M_PI * r / (2.0 * h[j])), 6.0);", 1, ["test_density_uses_own_h_only"]),
    ("IAD adjugate transposed entry", "Ci[1] = (t13 * t23 - t12 * t33) / det;", "Ci[1] = (t12 * t23 - t13 * t33) / det;", 1,
     ["test_iad_linear_exactness_variable_h"]),
]


def _mutant_lib(tmp_path, src, idx):
    path = str(tmp_path / f"liboracle_mutant{idx}.so")
    c = tmp_path / f"mutant{idx}.c"
    c.write_text(src)
    subprocess.check_call(["gcc", *oracle.CFLAGS, str(c), "-o", path, "-lm"])
    return path


def _run_pin(name, golden):
    fn = getattr(phys, name)
    if name == "test_iad_linear_exactness_variable_h":
        for kind in ("mutual_lattice", "jittered_varh"):
            fn(kind)
    elif name in ("test_density_uses_own_h_only",):
        fn(golden)
    else:
        fn()


@pytest.mark.parametrize("k", range(len(MUTANTS)), ids=[m[0] for m in MUTANTS])
def test_mutant_is_killed(k, tmp_path, golden):
    name, old, new, occ, killers = MUTANTS[k]
    src = open(SRC).read()
    parts = src.split(old)
    assert len(parts) > occ, f"mutation site not found: {old}"
    mutated = old.join(parts[:occ]) + new + old.join(parts[occ:])
    lib = _mutant_lib(tmp_path, mutated, k)
    with oracle.use_library(lib):
        for pin in killers:
            with pytest.raises(AssertionError):
                _run_pin(pin, golden)
    # and the real oracle passes the same pins
    for pin in killers:
        _run_pin(pin, golden)
