"""bench.py's JSON line (the driver's contract): the reference arm on CPU (the
oracle on the host cores), and the libsph arm on a GPU with a small workload."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, timeout=600):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True,
                         text=True, timeout=timeout, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    return json.loads(lines[0])


def test_reference_arm_line():
    d = _run(["--impl", "reference", "--workload", "turbulence16", "--steps", "1", "--warmup", "3",
              "--cpu-sample", "4"])
    assert d["impl"] == "reference" and d["metric"] and d["unit"] == "particle-updates/s"
    assert d["value"] > 0 and d["higher_is_better"] is True and d["steps"] == 1 and d["warmup"] == 3
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]


@pytest.mark.gpu
def test_libsph_arm_line():
    d = _run(["--workload", "turbulence40", "--steps", "3", "--warmup", "3", "--e2e-steps", "1",
              "--energy-seconds", "1.5", "--energy-repeats", "1", "--trace-seconds", "0", "--cpu-sample", "4"])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "dtype", "data", "config", "roofline", "e2e", "cpu_baseline", "clocks",
              "gpu_launches", "phases"):
        assert k in d, k
    assert d["n_gpus"] == 1 and d["dtype"] == "f64" and d["config"]["workload"] == "turbulence40"
    r = d["roofline"]
    assert r["bound"] == "alu" and 0 < r["frac"] < 1 and r["achieved"] > 0 and r["peak"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert 0 < d["e2e"]["value"] <= d["value"] * 1.05
    assert d["gpu_launches"] > 0 and d["cpu_baseline"]["kind"] == "oracle"
    assert d["phases"]["momentum_energy"]["bound"] == "fp64" and d["phases"]["update"]["GBps"] > 0
    assert d["repeats"]["blocks"] >= 4 and d["repeats"]["cv"] >= 0
    e = d["energy"]
    assert e["available"] and e["step"]["J_median"] > 0 and e["phases"]["momentum_energy"]["J"] > 0
    assert d["cpu_baseline"]["physics_only"]["s_per_particle"] > 0
    assert d["roofline"]["flops_per_pair"] == 171
    assert d["parity"]["order_exact"] and d["parity"]["nbr_exact"] and d["parity"]["pass"], d["parity"]
    assert d["e2e"]["sequential"]["value"] > 0


@pytest.mark.gpu
def test_decomposed_arm_line():
    """The N > 1 path of bench.py (SFC decomposition, halos, dt all-reduce) on one
    GPU: a one-rank NCCL group with every collective issued (--force-decomp)."""
    d = _run(["--force-decomp", "--workload", "turbulence40", "--steps", "3", "--warmup", "3", "--e2e-steps", "1"])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "dtype", "config", "roofline", "e2e", "clocks", "gpu_launches"):
        assert k in d, k
    assert d["scaling"] == "weak" and d["dtype"] == "f64" and d["value"] > 0
    assert "NCCL" in d["config"]["parallelism"] and d["config"]["n_particles_total"] == 40 ** 3
    r = d["roofline"]
    assert r["bound"] == "alu" and r["scope"] == "rank 0" and 0 < r["frac"] < 1
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["value"] > 0
    assert d["gpu_launches"] > 0
