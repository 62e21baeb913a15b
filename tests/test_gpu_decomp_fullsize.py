"""SURVEY 8(d) config 4 at its full size: Noh implosion 300^3 (27M particles,
open box: the global key box) decomposed over two ranks that share cuda:0
(gloo), bit-identical to the single-rank run after two steps
(tools/decomp_fullsize.py; 4 ranks in profiles/r02_decomp_fullsize_noh300_w4.json)."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_noh300_two_ranks_bit_identical_to_one(tmp_path):
    out = tmp_path / "df.json"
    r = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "decomp_fullsize.py"), "--workload", "noh300",
                        "--world", "2", "--steps", "2", "--out", str(out)],
                       cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    rec = json.loads(out.read_text())
    assert rec["n"] == 300 ** 3
    assert rec["dt_equal"] and rec["all_bit_identical"], rec
    assert rec["rank0_ghosts"] > 0
