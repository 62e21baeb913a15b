"""The NCCL data plane of the decomposed step on one GPU: a one-rank NCCL
process group with the decomposition's collectives issued anyway (Comm
always=True: all-reduces of the box / h_max / dt, the all-to-alls of migrants
and ghosts, the halo exchanges, async starts and waits on the libsph stream).
The result must equal the plain single-GPU step bit for bit.  (Several ranks
need several GPUs; their routing is covered by the gloo tests.)"""
import os
import subprocess
import sys
import textwrap

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = textwrap.dedent("""
    import os, sys
    sys.path.insert(0, sys.argv[1])
    import numpy as np, torch, torch.distributed as dist
    from paper_conf_sc_simsekpc24_b200 import decomp, ics, sph
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", init_method="env://", device_id=torch.device("cuda", 0))
    assert dist.get_backend() == "nccl" and dist.get_world_size() == 1
    for name, w in (("turbulence16", ics.turbulence(16)), ("noh14_open", ics.noh(14))):
        ds = decomp.DistributedSim(w.params, w.state, n_capacity=w.n, device=0, force_exchange=True,
                                   comm_always=True)
        assert not ds.comm._local and not ds.comm.host
        dts = [ds.step() for _ in range(4)]
        st = ds.gather_state()
        sim = sph.Simulation(w.params, n_capacity=w.n)
        sim.set_particles({k: np.ascontiguousarray(v) for k, v in w.state.items()})
        sim.set_time(0.0, w.params.dt_first, True)
        dts1 = [sim.step()["dt"] for _ in range(4)]
        st1 = sim.get_state()
        o1 = np.argsort(st1["id"])
        o = np.argsort(st["id"])
        assert dts == dts1, (name, dts, dts1)
        for k in ("x", "y", "z", "vx", "vy", "vz", "u", "h"):
            assert np.array_equal(st[k][o], st1[k][o1]), (name, k)
        sim.finalize()
    dist.destroy_process_group()
    print("NCCL-OK")
""")


def test_one_rank_nccl_collectives_equal_plain():
    env = dict(os.environ, RANK="0", WORLD_SIZE="1", LOCAL_RANK="0", MASTER_ADDR="127.0.0.1",
               MASTER_PORT=str(29000 + os.getpid() % 1000))
    out = subprocess.run([sys.executable, "-c", SCRIPT, ROOT], capture_output=True, text=True, env=env,
                         timeout=600, cwd=ROOT)
    assert out.returncode == 0 and "NCCL-OK" in out.stdout, (out.stdout[-2000:], out.stderr[-3000:])
