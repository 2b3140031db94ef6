"""Multi-process device mode: torchrun ranks bootstrap over gloo, map each other's slabs with
CUDA IPC and run the fused put/signal protocol across processes (all on cuda:0 here, the
box has one GPU; on an NVSwitch node each rank would own a GPU and the same code path runs
over NVLink).  Grid bit-exact vs the oracle, norms within 1e-5."""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

import oracle
from gpu_harness import assert_slabs_equal_global
from inputs import gen

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("P,topology,mode", [(2, "ring", "device"), (3, "dirichlet", "device"), (4, "ring", "device"),
                                             (3, "ring", "partial")])
def test_multiprocess_ipc_device_mode(tmp_path, P, topology, mode):
    nx, ny, iters = 520, 16 * P, 20
    ne = 5 if mode == "device" else 0  # partial-mode norms need NCCL: one GPU per rank
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={P}",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()),
           os.path.join(ROOT, "tests", "mp_worker.py"), "--nx", str(nx), "--ny", str(ny), "--iters", str(iters),
           "--norm-every", str(ne), "--topology", topology, "--mode", mode, "--same-device", "--out", str(tmp_path)]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=240, cwd=ROOT)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    res = [np.load(os.path.join(tmp_path, f"rank{q}.npz")) for q in range(P)]
    g = gen.global_field(nx, ny, topology)
    want, sums = oracle.jacobi_run(g, iters, topology, ne)
    assert_slabs_equal_global([x["slab"] for x in res], want, P, topology)
    for x in res:
        assert np.allclose(x["norms"], np.sqrt(sums), rtol=1e-5, atol=0)
        assert np.array_equal(x["norms"], res[0]["norms"])
