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


def _run(tmp_path, P, nx, ny, iters, ne, topology, mode, same_device=True, host_path=(0, 0)):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={P}",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()),
           os.path.join(ROOT, "tests", "mp_worker.py"), "--nx", str(nx), "--ny", str(ny), "--iters", str(iters),
           "--norm-every", str(ne), "--topology", topology, "--mode", mode, "--out", str(tmp_path),
           "--host-path", f"{host_path[0]},{host_path[1]}"]
    if same_device:
        cmd.append("--same-device")
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    res = [np.load(os.path.join(tmp_path, f"rank{q}.npz")) for q in range(P)]
    g = gen.global_field(nx, ny, topology)
    want, sums = oracle.jacobi_run(g, iters, topology, ne)
    assert_slabs_equal_global([x["slab"] for x in res], want, P, topology)
    for x in res:
        assert np.allclose(x["norms"], np.sqrt(sums), rtol=1e-5, atol=0)
        assert np.array_equal(x["norms"], res[0]["norms"])
    return res


@pytest.mark.parametrize("P,topology,mode", [(2, "ring", "device"), (3, "dirichlet", "device"), (4, "ring", "device"),
                                             (3, "ring", "partial")])
def test_multiprocess_ipc_device_mode(tmp_path, P, topology, mode):
    ne = 5 if mode == "device" else 0  # partial-mode norms need NCCL: one GPU per rank
    _run(tmp_path, P, 520, 16 * P, 20, ne, topology, mode)


@pytest.mark.parametrize("P,topology", [(2, "ring"), (3, "ring"), (4, "ring"), (3, "dirichlet")])
def test_multiprocess_ipc_deep(tmp_path, P, topology):
    """The shipped jacobi_t_kernel<8, 2> across PROCESSES (CUDA IPC peers): 24 iterations with a
    norm every 8 are three launches of 8 on every rank (device counters); with a norm every 6 the
    launches demote to <6, 2>: 6, 6, 6, 6."""
    res = _run(tmp_path, P, 1028, 16 * P, 24, 8, topology, "device")
    for x in res:
        c = list(x["counts"])
        assert c[8] == 3 and sum(c[:15]) == 3, c
    res = _run(tmp_path, P, 1028, 16 * P, 24, 6, topology, "device")
    for x in res:
        c = list(x["counts"])
        assert c[6] == 4 and sum(c[:15]) == 4, c


# ---- one GPU per rank (NCCL allows one rank per GPU): run where the box has >= 2 GPUs
def _gpus():
    import torch
    return torch.cuda.device_count()


@pytest.mark.skipif("_gpus() < 2", reason="needs >= 2 GPUs (one rank per GPU)")
@pytest.mark.parametrize("mode", ["host", "device", "partial"])
def test_two_gpus_each_mode(tmp_path, mode):
    """Host mode (grouped NCCL send/recv, ncclAllReduce norms) and device / partial mode over
    NVLink peer memory, P = 2 ranks on 2 GPUs, configs[1]-like grid."""
    _run(tmp_path, 2, 4096, 512, 40, 6, "ring", mode, same_device=False)


@pytest.mark.skipif("_gpus() < 2", reason="needs >= 2 GPUs (one rank per GPU)")
@pytest.mark.parametrize("deep,overlap", [(1, 0), (0, 1), (1, 1)])
@pytest.mark.parametrize("P,topology", [(2, "ring"), (3, "dirichlet"), (4, "ring")])
def test_host_paths_multi_gpu(tmp_path, deep, overlap, P, topology):
    """Deep-halo and overlapped host paths with real NCCL peers (one GPU per rank)."""
    if _gpus() < P:
        pytest.skip(f"needs {P} GPUs")
    res = _run(tmp_path, P, 2052, 96 * P, 25, 6, topology, "host", same_device=False, host_path=(deep, overlap))
    if deep:
        for x in res:
            assert list(x["counts"])[6] == 3, list(x["counts"])


@pytest.mark.skipif("_gpus() < 4", reason="needs >= 4 GPUs")
def test_four_gpus_t6_chain(tmp_path):
    res = _run(tmp_path, 4, 4096, 4 * 128, 24, 6, "dirichlet", "device", same_device=False)
    for x in res:
        assert list(x["counts"])[6] == 4
