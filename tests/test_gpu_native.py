"""GPU parity of the in-box native comparator (benchmarks/native/nccl_dev_jacobi.cu: the paper's
Listing-3 structure, on NCCL 2.28's device API -- LSA peer stores + LSA barrier) against
the CPU oracle: the comparator computes the same Jacobi, so its grids must be bit-exact too,
which makes the timing comparison in benchmarks/nccl_dev_bench.py one of equals.  P = 1 (NCCL
allows one rank per GPU): ring topology exchanges the halo rows with itself through the
window's LSA pointer; dirichlet keeps them fixed."""
import numpy as np
import pytest

from gpu_harness import bits
from test_gpu_jacobi import _oracle

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
@pytest.mark.parametrize("nx,ny,iters", [(256, 256, 100), (1028, 64, 37), (4100, 9, 12), (64, 2, 9), (64, 1, 5)])
def test_nccl_device_api_comparator_bit_exact(topology, nx, ny, iters):
    import torch

    from benchmarks.nccl_dev_bench import single_rank
    torch.cuda.set_device(0)
    g0, want, _ = _oracle(nx, ny, topology, iters, 0)
    J = single_rank(nx, ny, topology)
    try:
        J.copy_in(g0)
        J.run(iters)
        got = J.copy_out()
    finally:
        J.destroy()
    if not np.array_equal(bits(got), bits(want)):
        j, i = np.argwhere(bits(got) != bits(want))[0]
        raise AssertionError(f"differs at (row {j}, col {i}): {got[j, i]!r} vs oracle {want[j, i]!r}")
