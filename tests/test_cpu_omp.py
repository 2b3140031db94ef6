"""The multi-core host baseline (benchmarks/cpu_omp, bench.py's cpu_parallel) computes the
oracle's grid bit for bit, and its norms within the reduction-order tolerance."""
import numpy as np
import pytest

import oracle
from inputs import gen


@pytest.mark.parametrize("nx,ny,iters,topology,ne", [(256, 256, 100, "ring", 10), (130, 77, 31, "dirichlet", 7),
                                                    (4, 2, 25, "dirichlet", 1), (1028, 96, 13, "ring", 6)])
def test_omp_baseline_matches_oracle(nx, ny, iters, topology, ne):
    from benchmarks import cpu_omp
    g = gen.global_field(nx, ny, topology)
    want, wsums = oracle.jacobi_run(g, iters, topology, ne)
    got, sums = cpu_omp.jacobi_run(g, iters, topology, ne)
    assert np.array_equal(got.view(np.uint32), want.view(np.uint32))
    assert np.allclose(sums, wsums, rtol=1e-12, atol=0)
    assert cpu_omp.threads() >= 1
