"""The C-ABI used from plain C (examples/jacobi_c.c: no Python, no torch in the process):
the grid it writes is bit-exact vs the oracle and its norms within 1e-5, in every launch mode."""
import os
import subprocess

import numpy as np
import pytest

import oracle
from gpu_harness import bits
from inputs import gen

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("mode", [0, 1, 2])
def test_plain_c_driver(tmp_path, mode):
    exe = os.path.join(ROOT, "examples", "jacobi_c")
    assert os.path.exists(exe), "run __graft_entry__.build() first"
    nx, ny, iters, ne = 1028, 96, 21, 4
    out = os.path.join(tmp_path, "out.bin")
    r = subprocess.run([exe, str(nx), str(ny), str(iters), str(ne), str(mode), out], capture_output=True,
                       text=True, timeout=120)
    assert r.returncode == 0, r.stdout + r.stderr
    raw = open(out, "rb").read()
    slab = np.frombuffer(raw[:(ny + 2) * nx * 4], dtype=np.float32).reshape(ny + 2, nx)
    norms = np.frombuffer(raw[(ny + 2) * nx * 4:], dtype=np.float64)
    want, sums = oracle.jacobi_run(gen.global_field(nx, ny, "ring"), iters, "ring", ne)
    assert np.array_equal(bits(slab), bits(want))
    assert np.allclose(norms, np.sqrt(sums), rtol=1e-5, atol=0)
