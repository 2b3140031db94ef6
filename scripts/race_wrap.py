"""racecheck probe: the one-iteration staged kernel (variant 1) with enough rows per block that
its TMA ring wraps (stage reuse), to compare with the multi-iteration kernels' reports."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import oracle  # noqa: E402
from gpu_harness import assert_slabs_equal_global, solve_gpu  # noqa: E402
from inputs import gen  # noqa: E402
import gpu_harness  # noqa: E402

gpu_harness.TIMEOUT_S = 600.0
nx, ny, it = 132, 1200, 3
res = solve_gpu(nx, ny, 1, "ring", "device", it, 0, variant=1, blocks_per_sm=1, use_graph=False)
want, _ = oracle.jacobi_run(gen.global_field(nx, ny, "ring"), it, "ring")
assert_slabs_equal_global(res["final"], want, 1, "ring")
print("ok variant 1 wrapped ring", res["launch"], flush=True)
