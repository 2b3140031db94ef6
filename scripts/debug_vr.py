"""Debug helper: run P virtual ranks on one GPU with various options and report failures."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402

from gpu_harness import solve_gpu  # noqa: E402


def attempt(**kw):
    t = time.time()
    try:
        r = solve_gpu(**kw)
        print("OK  ", kw, f"{time.time() - t:.1f}s", r["launch"], flush=True)
    except Exception as e:  # noqa: BLE001
        print("FAIL", kw, f"{time.time() - t:.1f}s", str(e)[:300], flush=True)


if __name__ == "__main__":
    base = dict(nx=520, ny=72, P=3, topology="ring", mode="device", iters=25)
    attempt(**{**base, "norm_every": 0, "use_graph": False})
    attempt(**{**base, "norm_every": 0, "use_graph": True})
    attempt(**{**base, "norm_every": 5, "use_graph": False})
    attempt(**{**base, "iters": 1, "norm_every": 0, "use_graph": False})
    attempt(**{**base, "iters": 2, "norm_every": 0, "use_graph": False})
    attempt(**{**base, "P": 3, "topology": "dirichlet", "norm_every": 0, "use_graph": False})
    attempt(**{**base, "P": 4, "ny": 96, "norm_every": 0, "use_graph": False})
    attempt(**{**base, "P": 2, "ny": 48, "norm_every": 5, "use_graph": True})
