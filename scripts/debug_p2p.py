"""Debug helper for uc_p2p_bench with virtual ranks (not a test)."""
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import torch  # noqa: E402

import paper_conf_cluster_sagbilieinu25_b200 as U  # noqa: E402
from vranks import run_ranks  # noqa: E402


def attempt(P, plan, nbytes=4096):
    def body(rank, P, ag):
        env = U.Env(rank, P, 0, ag)
        comm = U.Comm(env, *U.ring_neighbours(rank, P))
        st = torch.cuda.Stream()
        co = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
        co.set_timeout(2.0)
        buf = U.SymMem(comm, 3 * nbytes)
        sig = U.SymMem(comm, 64)
        err = None
        try:
            for step in plan:
                if step == "pp" and rank in (0, 1):
                    co.p2p_bench(U.UC_P2P_PINGPONG, buf, sig, nbytes, 3, 1, 1 - rank, rank, 0)
                if step == "win" and rank in (0, 1):
                    co.p2p_bench(U.UC_P2P_WINDOW, buf, sig, nbytes, 2, 4, 1 - rank, rank, 0)
                if step == "halo":
                    co.p2p_bench(U.UC_P2P_HALO, buf, sig, nbytes, 3, 1, 0, 0, 0)
                if step == "sync":
                    co.sync()
                if step == "bar":
                    comm.barrier()
        except Exception as e:  # noqa: BLE001
            err = str(e)[:120]
        try:
            co.sync()
        except Exception as e:  # noqa: BLE001
            err = (err or "") + " | final " + str(e)[:80]
        comm.barrier()
        buf.free()
        sig.free()
        co.destroy()
        comm.destroy()
        env.finalize()
        return err

    t = time.time()
    r = run_ranks(P, body, timeout=120)
    print(P, plan, f"{time.time() - t:.1f}s", r, flush=True)


if __name__ == "__main__":
    attempt(3, ["halo", "sync"])
    attempt(3, ["pp", "sync"])
    attempt(3, ["win", "sync"])
    attempt(3, ["pp", "win", "sync", "bar", "halo", "sync"])
    attempt(3, ["pp", "win", "halo", "sync"])
    attempt(2, ["pp", "win", "halo", "sync"])
    attempt(4, ["halo", "sync"])
