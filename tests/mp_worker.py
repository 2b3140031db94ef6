"""One rank of a multi-PROCESS Jacobi run (launched by torchrun from test_gpu_multiprocess.py).

Exercises the production bootstrap: torch.distributed gloo allgather -> uc_comm_create ->
CUDA IPC handle exchange in uc_mem_alloc_symmetric -> device-mode put/signal across processes.
All ranks may share cuda:0 (--same-device) since the test box has one GPU.
Writes <out>/rank<r>.npz with the final slab and the norms.
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import paper_conf_cluster_sagbilieinu25_b200 as U  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--nx", type=int, default=520)
    ap.add_argument("--ny", type=int, default=64)
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--norm-every", type=int, default=5)
    ap.add_argument("--mode", default="device")
    ap.add_argument("--topology", default="ring")
    ap.add_argument("--same-device", action="store_true")
    ap.add_argument("--variant", type=int, default=-1)
    ap.add_argument("--tile-rows", type=int, default=0)
    ap.add_argument("--host-path", default="0,0", help="deep_halo,overlap (host mode)")
    ap.add_argument("--out", required=True)
    a = ap.parse_args()
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    local = 0 if a.same_device else int(os.environ["LOCAL_RANK"])
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(local)
    env = U.Env(rank, world, local, U.torch_allgather())
    neigh = U.ring_neighbours if a.topology == "ring" else U.chain_neighbours
    comm = U.Comm(env, *neigh(rank, world))
    stream = torch.cuda.Stream()
    mode = {"device": U.UC_MODE_DEVICE, "host": U.UC_MODE_HOST, "partial": U.UC_MODE_PARTIAL}[a.mode]
    coord = U.Coord(comm, mode, stream.cuda_stream)
    coord.set_timeout(20.0)
    J = U.Jacobi(comm, a.nx, a.ny)
    if a.variant >= 0:
        J.set_launch(a.variant, 0, 0, 0, a.tile_rows)
    deep, overlap = (int(x) for x in a.host_path.split(","))
    J.set_host_path(deep, overlap)
    norms = J.run(coord, a.iters, a.norm_every, use_graph=True)
    coord.sync()
    slab = J.copy_out(coord)
    counts = np.array(J.launch_counts(), np.uint64)
    np.savez(os.path.join(a.out, f"rank{rank}.npz"), slab=slab, norms=norms, counts=counts)
    comm.barrier()
    J.destroy()
    coord.destroy()
    comm.destroy()
    env.finalize()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
