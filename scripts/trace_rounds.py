"""Where the time of a jacobi_t_kernel<6, 2> launch goes, per block (A/B instrumentation build):

    python paper_conf_cluster_sagbilieinu25_b200/build.py --define UC_TRACE=1 --out build/ab/lib_trace.so
    UC_LIB_PATH=build/ab/lib_trace.so python scripts/trace_rounds.py [--ny 16384] [--shrink S]

%globaltimer stamps (ns) per block: 0 start, 1 after round 1, 2 after the march, 1+j after round j
(j = 2..T), 14 the SM id, 15 end.  Prints the launch span and, for interior and edge (boundary-round) blocks, the
phase durations relative to the launch start."""
import argparse
import ctypes as C
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_cluster_sagbilieinu25_b200 as U  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--nx", type=int, default=16384)
    ap.add_argument("--ny", type=int, default=16384)
    ap.add_argument("--topology", default="ring")
    a = ap.parse_args()
    env = U.Env(0, 1, 0)
    nb = U.ring_neighbours if a.topology == "ring" else U.chain_neighbours
    comm = U.Comm(env, *nb(0, 1))
    st = torch.cuda.Stream()
    co = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
    J = U.Jacobi(comm, a.nx, a.ny)
    info = J.launch_info()
    T = info["tile_rows"]
    for _ in range(4):
        J.run(co, 2 * T, 0, use_graph=False)
    co.sync()
    U.lib.uc_debug_trace_buffer.restype = C.c_void_p
    ptr = U.lib.uc_debug_trace_buffer()
    buf = np.ctypeslib.as_array((C.c_uint64 * (16 * info["grid"])).from_address(ptr)).reshape(info["grid"], 16)
    t = buf.astype(np.int64)
    t0 = t[:, 0].min()
    span = t[:, 15].max() - t0
    S, Q = info["strips"], info["chunks"]
    q = np.arange(info["grid"]) // S
    edge = (q == 0) | (q == Q - 1)
    mid = ~edge
    us = lambda x: x / 1e3  # noqa: E731
    print(f"launch {info}, span {us(span):.1f} us")
    print(f"interior blocks: start +{us(np.median(t[mid,0]-t0)):.1f}, march end +{us(np.median(t[mid,2]-t0)):.1f} "
          f"(max {us(np.max(t[mid,2]-t0)):.1f}), end max +{us(np.max(t[mid,15]-t0)):.1f} us")
    e = t[edge]
    print(f"edge blocks ({e.shape[0]}): round 1 done +{us(np.median(e[:,1]-t0)):.1f}, march end +{us(np.median(e[:,2]-t0)):.1f} "
          f"(max {us(np.max(e[:,2]-t0)):.1f})")
    for j in range(2, T + 1):
        d = e[:, 1 + j] - e[:, j]
        print(f"  round {j}: median {us(np.median(d)):.1f} us, max {us(np.max(d)):.1f}; done +{us(np.median(e[:,1+j]-t0)):.1f} "
              f"(max {us(np.max(e[:,1+j]-t0)):.1f})")
    print(f"edge end max +{us(np.max(e[:,15]-t0)):.1f} us")
    # per SM: what shares it, and when its blocks finish their march
    sm = t[:, 14]
    kinds = {}
    for b in range(info["grid"]):
        kinds.setdefault(int(sm[b]), []).append(b)
    by = {}
    for smid, bl in kinds.items():
        key = "+".join(sorted("E" if edge[b] else "I" for b in bl))
        for b in bl:
            if mid[b]:
                by.setdefault(key, []).append(t[b, 2] - t0)
    for key, v in sorted(by.items()):
        v = np.array(v)
        print(f"interior blocks on SMs holding [{key}]: n={len(v)} march end median {us(np.median(v)):.1f} max {us(v.max()):.1f}")
    lo = [us(t[b, 2] - t0) for b in range(info["grid"]) if mid[b] and sm[b] < 74]
    hi = [us(t[b, 2] - t0) for b in range(info["grid"]) if mid[b] and sm[b] >= 74]
    print(f"interior blocks by SM id < 74: median {np.median(lo):.1f} max {max(lo):.1f}; >= 74: median {np.median(hi):.1f} max {max(hi):.1f}")
    order = np.argsort(t[mid, 2])
    ids = np.nonzero(mid)[0][order]
    print("slowest interior blocks (block, sm, march end us):", [(int(b), int(sm[b]), round(us(t[b, 2] - t0), 1)) for b in ids[-12:]])
    print("fastest interior blocks:", [(int(b), int(sm[b]), round(us(t[b, 2] - t0), 1)) for b in ids[:12]])
    J.destroy()
    co.destroy()
    comm.destroy()
    env.finalize()


if __name__ == "__main__":
    main()
