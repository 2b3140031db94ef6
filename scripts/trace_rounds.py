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
    ap.add_argument("--balance", action="store_true", help="balanced chunks on (default off here)")
    a = ap.parse_args()
    env = U.Env(0, 1, 0)
    nb = U.ring_neighbours if a.topology == "ring" else U.chain_neighbours
    comm = U.Comm(env, *nb(0, 1))
    st = torch.cuda.Stream()
    co = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
    J = U.Jacobi(comm, a.nx, a.ny)
    J.set_balance(a.balance)  # off: the static chunking (the estimate below assumes its rows per block)
    info = J.launch_info()
    T = info["tile_rows"]
    for _ in range(4 if not a.balance else 40):
        J.run(co, 2 * T, 0, use_graph=False)
        if a.balance:
            co.sync()
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
    # is a block's speed a property of its SM?  Repeat the launch and compare the per-SM mean
    # interior march time across repetitions (and the block -> SM placement across them)
    reps = []
    for _ in range(3):
        J.run(co, T, 0, use_graph=False)
        co.sync()
        tr = buf.astype(np.int64).copy()
        reps.append(tr)
    per_sm = []
    for tr in [t] + reps:
        d = (tr[:, 2] - tr[:, 0]).astype(np.float64)
        m = np.full(200, np.nan)
        for smid in np.unique(tr[:, 14]):
            sel = (tr[:, 14] == smid) & mid
            if sel.any():
                m[int(smid)] = d[sel].mean()
        per_sm.append(m)
        same = np.mean(tr[:, 14] == t[:, 14])
    ok = ~np.isnan(per_sm[0]) & ~np.isnan(per_sm[1])
    cc = [np.corrcoef(per_sm[0][ok], per_sm[i][ok])[0, 1] for i in range(1, len(per_sm))]
    print(f"block -> SM placement identical across launches: {same:.3f}; per-SM mean interior march time "
          f"correlation launch 0 vs 1..3: {[round(c, 3) for c in cc]}")
    allm = np.nanmean(np.array(per_sm), axis=0)
    okm = ~np.isnan(allm)
    ids_sm = np.nonzero(okm)[0]
    v = allm[okm] / 1e3
    print(f"per-SM mean interior march (us, 4 launches): min {v.min():.1f} median {np.median(v):.1f} max {v.max():.1f}; "
          f"slowest SMs {[int(x) for x in ids_sm[np.argsort(v)[-10:]]]}, fastest {[int(x) for x in ids_sm[np.argsort(v)[:10]]]}")
    print("per-SM mean interior march (us) by SM id:", " ".join(f"{int(i)}:{x:.0f}" for i, x in zip(ids_sm, v)))
    # what balancing could buy: per block rate = march rows / march time (mean over the launches);
    # (a) the launch now (slowest march end), (b) rows re-cut within each strip (blocks keep their
    # strips), (c) fully balanced (total rows / summed rates)
    d = np.mean([(tr[:, 2] - tr[:, 0]).astype(np.float64) for tr in [t] + reps], axis=0) / 1e3
    rows = np.zeros(info["grid"])
    n = J.n
    for b in range(info["grid"]):
        qb = b // S
        lo = 1 + max(0, min(qb * (n + 2 * 160) // Q - 160, n)) if Q > 2 else 1 + qb * n // Q
        hi = max(0, min((qb + 1) * (n + 2 * 160) // Q - 160, n)) if Q > 2 else (qb + 1) * n // Q
        rows[b] = hi - lo + 1
    rate = rows / d
    strip_t = [rows[q * S + s_] .sum() if False else None for s_ in range(S) for q in range(1)]
    per_strip = [rows[np.arange(s_, info["grid"], S)].sum() / rate[np.arange(s_, info["grid"], S)].sum() for s_ in range(S)]
    print(f"balancing estimate (march us): now max {d.max():.1f} (median {np.median(d):.1f}); rows re-cut within "
          f"strips: {max(per_strip):.1f}; fully balanced: {rows.sum() / rate.sum():.1f}")
    J.destroy()
    co.destroy()
    comm.destroy()
    env.finalize()


if __name__ == "__main__":
    main()
