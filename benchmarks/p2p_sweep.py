#!/usr/bin/env python
"""Halo put-signal P2P sweep (BASELINE.json configs[4]): message sizes 4 KiB ..
256 MiB, device-initiated put + signal (uc_p2p_bench, one persistent kernel per rank) vs NCCL
send/recv (host mode, uc_put_signal / uc_signal_wait), latency and bandwidth, following the
paper's OSU-derived protocol (§VI-B):
  latency: ping-pong, 100K iterations + 10K warm-up below 8 KiB, 10K + 1K from 8 KiB;
  bandwidth: 64 messages in flight, 1000 + 100 below 8 KiB, 200 + 20 from 8 KiB;
  halo: every rank puts to top and bottom at once (the Jacobi pattern), same counts as latency;
  timing: CUDA events on the coordinator's stream, 10 repetitions, drop min and max, mean.

    torchrun --nproc-per-node N --master-addr 127.0.0.1 benchmarks/p2p_sweep.py [--scale 0.1]
    python benchmarks/p2p_sweep.py --vr 2          # virtual ranks on ONE GPU (no NVLink: a
                                                   # same-device copy; checks the machinery only)
One JSON line per (pattern, size) on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def osu_counts(nbytes, pattern, scale):
    if pattern == "bw":
        it, wu = (1000, 100) if nbytes < 8192 else (200, 20)
    else:
        it, wu = (100000, 10000) if nbytes < 8192 else (10000, 1000)
    return max(1, int(it * scale)), max(1, int(wu * scale))


def trimmed_mean(xs):
    xs = sorted(xs)
    if len(xs) > 2:
        xs = xs[1:-1]
    return statistics.mean(xs)


def rank_main(rank, P, device, ag, a, barrier):
    import torch

    import paper_conf_cluster_sagbilieinu25_b200 as U
    torch.cuda.set_device(device)
    env = U.Env(rank, P, device, ag)
    comm = U.Comm(env, *U.ring_neighbours(rank, P))
    st = torch.cuda.Stream()
    dev = U.Coord(comm, U.UC_MODE_DEVICE, st.cuda_stream)
    dev.set_timeout(30.0)
    host = U.Coord(comm, U.UC_MODE_HOST, st.cuda_stream) if a.nccl else None
    sizes = [4096 << i for i in range(17) if (4096 << i) <= a.max_bytes]
    maxb = max(sizes)
    buf = U.SymMem(comm, 3 * maxb)
    sig = U.SymMem(comm, 64)
    sig2 = U.SymMem(comm, 64)  # signals of the library-call legs (monotone per slot)
    sigv = [0, 0, 0]
    out = []

    def timed(fn, reps, all_ranks=False):
        ts = []
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            if all_ranks:
                barrier()
            e0.record(st)
            fn()
            e1.record(st)
            dev.sync()
            ts.append(e0.elapsed_time(e1))
        return trimmed_mean(ts)

    for S in sizes:
        rec = {"bytes": S}
        # ---- device put-signal ping-pong latency (ranks 0 <-> 1)
        if P >= 2 and rank in (0, 1):
            it, wu = osu_counts(S, "lat", a.scale)
            peer, role = 1 - rank, rank
            dev.p2p_bench(U.UC_P2P_PINGPONG, buf, sig, S, wu, 1, peer, role, a.blocks)
            ms = timed(lambda: dev.p2p_bench(U.UC_P2P_PINGPONG, buf, sig, S, it, 1, peer, role, a.blocks), a.reps)
            rec["put_signal_latency_us"] = ms * 1e3 / (2 * it)
            # ---- device put-signal bandwidth, window of 64
            itb, wub = osu_counts(S, "bw", a.scale)
            dev.p2p_bench(U.UC_P2P_WINDOW, buf, sig, S, wub, 64, peer, role, a.blocks)
            ms = timed(lambda: dev.p2p_bench(U.UC_P2P_WINDOW, buf, sig, S, itb, 64, peer, role, a.blocks), a.reps)
            rec["put_signal_GBps"] = S * 64 * itb / (ms / 1e3) / 1e9
        # ---- the library calls themselves (one launch / copy per message, host-enqueued):
        # uc_put_signal + uc_signal_wait ping-pong and a 64-message window, per transport --
        # SM stores + spin-kernel wait, copy engine + spin-kernel wait, copy engine +
        # cuStreamWaitValue64 (SURVEY §8 a7 paths (i), (ii) and the stream-side Acknowledge)
        if P >= 2 and rank in (0, 1) and not a.no_calls:
            peer = 1 - rank
            src = buf.ptr()
            for tag, (pp, wp) in (("sm", (0, 0)), ("ce", (1, 0)), ("ce_streamwait", (1, 1))):
                dev.set_p2p_path(pp, wp)
                itc = max(1, osu_counts(S, "lat", a.scale)[0] // 100)

                def call_pingpong(n):
                    for _ in range(n):
                        sigv[0] += 1
                        v = sigv[0]
                        if rank == 0:
                            dev.put_signal(src, buf, S, S, sig2, 0, v, peer)
                            dev.signal_wait(buf, S, S, sig2, 0, v, peer)
                        else:
                            dev.signal_wait(buf, S, S, sig2, 0, v, peer)
                            dev.put_signal(src, buf, S, S, sig2, 0, v, peer)

                def call_window(n):
                    for _ in range(n):
                        for _w in range(64):
                            sigv[1] += 1
                            if rank == 0:
                                dev.put_signal(src, buf, S, S, sig2, 1, sigv[1], peer)
                        sigv[2] += 1
                        if rank == 0:
                            dev.signal_wait(buf, S, S, sig2, 2, sigv[2], peer)
                        else:
                            dev.signal_wait(buf, S, S, sig2, 1, sigv[1], peer)
                            dev.put_signal(src, buf, 2 * S, 16, sig2, 2, sigv[2], peer)

                call_pingpong(2)
                ms = timed(lambda: call_pingpong(itc), a.reps)
                rec[f"{tag}_call_latency_us"] = ms * 1e3 / (2 * itc)
                itw = max(1, osu_counts(S, "bw", a.scale)[0] // 20)
                call_window(1)
                ms = timed(lambda: call_window(itw), a.reps)
                rec[f"{tag}_call_GBps"] = S * 64 * itw / (ms / 1e3) / 1e9
            dev.set_p2p_path(0, 0)
        # ---- halo pattern: every rank to top and bottom
        it, wu = osu_counts(S, "lat", a.scale)
        it = max(1, it // 10)
        dev.p2p_bench(U.UC_P2P_HALO, buf, sig, S, max(1, wu // 10), 1, 0, 0, a.blocks)
        ms = timed(lambda: dev.p2p_bench(U.UC_P2P_HALO, buf, sig, S, it, 1, 0, 0, a.blocks), a.reps, True)
        rec["halo_us"] = ms * 1e3 / it
        rec["halo_egress_GBps_per_rank"] = 2 * S * it / (ms / 1e3) / 1e9
        # ---- NCCL send/recv (host mode), ping-pong latency and window bandwidth
        if host is not None and P >= 2 and rank in (0, 1):
            peer = 1 - rank
            src = buf.ptr()
            it, wu = osu_counts(S, "lat", a.scale)
            it = max(1, it // 10)  # host-launched: each message is one NCCL launch

            def pingpong(n):
                for _ in range(n):
                    if rank == 0:
                        host.put_signal(src, buf, S, S, sig, 0, 0, peer)
                        host.signal_wait(buf, S, S, sig, 0, 0, peer)
                    else:
                        host.signal_wait(buf, S, S, sig, 0, 0, peer)
                        host.put_signal(src, buf, S, S, sig, 0, 0, peer)

            pingpong(max(1, wu // 10))
            ms = timed(lambda: pingpong(it), a.reps)
            rec["nccl_latency_us"] = ms * 1e3 / (2 * it)
            itb, _ = osu_counts(S, "bw", a.scale)
            itb = max(1, itb // 4)

            def window(n):
                for _ in range(n):
                    host.group_start()
                    for _w in range(64):
                        if rank == 0:
                            host.put_signal(src, buf, S, S, sig, 0, 0, peer)
                        else:
                            host.signal_wait(buf, S, S, sig, 0, 0, peer)
                    host.group_end()

            window(1)
            ms = timed(lambda: window(itb), a.reps)
            rec["nccl_GBps"] = S * 64 * itb / (ms / 1e3) / 1e9
        out.append(rec)
    comm.barrier()
    buf.free()
    sig.free()
    sig2.free()
    if host is not None:
        host.destroy()
    dev.destroy()
    comm.destroy()
    env.finalize()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--vr", type=int, default=0, help="virtual ranks on one GPU (threads)")
    ap.add_argument("--scale", type=float, default=1.0, help="multiply the OSU iteration counts")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--max-bytes", type=int, default=256 << 20)
    ap.add_argument("--blocks", type=int, default=0)
    ap.add_argument("--no-nccl", action="store_true")
    ap.add_argument("--no-calls", action="store_true", help="skip the per-call uc_put_signal legs")
    a = ap.parse_args()
    if a.vr:
        import threading

        import paper_conf_cluster_sagbilieinu25_b200 as U
        a.nccl = False  # NCCL cannot put two ranks on one GPU
        P = a.vr
        tg = U.ThreadAllgather(P)
        bar = threading.Barrier(P)
        res = [None] * P

        def th(r):
            res[r] = rank_main(r, P, 0, tg.for_rank(r), a, lambda: bar.wait(120))

        ts = [threading.Thread(target=th, args=(r,)) for r in range(P)]
        [t.start() for t in ts]
        [t.join() for t in ts]
        out, ranks, note = res[0], P, "virtual ranks on one GPU: same-device copies, not NVLink"
    else:
        import torch.distributed as dist

        import paper_conf_cluster_sagbilieinu25_b200 as U
        rank, P, local = int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), \
            int(os.environ.get("LOCAL_RANK", 0))
        a.nccl = not a.no_nccl
        dist.init_process_group("gloo", rank=rank, world_size=P)
        out = rank_main(rank, P, local, U.torch_allgather() if P > 1 else None, a, dist.barrier)
        dist.destroy_process_group()
        if rank != 0:
            return
        ranks, note = P, "one process per GPU"
    for rec in out:
        rec.update({"config": "configs[4] halo put-signal P2P sweep", "ranks": ranks, "note": note,
                    "scale": a.scale})
        print(json.dumps(rec))


if __name__ == "__main__":
    main()
