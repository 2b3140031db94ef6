"""Virtual-rank harness: P ranks as host threads in one process.

Each thread is one rank with its own Env/Comm/Coord/stream; the bootstrap allgather is an
in-memory barrier and peer buffers are plain pointers (the library detects same-process
peers), so the device-mode put/signal protocol runs for real on ONE GPU.
"""
from __future__ import annotations

import threading


def run_ranks(P: int, fn, timeout: float = 600.0):
    """Run fn(rank, P, allgather_impl_or_None) in P threads; return the per-rank results."""
    from paper_conf_cluster_sagbilieinu25_b200 import ThreadAllgather

    tg = ThreadAllgather(P, timeout=timeout) if P > 1 else None
    results = [None] * P
    errors = [None] * P
    order = []

    def wrap(r):
        try:
            results[r] = fn(r, P, tg.for_rank(r) if tg else None)
        except BaseException as e:  # noqa: BLE001
            errors[r] = e
            order.append(r)
            if tg is not None:
                tg._barrier.abort()

    threads = [threading.Thread(target=wrap, args=(r,), daemon=True) for r in range(P)]
    for t in threads:
        t.start()
    for t in threads:
        t.join(timeout)
    if order:  # the first failure in time caused the others (aborted barrier)
        raise errors[order[0]]
    if any(t.is_alive() for t in threads):
        raise TimeoutError("virtual ranks did not finish")
    return results
