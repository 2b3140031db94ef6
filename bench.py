#!/usr/bin/env python
"""Benchmark of the Jacobi halo/stencil hot path (BASELINE.json metric: "Jacobi GLUPS and % HBM
roofline at 1/2/4/8 B200; halo hidden fraction").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--mode device|host] [--impl ours|reference]
    torchrun --nproc-per-node N --master-addr 127.0.0.1 ... bench.py --gpus N ...

Workload (BASELINE.json configs[3], weak scaling): 16384 x 16384 fp32 points per GPU, ring in y
(rank r owns rows r*16384..), device-initiated halo exchange fused into the stencil, the global
L2 norm every 100 iterations.  At N = 1 this is also configs[2]'s single-GPU point.
A "step" = one pass of the whole hot path: 100 Jacobi iterations (stencil + halo exchange on
every iteration, the norm allreduce on the first), launched as one cached CUDA graph of 17
launches of the default kernel (variant 5: six iterations per launch -- 16 x 6 + 4 -- every
iteration's boundary rows exchanged; --tile-rows T picks T = 1..8 iterations per launch;
--variant 1 = one iteration per launch, the paper's structure).
GLUPS = NY * (NX - 2) * 100 * K / t / 1e9 over all ranks; t = max over ranks of the CUDA-event
time of the K timed steps (inputs > L2: 2 GiB working set per GPU vs 126 MB L2, no flush needed).

Timing protocol: barrier + synchronize on both sides of the timed region, W >= 3 warm-up steps.
Extra objects on the JSON line: roofline (dominant kernel = jacobi_t_kernel<6, 2>, per-launch CUDA
events, algorithmic bytes = 8 B per point per launch; roofline.alu = the same launch against the
FP32-pipe peak), cpu_baseline (the oracle on this host, rank 0, N = 1), e2e (host-buffer end-to-end through
the C-ABI), clocks (nvidia-smi during the timed region), halo (exchange overlap).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "Jacobi GLUPS and % HBM roofline at 1/2/4/8 B200; halo hidden fraction"
UNIT = "GLUPS"
NX = 16384
NY_PER_GPU = 16384
ITERS_PER_STEP = 100
NORM_EVERY = 100


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--mode", default="device", choices=["device", "host"])
    ap.add_argument("--host-path", default="1,0",
                    help="host mode: deep_halo,overlap (uc_jacobi_set_host_path); 0,0 = the paper's Listing 1")
    ap.add_argument("--nx", type=int, default=NX)
    ap.add_argument("--ny-per-gpu", type=int, default=NY_PER_GPU)
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"])
    ap.add_argument("--iters-per-step", type=int, default=ITERS_PER_STEP)
    ap.add_argument("--norm-every", type=int, default=NORM_EVERY)
    ap.add_argument("--no-graph", action="store_true")
    ap.add_argument("--inject-delay-us", type=float, default=0.0,
                    help="MEASUREMENT ONLY: release every boundary-round flag this much later (NVLink-like "
                         "latency on one GPU) to measure how much of it the launch hides")
    ap.add_argument("--same-device", action="store_true",
                    help="TEST ONLY: put every rank on cuda:0 (exercises the multi-process path on a 1-GPU box; "
                         "ranks time-slice the GPU, so the numbers are not a benchmark)")
    ap.add_argument("--no-extras", action="store_true", help="skip e2e / cpu_baseline / halo legs")
    ap.add_argument("--e2e-streams", type=int, default=3,
                    help="e2e leg: solvers (one stream each) whose steps are in flight at once")
    ap.add_argument("--balance", action="store_true",
                    help="balanced row chunks (uc_jacobi_set_balance 1; default: static equal chunks)")
    ap.add_argument("--halo-only", action="store_true", help="skip e2e / cpu_baseline, keep the halo leg")
    ap.add_argument("--cpu-sample-iters", type=int, default=12)
    ap.add_argument("--variant", type=int, default=-1,
                    help="0 register march, 1 TMA-staged, 2 dynamic tiles, 3 persistent, 4 two iterations per "
                         "launch, 5 T iterations per launch (T = --tile-rows; -1: library default = 5, T = 8)")
    ap.add_argument("--stages", type=int, default=0)
    ap.add_argument("--tile-rows", type=int, default=0)
    ap.add_argument("--block-x", type=int, default=0)
    ap.add_argument("--blocks-per-sm", type=int, default=0)
    return ap.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def init_pg(rank, world):
    import torch.distributed as dist
    if world > 1 and not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        dist.init_process_group("gloo", rank=rank, world_size=world)
    return dist if world > 1 else None


def allreduce_max(dist, x: float) -> float:
    if dist is None:
        return x
    import torch
    t = torch.tensor([x], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def barrier(dist):
    if dist is not None:
        dist.barrier()


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, torch copy)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def sm_max_mhz():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        if d.get("sm_max_mhz"):
            return float(d["sm_max_mhz"])
    return 1965.0  # B200 max SM clock (B200_PROFILING.md)


def ncu_traffic(nx, n, kernel="jacobi_iter_kernel"):
    """Per-launch DRAM bytes of the kernel from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    with open(p) as f:
        d = json.load(f)
    e = d.get(f"{kernel}:{nx}x{n}") or (d.get(f"{nx}x{n}") if kernel == "jacobi_iter_kernel" else None)
    return None if e is None else float(e["dram_bytes_per_launch"])


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region (B200_PROFILING.md)."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []   # (arrival time, line)
        self.t0 = self.t1 = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "20"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except (OSError, FileNotFoundError):
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append((time.time(), line.strip()))

    def wait_ready(self, timeout=5.0):
        """nvidia-smi needs a few hundred ms before its first sample; a short timed region that
        starts earlier records no clocks at all."""
        t = time.time()
        while self.proc is not None and not self.lines and time.time() - t < timeout:
            time.sleep(0.02)

    def mark_start(self):
        """Started before the warm-up (nvidia-smi needs ~0.1-0.3 s to start); the timed region is
        [mark_start, mark_stop] and only samples that arrive inside it count."""
        self.t0 = time.time()

    def mark_stop(self):
        self.t1 = time.time()

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sms, maxs, reasons, power = [], [], set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        lines = self.lines
        if self.t0 is not None and self.t1 is not None:
            lines = [l for t, l in self.lines if self.t0 <= t <= self.t1 + 0.025]
        else:
            lines = [l for _, l in self.lines]
        for l in lines:
            f = [x.strip() for x in l.split(",")]
            if len(f) < 9:
                continue
            try:
                sms.append(float(f[1]))
                maxs.append(float(f[2]))
                power.append(float(f[3]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sms) if sms else None, "sm_max_mhz": max(maxs) if maxs else None,
                "reasons": sorted(reasons), "samples": len(sms), "power_w_max": max(power) if power else None}


# ----------------------------------------------------------------------------- our implementation
def run_ours(a):
    import numpy as np
    import torch

    if a.inject_delay_us > 0:
        os.environ["UC_INJECT_PUT_DELAY_NS"] = str(int(a.inject_delay_us * 1000))
    import paper_conf_cluster_sagbilieinu25_b200 as U

    rank, world, local = dist_env()
    if a.same_device:
        local = 0
    if world != a.gpus:
        raise SystemExit(f"--gpus {a.gpus} but WORLD_SIZE={world}")
    dist = init_pg(rank, world)
    torch.cuda.set_device(local)
    ny = a.ny_per_gpu * world if a.scaling == "weak" else a.ny_per_gpu
    nx = a.nx
    mode = U.UC_MODE_DEVICE if a.mode == "device" else U.UC_MODE_HOST
    env = U.Env(rank, world, local, U.torch_allgather() if world > 1 else None)
    comm = U.Comm(env, *U.ring_neighbours(rank, world))
    stream = torch.cuda.Stream()
    coord = U.Coord(comm, mode, stream.cuda_stream)
    J = U.Jacobi(comm, nx, ny)
    if a.block_x or a.blocks_per_sm or a.variant >= 0 or a.stages or a.tile_rows:
        J.set_launch(a.variant, a.block_x, a.blocks_per_sm, a.stages, a.tile_rows)
    host_path = tuple(int(x) for x in a.host_path.split(","))
    if a.mode == "host":
        J.set_host_path(*host_path)
    if a.balance:
        J.set_balance(True)
    n = J.n
    launch_info = J.launch_info()
    use_graph = not a.no_graph
    ips = a.iters_per_step
    pts_rank = n * (nx - 2)
    norms_buf = np.zeros(max(1, ips // max(1, a.norm_every) + 1), np.float64)

    def step():
        J.run(coord, ips, a.norm_every, use_graph, norms_out=norms_buf)

    clocks = ClockSampler(local)
    clocks.start()  # sampling from the warm-up on; only samples inside the timed region count
    for _ in range(a.warmup):
        step()
    coord.sync()
    clocks.wait_ready()
    counts0 = J.launch_counts()

    # ---------------- timed region: K steps, events on the coordinator's stream
    barrier(dist)
    torch.cuda.synchronize()
    clocks.mark_start()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(a.steps):
        step()
    e1.record(stream)
    coord.sync()
    torch.cuda.synchronize()
    clocks.mark_stop()
    barrier(dist)
    clk = clocks.stop()
    counts1 = J.launch_counts()
    t_ms = e0.elapsed_time(e1)
    t_max = allreduce_max(dist, t_ms)
    ms_per_step = t_max / a.steps
    total_pts = pts_rank * world * ips * a.steps
    glups = total_pts / (t_max / 1e3) / 1e9
    # ---------------- the launches a step really runs (uc_jacobi_launch_plan; device counters agree)
    v = launch_info["variant"]
    levels = launch_info["tile_rows"] if v == 5 else 1
    plan = J.plan(mode, ips, a.norm_every)
    per_launch = max(plan)
    # our kernels in the timed region, from the device launch counters (host mode adds one
    # norm_finish kernel per norm round; NCCL's own kernels are not counted)
    ran = [c1 - c0 for c0, c1 in zip(counts0, counts1)]
    reruns = ran[15] if len(ran) > 15 else 0  # blocks whose scaled march re-ran unscaled
    ran = ran[:15]
    assert ran == [sum(1 for t in plan if t == d) * a.steps for d in range(len(ran))], (ran, plan)
    launches = sum(ran) + (a.steps * len(range(0, ips, a.norm_every)) if a.mode == "host" and a.norm_every > 0 else 0)
    # which launches of a step carry the norm round (steps start at k = 0 mod ips)
    norm_launch = []
    kk = 0
    for t in plan:
        norm_launch.append(a.norm_every > 0 and any((kk + j) % a.norm_every == 0 for j in range(t)))
        kk += t
    ghosts = 2 if v == 5 and levels > 4 else 1
    kname = (f"jacobi_t_kernel<{per_launch}, {ghosts}>" if v == 5 else
             {4: "jacobi_two_step_kernel"}.get(v, "jacobi_iter_kernel"))

    # ---------------- dominant kernel timed INSIDE a graph replay: a cached graph of L launches of
    # depth per_launch (norm_every 0 / norm_every = depth: every launch with its norm round),
    # replayed R times between CUDA events on the launching stream
    def graph_kernel_ms(depth, with_norm, L=16, R=5):
        iters = depth * L
        ne = depth if with_norm else 0
        buf = np.zeros(max(1, L), np.float64)
        assert J.plan(mode, iters, ne) == [depth] * L
        for _ in range(2):
            J.run(coord, iters, ne, True, norms_out=buf if with_norm else None)
        coord.sync()
        barrier(dist)
        g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        g0.record(stream)
        for _ in range(R):
            J.run(coord, iters, ne, True, norms_out=buf if with_norm else None)
        g1.record(stream)
        coord.sync()
        return g0.elapsed_time(g1) / (R * L)

    k_plain = allreduce_max(dist, graph_kernel_ms(per_launch, False))
    k_norm = allreduce_max(dist, graph_kernel_ms(per_launch, True))
    n_dom = sum(1 for t in plan if t == per_launch)
    n_dom_norm = sum(1 for t, nl in zip(plan, norm_launch) if t == per_launch and nl)
    dom_ms = k_plain * (n_dom - n_dom_norm) + k_norm * n_dom_norm
    peak, peak_src = measured_peaks()
    # algorithmic bytes per launch: every point of A_k read once, every point of A_{k+T} written
    # once -- 8 B per point per launch = 8/T B per point-iteration
    alg_bytes = 8.0 * pts_rank
    achieved = alg_bytes / (k_plain / 1e3) / 1e9
    sms = torch.cuda.get_device_properties(local).multi_processor_count
    alu_peak = sms * 128 * sm_max_mhz() * 1e6 / 1e12
    # FP32 work: the method does 4 operations per point-iteration (3 FADD + 1 FMUL, never fused).
    # The T-level kernel's norm-free launches run the scaled march: 3 adds per level,
    # the 4^-T product once on the last level, one exact permutation add (x + -0) as a row leaves
    # the ring -- 3T + 2 operations per point and launch; ghost lanes compute too (x 32 / (32 - 2G))
    alg_ops = 4.0 * pts_rank * per_launch
    ops = ((3.0 * per_launch + 2.0) * pts_rank * 32.0 / (32 - 2 * ghosts)) if v == 5 else alg_ops
    alu = ops / (k_plain / 1e3) / 1e12
    # the two roofs as GLUPS ceilings at this depth: HBM moves 8/T B per point-iteration; the
    # FP32 pipe does (3T + 2)/T (x ghost share) operations per point-iteration.  bound = the tighter one.
    hbm_glups = peak / (8.0 / per_launch)
    alu_glups = alu_peak * 1e3 / (ops / (pts_rank * per_launch))
    tighter = "hbm" if hbm_glups <= alu_glups else "alu"
    roof = {"bound": tighter, "kernel": kname, "achieved": round(achieved, 1), "peak": peak,
            "unit": "GB/s", "frac": round(achieved / peak, 4), "traffic": ncu_traffic(nx, n, kname),
            "alg_bytes_per_launch": alg_bytes, "iterations_per_launch": per_launch,
            "hbm_bytes_per_point_iteration": 8.0 / per_launch,
            "roof_glups": {"hbm": round(hbm_glups * world, 1), "alu": round(alu_glups * world, 1),
                           "note": "ceilings at this launch depth (all ranks): HBM = peak / (8/T B per "
                                   "point-iteration); ALU = FP32 peak / FP32 operations per point-iteration"},
            "kernel_ms": round(k_plain, 5), "kernel_norm_ms": round(k_norm, 5),
            "kernel_timing": "inside a CUDA-graph replay of 16 launches (events on the launching stream)",
            "launch_plan_per_step": plan,
            "kernel_share_of_step": round(dom_ms / ms_per_step, 4), "peak_source": peak_src}
    if tighter == "alu":  # report the FP32 roof as the primary figure
        roof.update({"achieved": round(alu, 3), "peak": round(alu_peak, 2), "unit": "TFLOP/s",
                     "frac": round(alu / alu_peak, 4)})
    roof["alu"] = {"bound": "alu", "achieved": round(alu, 3), "peak": round(alu_peak, 2), "unit": "TFLOP/s",
                   "frac": round(alu / alu_peak, 4), "flops_per_launch": ops, "alg_flops_per_launch": alg_ops,
                   "peak_source": f"{sms} SMs x 128 FP32 lanes x {sm_max_mhz():.0f} MHz (derived, DESIGN.md §5)"}
    roof["hbm"] = {"achieved": round(achieved, 1), "peak": peak, "unit": "GB/s", "frac": round(achieved / peak, 4)}

    # ---------------- halo exchange overlap (differential, §8 d): same slab, no neighbours
    halo = None
    if not a.no_extras:
        def full_launch():  # one launch of the timed configuration (T iterations, no norm)
            if per_launch > 1:
                J.run(coord, per_launch, 0, False)
            else:
                J.step(coord, False, None)

        halo = halo_overlap(a, U, torch, dist, env, rank, world, local, nx, n, mode, k_plain, per_launch,
                            launch_info, full_launch, stream)

    # ---------------- e2e through the C-ABI with pinned host buffers
    # Every step: H2D of the step's input slab (pinned), the 100 iterations, D2H of the final slab
    # and the norms.  Two solvers on two streams alternate steps, so step i+1's H2D overlaps step
    # i's compute and D2H (both copy engines busy); the serial single-stream figure is kept too.
    e2e = None
    if not a.no_extras and not a.halo_only:
        slab_elems = (n + 2) * nx
        S = max(1, a.e2e_streams)  # solvers in flight, one stream each
        ke = max(2 * S, min(a.steps, 3 * S))
        solvers = [(J, coord, stream)]
        for _ in range(S - 1):
            Jx = U.Jacobi(comm, nx, ny)
            if a.block_x or a.blocks_per_sm or a.variant >= 0 or a.stages or a.tile_rows:
                Jx.set_launch(a.variant, a.block_x, a.blocks_per_sm, a.stages, a.tile_rows)
            if a.mode == "host":
                Jx.set_host_path(*host_path)
            if a.balance:
                Jx.set_balance(True)
            sx = torch.cuda.Stream()
            solvers.append((Jx, U.Coord(comm, mode, sx.cuda_stream), sx))
        h_in = torch.empty(slab_elems, dtype=torch.float32, pin_memory=True)
        h_in.numpy()[:] = J.copy_out(coord).ravel()
        h_out = [torch.empty(slab_elems, dtype=torch.float32, pin_memory=True) for _ in range(S)]
        h_norm = [torch.zeros(8, dtype=torch.float64, pin_memory=True) for _ in range(S)]

        def e2e_step(i, pipelined):
            b = i % S if pipelined else 0
            Jx, cx, _ = solvers[b]
            Jx.copy_in_async(cx, h_in.data_ptr())
            Jx.run(cx, ips, a.norm_every, use_graph, norms_out=h_norm[b].numpy())
            Jx.copy_out_async(cx, h_out[b].data_ptr())

        for pipelined in (False, True):  # warm-up (graph builds are collective and synchronous)
            for i in range(S):
                e2e_step(i, pipelined)
        for _, cx, _ in solvers:
            cx.sync()
        times = {}
        for pipelined in (False, True):
            barrier(dist)
            torch.cuda.synchronize()
            f0 = torch.cuda.Event(enable_timing=True)
            f0.record(stream)
            for _, _, sx in solvers[1:]:
                sx.wait_event(f0)
            for i in range(ke):
                e2e_step(i, pipelined)
            ends = []
            for _, _, sx in solvers:
                f = torch.cuda.Event(enable_timing=True)
                f.record(sx)
                ends.append(f)
            for _, cx, _ in solvers:
                cx.sync()
            barrier(dist)
            times[pipelined] = allreduce_max(dist, max(f0.elapsed_time(f) for f in ends))
        te, ts = times[True], times[False]
        e2e = {"value": round(pts_rank * world * ips * ke / (te / 1e3) / 1e9, 3), "unit": UNIT,
               "h2d_bytes_per_step": slab_elems * 4, "d2h_bytes_per_step": slab_elems * 4 + 8 * (len(range(0, ips, a.norm_every)) if a.norm_every > 0 else 0),
               "steps": ke, "ms_per_step": round(te / ke, 3),
               "pipeline": f"{S} solvers on {S} streams take turns (step i+1's H2D overlaps step i's compute and D2H)",
               "serial_value": round(pts_rank * world * ips * ke / (ts / 1e3) / 1e9, 3),
               "serial_ms_per_step": round(ts / ke, 3)}
        comm.barrier()
        for Jx, cx, _ in solvers[1:]:
            Jx.destroy()
            cx.destroy()

    comm.barrier()
    J.destroy()
    coord.destroy()
    comm.destroy()
    env.finalize()

    # ---------------- oracle on the host cores (rank 0, N = 1)
    cpu = cpu_par = None
    if rank == 0 and world == 1 and not a.no_extras and not a.halo_only:
        cpu = cpu_baseline(nx, a.ny_per_gpu, a.cpu_sample_iters, a.norm_every)
        cpu_par = cpu_parallel(nx, a.ny_per_gpu, 10, a.norm_every)

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(glups, 3), "unit": UNIT, "n_gpus": world, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": round(ms_per_step, 4), "higher_is_better": True,
            "scaling": a.scaling, "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": f"jacobi2d_{nx}x{a.ny_per_gpu}_per_gpu_{a.mode}_ring" if a.scaling == "weak"
                       else f"jacobi2d_{nx}x{ny}_strong_{a.mode}_ring",
                       "baseline_config": "configs[3] (weak, 16384^2 per GPU)" if a.scaling == "weak"
                       else "configs[2] (strong, 16384^2 total)",
                       "nx": nx, "ny_global": ny, "rows_per_gpu": n, "iters_per_step": ips,
                       "norm_every": a.norm_every, "mode": a.mode, "cuda_graph": use_graph,
                       "injected_flag_delay_us": a.inject_delay_us or None,
                       "host_path": ({"deep_halo": host_path[0], "overlap": host_path[1]} if a.mode == "host"
                                     else None),
                       "parallelism": f"y-slab x{world}", "l2": "inputs > L2 (2 slabs x "
                       f"{(n + 2) * nx * 4 / 2**20:.0f} MiB per GPU vs 126 MB L2), no flush",
                       "launch": launch_info, "balanced_chunks": bool(v == 5 and a.mode == "device" and a.balance)},
            "roofline": roof, "cpu_baseline": cpu, "cpu_parallel": cpu_par, "e2e": e2e, "clocks": clk, "gpu_launches": launches,
            "gpu_launches_by_depth": {str(d): c for d, c in enumerate(ran) if c},
            "scaled_march_reruns": reruns,
            "halo": halo, "pct_hbm_roofline": round(100 * glups / (world * peak / 8.0), 2),
            "pct_hbm_roofline_note": "GLUPS vs the one-iteration-per-sweep roofline (8 B per point-iteration at the measured copy peak); above 100 because temporal blocking moves 8/T B per point-iteration; the kernel's own bandwidth fraction is roofline.frac",
        }
        print(json.dumps(line))
    if dist is not None:
        dist.destroy_process_group()


def halo_overlap(a, U, torch, dist, env, rank, world, local, nx, n, mode, k_full, per_launch, launch_info,
                 full_launch=None, full_stream=None):
    """hidden = clamp(1 - (T_full - T_compute) / T_xchg, 0, 1) (SURVEY §8 d).  T_compute: the same
    slab and kernel with no neighbours (chain-less comm: top = bottom = -1 is not a valid Jacobi
    topology for P > 1, so we time a P = 1 dirichlet-chain solver of the same n rows in its own
    communicator); T_xchg: the exchange alone = put_signal of one row to each neighbour.
    T_full and T_compute are timed in alternation (10 repetitions of 5 launches each, the
    lowest and highest dropped, the mean of the rest), so clock drift cancels."""
    # T_compute: independent single-rank chain (no waits, no puts) on this GPU
    env1 = U.Env(0, 1, local)
    comm1 = U.Comm(env1, -1, -1)
    st = torch.cuda.Stream()
    co1 = U.Coord(comm1, mode, st.cuda_stream)
    J1 = U.Jacobi(comm1, nx, n)
    J1.set_launch(launch_info["variant"], 0, 0, launch_info["stages"], launch_info["tile_rows"])

    def comp_launch():
        if per_launch > 1:
            J1.run(co1, per_launch, 0, False)
        else:
            J1.step(co1, False, None)

    def timed(fn, stream, k=5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(k):
            fn()
        e1.record(stream)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / k

    def trimmed(xs):
        xs = sorted(xs)[1:-1] if len(xs) > 2 else xs
        return statistics.mean(xs)

    for _ in range(3):
        comp_launch()
    fulls, comps = [], []
    for _ in range(10):
        if full_launch is not None:
            barrier(dist)
            fulls.append(timed(full_launch, full_stream))
        comps.append(timed(comp_launch, st))
    t_comp = trimmed(comps)
    t_full = trimmed(fulls) if fulls else k_full
    J1.destroy()
    co1.destroy()
    comm1.destroy()
    env1.finalize()
    # T_xchg: two row puts + signal waits (device mode), the same message size
    comm = U.Comm(env, *U.ring_neighbours(rank, world))
    st2 = torch.cuda.Stream()
    co = U.Coord(comm, U.UC_MODE_DEVICE, st2.cuda_stream)
    row = U.SymMem(comm, 2 * nx * 4)
    sig = U.SymMem(comm, 256)
    with torch.cuda.stream(st2):
        src = torch.zeros(nx, dtype=torch.float32, device="cuda")
    reps = 50
    barrier(dist)
    x0, x1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    x0.record(st2)
    for i in range(1, reps + 1):
        co.put_signal(src.data_ptr(), row, 0, nx * 4, sig, 0, i, comm.top)
        co.put_signal(src.data_ptr(), row, nx * 4, nx * 4, sig, 16, i, comm.bottom)
        co.signal_wait(row, 0, nx * 4, sig, 0, i, comm.bottom)
        co.signal_wait(row, nx * 4, nx * 4, sig, 16, i, comm.top)
    x1.record(st2)
    co.sync()
    # a launch of T iterations exchanges T rounds of boundary rows; under injected flag latency
    # (--inject-delay-us) every round of the exchange alone costs that much more
    t_x = x0.elapsed_time(x1) / reps * per_launch + per_launch * a.inject_delay_us / 1e3
    comm.barrier()
    row.free()
    sig.free()
    co.destroy()
    comm.destroy()
    t_full = allreduce_max(dist, t_full)
    t_comp = allreduce_max(dist, t_comp)
    t_x = allreduce_max(dist, t_x)
    hidden = max(0.0, min(1.0, 1.0 - (t_full - t_comp) / t_x)) if t_x > 0 else None
    return {"hidden_fraction": None if hidden is None else round(hidden, 4), "t_full_ms": round(t_full, 5),
            "t_compute_ms": round(t_comp, 5), "t_xchg_ms": round(t_x, 5),
            "note": f"per launch ({per_launch} iteration(s)); t_xchg = standalone put_signal of both boundary "
                    f"rows + waits, x{per_launch} rounds" + (f", + {a.inject_delay_us} us injected flag latency per "
                                                             "round" if a.inject_delay_us else "")}


def cpu_baseline(nx, ny, iters, norm_every):
    """The oracle as it stands (single-threaded C, -O2) on a bounded sample of the workload: one
    oracle_jacobi_run of `iters` iterations of the full rank-0 grid (the norm every norm_every
    iterations, as in the timed steps), timed around the C call only."""
    import oracle
    from inputs import gen
    oracle.build()
    g = gen.global_field(nx, ny, "ring")
    t = time.perf_counter()
    oracle.jacobi_run(g, iters, "ring", norm_every)
    dt = time.perf_counter() - t
    return {"value": round(ny * (nx - 2) * iters / dt / 1e9, 4), "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"one oracle run of {iters} iterations (norm every {norm_every}) of the full {nx}x{ny} ring "
                      f"grid, {dt:.1f} s incl. the wrapper's copy of the 1 GiB array; host {os.cpu_count()} "
                      "cores visible, 1 used (the oracle is single-threaded by design)"}


def cpu_parallel(nx, ny, iters, norm_every):
    """The same loop on every host core (benchmarks/cpu_omp, OpenMP C, bit-identical grid --
    tests/test_cpu_omp.py): the multi-core host baseline beside the single-core oracle."""
    import numpy as np

    from benchmarks import cpu_omp
    from inputs import gen
    cpu_omp.build()
    g = np.ascontiguousarray(gen.global_field(nx, ny, "ring"), dtype=np.float32)
    cpu_omp.jacobi_run(g, 1, "ring", 0, inplace=True)  # page in, spin up the thread pool
    t = time.perf_counter()
    cpu_omp.jacobi_run(g, iters, "ring", norm_every, inplace=True)
    dt = time.perf_counter() - t
    return {"value": round(ny * (nx - 2) * iters / dt / 1e9, 4), "unit": UNIT, "cores": cpu_omp.threads(),
            "kind": "openmp (same loop as the oracle, bit-identical grid)",
            "sample": f"{iters} iterations (norm every {norm_every}) of the full {nx}x{ny} ring grid, {dt:.2f} s"}


# ----------------------------------------------------------------------------- reference arm
def run_reference(a):
    """The oracle (plain single-threaded C over the global grid) on the host cores, as the
    reference arm: rank 0 only.  The warm-up is one oracle run of W iterations, the timed region
    ONE oracle run of K iterations (each "step" = one iteration of the 16384^2 rank-0 grid with
    the step's norm cadence), so the wrapper's array copies are paid once, not per step."""
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import numpy as np

    import oracle
    from inputs import gen
    oracle.build()
    nx, ny = a.nx, a.ny_per_gpu
    g = gen.global_field(nx, ny, "ring")
    g, _s = oracle.jacobi_run(g, a.warmup, "ring", a.norm_every)
    t = time.perf_counter()
    g, _s = oracle.jacobi_run(g, a.steps, "ring", a.norm_every)
    dt = time.perf_counter() - t
    assert np.isfinite(g[1, 1])
    v = ny * (nx - 2) * a.steps / dt / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": round(v, 4), "unit": UNIT, "n_gpus": world,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": round(dt / a.steps * 1e3, 2),
            "higher_is_better": True, "scaling": a.scaling, "vs_baseline": None, "dtype": "f32",
            "data": "synthetic",
            "config": {"workload": f"jacobi2d_{nx}x{ny}_per_gpu_{a.mode}_ring", "nx": nx, "ny_global": ny,
                       "sample": f"1 iteration per step of the rank-0 {nx}x{ny} grid (norm every {a.norm_every}); "
                                 "K steps timed as one oracle run"},
            "cpu_baseline": {"value": round(v, 4), "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"one oracle run of {a.steps} iterations of {nx}x{ny}, {dt:.1f} s"},
            "e2e": {"value": round(v, 4), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))


def spawn_ranks(a):
    """`bench.py --gpus N` without a torchrun environment: launch N ranks (one per GPU) with
    torch.distributed.run on 127.0.0.1 and relay their output (rank 0 prints the JSON line)."""
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={a.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd, cwd=ROOT)


def main():
    a = parse()
    if a.warmup < 3:
        raise SystemExit("--warmup must be >= 3")
    if a.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn_ranks(a))
    if a.impl == "reference":
        run_reference(a)
    else:
        run_ours(a)


if __name__ == "__main__":
    main()
