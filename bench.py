#!/usr/bin/env python
"""Benchmark of the hybrid tridiagonal solve (tiled PCR + p-Thomas) on B200.

Contract (driver): `python bench.py --gpus N --steps K --warmup W` prints ONE
JSON line on rank 0.  A "step" is one pass of the whole hot path (one tri_solve
of the full batch).  Default workload = BASELINE config 5 (fp64, m = 16384
systems of n = 16384, contiguous), the config the metric's 1/2/4/8-GPU figures
are quoted on; other configs via --config.  Inputs are synthetic (trigen,
seeded), generated on the host and resident in HBM before the timed region.

N > 1 (torchrun, one rank per GPU, NCCL): the m systems of the batched
configs (c2, c4, c5) are sharded into contiguous ranges through
paper_conf_icpp_kimwch11_b200.dist (strong scaling: rank r solves m/N systems;
no collective inside the solve; time = max over ranks); the one-system configs
(c1, c3) run as replicas (weak scaling).  The edge collectives (NCCL scatter of
a, b, c, d from rank 0, gather of x) run on the real shards after the timed
region and are reported in `collectives`, with a check of the gathered x.

--impl reference times the CPU oracle (plain sequential Thomas, oracle/) on a
bounded sample of the same workload -- the tier's reference arm.
"""
import argparse
import glob
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIGS = {
    # name: (n, m, dtype, layout, description)  -- BASELINE.json configs[0..4]
    "c1": (1024, 1, "f64", 0, "single fp64 diagonally dominant system n=1024"),
    "c2": (1024, 1024, "f64", 1, "batched fp64 m=1024 systems of n=1024, interleaved"),
    "c3": (1 << 24, 1, "f64", 0, "single large fp64 system n=2^24"),
    "c4": (256, 1 << 20, "f32", 0, "many small fp32 systems m=2^20, n=256, contiguous"),
    "c5": (16384, 16384, "f64", 0, "batched fp64 m=16384 systems of n=16384, contiguous"),
}
METRIC = "Munknowns/s fp64/fp32 and % of HBM roofline at 1/2/4/8 B200"
FALLBACK_HBM_GBS = 6650.0  # /opt/skills/guides/B200_PROFILING.md fallback


def config_of(args):
    """(n, m, dtype, layout, desc) of --config, with the --n / --m / --layout overrides
    (an overridden shape is a side measurement, not a BASELINE config)."""
    n, m, dt, layout, desc = CONFIGS[args.config]
    if args.layout is not None:
        layout = args.layout
    if args.n is not None or args.m is not None:
        n, m = args.n or n, args.m or m
        desc = f"custom shape n={n} m={m} ({dt}, layout {layout}); not a BASELINE config"
    return n, m, dt, layout, desc


def workload_of(args):
    return args.config if args.n is None and args.m is None else args.config + "-custom"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c5", choices=sorted(CONFIGS))
    ap.add_argument("--layout", type=int, default=None, help="override layout (0 contiguous, 1 interleaved)")
    ap.add_argument("--n", type=int, default=None, help="override n (side measurement: workload named custom)")
    ap.add_argument("--m", type=int, default=None, help="override m (side measurement: workload named custom)")
    ap.add_argument("--family", default="dd")
    ap.add_argument("--k", type=int, default=None, help="force the transition point k")
    ap.add_argument("--variant", type=int, default=None, help="force variant (1 onchip, 2 split, 3 fused)")
    ap.add_argument("--scaling", default=None, choices=["strong", "weak"],
                    help="strong (default for the batched configs): the config's m systems are sharded over the "
                         "ranks; weak (default for the one-system configs c1 / c3): every rank solves a replica")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-check", action="store_true")
    ap.add_argument("--no-graph", action="store_true", help="time direct solve calls instead of graph replays")
    ap.add_argument("--no-collectives", action="store_true", help="N > 1: skip the scatter/gather measurement")
    return ap.parse_args()


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as fh:
            j = json.load(fh)
        return float(j["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy test)"
    return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """Polls NVML (SM clock, throttle reasons) every 10 ms during the timed region."""

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, index):
        self.samples, self.reasons, self.ok = [], set(), False
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            self.max_mhz = None

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.01)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *exc):
        if self.ok:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": float(statistics.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def method_arrays(plan, tri, l2_bytes):
    """Arrays of n*m*s bytes the plan's method moves per solve (SURVEY 8(d)
    model): compulsory 5 + every materialised PCR pass + spilled Thomas
    intermediates.  Superseded by the ncu-measured DRAM bytes when a traffic
    file for this exact plan exists (roofline.method_source says which)."""
    v = plan.variant
    if v in (tri.VARIANT_WARP, tri.VARIANT_ONCHIP):
        return 5
    if v in (tri.VARIANT_FUSED, tri.VARIANT_STREAM, tri.VARIANT_SCAN):
        return 5  # c', d' stay in smem or in per-CTA scratch that stays in L2 (ncu: 5.0 arrays of DRAM traffic)
    if v == tri.VARIANT_SCAN_MC:
        return 9 if "lookback=0" not in plan.describe() else 13  # look-back: 4 + 2 + 2 + 1; three passes: + 4
    if plan.k == 0:
        return 9  # read a, b, c, d; write + read c', d' (materialised); write x -- ncu bytes override when known
    # pass 1: read 4 + write 3; each later pass: read 3 + write 3; p-Thomas: read 3, c', d' 2 + 2, write x
    return 7 + 6 * (plan.launches - 2) + 8


def cpu_oracle_time(n, mr, arrs, layout, budget_s=20.0):
    """Time the oracle (as it stands) on the host cores over a bounded sample,
    with every core the process may use and with one thread."""
    import oracle
    cores = len(os.sched_getaffinity(0))
    # sample: whole systems, as many as fit ~budget_s at ~50 Munk/s/core
    est_rate = 50e6 * cores
    qs = int(max(1, min(mr, budget_s * est_rate / n)))
    if layout == 1 and qs < mr:
        qs = mr  # interleaved sample would read strided rows; use the full (small) batch
    t0 = time.perf_counter()
    oracle.solve_batch(n, mr, *arrs, layout=layout, q_begin=0, q_end=qs, nthreads=cores)
    dt = time.perf_counter() - t0
    # one thread: a smaller sample (~3 s at ~50 Munk/s)
    q1 = int(max(1, min(qs, 3.0 * 50e6 / n))) if layout == 0 else qs
    t0 = time.perf_counter()
    oracle.solve_batch(n, mr, *arrs, layout=layout, q_begin=0, q_end=q1, nthreads=1)
    dt1 = time.perf_counter() - t0
    return {"value": n * qs / dt / 1e6, "unit": "Munknowns/s", "cores": cores, "kind": "oracle",
            "hardware_concurrency": os.cpu_count(),
            "sample": f"{qs} of {mr} systems x n={n} (whole systems, {dt:.2f} s, {cores} threads over systems)",
            "t1": {"value": n * q1 / dt1 / 1e6, "unit": "Munknowns/s", "cores": 1,
                   "sample": f"{q1} systems x n={n} ({dt1:.2f} s, one thread)"}}


def run_reference(args):
    """--impl reference: the CPU oracle on the box's host cores."""
    world, rank, _ = dist_env()
    n, m, dt, layout, desc = config_of(args)
    if rank != 0:
        return  # rank 0 alone runs and prints it
    import oracle
    import trigen
    cores = len(os.sched_getaffinity(0))
    # bounded sample per step: ~10 s of CPU work across all steps
    total_budget = 60.0
    per_step = total_budget / max(1, args.steps + args.warmup)
    qs = int(max(1, min(m, per_step * 50e6 * cores / n)))
    if layout == 1:
        qs = m
    arrs = trigen.generate(n, qs, dt, layout, args.family, seed=trigen.SEED_BASE + int(args.config[1]))
    for _ in range(args.warmup):
        oracle.solve_batch(n, qs, *arrs, layout=layout, nthreads=cores)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.solve_batch(n, qs, *arrs, layout=layout, nthreads=cores)
        times.append(time.perf_counter() - t0)
    t = sum(times) / len(times)
    v = n * qs / t / 1e6
    out = {"metric": METRIC, "value": v, "unit": "Munknowns/s", "impl": "reference", "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
           "scaling": args.scaling or ("weak" if m == 1 else "strong"), "vs_baseline": None, "dtype": dt,
           "data": "synthetic",
           "config": {"workload": workload_of(args), "desc": desc, "n": n, "m": m, "layout": layout,
                      "family": args.family},
           "cpu_baseline": {"value": v, "unit": "Munknowns/s", "cores": cores, "kind": "oracle",
                            "sample": f"{qs} of {m} systems x n={n} per step (whole systems)"},
           "e2e": {"value": v, "unit": "Munknowns/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist

    import trigen
    import paper_conf_icpp_kimwch11_b200 as tri
    from paper_conf_icpp_kimwch11_b200 import dist as tdist

    world, rank, local = dist_env()
    ngpu = torch.cuda.device_count()
    backend = "nccl"
    if world > 1 and ngpu >= world:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    elif world > 1:
        # fewer GPUs than ranks (a code-path check on a 1-GPU box, not a scaling
        # measurement): ranks share devices, collectives over gloo; the line says so
        backend = "gloo"
        torch.cuda.set_device(local % ngpu)
        dist.init_process_group("gloo")
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    rdev = dev if backend == "nccl" else torch.device("cpu")  # device of the all-reduce scalars

    n, m, dt, layout, desc = config_of(args)
    s = 8 if dt == "f64" else 4
    tdt = torch.float64 if dt == "f64" else torch.float32
    td = tri.F64 if dt == "f64" else tri.F32
    # strong scaling for the batched configs (the m systems sharded over the ranks,
    # dist.shard_range); the one-system configs run as replicas (system q = rank)
    scaling = args.scaling or ("weak" if m == 1 else "strong")
    if scaling == "strong":
        q0, mr = tdist.shard_range(m, world, rank)
        m_all = m
    else:
        q0, mr = rank * m, m
        m_all = m * world
    if mr == 0:
        raise SystemExit(f"rank {rank}: no systems in its shard (m = {m} < N = {world}); use --scaling weak")
    seed = trigen.SEED_BASE + int(args.config[1])

    # ---- inputs: seeded host generation of this rank's shard (global system
    # indices q0 ..), then resident in HBM before the timed region
    pin = not args.no_e2e
    host = [torch.empty(n * mr, dtype=tdt, pin_memory=pin) for _ in range(4)]
    trigen.generate(n, mr, dt, layout, args.family, seed=seed, q0=q0, out=[t.numpy() for t in host])
    a, b, c, d = (t.to(dev, non_blocking=False) for t in host)
    x = torch.empty_like(b)
    plan = tri.Plan(n, mr, td, layout)
    if args.variant is not None:
        plan.variant = args.variant
    if args.k is not None:
        plan.k = args.k
    stream = torch.cuda.current_stream()
    n_unknowns = n * mr

    # L2 policy: flush between timed steps when this rank's working set could sit in L2
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    ws = 5 * n_unknowns * s + plan.scratch_bytes
    flush = ws < 4 * l2
    flush_buf = torch.empty(2 * l2 // 4 + 1024, dtype=torch.int32, device=dev) if flush else None
    clean_buf = torch.ones(2 * l2 // 4 + 1024, dtype=torch.int32, device=dev) if flush else None

    def flush_l2():
        # outside the timed interval: write 2x L2 worth of bytes (evicts our data),
        # then read another 2x L2 so the dirty lines are written back before the
        # step instead of during it
        flush_buf.add_(1)
        clean_buf.sum()

    for _ in range(args.warmup):
        plan.solve(a, b, c, d, out=x, stream=stream)
    torch.cuda.synchronize()
    # the timed step replays the solve from a CUDA graph captured once: the same
    # kernels, without the per-call host latency that would otherwise sit inside
    # the device-timed window of the small configs (reported separately: `direct`)
    graph = None
    if not args.no_graph:
        cap = torch.cuda.Stream()
        cap.wait_stream(stream)
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph, stream=cap):
            plan.solve(a, b, c, d, out=x, stream=cap)
        torch.cuda.synchronize()
        for _ in range(args.warmup):
            graph.replay()
        torch.cuda.synchronize()

    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(dev.index) as clk:
        for i in range(args.steps):
            if flush:
                flush_l2()
            ev[i][0].record(stream)
            if graph is not None:
                graph.replay()
            else:
                plan.solve(a, b, c, d, out=x, stream=stream)
            ev[i][1].record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    step_ms = [e0.elapsed_time(e1) for e0, e1 in ev]
    t_step = sum(step_ms) / len(step_ms)
    t_step_max = tdist.max_over_ranks(t_step, device=rdev)
    value = m_all * n / (t_step_max * 1e-3) / 1e6  # whole-job Munknowns/s

    # ---- per-call latency of a direct (non-graph) tri_solve: idle GPU, events
    # around one call, so the host-side cost of the call (ctypes, argument checks,
    # launches) is inside the window; plus the host time of one call
    direct = None
    if graph is not None:
        reps = max(3, min(args.steps, 20))
        dms, hus = [], []
        for _ in range(reps):
            if flush:
                flush_l2()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            th0 = time.perf_counter()
            plan.solve(a, b, c, d, out=x, stream=stream)
            hus.append((time.perf_counter() - th0) * 1e6)
            e1.record(stream)
            torch.cuda.synchronize()
            dms.append(e0.elapsed_time(e1))
        direct = {"ms_per_step": statistics.median(dms), "host_us_per_call": statistics.median(hus),
                  "how": "one Plan.solve (ctypes -> tri_solve) per step on an idle GPU, CUDA events around the call; "
                         "host_us = Python + C host time of the call"}

    # ---- back to back (small working sets only, where each timed step above is one
    # graph replay after an L2 flush and so carries the replay's fixed device-side
    # cost, ~2-3 us): the K steps as ONE graph of K solves, solve i on its own copy
    # of the inputs and x (K x the working set > L2, flushed once before), so every
    # solve still reads its inputs from HBM and writes x back; per step = total / K
    b2b = None
    if flush and graph is not None and rank == 0:
        try:
            kk = int(max(2, min(args.steps, 8e9 // max(1, 5 * n_unknowns * s))))  # <= ~8 GB of copies
            cps = [[t.clone() for t in (a, b, c, d, x)] for _ in range(kk)]
            cap2 = torch.cuda.Stream()
            cap2.wait_stream(stream)
            g2 = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g2, stream=cap2):
                for cp in cps:
                    plan.solve(*cp[:4], out=cp[4], stream=cap2)
            torch.cuda.synchronize()
            g2.replay()
            tot = []
            for _ in range(3):
                flush_l2()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                g2.replay()
                e1.record(stream)
                torch.cuda.synchronize()
                tot.append(e0.elapsed_time(e1))
            bms = statistics.median(tot) / kk
            b2b = {"ms_per_step": bms, "value": n_unknowns / (bms * 1e-3) / 1e6, "unit": "Munknowns/s",
                   "steps": kk, "roofline_frac": 5 * n_unknowns * s / (bms * 1e-3) / 1e9 / measured_peaks()[0],
                   "how": f"{kk} solves in one CUDA graph, solve i on its own copy of a, b, c, d, x "
                          f"({kk} x {5 * n_unknowns * s / 1e6:.3f} MB; L2 flushed once before, so every copy is "
                          "read cold, once); per step = total / steps; median of 3"}
            del cps
        except Exception as exc:
            b2b = {"error": repr(exc)[:200]}

    # ---- sampled parity vs the oracle (rank 0's shard, a few whole systems)
    parity = None
    if not args.no_check and rank == 0:
        import oracle
        xs = x.cpu().numpy()
        qs = sorted(set([0, mr // 3, mr // 2, mr - 1]))
        errs = []
        for qq in qs:
            sa = trigen.generate(n, 1, dt, 0, args.family, seed=seed, q0=q0 + qq)
            xo = oracle.solve_batch(n, 1, *sa)
            xg = xs.reshape(mr, n)[qq] if layout == 0 else xs.reshape(n, mr)[:, qq]
            errs.append(float(np.max(np.abs(xg.astype(np.float64) - xo) / np.abs(xo))))
        parity = {"systems": len(qs), "max_rel_err": max(errs)}

    # ---- end to end through the C ABI with HOST buffers (copies inside the timed region)
    e2e = None
    if not args.no_e2e:
        xh = torch.empty(n * mr, dtype=tdt, pin_memory=True)
        plan.solve_host(*host, xh, stream=stream)  # warm (allocates staging)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(args.e2e_steps):
            plan.solve_host(*host, xh, stream=stream)  # synchronises its stream
        te = tdist.max_over_ranks((time.perf_counter() - t0) / args.e2e_steps, device=rdev)
        e2e = {"value": m_all * n / te / 1e6, "unit": "Munknowns/s",
               "h2d_bytes_per_step": 4 * n_unknowns * s, "d2h_bytes_per_step": n_unknowns * s,
               "steps": args.e2e_steps, "ms_per_step": te * 1e3,
               "how": "tri_solve_host per rank: pinned host a,b,c,d -> device, solve, x -> pinned host, per step; "
                      "max over ranks"}
        del xh

    # ---- edge collectives (N > 1, sharded batch): NCCL scatter of the input
    # shards from rank 0 and gather of x to rank 0, through dist.py on the real
    # data, checked against the resident shards and the oracle
    coll = None
    if world > 1 and scaling == "strong" and not args.no_collectives:
        try:
            coll = edge_collectives(args, tdist, trigen, n, m, dt, layout, seed, q0, mr, (a, b, c, d), x, s, world,
                                    rank, dev, tdt, rdev)
        except Exception as exc:  # never let the edge measurement cost the solve numbers
            coll = {"error": repr(exc)[:300]}

    # ---- the copy bandwidth of this GPU in this run (re-measure the
    # denominator in the same session; the roofline keeps MEASURED_PEAKS.json's)
    copy_gbs = None
    if rank == 0:
        try:
            src = torch.empty(1 << 30, dtype=torch.uint8, device=dev)
            dst = torch.empty_like(src)
            for _ in range(2):
                dst.copy_(src)
            best = None
            for _ in range(5):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                dst.copy_(src)
                e1.record()
                torch.cuda.synchronize()
                t = e0.elapsed_time(e1)
                best = t if best is None else min(best, t)
            copy_gbs = 2 * src.numel() / (best * 1e-3) / 1e9
            del src, dst
            torch.cuda.empty_cache()
        except Exception:  # never let the side measurement cost the line
            copy_gbs = None

    # ---- CPU oracle baseline (rank 0 at N=1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_oracle_time(n, mr, [t.numpy() for t in host], layout)

    if rank != 0:
        dist.destroy_process_group()
        return
    peak, peak_src = measured_peaks()
    algo_bytes = 5 * n_unknowns * s          # compulsory 5 arrays per unknown
    achieved = algo_bytes / (t_step * 1e-3) / 1e9
    marr = method_arrays(plan, tri, l2)
    method_bytes = marr * n_unknowns * s
    method_src = "model (SURVEY 8(d))"
    traffic, traffic_src = None, None
    # profiles/traffic_<config>*.json: one ncu capture per plan (n, m, k, variant, layout)
    for tf in sorted(glob.glob(os.path.join(ROOT, "profiles", f"traffic_{args.config}*.json"))):
        with open(tf) as fh:
            tj = json.load(fh)
        if tj.get("n") == n and tj.get("m") == mr and tj.get("k") == plan.k and \
                tj.get("variant", plan.variant) == plan.variant and tj.get("layout", layout) == layout and \
                all(t in plan.describe().split() for t in tj.get("describe_has", [])):
            traffic = tj.get("dram_bytes_per_launch")
            traffic_src = tj.get("source", tf)
            break
    if traffic:
        method_bytes, method_src = traffic, "ncu dram bytes of this plan (" + str(traffic_src) + ")"
    out = {
        "metric": METRIC, "value": value, "unit": "Munknowns/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": t_step_max, "higher_is_better": True, "scaling": scaling,
        "vs_baseline": None, "dtype": dt, "data": "synthetic",
        "config": {"workload": workload_of(args), "desc": desc, "n": n, "m": m, "m_per_rank": mr, "layout": layout,
                   "family": args.family,
                   "parallelism": (f"dp{world}: the m systems sharded over the ranks (contiguous ranges, "
                                   "dist.shard_range), no collective in the solve" if scaling == "strong" else
                                   f"dp{world}: replicas (every rank solves its own {m} system(s))") +
                                  ("" if backend == "nccl" or world == 1 else
                                   f" [code-path check: {world} ranks on {ngpu} GPU(s), gloo collectives]"),
                   "timing": "CUDA graph replay of one solve per step" if graph is not None else "direct solve call",
                   "l2": "flushed between timed steps (2x L2 write + 2x L2 read)" if flush else
                         f"inputs larger than L2 ({ws / 2**30:.1f} GiB working set vs {l2 / 2**20:.0f} MiB L2)",
                   "plan": plan.describe()},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                     "traffic": traffic, "traffic_source": traffic_src, "peak_source": peak_src,
                     "copy_gbs_same_run": copy_gbs,
                     "algorithmic_bytes_per_launch": algo_bytes,
                     "method_arrays": method_bytes / (n_unknowns * s), "method_source": method_src,
                     "method_bytes_per_launch": method_bytes,
                     "method_frac": method_bytes / (t_step * 1e-3) / 1e9 / peak,
                     "excess_traffic": (traffic / algo_bytes) if traffic else None,
                     "kernel": "whole solve (%d launch%s)" % (plan.launches, "" if plan.launches == 1 else "es")},
        "clocks": clk.summary(),
        "e2e": e2e,
        "direct": direct,
        "b2b": b2b,
        "gpu_launches": args.steps * plan.launches,
        "cpu_baseline": cpu,
        "collectives": coll,
        "parity": parity,
        "step_ms_min": min(step_ms), "step_ms_median": statistics.median(step_ms),
    }
    print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


def edge_collectives(args, tdist, trigen, n, m, dt, layout, seed, q0, mr, local, x_local, s, world, rank, dev, tdt,
                     rdev):
    """SURVEY 8(e) edge collectives through dist.py on the real shards: rank 0
    scatters a, b, c, d (dist.scatter_inputs) and gathers x (dist.gather_x);
    CUDA events, max over ranks.  Checks: every rank's scattered shard equals
    its resident one bitwise; the gathered x matches the oracle on sampled
    systems of every shard."""
    import torch
    import torch.distributed as dist
    full = None
    if rank == 0:
        full = [torch.from_numpy(t).to(dev) for t in trigen.generate(n, m, dt, layout, args.family, seed=seed)]
    res = {}
    for what in ("scatter", "gather"):
        for it in range(2):  # one warm-up round
            dist.barrier()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            if what == "scatter":
                got = tdist.scatter_inputs(n, m, full, layout, dtype=tdt, device=dev)
            else:
                xfull = tdist.gather_x(x_local, n, m, layout)
            e1.record()
            torch.cuda.synchronize()
        res[what] = tdist.max_over_ranks(e0.elapsed_time(e1), device=rdev)
    same = all(torch.equal(g, l) for g, l in zip(got, local))
    ok = tdist.max_over_ranks(0.0 if same else 1.0, device=rdev) == 0.0
    per = -(-m // world)
    moved = (world - 1) * n * per * s  # bytes of one array leaving / entering rank 0
    out = {"scatter_ms": res["scatter"], "gather_ms": res["gather"], "scatter_bytes": 4 * moved, "gather_bytes": moved,
           "scatter_gbs": 4 * moved / (res["scatter"] * 1e-3) / 1e9, "gather_gbs": moved / (res["gather"] * 1e-3) / 1e9,
           "scattered_shards_equal_resident": ok,
           "how": "dist.scatter_inputs (4 arrays, NCCL scatter from rank 0) / dist.gather_x (NCCL gather to rank 0), "
                  "padding and unpacking included, CUDA events, max over ranks; after the timed solve"}
    if rank == 0:
        import oracle
        xs = xfull.cpu().numpy()
        errs = []
        for r in range(world):
            rq0, rmr = tdist.shard_range(m, world, r)
            for qq in sorted({rq0, rq0 + rmr - 1}):
                sa = trigen.generate(n, 1, dt, 0, args.family, seed=seed, q0=qq)
                xo = oracle.solve_batch(n, 1, *sa)
                xg = xs.reshape(m, n)[qq] if layout == 0 else xs.reshape(n, m)[:, qq]
                errs.append(float(np.max(np.abs(xg.astype(np.float64) - xo) / np.abs(xo))))
        out["gathered_parity"] = {"systems": len(errs), "max_rel_err": max(errs)}
    del full
    torch.cuda.empty_cache()
    return out


if __name__ == "__main__":
    main()
