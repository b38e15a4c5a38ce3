"""Transition-point sweep: for shapes like the
paper's Figs 12-13 (fixed n with m swept, fixed m with n swept), time every
feasible (variant, k) with CUDA-graph replays and record the best against the
planner's automatic choice.  Writes JSON lines to stdout.

usage: python scripts/sweep_k.py [f64|f32] [--quick]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402

DT = sys.argv[1] if len(sys.argv) > 1 and not sys.argv[1].startswith("-") else "f64"
QUICK = "--quick" in sys.argv
TD = tri.F64 if DT == "f64" else tri.F32
MAX_ELEMS = (1 << 26) if DT == "f64" else (1 << 27)   # keep every case well inside HBM and quick

SHAPES = []
for n in (512, 2048, 16384):                      # Fig 12: fixed N, M swept
    for m in (1, 16, 256, 2048, 16384):
        if n * m <= MAX_ELEMS:
            SHAPES.append((n, m))
for m in (1, 16, 256, 2048):                      # Fig 13: fixed M, N swept
    for n in (1024, 8192, 65536, 1 << 20, 1 << 22):
        if n * m <= MAX_ELEMS and (n, m) not in SHAPES:
            SHAPES.append((n, m))
if QUICK:
    SHAPES = SHAPES[::3]


def time_plan(plan, a, b, c, d, x, reps):
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        plan.solve(a, b, c, d, out=x, stream=s)
    torch.cuda.synchronize()
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        g.replay()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3  # us


def candidates(n, m):
    out = []
    kmax = n.bit_length() - 1
    if 32 <= n <= 1024:
        out.append((tri.VARIANT_WARP, None))
    if n <= (3072 if DT == "f64" else 6144):
        for k in range(0, min(kmax, 10) + 1):
            out.append((tri.VARIANT_ONCHIP, k))
    for k in range(0, min(kmax, 15) + 1):
        out.append((tri.VARIANT_SPLIT, k))
    if n >= 512:
        out.append((tri.VARIANT_FUSED, None))
    return out


for n, m in SHAPES:
    arrs = trigen.generate(n, m, DT, 0, "dd")
    a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
    x = torch.empty_like(b)
    reps = max(3, min(100, int(4e8 // max(1, n * m * 8 * 5))))
    auto = tri.Plan(n, m, TD, 0)
    t_auto = time_plan(auto, a, b, c, d, x, reps)
    rec = {"n": n, "m": m, "dtype": DT, "auto": {"variant": auto.variant, "k": auto.k, "us": t_auto}, "all": []}
    best = None
    for v, k in candidates(n, m):
        try:
            p = tri.Plan(n, m, TD, 0)
            p.variant = v
            if k is not None:
                p.k = k
            t = time_plan(p, a, b, c, d, x, reps)
        except Exception as exc:  # infeasible combination (smem, scratch)
            rec["all"].append({"variant": v, "k": k, "error": str(exc)[:80]})
            continue
        rec["all"].append({"variant": v, "k": p.k, "us": t})
        if best is None or t < best["us"]:
            best = {"variant": v, "k": p.k, "us": t}
    rec["best"] = best
    rec["auto_over_best"] = t_auto / best["us"] if best else None
    print(json.dumps(rec), flush=True)
    del a, b, c, d, x
    torch.cuda.empty_cache()
