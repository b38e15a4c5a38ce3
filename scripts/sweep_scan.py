"""Planner calibration for the SCAN variant: over a grid of
contiguous shapes like the paper's (Figs 12-13), time the planner's choice and
every competing whole-solve variant (SCAN, SCAN_MC, STREAM, SPLIT (k = 0 from
148 systems, else its planned k), FUSED, WARP, ONCHIP at its planned k) with CUDA-graph replays; JSON lines to stdout.
usage: python scripts/sweep_scan.py [f64|f32]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402


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


DT = sys.argv[1] if len(sys.argv) > 1 else "f64"
LAYOUT = int(sys.argv[2]) if len(sys.argv) > 2 else 0
TD = tri.F64 if DT == "f64" else tri.F32
MAXE = (1 << 27) if DT == "f64" else (1 << 28)
SHAPES = []
if LAYOUT == 0:
    for n in (256, 512, 1024, 2048, 4096, 8192, 16384, 65536, 1 << 20):
        for m in (1, 16, 148, 592, 2368, 9472, 37888, 151552, 1 << 20):
            if n * m <= MAXE and n * m >= 4096:
                SHAPES.append((n, m))
else:  # interleaved: m a multiple of 8
    for n in (64, 256, 1024, 2048, 4096, 8192, 16384):
        for m in (64, 296, 1024, 2368, 4096, 9472, 16384, 37888, 151552, 1 << 20):
            if n * m <= MAXE and n * m >= 4096:
                SHAPES.append((n, m))
VARS = [tri.VARIANT_SCAN, tri.VARIANT_SCAN_MC, tri.VARIANT_STREAM, tri.VARIANT_SPLIT, tri.VARIANT_FUSED, tri.VARIANT_WARP, tri.VARIANT_ONCHIP]
for n, m in SHAPES:
    arrs = trigen.generate(n, m, DT, LAYOUT, "dd")
    a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
    x = torch.empty_like(b)
    reps = max(3, min(200, int(4e9 / max(1, n * m * b.element_size() * 5))))
    plan = tri.Plan(n, m, TD, LAYOUT)
    rec = {"n": n, "m": m, "dtype": DT, "layout": LAYOUT, "auto": {"variant": plan.variant, "k": plan.k, "us": time_plan(plan, a, b, c, d, x, reps)}}
    allv = []
    for v in VARS:
        p = tri.Plan(n, m, TD, LAYOUT)
        try:
            p.variant = v
            if v == tri.VARIANT_SPLIT and m >= 148:
                p.k = 0
        except tri.TriError:
            continue
        allv.append({"variant": v, "k": p.k, "us": time_plan(p, a, b, c, d, x, reps)})
        del p
    rec["all"] = allv
    best = min(allv, key=lambda r: r["us"])
    rec["best"] = best
    rec["auto_over_best"] = rec["auto"]["us"] / best["us"]
    print(json.dumps(rec), flush=True)
    del a, b, c, d, x, plan
    torch.cuda.empty_cache()
