"""Run one configuration's solve a few times (for ncu / compute-sanitizer).
usage: python scripts/prof_one.py N M [f64|f32] [layout] [variant] [k] [iters]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402

n, m = int(sys.argv[1]), int(sys.argv[2])
dt = sys.argv[3] if len(sys.argv) > 3 else "f64"
layout = int(sys.argv[4]) if len(sys.argv) > 4 else 0
variant = int(sys.argv[5]) if len(sys.argv) > 5 else 0
k = int(sys.argv[6]) if len(sys.argv) > 6 and sys.argv[6] != "-" else None
iters = int(sys.argv[7]) if len(sys.argv) > 7 else 3
arrs = trigen.generate(n, m, dt, layout, "dd")
a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
plan = tri.Plan(n, m, tri.F64 if dt == "f64" else tri.F32, layout)
if variant:
    plan.variant = variant
if k is not None:
    plan.k = k
print(plan.describe(), flush=True)
x = torch.empty_like(b)
for _ in range(iters):
    plan.solve(a, b, c, d, out=x)
torch.cuda.synchronize()
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
s.record()
plan.solve(a, b, c, d, out=x)
e.record()
torch.cuda.synchronize()
ms = s.elapsed_time(e)
print(f"time {ms:.3f} ms  {n * m / ms / 1e3:.1f} Munk/s  {5 * n * m * b.element_size() / ms / 1e6:.1f} GB/s(5 arrays)")
if os.environ.get("PROF_GRAPH", "1") == "1":
    # device-only time: the solve captured in a CUDA graph, replayed back to back
    stream = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=stream):
        plan.solve(a, b, c, d, out=x, stream=stream)
    reps = max(3, min(200, int(2e9 / max(1, n * m * b.element_size() * 5))))
    g.replay()
    torch.cuda.synchronize()
    s.record()
    for _ in range(reps):
        g.replay()
    e.record()
    torch.cuda.synchronize()
    ms = s.elapsed_time(e) / reps
    print(f"graph {ms * 1e3:.1f} us  {n * m / ms / 1e3:.1f} Munk/s  "
          f"{5 * n * m * b.element_size() / ms / 1e6:.1f} GB/s(5 arrays)  reps={reps}")
