"""Phase timeline of k_scan_grid (tri_debug_set_profile: [CTAs][8] %globaltimer
stamps at the kernel's phase barriers).  usage: python scripts/prof_grid.py N M [f64|f32]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402

n, m = int(sys.argv[1]), int(sys.argv[2])
dt = sys.argv[3] if len(sys.argv) > 3 else "f64"
arrs = trigen.generate(n, m, dt, 1, "dd")
a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
plan = tri.Plan(n, m, tri.F64 if dt == "f64" else tri.F32, 1)
print(plan.describe())
x = torch.empty_like(b)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
cnt = torch.zeros(148 * 16 * 16, dtype=torch.int64, device="cuda")
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
if os.environ.get("TRI_FUSED_DBG_MODE") in ("3", "4"):  # launch cost alone (graph replay, L2 flushed)
    tri.lib().tri_debug_set_profile(None)
    g = torch.cuda.CUDAGraph()
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        plan.solve(a, b, c, d, out=x)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=st):
            plan.solve(a, b, c, d, out=x)
    ts, tn = [], []
    for _ in range(20):
        g.replay()
        s.record()
        g.replay()
        e.record()
        torch.cuda.synchronize()
        tn.append(s.elapsed_time(e) * 1e3)
    print(f"no flush: median {sorted(tn)[10]:.2f} us")
    for _ in range(20):
        torch.cuda.synchronize()
        flush.zero_()  # the GPU is busy with the flush while the host enqueues the replay (bench.py)
        s.record()
        g.replay()
        e.record()
        torch.cuda.synchronize()
        ts.append(s.elapsed_time(e) * 1e3)
    print(f"dbg {os.environ['TRI_FUSED_DBG_MODE']} (prologue only), flushed: median {sorted(ts)[10]:.2f} us, min {min(ts):.2f} us")
    sys.exit(0)
for prof in (False, True, True):
    tri.lib().tri_debug_set_profile(cnt.data_ptr() if prof else None)
    plan.solve(a, b, c, d, out=x)
    flush.zero_()
    torch.cuda.synchronize()
    s.record()
    plan.solve(a, b, c, d, out=x)
    e.record()
    torch.cuda.synchronize()
    print(f"{'profiled' if prof else 'plain'}: {s.elapsed_time(e) * 1e3:.1f} us (L2 flushed)")
tri.lib().tri_debug_set_profile(None)
Q = int(dict(kv.split("=") for kv in plan.describe().split() if "=" in kv)["grid_Q"])
v = cnt.cpu().numpy().reshape(148, 16, 16).astype(np.float64)
live = v[:, 0, 0] > 0
v = v[live]
t0 = v[:, :, 0][v[:, :, 0] > 0].min()
v = (v - t0) / 1e3
names = {0: "start", 6: "A loop done", 1: "A barrier", 15: "scan done", 13: "cluster bar",
         14: "folded", 2: "state in", 8: "C0", 9: "C1", 10: "C2", 11: "C3",
         7: "replay loop", 3: "replay barrier", 4: "x after", 5: "end"}
print(f"{len(v)} CTAs, Q = {Q}; us after the first start: median over CTAs of (min / median / max over warps)")
for q in range(Q):
    row = []
    for k in (0, 6, 1, 15, 13, 14, 2, 8, 9, 10, 11, 7, 3, 4, 5):
        w = v[q::Q, :, k]
        row.append(f"  {names[k]:15s} {np.median(w.min(1)):6.2f} {np.median(np.median(w, 1)):6.2f} {np.median(w.max(1)):6.2f}")
    print(f"q={q}:\n" + "\n".join(row))
