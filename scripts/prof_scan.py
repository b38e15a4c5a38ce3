"""Per-phase cycle breakdown of the SCAN kernel (tri_debug_set_profile; env
TRI_FUSED_DBG_MODE=1 drops the chain handover: wrong results, timing only).
usage: python scripts/prof_scan.py N M [f64|f32]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402

n, m = int(sys.argv[1]), int(sys.argv[2])
dt = sys.argv[3] if len(sys.argv) > 3 else "f64"
lay = int(sys.argv[4]) if len(sys.argv) > 4 else 0
arrs = trigen.generate(n, m, dt, lay, "dd")
a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
plan = tri.Plan(n, m, tri.F64 if dt == "f64" else tri.F32, lay)
plan.variant = tri.VARIANT_SCAN
x = torch.empty_like(b)
plan.solve(a, b, c, d, out=x)
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for prof in (False, True):
    cnt = torch.zeros(8, dtype=torch.int64, device="cuda")
    tri.lib().tri_debug_set_profile(cnt.data_ptr() if prof else None)
    plan.solve(a, b, c, d, out=x)
    torch.cuda.synchronize()
    cnt.zero_()
    s.record()
    plan.solve(a, b, c, d, out=x)
    e.record()
    torch.cuda.synchronize()
    ms = s.elapsed_time(e)
    print(f"{'profiled' if prof else 'plain'}: {ms:.3f} ms  dbg={os.environ.get('TRI_FUSED_DBG_MODE', '0')}")
tri.lib().tri_debug_set_profile(None)
v = cnt.cpu().tolist()
S = 8 if lay == 1 else 1
ncta = min(-(-m // S), 148)
nw = int(os.environ.get("SC_NW", "12"))
steps = -(-m // S) * ((n + 256 // S - 1) // (256 // S)) / ncta
names = ["total", "wait input", "wait bar.sync", "handover section", "wait slot counter", "pre-handover compute",
         "post-handover (replays, stores)"]
print(f"{ms * 1.965e6:.0f} cycles @1.965GHz, {steps:.0f} steps per CTA, {ms * 1.965e6 / steps:.0f} cycles/step; "
      f"per warp-step (cycles):")
for i, nm in enumerate(names):
    per = v[i] / ncta / nw / (steps / nw)
    print(f"  {nm:32s} {per:10.0f}")
