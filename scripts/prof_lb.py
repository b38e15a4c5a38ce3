"""Per-chunk %globaltimer stamps of the SCAN_MC look-back kernel (diagnostics:
tri_debug_set_profile).  usage: python scripts/prof_lb.py N [M] [dtype]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402

n = int(sys.argv[1]); m = int(sys.argv[2]) if len(sys.argv) > 2 else 1
dt = sys.argv[3] if len(sys.argv) > 3 else "f64"
arrs = trigen.generate(n, m, dt, 0, "dd")
a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
plan = tri.Plan(n, m, tri.F64 if dt == "f64" else tri.F32, 0)
plan.variant = tri.VARIANT_SCAN_MC
print(plan.describe())
x = plan.solve(a, b, c, d)
nch = m * ((n // 256 + 31) // 32)
prof = torch.zeros(nch * 8 + 64, dtype=torch.int64, device="cuda")
tri.lib().tri_debug_set_profile(prof.data_ptr())
for _ in range(3):
    prof.zero_()
    plan.solve(a, b, c, d, out=x)
    torch.cuda.synchronize()
tri.lib().tri_debug_set_profile(None)
P = prof[: nch * 8].view(nch, 8).cpu().numpy().astype(np.int64)
t0 = P[:, 0].min()
P[:, :7] -= t0
names = ["A start", "A maps done", "L got maps", "L state out", "B ready", "B got state", "B done"]
print("kernel span us", (P[:, 6].max()) / 1e3)
for k in range(1, 7):
    dd = (P[:, k] - P[:, k - 1]) / 1e3
    print(f"{names[k-1]:>12} -> {names[k]:<12}: median {np.median(dd):7.2f} us  p90 {np.percentile(dd, 90):7.2f}  max {dd.max():7.2f}")
print("per-chunk total (A start -> B done) median us", np.median((P[:, 6] - P[:, 0]) / 1e3))
for cta in (0, 1, 147):
    rows = P[P[:, 7] == cta]
    rows = rows[np.argsort(rows[:, 0])]
    print("cta", cta, "chunks", len(rows))
    for r in rows[:16]:
        print("   ", " ".join(f"{v/1e3:8.1f}" for v in r[:7]))
