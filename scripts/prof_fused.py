"""Per-role cycle breakdown of the fused kernel (tri_debug_set_profile).
usage: python scripts/prof_fused.py N M"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402

n, m = int(sys.argv[1]), int(sys.argv[2])
arrs = trigen.generate(n, m, "f64", 0, "dd")
a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
plan = tri.Plan(n, m, tri.F64, 0)
plan.variant = tri.VARIANT_FUSED
x = torch.empty_like(b)
plan.solve(a, b, c, d, out=x)
cnt = torch.zeros(16, dtype=torch.int64, device="cuda")
tri.lib().tri_debug_set_profile(cnt.data_ptr())
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
s.record()
plan.solve(a, b, c, d, out=x)
e.record()
torch.cuda.synchronize()
tri.lib().tri_debug_set_profile(None)
ms = s.elapsed_time(e)
v = cnt.cpu().tolist()
ncta = min(m, 148)
names = ["TC wait full", "TC total", "TR wait TB", "TR store", "PCR wait empty (all warps)", "PCR total (all warps)",
         "TB total", "TB wait TR", "TR total", "TC wait sempty", "TR wait sfull", "PCR wait loads (all warps)", "TB on-chip segments", "TB spilled segments"]
print(f"time {ms:.3f} ms, {ms * 1.965e6:.0f} cycles @1.965GHz; per CTA:")
for nm, val in zip(names, v):
    print(f"  {nm:28s} {val / ncta:14.0f}")
