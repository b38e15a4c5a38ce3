"""Per-role cycle breakdown of the STREAM kernel (tri_debug_set_profile; env
TRI_FUSED_DBG_MODE=1 skips the PCR math).  usage: python scripts/prof_stream.py N M"""
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
plan.variant = tri.VARIANT_STREAM
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
nwin = m * ((n + 239) // 240) / ncta
names = ["total (8 warps)", "wait input", "wait fwd state", "wait bwd x", "wait slot stored", "ph replays+store", "ph wait+load+norm", "ph PCR", "ph bwd load", "ph transpose", "ph pass1+scans", "ph serial steps"]
print(f"time {ms:.3f} ms, {ms * 1.965e6:.0f} cycles @1.965GHz, {nwin:.0f} windows per CTA; per CTA (per window):")
for i, nm in enumerate(names):
    per = v[i] / ncta / 12
    print(f"  {nm:24s} {per:14.0f}  ({per / nwin:8.1f}/window per warp)")
