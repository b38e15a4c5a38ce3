"""One fused solve for ncu (env TRI_FUSED_DBG_MODE honoured via tri_debug_set_profile)."""
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
cnt = torch.zeros(8, dtype=torch.int64, device="cuda")
tri.lib().tri_debug_set_profile(cnt.data_ptr())
plan.solve(a, b, c, d, out=x)
plan.solve(a, b, c, d, out=x)
torch.cuda.synchronize()
