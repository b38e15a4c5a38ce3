"""fp32 contiguous many-system shapes: SCAN vs SPLIT k = 0 after the round-2 k_scan instruction cuts."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402
from scripts.sweep_grid import time_plan  # noqa: E402

for n, m in ((512, 151552), (512, 37888), (1024, 37888), (1024, 151552 // 2), (768, 65536), (2048, 37888)):
    arrs = trigen.generate(n, m, "f32", 0, "dd")
    a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
    x = torch.empty_like(b)
    r = {}
    for name, v in (("scan", tri.VARIANT_SCAN), ("split", tri.VARIANT_SPLIT)):
        p = tri.Plan(n, m, tri.F32, 0)
        p.variant = v
        if v == tri.VARIANT_SPLIT:
            p.k = 0
        r[name] = round(time_plan(p, a, b, c, d, x, reps=5), 1)
    print(n, m, r, "auto", tri.Plan(n, m, tri.F32, 0).variant, flush=True)
