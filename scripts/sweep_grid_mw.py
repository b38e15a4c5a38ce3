"""k_scan_grid over several waves (TRI_OPT_SCAN_GRID 1) vs the chained interleaved
kernel (option 0) on mid-size interleaved batches; L2 flushed per replay.
usage: python scripts/sweep_grid_mw.py [f64|f32]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402
from scripts.sweep_grid import time_plan  # noqa: E402

DT = sys.argv[1] if len(sys.argv) > 1 else "f64"
TD = tri.F64 if DT == "f64" else tri.F32
for n in (512, 1024, 2048):
    for m in (1024, 2048, 4096, 8192, 16384):
        arrs = trigen.generate(n, m, DT, 1, "dd")
        a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
        x = torch.empty_like(b)
        plan = tri.Plan(n, m, TD, 1)
        plan.variant = tri.VARIANT_SCAN
        plan.set_option(tri.OPT_SCAN_GRID, 1)
        dd = dict(kv.split("=") for kv in plan.describe().split() if "=" in kv)
        tg = time_plan(plan, a, b, c, d, x)
        plan.set_option(tri.OPT_SCAN_GRID, 0)
        tc = time_plan(plan, a, b, c, d, x)
        auto = tri.Plan(n, m, TD, 1)
        ta = time_plan(auto, a, b, c, d, x)
        print(json.dumps({"n": n, "m": m, "dtype": DT, "Q": int(dd["grid_Q"]), "R": int(dd["grid_R"]),
                          "grid_us": round(tg, 2), "chained_us": round(tc, 2), "auto_variant": auto.variant,
                          "auto_us": round(ta, 2)}), flush=True)
