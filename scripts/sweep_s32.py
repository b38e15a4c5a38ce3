"""Interleaved SCAN with 32 systems per window (one system per lane) vs the
planner's pick on many short interleaved systems; back-to-back graph replays of
one solve (inputs > L2 except the smallest).  usage: python scripts/sweep_s32.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402
from scripts.sweep_grid import time_plan  # noqa: E402

DTS = sys.argv[1].split(",") if len(sys.argv) > 1 else ["f32", "f64"]
NS = [int(v) for v in sys.argv[2].split(",")] if len(sys.argv) > 2 else [32, 64, 128, 256, 512, 1024]
for dt in DTS:
    TD = tri.F64 if dt == "f64" else tri.F32
    for n in NS:
        for m in (8192, 65536, 1 << 20):
            if n * m > (1 << 28):
                continue
            arrs = trigen.generate(n, m, dt, 1, "dd")
            a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
            x = torch.empty_like(b)
            auto = tri.Plan(n, m, TD, 1)
            ta = time_plan(auto, a, b, c, d, x, reps=5)
            sp = tri.Plan(n, m, TD, 1)
            sp.variant = tri.VARIANT_SCAN
            dd = dict(kv.split("=") for kv in sp.describe().split() if "=" in kv)
            ts = time_plan(sp, a, b, c, d, x, reps=5)
            spl = tri.Plan(n, m, TD, 1)
            spl.variant = tri.VARIANT_SPLIT
            tsp = time_plan(spl, a, b, c, d, x, reps=5)
            print(json.dumps({"n": n, "m": m, "dtype": dt, "auto_variant": auto.variant, "auto_k": auto.k,
                              "auto_us": round(ta, 2), "scan_us": round(ts, 2), "scan_nc": int(dd["sk_nc"]),
                              "split_us": round(tsp, 2)}), flush=True)
            del a, b, c, d, x
            torch.cuda.empty_cache()
