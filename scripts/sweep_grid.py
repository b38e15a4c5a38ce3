"""Interleaved SCAN: k_scan_grid (TRI_OPT_SCAN_GRID auto) vs the chained 8-system
kernel (option 0) on the shapes where the grid kernel fits; graph replays timed
one by one after an L2 flush (bench.py's method).  JSON lines to stdout.
usage: python scripts/sweep_grid.py [f64|f32]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402

DT = sys.argv[1] if len(sys.argv) > 1 else "f64"
TD = tri.F64 if DT == "f64" else tri.F32
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")


def time_plan(plan, a, b, c, d, x, reps=15):
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    g = torch.cuda.CUDAGraph()
    plan.solve(a, b, c, d, out=x)
    torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=s):
        plan.solve(a, b, c, d, out=x, stream=s)
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        flush.add_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    return sorted(ts)[len(ts) // 2]


def main():
    for n in (64, 128, 256, 512, 1024, 2048):
      for m in (64, 128, 256, 512, 1024, 2048, 4096):
          plan = tri.Plan(n, m, TD, 1)
          plan.variant = tri.VARIANT_SCAN
          d_ = dict(kv.split("=") for kv in plan.describe().split() if "=" in kv)
          if int(d_["grid_Q"]) == 0:
              continue
          arrs = trigen.generate(n, m, DT, 1, "dd")
          a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
          x = torch.empty_like(b)
          tg = time_plan(plan, a, b, c, d, x)
          plan.set_option(tri.OPT_SCAN_GRID, 0)
          tc = time_plan(plan, a, b, c, d, x)
          auto = tri.Plan(n, m, TD, 1)
          ta = time_plan(auto, a, b, c, d, x)
          print(json.dumps({"n": n, "m": m, "dtype": DT, "Q": int(d_["grid_Q"]), "R": int(d_["grid_R"]), "grid_us": round(tg, 2),
                            "chained_us": round(tc, 2), "auto_variant": auto.variant, "auto_us": round(ta, 2)}), flush=True)


if __name__ == "__main__":
    main()
