"""STREAM vs the other variants on fp64 contiguous batches (planner calibration
for TRI_VARIANT_STREAM): for each (n, m) time the STREAM
kernel, the k = 0 TMA p-Thomas (SPLIT k = 0) and the FUSED kernel with CUDA-graph
replays; print one JSON line per shape.

usage: python scripts/sweep_stream.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402
from scripts.sweep_k import time_plan  # noqa: E402

MAX_ELEMS = 1 << 28
SHAPES = [(n, m) for n in (1928, 2048, 4096, 8192, 16384, 65536, 245760)
          for m in (37, 74, 148, 296, 592, 1184, 2368, 4736, 16384) if n * m <= MAX_ELEMS]


def main():
    torch.cuda.set_device(0)
    g = torch.Generator(device="cuda").manual_seed(7)
    for (n, m) in SHAPES:
        N = n * m
        a = torch.rand(N, dtype=torch.float64, device="cuda", generator=g) - 0.5
        c = torch.rand(N, dtype=torch.float64, device="cuda", generator=g) - 0.5
        b = a.abs() + c.abs() + 1.0
        d = torch.rand(N, dtype=torch.float64, device="cuda", generator=g)
        x = torch.empty_like(d)
        reps = max(3, min(100, int(4e9 / (40 * N))))
        res = {"n": n, "m": m}
        for name, v, k in (("stream", tri.VARIANT_STREAM, None), ("k0", tri.VARIANT_SPLIT, 0),
                           ("fused", tri.VARIANT_FUSED, None), ("auto", None, None)):
            try:
                plan = tri.Plan(n, m, tri.F64, 0)
                if v is not None:
                    plan.variant = v
                if k is not None:
                    plan.k = k
                res[name] = round(time_plan(plan, a, b, c, d, x, reps), 2)
                if name == "auto":
                    res["auto_variant"] = plan.variant
                    res["auto_k"] = plan.k
                del plan
            except tri.TriError:
                res[name] = None
        res["munk_s_stream"] = round(N / res["stream"], 1) if res.get("stream") else None
        print(json.dumps(res), flush=True)
        del a, b, c, d, x
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
