"""Small shapes of every kernel family for compute-sanitizer (memcheck,
racecheck, synccheck, initcheck): each case solves through the C ABI and is
checked against the oracle.  Shapes are chosen to exercise the chained paths
(several windows per system, several systems per CTA, ragged tails) with a
grid of a few CTAs so the sanitizers finish in minutes.

usage: python scripts/sanitize_cases.py [family ...]   (default: all)
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402  (test infrastructure: the checker)
import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402

V = tri
CASES = {
    # family: [(n, m, dtype, layout, variant, k)]
    "scan": [(2048, 3, "f64", 0, V.VARIANT_SCAN, None),      # NC = 8 chained windows, 3 systems (3 CTAs)
             (16384, 2, "f64", 0, V.VARIANT_SCAN, None),     # NC = 64 > on-chip slots: spill path
             (1024, 5, "f32", 0, V.VARIANT_SCAN, None),
             (256, 40, "f64", 0, V.VARIANT_SCAN, None),      # one-window systems, several per warp
             (128, 40, "f32", 0, V.VARIANT_SCAN, None)],     # short one-window systems (k_scan1)
    "scan_il": [(1024, 16, "f64", 1, V.VARIANT_SCAN, None),  # interleaved, S = 8: two 8-system groups
                (520, 24, "f32", 1, V.VARIANT_SCAN, None)],  # ragged last window
    "scan_mc": [(1 << 16, 1, "f64", 0, V.VARIANT_SCAN_MC, None),
                (40960, 2, "f32", 0, V.VARIANT_SCAN_MC, None)],
    "stream": [(4096, 3, "f64", 0, V.VARIANT_STREAM, None)],
    "fused": [(2048, 3, "f64", 0, V.VARIANT_FUSED, None), (2000, 2, "f32", 0, V.VARIANT_FUSED, None)],
    "warp": [(512, 16, "f64", 0, V.VARIANT_WARP, None), (256, 16, "f32", 1, V.VARIANT_WARP, None)],
    "onchip": [(1000, 3, "f64", 0, V.VARIANT_ONCHIP, None)],
    "split": [(4096, 2, "f64", 0, V.VARIANT_SPLIT, 3), (1 << 14, 1, "f64", 0, V.VARIANT_SPLIT, 12),
              (2048, 64, "f64", 0, V.VARIANT_SPLIT, 0), (1000, 64, "f32", 1, V.VARIANT_SPLIT, 0)],
}


def main():
    import torch
    fams = sys.argv[1:] or list(CASES)
    torch.cuda.set_device(0)
    worst = 0.0
    for f in fams:
        for (n, m, dt, layout, v, k) in CASES[f]:
            arrs = trigen.generate(n, m, dt, layout, "dd")
            plan = tri.Plan(n, m, tri.F64 if dt == "f64" else tri.F32, layout)
            plan.variant = v
            if k is not None:
                plan.k = k
            a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
            x = plan.solve(a, b, c, d)
            torch.cuda.synchronize()
            xo = oracle.solve_batch(n, m, *arrs, layout=layout)
            err = float(np.max(np.abs(x.cpu().numpy().astype(np.float64) - xo) / np.abs(xo)))
            tol = 1e-10 if dt == "f64" else 1e-4
            worst = max(worst, err / tol)
            print(f"{f}: n={n} m={m} {dt} layout={layout} err={err:.2e} [{plan.describe()}]", flush=True)
            assert err <= tol
    print(f"sanitize cases ok (worst err / tol = {worst:.2e})")


if __name__ == "__main__":
    main()
