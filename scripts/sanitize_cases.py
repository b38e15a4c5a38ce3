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
             (128, 40, "f32", 0, V.VARIANT_SCAN, None),      # short one-window systems (k_scan1)
             (1002, 3, "f64", 0, V.VARIANT_SCAN, None),      # ragged n, 16-byte pitch: tail rows from global
             (5003, 1, "f32", 0, V.VARIANT_SCAN, None)],     # ragged n, one system
    "scan_il": [(1024, 16, "f64", 1, V.VARIANT_SCAN, "grid0"),  # interleaved, S = 8: two 8-system groups
                (520, 24, "f32", 1, V.VARIANT_SCAN, "grid0")],  # ragged last window (chained kernel)
    # k_scan_grid: clusters of Q CTAs exchanging aggregates through DSMEM; ragged
    # blocks (m % 32), rows past n, 1 / 3 / 4 stages per warp, Q = 1 .. 8
    "scan_grid": [(1024, 40, "f64", 1, V.VARIANT_SCAN, None), (700, 36, "f32", 1, V.VARIANT_SCAN, None),
                  (60, 12, "f64", 1, V.VARIANT_SCAN, None), (2000, 32, "f64", 1, V.VARIANT_SCAN, None)],
    # k_scan_w512: 512-row fp64 windows (contiguous); several windows, ragged n,
    # one system per CTA (back-substitution lag 0) and more systems than SMs (lag 8)
    "scan_w512": [(2048, 3, "f64", 0, V.VARIANT_SCAN, "w512"), (1000, 5, "f64", 0, V.VARIANT_SCAN, "w512"),
                  (1024, 1, "f64", 0, V.VARIANT_SCAN, "w512"), (1536, 200, "f64", 0, V.VARIANT_SCAN, "w512")],
    "scan_r16": [(256, 40, "f32", 0, V.VARIANT_SCAN, None), (224, 33, "f32", 0, V.VARIANT_SCAN, None)],
    "scan_mc": [(1 << 16, 1, "f64", 0, V.VARIANT_SCAN_MC, None),
                (40960, 2, "f32", 0, V.VARIANT_SCAN_MC, None),
                (65537, 1, "f64", 0, V.VARIANT_SCAN_MC, None)],  # ragged n
    "scan_mc_lb": [(1 << 16, 1, "f64", 0, V.VARIANT_SCAN_MC, "lb32"), (40960, 2, "f32", 0, V.VARIANT_SCAN_MC, "lb16")],
    "stream": [(4096, 3, "f64", 0, V.VARIANT_STREAM, None)],
    "fused": [(2048, 3, "f64", 0, V.VARIANT_FUSED, None), (2000, 2, "f32", 0, V.VARIANT_FUSED, None)],
    "warp": [(512, 16, "f64", 0, V.VARIANT_WARP, None), (256, 16, "f32", 1, V.VARIANT_WARP, None)],
    "onchip": [(1000, 3, "f64", 0, V.VARIANT_ONCHIP, None)],
    # register-tile passes: rows kernel (contiguous, ragged, several systems), chain
    # passes by TMA and by cp.async (interleaved odd pitch), RAW first pass
    "split": [(4096, 2, "f64", 0, V.VARIANT_SPLIT, 3), (1 << 14, 1, "f64", 0, V.VARIANT_SPLIT, 12),
              (5003, 3, "f64", 0, V.VARIANT_SPLIT, 9), (3001, 4, "f32", 0, V.VARIANT_SPLIT, 7),
              (1000, 37, "f64", 1, V.VARIANT_SPLIT, 7), (1024, 40, "f32", 1, V.VARIANT_SPLIT, 5),
              (2048, 64, "f64", 0, V.VARIANT_SPLIT, 0), (1000, 64, "f32", 1, V.VARIANT_SPLIT, 0)],
    # the paper's shared-memory sliding window (TRI_OPT_TMA off)
    "split_sw": [(4096, 2, "f64", 0, V.VARIANT_SPLIT, "tma0:3"), (1 << 14, 1, "f64", 0, V.VARIANT_SPLIT, "tma0:12"),
                 (1000, 37, "f64", 1, V.VARIANT_SPLIT, "tma0:7")],
}


def main():
    import torch
    fams = sys.argv[1:] or list(CASES)
    torch.cuda.set_device(0)
    worst = 0.0
    for f in fams:
        for (n, m, dt, layout, v, k) in CASES.get(f, []):
            arrs = trigen.generate(n, m, dt, layout, "dd")
            plan = tri.Plan(n, m, tri.F64 if dt == "f64" else tri.F32, layout)
            plan.variant = v
            if isinstance(k, str) and k.startswith("tma0:"):  # TRI_OPT_TMA off, then k
                plan.set_option(tri.OPT_TMA, 0)
                plan.k = int(k[5:])
            elif k == "grid0":  # interleaved SCAN through the chained kernel
                plan.set_option(tri.OPT_SCAN_GRID, 0)
            elif k == "w512":  # fp64 contiguous SCAN through k_scan_w512
                plan.set_option(tri.OPT_SCAN_W512, 1)
            elif isinstance(k, str):  # "lbW": SCAN_MC look-back with W-window chunks
                plan.set_option(tri.OPT_SCAN_MC_LOOKBACK, int(k[2:]))
            elif k is not None:
                plan.k = k
            a, b, c, d = (torch.from_numpy(t).cuda() for t in arrs)
            # x pre-filled with NaN: the element-wise parity check below then proves
            # every element was written (initcheck does not see the TMA tensor stores
            # of k_pthomas_il_tma's x path, so an uninitialised x would be flagged there)
            x = torch.full_like(b, float("nan"))
            plan.solve(a, b, c, d, out=x)
            torch.cuda.synchronize()
            xo = oracle.solve_batch(n, m, *arrs, layout=layout)
            xh = x.cpu().numpy().astype(np.float64)
            assert np.all(np.isfinite(xh)), "unwritten x elements"
            err = float(np.max(np.abs(xh - xo) / np.abs(xo)))
            tol = 1e-10 if dt == "f64" else 1e-4
            worst = max(worst, err / tol)
            print(f"{f}: n={n} m={m} {dt} layout={layout} err={err:.2e} [{plan.describe()}]", flush=True)
            assert err <= tol
    if "strided" in fams:
        # pitched views of a [5][24][72] array: x-lines (TMA path) and an odd-pitch packed case
        for (n, ms, nb, es, ss, bs, off) in [(64, 20, 4, 1, 72, 24 * 72, 72 + 8), (20, 60, 4, 72, 1, 24 * 72, 1)]:
            m = ms * nb
            arrs = trigen.generate(n, m, "f64", 0, "dd")
            q = np.arange(m)
            flat = (off + (q % ms)[:, None] * ss + (q // ms)[:, None] * bs + np.arange(n)[None, :] * es).reshape(-1)
            par = []
            for t in arrs:
                P = np.zeros(5 * 24 * 72, dtype=np.float64)
                P[flat] = t
                par.append(torch.from_numpy(P).cuda())
            xd = torch.zeros_like(par[0])
            plan = tri.Plan.strided(n, ms, nb, es, ss, bs, tri.F64)
            plan.solve(*[t[off:] for t in par], out=xd[off:])
            torch.cuda.synchronize()
            xo = oracle.solve_batch(n, m, *arrs)
            err = float(np.max(np.abs(xd.cpu().numpy()[flat] - xo) / np.abs(xo)))
            print(f"strided: n={n} ms={ms} nb={nb} err={err:.2e} [{plan.describe()}]", flush=True)
            assert err <= 1e-10
    print(f"sanitize cases ok (worst err / tol = {worst:.2e})")


if __name__ == "__main__":
    main()
