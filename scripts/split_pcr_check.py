"""debug_pcr of SPLIT at small k on a long system vs a vectorised numpy PCR (fp64)."""
import sys
import numpy as np
import torch
sys.path.insert(0, __file__.rsplit("/scripts/", 1)[0])
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402


def pcr_np(a, b, c, d, k):
    n = len(a)
    A, C, D = a / b, c / b, d / b
    A[0] = 0.0
    C[-1] = 0.0
    for j in range(k):
        s = 1 << j
        Am = np.concatenate([np.zeros(s), A[:-s]]); Cm = np.concatenate([np.zeros(s), C[:-s]]); Dm = np.concatenate([np.zeros(s), D[:-s]])
        Ap = np.concatenate([A[s:], np.zeros(s)]); Cp = np.concatenate([C[s:], np.zeros(s)]); Dp = np.concatenate([D[s:], np.zeros(s)])
        bp = 1.0 - A * Cm - C * Ap
        A, C, D = -A * Am / bp, -C * Cp / bp, (D - A * Dm - C * Dp) / bp
    return A, C, D


n = int(sys.argv[1]); m = 1
g = np.random.default_rng(0)
a, c = g.random(n) - 0.5, g.random(n) - 0.5
b, d = 2.0 + g.random(n), g.random(n)
dev = [torch.from_numpy(t).cuda() for t in (a, b, c, d)]
for k in [int(x) for x in sys.argv[2:]]:
    p = tri.Plan(n, m, tri.F64, 0)
    p.variant = tri.VARIANT_SPLIT
    p.k = k
    got = [t.cpu().numpy() for t in p.debug_pcr(*dev)]
    ref = pcr_np(a.copy(), b, c.copy(), d, k)
    errs = [float(np.max(np.abs(x - y))) for x, y in zip(got, ref)]
    bad = [int(np.argmax(np.abs(x - y))) for x, y in zip(got, ref)]
    print("k", k, "err", errs, "worst rows", bad, p.describe()[:80], flush=True)
