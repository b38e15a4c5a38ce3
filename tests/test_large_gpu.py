"""Arrays past 2^31 elements (n m <= 2^40, 64-bit element offsets
wherever n m s exceeds 2^31 bytes): one solve per kernel family with
n m = 2^31 + a bit, fp32 (8.6 GB per array), inputs generated on the device.
Batched shapes are checked against the oracle on sampled whole systems; single
systems of 2^31 rows through the relative residual computed on the device in
fp64 (a property that holds at any size)."""
import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu
tri = pytest.importorskip("paper_conf_icpp_kimwch11_b200")


def _inputs(N, seed):
    import torch
    g = torch.Generator(device="cuda").manual_seed(seed)
    a = torch.rand(N, generator=g, device="cuda", dtype=torch.float32) - 0.5
    c = torch.rand(N, generator=g, device="cuda", dtype=torch.float32) - 0.5
    b = torch.rand(N, generator=g, device="cuda", dtype=torch.float32) + 2.0
    d = torch.rand(N, generator=g, device="cuda", dtype=torch.float32) - 0.5
    return a, b, c, d


def _residual_one_system(a, b, c, d, x):
    """max |a_i x_{i-1} + b_i x_i + c_i x_{i+1} - d_i| / max |d| over one system
    (a_0 and c_{n-1} ignored), in fp64 chunks on the device."""
    import torch
    n = x.numel()
    step = 1 << 27
    rmax, dmax = 0.0, float(d.abs().max())
    for s0 in range(0, n, step):
        s1 = min(n, s0 + step)
        lo, hi = max(0, s0 - 1), min(n, s1 + 1)
        xx = x[lo:hi].double()
        xi = xx[s0 - lo:s0 - lo + (s1 - s0)]
        xm = torch.zeros_like(xi)
        xp = torch.zeros_like(xi)
        if s0 > 0:
            xm[:] = xx[s0 - lo - 1:s0 - lo - 1 + (s1 - s0)]
        else:
            xm[1:] = xi[:-1]
        if s1 < n:
            xp[:] = xx[s0 - lo + 1:s0 - lo + 1 + (s1 - s0)]
        else:
            xp[:-1] = xi[1:]
        r = a[s0:s1].double() * xm + b[s0:s1].double() * xi + c[s0:s1].double() * xp - d[s0:s1].double()
        rmax = max(rmax, float(r.abs().max()))
    return rmax / dmax


@pytest.mark.parametrize("layout,variant", [(0, None), (1, None), (1, "SCAN")])
def test_batched_past_2_31(cuda_ok, layout, variant):
    import torch
    n, m = 65536, 32776  # n m = 2^31 + 2^19
    N = n * m
    a, b, c, d = _inputs(N, 11 + layout)
    plan = tri.Plan(n, m, tri.F32, layout)
    if variant:
        plan.variant = getattr(tri, "VARIANT_" + variant)
    x = plan.solve(a, b, c, d)
    torch.cuda.synchronize()
    for q in [0, 1, 12345, m - 1]:
        if layout == 0:
            sl = [t[q * n:(q + 1) * n].cpu().numpy() for t in (a, b, c, d, x)]
        else:
            sl = [t.view(n, m)[:, q].contiguous().cpu().numpy() for t in (a, b, c, d, x)]
        xo = oracle.solve_batch(n, 1, *sl[:4])
        # normwise (d is centred on 0 here, so x crosses zero: elementwise relative
        # error is not the fp32 gate's quantity for these inputs)
        err = float(np.max(np.abs(sl[4].astype(np.float64) - xo)) / np.max(np.abs(xo)))
        assert err <= 1e-5, (q, err, plan.describe())
    del a, b, c, d, x, plan
    torch.cuda.empty_cache()


@pytest.mark.parametrize("n,variant,k", [((1 << 31) + (1 << 20) + 3, "SCAN_MC", None),
                                         ((1 << 31) + 77, "SPLIT", 14)])
def test_one_system_past_2_31(cuda_ok, n, variant, k):
    import torch
    a, b, c, d = _inputs(n, 21)
    plan = tri.Plan(n, 1, tri.F32, 0)
    plan.variant = getattr(tri, "VARIANT_" + variant)
    if k is not None:
        plan.k = k
    x = plan.solve(a, b, c, d)
    torch.cuda.synchronize()
    assert bool(torch.isfinite(x).all())
    r = _residual_one_system(a, b, c, d, x)
    assert r <= 1e-5, (r, plan.describe())
    del a, b, c, d, x, plan
    torch.cuda.empty_cache()
