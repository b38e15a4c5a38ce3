"""Shared helpers for the GPU parity tests: seeded inputs (trigen) -> CUDA path
(through the C ABI) vs the CPU oracle, with the north-star tolerances."""
import numpy as np

import oracle
import trigen

# BASELINE.json north_star tolerances:
TOL = {"f64": dict(rel=1e-10, resid=1e-12), "f32": dict(rel=1e-4, resid=None)}


def gen(n, m, dtype="f64", layout=0, family="dd", eps=1e-2, seed=trigen.SEED_BASE, q0=0):
    return trigen.generate(n, m, dtype, layout, family, eps=eps, seed=seed, q0=q0)


def to_dev(*arrs):
    import torch
    return [torch.from_numpy(a).cuda() for a in arrs]


def gpu_solve(n, m, arrs, dtype="f64", layout=0, k=None, variant=None, plan=None):
    import paper_conf_icpp_kimwch11_b200 as tri
    if plan is None:
        plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, layout)
    if variant is not None:
        plan.variant = variant
    if k is not None:
        plan.k = k
    a, b, c, d = to_dev(*arrs)
    x = plan.solve(a, b, c, d)
    return x.cpu().numpy(), plan


def max_rel_err(x, xo):
    return float(np.max(np.abs(x.astype(np.float64) - xo) / np.abs(xo)))


def check_parity(n, m, arrs, x, dtype, layout, x_oracle=None, resid=True):
    """Element-by-element parity with the oracle + residual gate (fp64)."""
    a, b, c, d = arrs
    xo = oracle.solve_batch(n, m, a, b, c, d, layout=layout) if x_oracle is None else x_oracle
    assert np.all(np.isfinite(x)), "non-finite output"
    err = max_rel_err(x, xo)
    tol = TOL[dtype]
    assert err <= tol["rel"], f"max rel err {err:.3e} > {tol['rel']}"
    if resid and tol["resid"] is not None:
        r = oracle.residual_batch(n, m, a, b, c, d, x, layout=layout)
        assert r[:, 0].max() <= tol["resid"], f"max rel residual {r[:, 0].max():.3e}"
    return err
