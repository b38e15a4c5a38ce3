"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, element by
element on the same seeded inputs, with the north-star tolerances
(fp64: max rel err <= 1e-10 and rel residual <= 1e-12; fp32: rel err <= 1e-4).
Shapes span several tiles, ragged tails, every variant, both layouts and every
forced transition point k."""
import numpy as np
import pytest

import oracle
from tests._helpers import check_parity, gen, gpu_solve, to_dev

pytestmark = pytest.mark.gpu

tri = pytest.importorskip("paper_conf_icpp_kimwch11_b200")
ONCHIP, SPLIT, WARP = tri.VARIANT_ONCHIP, tri.VARIANT_SPLIT, tri.VARIANT_WARP


# ------------------------------------------------------------------ auto plan
@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("layout", [0, 1])
@pytest.mark.parametrize("n,m", [(1, 1), (1, 9), (2, 3), (5, 1), (17, 33), (64, 129), (255, 3), (1000, 37),
                                 (1024, 1), (1024, 300), (3000, 3), (5003, 2), (8191, 5), (20000, 3),
                                 (65536 + 37, 1)])
def test_auto_plan_parity(cuda_ok, dtype, layout, n, m):
    arrs = gen(n, m, dtype, layout)
    x, plan = gpu_solve(n, m, arrs, dtype, layout)
    check_parity(n, m, arrs, x, dtype, layout)


@pytest.mark.parametrize("family,eps", [("weak", 1e-2), ("weak", 1e-3), ("integer", 0.0)])
@pytest.mark.parametrize("n,m", [(1024, 64), (333, 17), (40000, 2)])
def test_families_fp64(cuda_ok, family, eps, n, m):
    arrs = gen(n, m, "f64", 0, family, eps=eps)
    x, _ = gpu_solve(n, m, arrs, "f64", 0)
    check_parity(n, m, arrs, x, "f64", 0)


@pytest.mark.parametrize("family", ["dd", "weak"])
def test_families_fp32(cuda_ok, family):
    n, m = 256, 4096
    arrs = gen(n, m, "f32", 0, family, eps=1e-2)
    x, _ = gpu_solve(n, m, arrs, "f32", 0)
    check_parity(n, m, arrs, x, "f32", 0)


# ------------------------------------------------------------------ forced k
@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("layout", [0, 1])
@pytest.mark.parametrize("n,m", [(1024, 5), (777, 3), (2048, 1)])
def test_onchip_every_k(cuda_ok, dtype, layout, n, m):
    """k-independence: every forced k in [0, floor(log2 n)]."""
    arrs = gen(n, m, dtype, layout, "weak", eps=1e-2)
    xo = oracle.solve_batch(n, m, *arrs, layout=layout)
    plan = None
    for k in range(0, int(np.log2(n)) + 1):
        x, plan = gpu_solve(n, m, arrs, dtype, layout, k=k, variant=ONCHIP, plan=plan)
        check_parity(n, m, arrs, x, dtype, layout, x_oracle=xo)


def split_launches(n, m, k, layout, dtype, tma=True):
    """tri_plan_launches of a SPLIT plan (l_split.cu split_geometry): p-Thomas plus
    the tiled-PCR passes -- register tiles (5 steps on CONTIGUOUS rows, 3 on
    INTERLEAVED rows, then passes of <= 3), else the sliding window (10 steps,
    then passes of <= 5)."""
    if k == 0:
        return 1
    if tma and layout == 0:
        return 2 + -(-max(0, k - 5) // 3)
    if tma and layout == 1:
        return 2 + -(-max(0, k - 3) // 3)
    return 2 + (0 if k <= 10 else -(-(k - 10) // 5))


@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("layout", [0, 1])
@pytest.mark.parametrize("n,m", [(10007, 3), (4099, 1), (70001, 1), (10007, 4), (3001, 40), (1 << 12, 64)])
def test_split_every_k(cuda_ok, dtype, layout, n, m):
    """Every k through both tiled-PCR kernel families (register tiles by
    default, the paper's shared-memory sliding window with TRI_OPT_TMA off):
    ragged n, m = 1 .. 64, chain blocks with idle lanes (m = 3, 40)."""
    arrs = gen(n, m, dtype, layout, "weak", eps=1e-2)
    xo = oracle.solve_batch(n, m, *arrs, layout=layout)
    dev = to_dev(*arrs)
    kmax = min(int(np.log2(n)), 15)
    for tma in (1, 0):
        plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, layout)
        plan.set_option(tri.OPT_TMA, tma)
        plan.variant = SPLIT
        for k in range(0, kmax + 1):
            plan.k = k
            assert plan.launches == split_launches(n, m, k, layout, dtype, bool(tma)), (k, plan.describe())
            x = plan.solve(*dev).cpu().numpy()
            check_parity(n, m, arrs, x, dtype, layout, x_oracle=xo)


@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("n,m,k", [(3001, 3, 7), (5003, 37, 8), (2001, 5, 10), (999, 1, 9)])
def test_split_chains_cp_async(cuda_ok, dtype, n, m, k):
    """INTERLEAVED rows whose pitch m s is not a 16-byte multiple (m = 1, 3, 5,
    37) go through the cp.async chain kernel instead of TMA boxes in the first
    pass (later passes: pitch m 2^k1 s)."""
    arrs = gen(n, m, dtype, 1, "weak", eps=1e-2)
    xo = oracle.solve_batch(n, m, *arrs, layout=1)
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, 1)
    plan.variant = SPLIT
    plan.k = k
    assert plan.launches == split_launches(n, m, k, 1, dtype)
    x = plan.solve(*to_dev(*arrs)).cpu().numpy()
    check_parity(n, m, arrs, x, dtype, 1, x_oracle=xo)


def test_split_on_small_systems(cuda_ok):
    """The streaming variant must also handle systems shorter than a tile."""
    for n, m in [(1, 4), (3, 7), (100, 9), (600, 2)]:
        arrs = gen(n, m, "f64", 0)
        for k in range(0, int(np.log2(n)) + 1):
            x, _ = gpu_solve(n, m, arrs, "f64", 0, k=k, variant=SPLIT)
            check_parity(n, m, arrs, x, "f64", 0)


# ------------------------------------------------------------------ PCR stage (row A2)
@pytest.mark.parametrize("variant,n,m,k,layout,tma", [
    (ONCHIP, 1024, 3, 3, 0, 1), (ONCHIP, 500, 2, 5, 0, 1), (SPLIT, 9000, 2, 4, 0, 1), (WARP, 1000, 3, 5, 0, 1),
    (WARP, 33, 2, 5, 0, 1), (WARP, 256, 4, 5, 0, 1), (SPLIT, 70001, 1, 13, 0, 1), (SPLIT, 20001, 2, 12, 0, 1),
    (SPLIT, 40000, 3, 15, 0, 1), (SPLIT, 20001, 1, 8, 0, 1), (SPLIT, 5000, 3, 1, 0, 1), (SPLIT, 9000, 2, 5, 0, 1),
    (SPLIT, 3001, 40, 7, 0, 1), (SPLIT, 3001, 4, 6, 1, 1), (SPLIT, 3001, 40, 9, 1, 1), (SPLIT, 4001, 4, 2, 1, 1),
    (SPLIT, 70001, 1, 13, 0, 0),
])
def test_pcr_stage_matches_oracle(cuda_ok, variant, n, m, k, layout, tma):
    """The reduced system after k PCR steps (Eqs 5-6) vs the oracle's plain PCR,
    normalised to unit diagonal, and satisfied by the oracle solution (both
    tiled-PCR kernel families, both layouts)."""
    arrs = gen(n, m, "f64", layout, "weak", eps=1e-2)
    plan = tri.Plan(n, m, tri.F64, layout)
    plan.set_option(tri.OPT_TMA, tma)
    plan.variant = variant
    plan.k = k
    A, C, D = (t.cpu().numpy() for t in plan.debug_pcr(*to_dev(*arrs)))
    xo = oracle.solve_batch(n, m, *arrs, layout=layout)
    s = 1 << k
    for q in range(m):
        sl = slice(q * n, (q + 1) * n) if layout == 0 else slice(q, None, m)
        ao, bo, co, do = oracle.pcr_k(*(t[sl] for t in arrs), k)
        An, Cn, Dn = ao / bo, co / bo, do / bo
        for got, ref in ((A[sl], An), (C[sl], Cn), (D[sl], Dn)):
            assert np.max(np.abs(got - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref)))
        # invariant: A_i x_{i-s} + x_i + C_i x_{i+s} - D_i = 0
        x = xo[sl]
        xm = np.concatenate([np.zeros(s), x[:-s]]) if s < n else np.zeros(n)
        xp = np.concatenate([x[s:], np.zeros(s)]) if s < n else np.zeros(n)
        r = A[sl] * xm + x + C[sl] * xp - D[sl]
        assert np.max(np.abs(r)) <= 1e-13 * np.max(np.abs(D[sl]))


# ------------------------------------------------------------------ edge cases / API
@pytest.mark.parametrize("variant,n,m", [(ONCHIP, 1024, 4), (SPLIT, 9000, 2), (SPLIT, 3000, 130), (WARP, 1000, 5),
                                         (WARP, 64, 9)])
@pytest.mark.parametrize("layout", [0, 1])
def test_ignored_entries_nan(cuda_ok, variant, n, m, layout):
    """a[q][0] and c[q][n-1] lie outside A (Eq 1, reading X1): NaN there must
    not change x (bitwise)."""
    import torch
    arrs = gen(n, m, "f64", layout)
    plan = tri.Plan(n, m, tri.F64, layout)
    plan.variant = variant
    a, b, c, d = to_dev(*arrs)
    x1 = plan.solve(a, b, c, d).clone()
    a2, c2 = a.clone(), c.clone()
    if layout == 0:
        a2.view(m, n)[:, 0] = float("nan")
        c2.view(m, n)[:, -1] = float("nan")
    else:
        a2.view(n, m)[0, :] = float("nan")
        c2.view(n, m)[-1, :] = float("nan")
    x2 = plan.solve(a2, b, c2, d)
    assert torch.equal(x1, x2)


def test_determinism_and_plan_reuse(cuda_ok):
    import torch
    for n, m in [(1024, 300), (16384, 64), (100000, 1)]:
        arrs = gen(n, m, "f64", 0)
        plan = tri.Plan(n, m, tri.F64, 0)
        a, b, c, d = to_dev(*arrs)
        x1 = plan.solve(a, b, c, d).clone()
        for _ in range(3):
            assert torch.equal(plan.solve(a, b, c, d), x1)


def test_batch_invariance(cuda_ok):
    """Identical systems give identical x (bitwise) wherever they sit."""
    import torch
    n, m = 700, 40
    a, b, c, d = gen(n, 1, "f64", 0)
    rep = [np.tile(t, m) for t in (a, b, c, d)]
    for variant in (ONCHIP, SPLIT):
        x, _ = gpu_solve(n, m, rep, "f64", 0, variant=variant)
        xs = x.reshape(m, n)
        assert np.all(xs == xs[0])


def test_power_of_two_row_scaling_bitwise(cuda_ok):
    """Scaling row i by 2^p_i leaves x unchanged bitwise; scaling d by 2^p scales
    x by 2^p bitwise (every rounding step is scale-covariant)."""
    n, m = 3000, 8
    a, b, c, d = gen(n, m, "f64", 0, "weak", eps=1e-2)
    rng = np.random.default_rng(0)
    p = 2.0 ** rng.integers(-20, 20, n * m)
    for variant, k in ((ONCHIP, 3), (SPLIT, 0), (SPLIT, 4)):
        x0, _ = gpu_solve(n, m, (a, b, c, d), "f64", 0, variant=variant, k=k)
        x1, _ = gpu_solve(n, m, (a * p, b * p, c * p, d * p), "f64", 0, variant=variant, k=k)
        assert np.array_equal(x0, x1)
        x2, _ = gpu_solve(n, m, (a, b, c, d * 1024.0), "f64", 0, variant=variant, k=k)
        assert np.array_equal(x2, x0 * 1024.0)


@pytest.mark.parametrize("variant,k,n,m,layout", [
    ("SCAN", None, 4096, 6, 0), ("SCAN", None, 1024, 64, 1), ("SCAN_MC", None, 1 << 16, 1, 0),
    ("SPLIT", 0, 3000, 40, 0), ("SPLIT", 4, 3000, 40, 0), ("SPLIT", 9, 20001, 3, 0), ("SPLIT", 6, 3000, 40, 1),
    ("STREAM", None, 4096, 6, 0), ("FUSED", None, 2048, 160, 0), ("WARP", None, 512, 160, 0),
    ("ONCHIP", 3, 1000, 3, 0)])
def test_degenerate_systems(cuda_ok, variant, k, n, m, layout):
    """Special cases with a plain answer, on every variant: a diagonal system
    (a = c = 0: x = d / b, within 2 ulp -- the path divides through reciprocals
    and scales by powers of two), d = 0 (x = 0 exactly, no NaN from 0 / 0 or
    inf * 0), and the identity (x = d bitwise)."""
    import torch
    g = torch.Generator().manual_seed(5)
    N = n * m
    b = (1.0 + torch.rand(N, generator=g, dtype=torch.float64)).cuda()
    d = (torch.rand(N, generator=g, dtype=torch.float64) - 0.5).cuda()
    zero = torch.zeros(N, dtype=torch.float64, device="cuda")
    plan = tri.Plan(n, m, tri.F64, layout)
    plan.variant = getattr(tri, "VARIANT_" + variant)
    if k is not None:
        plan.k = k
    x = plan.solve(zero, b, zero, d)
    ref = d / b
    assert float(((x - ref).abs() / ref.abs().clamp_min(1e-300)).max()) <= 4.5e-16, plan.describe()
    a = (torch.rand(N, generator=g, dtype=torch.float64) - 0.5).cuda() * 0.4
    c = (torch.rand(N, generator=g, dtype=torch.float64) - 0.5).cuda() * 0.4
    x0 = plan.solve(a, b, c, zero)
    assert bool((x0 == 0).all()), plan.describe()
    one = torch.ones(N, dtype=torch.float64, device="cuda")
    x1 = plan.solve(zero, one, zero, d)
    assert torch.equal(x1, d), plan.describe()


def test_flip(cuda_ok):
    """Reversing the rows and swapping a and c reverses x (within tolerance)."""
    n, m = 5000, 4
    a, b, c, d = gen(n, m, "f64", 0)
    rev = lambda t: t.reshape(m, n)[:, ::-1].copy().ravel()
    x0, _ = gpu_solve(n, m, (a, b, c, d), "f64", 0)
    x1, _ = gpu_solve(n, m, (rev(c), rev(b), rev(a), rev(d)), "f64", 0)
    assert np.max(np.abs(rev(x1) - x0) / np.abs(x0)) <= 1e-12


def test_api_errors(cuda_ok):
    import torch
    n, m = 1024, 4
    plan = tri.Plan(n, m, tri.F64, 0)
    a, b, c, d = to_dev(*gen(n, m, "f64", 0))
    x = torch.empty_like(b)
    L = tri.lib()
    h = plan._h
    assert L.tri_solve(h, a.data_ptr(), b.data_ptr(), c.data_ptr(), d.data_ptr(), x.data_ptr(), None) == 0
    assert L.tri_solve(h, None, b.data_ptr(), c.data_ptr(), d.data_ptr(), x.data_ptr(), None) == 1
    assert L.tri_solve(h, a.data_ptr() + 8, b.data_ptr(), c.data_ptr(), d.data_ptr(), x.data_ptr(), None) == 2
    assert L.tri_solve(h, a.data_ptr(), b.data_ptr(), c.data_ptr(), d.data_ptr(), d.data_ptr(), None) == 3
    big = torch.empty(2 * n * m, dtype=torch.float64, device="cuda")
    assert L.tri_solve(h, big.data_ptr(), b.data_ptr(), c.data_ptr(), d.data_ptr(),
                       big.data_ptr() + 8 * (n * m // 2), None) == 3  # partial overlap
    host = np.zeros(n * m)
    assert L.tri_solve(h, a.data_ptr(), b.data_ptr(), c.data_ptr(), d.data_ptr(), host.ctypes.data, None) == 4
    assert L.tri_plan_set_k(h, 11) == 1          # k > floor(log2 1024)
    assert L.tri_plan_set_k(h, -1) == 1
    assert L.tri_plan_set_variant(h, 9) == 1
    p1 = tri.Plan(1, 5, tri.F64, 0)
    with pytest.raises(tri.TriError):
        p1.k = 1                                  # n = 1: only k = 0
    with pytest.raises(tri.TriError):
        tri.Plan(0, 5)
    ps = tri.Plan(100000, 1, tri.F64, 0)
    with pytest.raises(tri.TriError):
        ps.variant = ONCHIP                       # does not fit one CTA


def test_concurrent_plans_two_streams(cuda_ok):
    import torch
    n, m = 20000, 8
    arrs = gen(n, m, "f64", 0)
    xo = oracle.solve_batch(n, m, *arrs)
    a, b, c, d = to_dev(*arrs)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    p1, p2 = tri.Plan(n, m, tri.F64, 0), tri.Plan(n, m, tri.F64, 0)
    p2.variant = SPLIT
    p2.k = 3
    torch.cuda.synchronize()
    x1, x2 = torch.empty_like(b), torch.empty_like(b)
    for _ in range(3):
        p1.solve(a, b, c, d, out=x1, stream=s1)
        p2.solve(a, b, c, d, out=x2, stream=s2)
    torch.cuda.synchronize()
    for x in (x1, x2):
        assert np.max(np.abs(x.cpu().numpy() - xo) / np.abs(xo)) <= 1e-10


@pytest.mark.parametrize("dtype,n,m,layout", [("f64", 4096, 16, 0), ("f64", 2048, 1000, 0), ("f32", 256, 5003, 0),
                                              ("f64", 1024, 1024, 1), ("f64", 16384, 33, 0)])
def test_solve_host(cuda_ok, dtype, n, m, layout):
    """tri_solve_host: one staged copy-solve-copy (small m, interleaved) and the
    pipelined chunked path (contiguous, m >= 32: 16 chunks of systems, ragged last
    chunk, two sub-plan sizes), reused twice on the same plan."""
    import torch
    arrs = gen(n, m, dtype, layout)
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, layout)
    pin = [torch.from_numpy(t).pin_memory() for t in arrs]
    out = torch.empty(n * m, dtype=pin[0].dtype).pin_memory()
    for _ in range(2):
        out.zero_()
        plan.solve_host(*pin, out)
        check_parity(n, m, arrs, out.numpy(), dtype, layout)


# ------------------------------------------------------------------ FUSED variant
FUSED = tri.VARIANT_FUSED


@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("n,m", [(512, 3), (2048, 5), (16384, 7), (4099, 2), (4100, 3), (100000, 2), (1001, 300),
                                 (16392, 150)])
def test_fused_parity(cuda_ok, dtype, n, m):
    arrs = gen(n, m, dtype, 0)
    x, plan = gpu_solve(n, m, arrs, dtype, 0, variant=FUSED)
    assert plan.k == 4
    check_parity(n, m, arrs, x, dtype, 0)


@pytest.mark.parametrize("family,eps", [("weak", 1e-2), ("weak", 1e-3), ("integer", 0.0), ("poisson", 0.0)])
def test_fused_families(cuda_ok, family, eps):
    n, m = 16384, 6
    arrs = gen(n, m, "f64", 0, family, eps=eps)
    x, _ = gpu_solve(n, m, arrs, "f64", 0, variant=FUSED)
    if family == "poisson":
        # Poisson is ill-conditioned (kappa ~ n^2/2): forward error vs oracle bounded by kappa*u
        xo = oracle.solve_batch(n, m, *arrs)
        assert np.max(np.abs(x - xo)) / np.max(np.abs(xo)) <= 2 * (n + 1) ** 2 / 2 * 2.2e-16
    else:
        check_parity(n, m, arrs, x, "f64", 0)


@pytest.mark.parametrize("n,m", [(4099, 2), (16384, 3)])
def test_fused_pcr_stage(cuda_ok, n, m):
    arrs = gen(n, m, "f64", 0, "weak", eps=1e-2)
    plan = tri.Plan(n, m, tri.F64, 0)
    plan.variant = FUSED
    A, C, D = (t.cpu().numpy() for t in plan.debug_pcr(*to_dev(*arrs)))
    for q in range(m):
        sl = slice(q * n, (q + 1) * n)
        ao, bo, co, do = oracle.pcr_k(*(t[sl] for t in arrs), plan.k)
        for got, ref in ((A[sl], ao / bo), (C[sl], co / bo), (D[sl], do / bo)):
            assert np.max(np.abs(got - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref)))


def test_fused_edges_and_scaling(cuda_ok):
    import torch
    n, m = 9000, 5
    a, b, c, d = gen(n, m, "f64", 0, "weak", eps=1e-2)
    plan = tri.Plan(n, m, tri.F64, 0)
    plan.variant = FUSED
    da, db, dc, dd = to_dev(a, b, c, d)
    x1 = plan.solve(da, db, dc, dd).clone()
    a2, c2 = da.clone(), dc.clone()
    a2.view(m, n)[:, 0] = float("nan")
    c2.view(m, n)[:, -1] = float("nan")
    assert torch.equal(plan.solve(a2, db, c2, dd), x1)
    p = 2.0 ** np.random.default_rng(1).integers(-20, 20, n * m)
    x2 = plan.solve(*to_dev(a * p, b * p, c * p, d * p))
    assert torch.equal(x2, x1)
    x3 = plan.solve(da, db, dc, dd * 4.0)
    assert torch.equal(x3, x1 * 4.0)
    plan.k = 2  # the fused kernel is built for k = 4: the plan moves to a variant that runs k = 2
    assert plan.k == 2 and plan.variant != tri.VARIANT_FUSED


# ------------------------------------------------------------------ STREAM variant
STREAM = tri.VARIANT_STREAM


@pytest.mark.parametrize("n,m", [(1928, 3), (1936, 2), (2048, 5), (16384, 7), (4104, 2), (16392, 150), (2400, 300),
                                 (6000, 149), (16384, 300), (100000, 2), (245760, 2)])
def test_stream_parity(cuda_ok, n, m):
    """Spans: NC from 9 (all slots resident) to 1024 (most slots spilled), a
    ragged last window (1928, 4104, 16392), one and several systems per CTA
    (both slot parities), m > #SMs (uneven systems per CTA)."""
    arrs = gen(n, m, "f64", 0)
    x, plan = gpu_solve(n, m, arrs, "f64", 0, variant=STREAM)
    assert plan.variant == STREAM and plan.k == 3
    check_parity(n, m, arrs, x, "f64", 0)


@pytest.mark.parametrize("family,eps", [("weak", 1e-2), ("weak", 1e-3), ("integer", 0.0), ("poisson", 0.0)])
def test_stream_families(cuda_ok, family, eps):
    n, m = 16384, 6
    arrs = gen(n, m, "f64", 0, family, eps=eps)
    x, _ = gpu_solve(n, m, arrs, "f64", 0, variant=STREAM)
    if family == "poisson":
        # Poisson is ill-conditioned (kappa ~ n^2/2): forward error vs oracle bounded by kappa*u
        xo = oracle.solve_batch(n, m, *arrs)
        assert np.max(np.abs(x - xo)) / np.max(np.abs(xo)) <= 2 * (n + 1) ** 2 / 2 * 2.2e-16
    else:
        check_parity(n, m, arrs, x, "f64", 0)


@pytest.mark.parametrize("n,m", [(1936, 2), (16384, 3)])
def test_stream_pcr_stage(cuda_ok, n, m):
    """Row A2 for the STREAM kernel: its 3-step reduced system (normalised) vs
    the oracle's plain PCR (Eqs 5-6)."""
    arrs = gen(n, m, "f64", 0, "weak", eps=1e-2)
    plan = tri.Plan(n, m, tri.F64, 0)
    plan.variant = STREAM
    A, C, D = (t.cpu().numpy() for t in plan.debug_pcr(*to_dev(*arrs)))
    for q in range(m):
        sl = slice(q * n, (q + 1) * n)
        ao, bo, co, do = oracle.pcr_k(*(t[sl] for t in arrs), plan.k)
        for got, ref in ((A[sl], ao / bo), (C[sl], co / bo), (D[sl], do / bo)):
            assert np.max(np.abs(got - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref)))


def test_stream_edges_and_scaling(cuda_ok):
    """X1 (NaN in a_0 / c_{n-1} ignored, bitwise), metamorphic row and rhs
    scaling by powers of two (bitwise), determinism across runs, and the
    variant's fixed k."""
    import torch
    n, m = 9000, 5
    a, b, c, d = gen(n, m, "f64", 0, "weak", eps=1e-2)
    plan = tri.Plan(n, m, tri.F64, 0)
    plan.variant = STREAM
    da, db, dc, dd = to_dev(a, b, c, d)
    x1 = plan.solve(da, db, dc, dd).clone()
    assert torch.equal(plan.solve(da, db, dc, dd), x1)
    a2, c2 = da.clone(), dc.clone()
    a2.view(m, n)[:, 0] = float("nan")
    c2.view(m, n)[:, -1] = float("nan")
    assert torch.equal(plan.solve(a2, db, c2, dd), x1)
    p = 2.0 ** np.random.default_rng(1).integers(-20, 20, n * m)
    x2 = plan.solve(*to_dev(a * p, b * p, c * p, d * p))
    assert torch.equal(x2, x1)
    x3 = plan.solve(da, db, dc, dd * 4.0)
    assert torch.equal(x3, x1 * 4.0)
    plan.k = 2  # the stream kernel is built for k = 3: the plan moves to a variant that runs k = 2
    assert plan.k == 2 and plan.variant != tri.VARIANT_STREAM


def test_stream_rejects_unsupported(cuda_ok):
    for (n, m, dt, layout) in [(1004, 3, tri.F64, 0), (16384, 3, tri.F32, 0), (16384, 3, tri.F64, 1), (256, 3, tri.F64, 0),
                               (1672, 3, tri.F64, 0), (245768, 2, tri.F64, 0)]:
        plan = tri.Plan(n, m, dt, layout)
        with pytest.raises(tri.TriError):
            plan.variant = STREAM


def test_stream_full_size_sampled(cuda_ok):
    """BASELINE c5 shape (m = n = 16384) in the launch configuration bench.py
    times: whole sampled systems (first/last of a CTA's sweep, both slot
    parities, the last system) vs the oracle element by element."""
    n, m = 16384, 16384
    arrs = gen(n, m, "f64", 0)
    plan = tri.Plan(n, m, tri.F64, 0)
    plan.variant = STREAM
    x = plan.solve(*to_dev(*arrs)).cpu().numpy()
    for q in (0, 1, 147, 148, 149, 8191, 16235, 16383):
        sl = slice(q * n, (q + 1) * n)
        sub = [t[sl] for t in arrs]
        check_parity(n, 1, sub, x[sl], "f64", 0)


# ------------------------------------------------------------------ SCAN variant
SCAN = tri.VARIANT_SCAN


@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("n,m", [(8, 5), (128, 3000), (192, 40), (248, 300), (256, 1000), (264, 3), (512, 7), (1936, 2), (2048, 5),
                                 (4104, 2), (16384, 7), (16392, 150), (2400, 300), (6000, 149), (100000, 2),
                                 (245760, 2), (1 << 20, 1)])
def test_scan_parity(cuda_ok, dtype, n, m):
    """Spans: one-window systems (n <= 256: no chain), NC = 2 with an 8-row last
    window, NC up to 4096 (most slots spilled), ragged last windows, one and
    several systems per CTA (both slot parities), m > #SMs."""
    arrs = gen(n, m, dtype, 0)
    x, plan = gpu_solve(n, m, arrs, dtype, 0, variant=SCAN)
    assert plan.variant == SCAN and plan.k == 0
    check_parity(n, m, arrs, x, dtype, 0)


@pytest.mark.parametrize("family,eps", [("weak", 1e-2), ("weak", 1e-3), ("integer", 0.0), ("poisson", 0.0)])
@pytest.mark.parametrize("n,m", [(16384, 6), (256, 40)])
def test_scan_families(cuda_ok, family, eps, n, m):
    arrs = gen(n, m, "f64", 0, family, eps=eps)
    x, _ = gpu_solve(n, m, arrs, "f64", 0, variant=SCAN)
    if family == "poisson":
        xo = oracle.solve_batch(n, m, *arrs)
        assert np.max(np.abs(x - xo)) / np.max(np.abs(xo)) <= 2 * (n + 1) ** 2 / 2 * 2.2e-16
    else:
        check_parity(n, m, arrs, x, "f64", 0)


@pytest.mark.parametrize("n,m", [(9000, 5), (200, 7)])
def test_scan_edges_and_scaling(cuda_ok, n, m):
    """X1 (NaN in a_0 / c_{n-1} ignored, bitwise), metamorphic row and rhs
    scaling by powers of two (bitwise: the continuant state and the segment maps
    rescale exactly), determinism across runs, and the variant's fixed k = 0."""
    import torch
    a, b, c, d = gen(n, m, "f64", 0, "weak", eps=1e-2)
    plan = tri.Plan(n, m, tri.F64, 0)
    plan.variant = SCAN
    da, db, dc, dd = to_dev(a, b, c, d)
    x1 = plan.solve(da, db, dc, dd).clone()
    assert torch.equal(plan.solve(da, db, dc, dd), x1)
    a2, c2 = da.clone(), dc.clone()
    a2.view(m, n)[:, 0] = float("nan")
    c2.view(m, n)[:, -1] = float("nan")
    assert torch.equal(plan.solve(a2, db, c2, dd), x1)
    p = 2.0 ** np.random.default_rng(1).integers(-20, 20, n * m)
    x2 = plan.solve(*to_dev(a * p, b * p, c * p, d * p))
    assert torch.equal(x2, x1)
    x3 = plan.solve(da, db, dc, dd * 4.0)
    assert torch.equal(x3, x1 * 4.0)
    with pytest.raises(tri.TriError):
        plan.debug_pcr(da, db, dc, dd)  # no PCR stage
    plan.k = 1  # the scan kernel is p-Thomas at k = 0: the plan moves to a k-capable variant
    assert plan.k == 1 and plan.variant not in (SCAN, tri.VARIANT_SCAN_MC)


def test_scan_rejects_unsupported(cuda_ok):
    for (n, m, dt, layout) in [(1001, 3, tri.F64, 0), (1002, 3, tri.F32, 0), (250, 3, tri.F64, 0),
                               (16384, 3, tri.F64, 1), (7, 3, tri.F32, 0), ((1 << 20) + 8, 1, tri.F64, 0),
                               (100, 6, tri.F32, 1)]:
        plan = tri.Plan(n, m, dt, layout)
        with pytest.raises(tri.TriError):
            # ragged n with unaligned system starts, or of one window; interleaved row
            # stride not a 16-byte multiple; > 4096 windows
            plan.variant = SCAN


@pytest.mark.parametrize("family", ["dd", "weak"])
@pytest.mark.parametrize("cfg,dtype,n,m,layout", [("c5", "f64", 16384, 16384, 0), ("c4", "f32", 256, 1 << 20, 0),
                                                  ("c5-il", "f64", 16384, 16384, 1), ("c4-il", "f32", 256, 1 << 20, 1)])
def test_full_size_every_system(cuda_ok, family, cfg, dtype, n, m, layout):
    """BASELINE c5 / c4 at full size through the auto plan -- the launch
    configuration bench.py times (SCAN on the contiguous layout) -- and the
    interleaved layout: EVERY system vs the oracle, element by
    element (the threaded oracle solves 2^28 unknowns in under a second), for
    the dd family and the weak family at eps = 1e-2 (the
    full-size fp32 gate uses dd and eps = 1e-2).  fp64 also gates the relative
    residual of every system."""
    import torch
    import trigen
    seed = trigen.SEED_BASE + int(cfg[1])
    arrs = gen(n, m, dtype, layout, family, eps=1e-2, seed=seed)
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, layout)
    x = plan.solve(*to_dev(*arrs)).cpu().numpy()
    torch.cuda.empty_cache()
    check_parity(n, m, arrs, x, dtype, layout)


@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("n,m", [(1, 8), (5, 12), (200, 64), (1024, 1024), (1000, 36), (333, 300), (4099, 148),
                                 (16384, 40), (70000, 4)])
def test_scan_interleaved_parity(cuda_ok, dtype, n, m):
    """SCAN on the INTERLEAVED layout (S adjacent systems per window, scans over
    32 / S lane segments): ragged rows and ragged last group of systems, one-row
    systems, c2's shape, NC from 1 to 1094 windows."""
    arrs = gen(n, m, dtype, 1)
    x, plan = gpu_solve(n, m, arrs, dtype, 1, variant=SCAN)
    assert plan.variant == SCAN and plan.k == 0
    check_parity(n, m, arrs, x, dtype, 1)


@pytest.mark.parametrize("family,eps", [("weak", 1e-3), ("integer", 0.0)])
def test_scan_interleaved_families(cuda_ok, family, eps):
    n, m = 5000, 64
    arrs = gen(n, m, "f64", 1, family, eps=eps)
    x, _ = gpu_solve(n, m, arrs, "f64", 1, variant=SCAN)
    check_parity(n, m, arrs, x, "f64", 1)


@pytest.mark.parametrize("dtype,emax", [("f32", 40), ("f32", 120), ("f64", 100), ("f64", 500), ("f64", 1000)])
@pytest.mark.parametrize("n,m,layout,variant", [(256, 300, 0, "SCAN"), (4096, 200, 0, "SCAN"),
                                                 (100000, 2, 0, "SCAN_MC"), (1024, 512, 1, "SCAN")])
def test_scan_row_scale_range(cuda_ok, dtype, emax, n, m, layout, variant):
    """Rows scaled by random powers of two up to 2^+-emax (exact: x unchanged;
    reading X21): the continuant of 8 raw rows would leave the dtype's range
    (fp32 beyond |b| ~ 2^16, fp64 beyond ~2^127), so fp32 rows are always
    renormalised by 2^-exponent(b) in the kernel and fp64 windows whose pivots
    leave 2^+-64 are (sc_range): any |b| in the dtype's range works."""
    a, b, c, d = gen(n, m, "f64", layout)
    p = 2.0 ** np.random.default_rng(5).integers(-emax, emax + 1, n * m)
    arrs = [(t * p).astype(np.float32 if dtype == "f32" else np.float64) for t in (a, b, c, d)]
    x, plan = gpu_solve(n, m, arrs, dtype, layout, variant=getattr(tri, "VARIANT_" + variant))
    check_parity(n, m, arrs, x, dtype, layout, resid=False)


@pytest.mark.parametrize("dtype,n,m,layout", [("f64", 2048, 300, 0), ("f32", 1000, 64, 1), ("f64", 4099, 3, 0)])
def test_autotune(cuda_ok, dtype, n, m, layout):
    """tri_plan_autotune: the kept (variant, k) is about as
    fast as the planner's pick or faster (timing slack) and still meets parity."""
    import torch
    arrs = gen(n, m, dtype, layout)
    a, b, c, d = to_dev(*arrs)
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, layout)
    x = torch.empty_like(b)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    # 20 solves per timing: CUDA events tick in ~2 us steps on this GPU, so 5-solve
    # timings of ~10 us shapes could not resolve 10 %
    def t_solve(p):
        p.solve(a, b, c, d, out=x)
        s.record()
        for _ in range(20):
            p.solve(a, b, c, d, out=x)
        e.record()
        torch.cuda.synchronize()
        return s.elapsed_time(e) * 1e3 / 20

    t_auto = min(t_solve(plan) for _ in range(3))
    best = plan.autotune(a, b, c, d, out=x, reps=20)
    t_tuned = min(t_solve(plan) for _ in range(3))  # the kept plan, timed exactly like the planner's pick
    assert best > 0
    assert t_tuned <= 1.1 * t_auto + 2.0, (t_tuned, t_auto, plan.describe())
    check_parity(n, m, arrs, plan.solve(a, b, c, d).cpu().numpy(), dtype, layout)


def _grid_lines(n, ms, nb, dtype, family="dd"):
    """Seeded systems for the y-lines of a grid [nb][n][ms]: generated as nb*ms
    contiguous systems (system q = b*ms + s), returned both ways."""
    arrs = gen(n, ms * nb, dtype, 0, family)
    grid = [np.ascontiguousarray(t.reshape(nb, ms, n).transpose(0, 2, 1)).reshape(-1) for t in arrs]
    return arrs, grid


@pytest.mark.parametrize("dtype,n,ms,nb", [("f64", 100, 64, 7), ("f64", 1000, 18, 5), ("f32", 333, 36, 9),
                                           ("f64", 16, 8, 300), ("f32", 4096, 12, 3), ("f64", 64, 1, 50),
                                           ("f64", 77, 50, 1)])
def test_batched_layout_adi_lines(cuda_ok, dtype, n, ms, nb):
    """TRI_LAYOUT_BATCHED: the y-lines of a row-major grid
    [nb][n][ms] solved in place, vs the oracle on the same systems laid out
    contiguously; ragged groups of 8 systems, ms = 1 / nb = 1 reductions."""
    import torch
    arrs, grid = _grid_lines(n, ms, nb, dtype)
    plan = tri.Plan.batched(n, ms, nb, tri.F64 if dtype == "f64" else tri.F32)
    xg = plan.solve(*to_dev(*grid)).cpu().numpy()
    x = np.ascontiguousarray(xg.reshape(nb, n, ms).transpose(0, 2, 1)).reshape(-1)
    check_parity(n, ms * nb, arrs, x, dtype, 0)


def test_batched_layout_rejects(cuda_ok):
    with pytest.raises(tri.TriError):
        tri.Plan.batched(100, 3, 4, tri.F64)   # row stride 24 B: not a 16-byte multiple
    with pytest.raises(tri.TriError):
        tri.Plan.batched(0, 8, 4, tri.F64)
    p = tri.Plan.batched(100, 8, 4, tri.F64)
    with pytest.raises(tri.TriError):
        p.variant = tri.VARIANT_SPLIT            # SCAN is the only kernel for this layout
    assert p.variant == tri.VARIANT_SCAN and p.k == 0


# ------------------------------------------------------------------ SCAN_MC variant
SCAN_MC = tri.VARIANT_SCAN_MC


@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("n,m", [(264, 1), (520, 1), (4104, 5), (65536, 16), (100008, 2), (1 << 20, 3), (16384, 200),
                                 (1 << 24, 1)])
def test_scan_mc_parity(cuda_ok, dtype, n, m):
    """Spans: chunks of one window, ragged last windows and chunks, one chunk per
    system (m > #SMs), several chunks per system, the c3 shape (2^24 rows: 148
    chunks of 443 windows)."""
    arrs = gen(n, m, dtype, 0)
    x, plan = gpu_solve(n, m, arrs, dtype, 0, variant=SCAN_MC)
    assert plan.variant == SCAN_MC and plan.k == 0 and plan.launches in (2, 3)
    check_parity(n, m, arrs, x, dtype, 0)


@pytest.mark.parametrize("family,eps", [("weak", 1e-2), ("weak", 1e-3), ("integer", 0.0), ("poisson", 0.0)])
def test_scan_mc_families(cuda_ok, family, eps):
    n, m = (16384, 2) if family == "poisson" else (1 << 20, 2)
    arrs = gen(n, m, "f64", 0, family, eps=eps)
    x, _ = gpu_solve(n, m, arrs, "f64", 0, variant=SCAN_MC)
    if family == "poisson":
        xo = oracle.solve_batch(n, m, *arrs)
        assert np.max(np.abs(x - xo)) / np.max(np.abs(xo)) <= 2 * (n + 1) ** 2 / 2 * 2.2e-16
    else:
        check_parity(n, m, arrs, x, "f64", 0)


def test_scan_mc_edges_and_scaling(cuda_ok):
    """X1 NaN edges ignored (bitwise), power-of-two row / rhs scaling (bitwise),
    determinism, k fixed at 0."""
    import torch
    n, m = 300000, 2
    a, b, c, d = gen(n, m, "f64", 0, "weak", eps=1e-2)
    plan = tri.Plan(n, m, tri.F64, 0)
    plan.variant = SCAN_MC
    da, db, dc, dd = to_dev(a, b, c, d)
    x1 = plan.solve(da, db, dc, dd).clone()
    assert torch.equal(plan.solve(da, db, dc, dd), x1)
    a2, c2 = da.clone(), dc.clone()
    a2.view(m, n)[:, 0] = float("nan")
    c2.view(m, n)[:, -1] = float("nan")
    assert torch.equal(plan.solve(a2, db, c2, dd), x1)
    p = 2.0 ** np.random.default_rng(2).integers(-20, 20, n * m)
    assert torch.equal(plan.solve(*to_dev(a * p, b * p, c * p, d * p)), x1)
    assert torch.equal(plan.solve(da, db, dc, dd * 4.0), x1 * 4.0)
    plan.k = 1
    assert plan.k == 1 and plan.variant == SPLIT


def test_scan_mc_rejects_unsupported(cuda_ok):
    for (n, m, dt, layout) in [(256, 3, tri.F64, 0), (1001, 3, tri.F64, 0), (16384, 3, tri.F64, 1)]:
        plan = tri.Plan(n, m, dt, layout)
        with pytest.raises(tri.TriError):
            plan.variant = SCAN_MC


def _sliced_solve_one_device(arrs, cuts, dtype):
    """NEXT-4 on one device: the system's row ranges [cuts[i], cuts[i+1]) as G
    'devices' (one plan each), phases run in order with the maps gathered by
    concatenation (what the all-gather of dist.solve_one_system_sliced does)."""
    import torch
    G = len(cuts) - 1
    td = tri.F64 if dtype == "f64" else tri.F32
    sl = [[torch.from_numpy(t[cuts[r]:cuts[r + 1]].copy()).cuda() for t in arrs] for r in range(G)]
    plans = []
    for r in range(G):
        p = tri.Plan(cuts[r + 1] - cuts[r], 1, td, 0)
        p.variant = tri.VARIANT_SCAN_MC
        plans.append(p)
    maps = torch.cat([plans[r].slice_phase(0, r, G, *sl[r]) for r in range(G)])
    bmaps = torch.cat([plans[r].slice_phase(1, r, G, *sl[r], maps=maps) for r in range(G)])
    return torch.cat([plans[r].slice_phase(2, r, G, maps=bmaps) for r in range(G)]).cpu().numpy()


@pytest.mark.parametrize("dtype,family,cuts", [
    ("f64", "dd", [0, 1 << 20]),
    ("f64", "dd", [0, 300000, 562144, 1000008, 1 << 21]),
    ("f64", "weak", [0, 65536, 131072, 196608, 262144, 327680, 393216, 458752, 524288]),
    ("f64", "poisson", [0, 4096, 8192, 12288, 16384]),
    ("f32", "dd", [0, 70000, 140000, 1000000]),
    ("f64", "dd", [0, 300003, 700001, 1000003]),  # ragged slice lengths (tail rows read directly)
])
def test_one_system_sliced_over_devices(cuda_ok, dtype, family, cuts):
    """one system split into row slices (ragged, 1 to 8
    slices), each solved by its own plan with only 8-value maps exchanged
    (tri_slice_solve); vs the oracle on the whole system."""
    n = cuts[-1]
    arrs = gen(n, 1, dtype, 0, family, eps=1e-2)
    x = _sliced_solve_one_device(arrs, cuts, dtype)
    if family == "poisson":
        xo = oracle.solve_batch(n, 1, *arrs)
        assert np.max(np.abs(x - xo)) / np.max(np.abs(xo)) <= 2 * (n + 1) ** 2 / 2 * 2.2e-16
    else:
        check_parity(n, 1, arrs, x, dtype, 0)


def test_one_system_sliced_rejects(cuda_ok):
    import torch
    p = tri.Plan(4096, 1, tri.F64, 0)
    p.variant = tri.VARIANT_SCAN  # not SCAN_MC
    a = torch.ones(4096, dtype=torch.float64, device="cuda")
    with pytest.raises(tri.TriError):
        p.slice_phase(0, 0, 2, a, a, a, a)
    p.variant = tri.VARIANT_SCAN_MC
    with pytest.raises(tri.TriError):
        p.slice_phase(0, 2, 2, a, a, a, a)  # slice out of range
    with pytest.raises(tri.TriError):
        p.slice_phase(1, 0, 2, a, a, a, a)  # phase 1 needs the gathered maps


# ------------------------------------------------------------------ WARP variant
@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("layout", [0, 1])
@pytest.mark.parametrize("n,m", [(32, 5), (33, 4), (63, 7), (64, 1), (100, 9), (128, 33), (200, 3), (256, 130),
                                 (511, 2), (512, 5), (700, 3), (1023, 4), (1024, 7)])
def test_warp_parity(cuda_ok, dtype, layout, n, m):
    """One warp per system (forced; auto picks WARP only when m >= #SMs), every
    register-slot count R = 1..32 and ragged n."""
    arrs = gen(n, m, dtype, layout, "weak", eps=1e-2)
    x, plan = gpu_solve(n, m, arrs, dtype, layout, variant=WARP)
    assert plan.variant == WARP and plan.k == 5
    check_parity(n, m, arrs, x, dtype, layout)


@pytest.mark.parametrize("family,eps", [("dd", 0.0), ("weak", 1e-3), ("integer", 0.0)])
def test_warp_families(cuda_ok, family, eps):
    n, m = 1000, 20
    arrs = gen(n, m, "f64", 0, family, eps=eps)
    x, plan = gpu_solve(n, m, arrs, "f64", 0, variant=WARP)
    check_parity(n, m, arrs, x, "f64", 0)


def test_warp_large_batch_sampled(cuda_ok):
    """Large batch through WARP (n = 256, fp32, m = 2^18; persistent warps with
    next-system prefetch): sampled systems vs the oracle."""
    n, m = 256, 1 << 18
    arrs = gen(n, m, "f32", 0)
    x, plan = gpu_solve(n, m, arrs, "f32", 0, variant=WARP)
    assert plan.variant == WARP
    rng = np.random.default_rng(5)
    for q in rng.choice(m, 64, replace=False).tolist() + [0, m - 1]:
        sl = slice(q * n, (q + 1) * n)
        sub = [t[sl] for t in arrs]
        check_parity(n, 1, sub, x[sl], "f32", 0)


@pytest.mark.parametrize("variant,n,m", [(WARP, 1000, 4), (ONCHIP, 2000, 3), (SPLIT, 5000, 2)])
def test_poisson_closed_form(cuda_ok, variant, n, m):
    """The [-1, 2, -1] Poisson system (only weakly dominant, cond ~ n^2, so the
    elementwise dd tolerance does not apply): normwise error against the
    manufactured exact solution within cond * eps, and the residual gate."""
    import trigen
    a, b, c, d, xs = trigen.generate(n, m, "f64", 0, "poisson", want_xstar=True)
    x, plan = gpu_solve(n, m, (a, b, c, d), "f64", 0, variant=variant)
    assert plan.variant == variant
    cond = (n + 1) ** 2 / 2.0  # ||A||_inf ||A^-1||_inf bound for the 1-D Laplacian
    for q in range(m):
        sl = slice(q * n, (q + 1) * n)
        err = np.max(np.abs(x[sl] - xs[sl])) / np.max(np.abs(xs[sl]))
        assert err <= 64 * cond * np.finfo(np.float64).eps, err
    # ||Ax - d|| / ||d|| is ~cond * eps here, so gate the normwise backward error
    # ||Ax - d|| / (||A|| ||x|| + ||d||) instead
    r = oracle.residual_batch(n, m, a, b, c, d, x, layout=0)
    assert r[:, 1].max() <= 1e-14


# ------------------------------------------------------------------ k = 0 contiguous, TMA path
@pytest.mark.parametrize("dtype,n,m", [("f64", 2, 32), ("f64", 16, 32), ("f64", 1000, 70), ("f64", 20000, 64),
                                       ("f64", 4096, 130), ("f32", 1000, 68), ("f32", 32, 4), ("f32", 5000, 100)])
def test_split_k0_tma(cuda_ok, dtype, n, m):
    """k = 0 on the contiguous layout through the TMA kernel (row strides are
    16-byte multiples): ragged last tile (n % R != 0), ragged last warp (m % 32
    != 0), one-tile systems; bitwise equal to the cp.async kernel (same
    arithmetic in the same order)."""
    import os
    import torch
    arrs = gen(n, m, dtype, 0, "weak", eps=1e-2)
    x, plan = gpu_solve(n, m, arrs, dtype, 0, k=0, variant=SPLIT)
    check_parity(n, m, arrs, x, dtype, 0)
    plan.set_option(tri.OPT_TMA, 0)
    x2 = plan.solve(*to_dev(*arrs)).cpu().numpy()
    assert np.array_equal(x, x2)
    torch.cuda.synchronize()


@pytest.mark.parametrize("dtype,n,m,layout,k", [("f64", 300, 5000, 1, 0), ("f64", 77, 4738, 1, 0),
                                               ("f32", 200, 4800, 1, 0), ("f64", 1 << 16, 1, 0, 13),
                                               ("f64", 70001, 1, 0, 13), ("f64", 3000, 3, 1, 11)])
def test_chain_interleaved_tma(cuda_ok, dtype, n, m, layout, k):
    """p-Thomas over chain-interleaved data through TMA (C = m 2^k >= 32 x SMs):
    raw interleaved input at k = 0 (MODE 1) and tiled-PCR output (MODE 0), x by
    TMA store where x is a 2D view; the fallback (ring kernel, continuant
    forward sweep X18: different rounding) is checked against the oracle too."""
    import os
    arrs = gen(n, m, dtype, layout, "weak", eps=1e-2)
    x, plan = gpu_solve(n, m, arrs, dtype, layout, k=k, variant=SPLIT)
    xo = oracle.solve_batch(n, m, *arrs, layout=layout)
    check_parity(n, m, arrs, x, dtype, layout, x_oracle=xo)
    plan.set_option(tri.OPT_TMA, 0)
    x2 = plan.solve(*to_dev(*arrs)).cpu().numpy()
    check_parity(n, m, arrs, x2, dtype, layout, x_oracle=xo)


@pytest.mark.parametrize("layout", [0, 1])
def test_c4_auto_plan_sampled(cuda_ok, layout):
    """BASELINE config c4 at full size (n = 256, m = 2^20, fp32) through the auto
    plan (M > P: k = 0; SCAN on both layouts -- the interleaved one with one
    system per lane, 32 per window, since round 2): sampled systems vs the oracle
    (every system: test_full_size_every_system)."""
    import trigen
    n, m = 256, 1 << 20
    arrs = gen(n, m, "f32", layout, seed=trigen.SEED_BASE + 4)
    x, plan = gpu_solve(n, m, arrs, "f32", layout)
    assert plan.variant == SCAN and plan.k == 0
    rng = np.random.default_rng(4)
    for q in rng.choice(m, 48, replace=False).tolist() + [0, m - 1]:
        sub = trigen.generate(n, 1, "f32", 0, "dd", seed=trigen.SEED_BASE + 4, q0=q)
        xs = x.reshape(m, n)[q] if layout == 0 else x.reshape(n, m)[:, q]
        check_parity(n, 1, sub, xs, "f32", 0)


@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("n,m", [(1024, 1024), (1000, 36), (4099, 148), (16384, 40), (600, 64), (1024, 8)])
def test_scan_cluster_option(cuda_ok, dtype, n, m):
    """Interleaved SCAN through thread-block clusters (TRI_OPT_SCAN_CLUSTER,
    k_scan_cl: windows of a group spread over 2-8 CTAs, forward state and x
    handed over through distributed shared memory): parity on 2-, 4- and 8-CTA
    clusters, ragged n, padded last groups, fewer windows than warps; the same
    plan without the option runs the chained kernel; repeated solves are
    bitwise identical (fixed composition order)."""
    arrs = gen(n, m, dtype, 1, "weak", eps=1e-2)
    xo = oracle.solve_batch(n, m, *arrs, layout=1)
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, 1)
    plan.variant = tri.VARIANT_SCAN
    plan.set_option(tri.OPT_SCAN_CLUSTER, 1)
    x, _ = gpu_solve(n, m, arrs, dtype, 1, plan=plan)
    check_parity(n, m, arrs, x, dtype, 1, x_oracle=xo)
    x2, _ = gpu_solve(n, m, arrs, dtype, 1, plan=plan)
    assert np.array_equal(x, x2)
    plan.set_option(tri.OPT_SCAN_CLUSTER, 0)
    x3, _ = gpu_solve(n, m, arrs, dtype, 1, plan=plan)
    check_parity(n, m, arrs, x3, dtype, 1, x_oracle=xo)


@pytest.mark.parametrize("dtype,n,m,variant", [
    ("f64", (1 << 20) + 3, 1, "SCAN_MC"), ("f64", 65537, 1, "SCAN_MC"), ("f64", 1000003, 1, "SCAN_MC"),
    ("f32", (1 << 20) + 5, 1, "SCAN_MC"), ("f64", 300, 1, "SCAN"), ("f64", 5003, 1, "SCAN"),
    ("f64", 1002, 64, "SCAN"), ("f32", 1004, 100, "SCAN"), ("f64", 514, 300, "SCAN"), ("f32", 4100, 3, "SCAN"),
    ("f64", 40002, 3, "SCAN_MC")])
def test_scan_ragged_n(cuda_ok, dtype, n, m, variant):
    """SCAN / SCAN_MC with n % 8 != 0 (one system, or a 16-byte system pitch):
    the TMA maps cover the full 8-row groups and the last rows of each system
    come from global memory (k_scan.cuh sc_patch_tail); every system vs the
    oracle, weak family, plus the SCAN_MC look-back path on one system."""
    arrs = gen(n, m, dtype, 0, "weak", eps=1e-2)
    xo = oracle.solve_batch(n, m, *arrs)
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, 0)
    plan.variant = getattr(tri, "VARIANT_" + variant)
    assert plan.variant == getattr(tri, "VARIANT_" + variant)
    x, _ = gpu_solve(n, m, arrs, dtype, 0, plan=plan)
    check_parity(n, m, arrs, x, dtype, 0, x_oracle=xo)
    if variant == "SCAN_MC" and m == 1:
        plan.set_option(tri.OPT_SCAN_MC_LOOKBACK, 32)
        x2, _ = gpu_solve(n, m, arrs, dtype, 0, plan=plan)
        check_parity(n, m, arrs, x2, dtype, 0, x_oracle=xo)


@pytest.mark.parametrize("w", [24, 32, 64, 0])
def test_scan_mc_lookback_variant(cuda_ok, w):
    """SCAN_MC with passes 0 and 1 fused by a look-back over small chunks
    (k_scan_mc_lb, tri_plan_set_option(TRI_OPT_SCAN_MC_LOOKBACK, w)): parity
    against the oracle on ragged chunk counts, fp64 / fp32, several systems, and
    bitwise-identical repeated solves (the look-back has a fixed composition
    order)."""
    import torch
    for dt, n, m in [('f64', 65536, 1), ('f64', 256 * 1000 + 8, 1), ('f32', 256 * 2100 - 16, 1),
                     ('f64', 256 * 130, 3), ('f64', 256 * 40 * 33, 2), ('f64', 1 << 22, 1), ('f64', 1 << 24, 1),
                     ('f32', 1 << 24, 1), ('f64', (1 << 22) + 8, 5)]:
        arrs = gen(n, m, dt, 0)
        plan = tri.Plan(n, m, tri.F64 if dt == "f64" else tri.F32, 0)
        plan.variant = tri.VARIANT_SCAN_MC
        plan.set_option(tri.OPT_SCAN_MC_LOOKBACK, w)
        x, _ = gpu_solve(n, m, arrs, dt, 0, plan=plan)
        check_parity(n, m, arrs, x, dt, 0)
        x2, _ = gpu_solve(n, m, arrs, dt, 0, plan=plan)
        assert np.array_equal(x, x2), (dt, n, m)


@pytest.mark.parametrize("cfg,dtype,n,m,layout", [("c1", "f64", 1024, 1, 0), ("c2", "f64", 1024, 1024, 1),
                                                  ("c3", "f64", 1 << 24, 1, 0), ("c4", "f32", 256, 4096, 0),
                                                  ("c5", "f64", 16384, 64, 0), ("ragged", "f64", 1000003, 1, 0),
                                                  ("c5-il", "f64", 16384, 40, 1)])
def test_set_k_every_k_on_default_plans(cuda_ok, cfg, dtype, n, m, layout):
    """tri_plan_set_k(plan, k) succeeds for every 0 <= k <=
    floor(log2 n) on the planner's default plan of each BASELINE config shape
    (reduced m), switching to a variant that runs k where the default one does
    not (k is the method's knob), and every k meets parity;
    k > floor(log2 n) is rejected and leaves the plan unchanged."""
    import torch
    import trigen
    arrs = gen(n, m, dtype, layout, "weak", eps=1e-2, seed=trigen.SEED_BASE + 9)
    xo = oracle.solve_batch(n, m, *arrs, layout=layout)
    dev = to_dev(*arrs)
    kmax = n.bit_length() - 1
    for k in range(0, kmax + 1):
        plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, layout)
        plan.k = k
        assert plan.k == k, (k, plan.describe())
        x = plan.solve(*dev).cpu().numpy()
        check_parity(n, m, arrs, x, dtype, layout, x_oracle=xo, resid=(n * m <= (1 << 22)))
        del plan
        torch.cuda.empty_cache()
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, layout)
    v0, k0 = plan.variant, plan.k
    with pytest.raises(tri.TriError):
        plan.k = kmax + 1
    assert plan.variant == v0 and plan.k == k0


@pytest.mark.parametrize("dtype,n,m,variant,k", [("f64", 1001, 48, None, None), ("f32", 1001, 33, None, None),
                                                 ("f64", 2048, 64, "STREAM", None), ("f64", 4096, 40, "SPLIT", 3),
                                                 ("f32", 1000, 64, "SPLIT", 2)])
def test_solve_host_chunks_and_forced_plans(cuda_ok, dtype, n, m, variant, k):
    """tri_solve_host's pipelined path (CONTIGUOUS, m >= 32) on chunk sizes whose
    byte offsets are not 16-byte multiples (odd n fp64, n % 4 != 0 fp32: every
    chunk gets its own 256-byte-aligned staging region), and with a forced
    variant / k, which the chunk sub-plans keep."""
    import torch
    arrs = gen(n, m, dtype, 0)
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, 0)
    if variant is not None:
        plan.variant = getattr(tri, "VARIANT_" + variant)
    if k is not None:
        plan.k = k
    host = [torch.from_numpy(t).pin_memory() for t in arrs]
    out = torch.empty(n * m, dtype=host[0].dtype).pin_memory()
    plan.solve_host(*host, out)
    check_parity(n, m, arrs, out.numpy(), dtype, 0)
    with pytest.raises(ValueError):
        plan.solve_host(*host[:3], host[3][:-1], out)  # short array: rejected before the C call
    with pytest.raises(ValueError):
        plan.solve_host(*host[:3], host[3].cuda(), out)  # device tensor: not a host buffer


@pytest.mark.parametrize("n,m,layout,variant,lookback", [(256, 1 << 18, 0, "SCAN", 0), (4096, 4096, 0, "SCAN", 0),
                                                         (1024, 8192, 1, "SCAN", 0), (1 << 22, 1, 0, "SCAN_MC", 0),
                                                         (1 << 22, 1, 0, "SCAN_MC", 64), (65536, 16, 0, "SCAN_MC", 0)])
def test_fp32_weak_accuracy(cuda_ok, n, m, layout, variant, lookback):
    """fp32 on the weakly dominant family (eps = 1e-2, same-sign couplings) over
    2^22 unknowns per case: the SCAN kernels compose their lane / window / chunk
    maps in fp64 (X22), so the error stays at textbook fp32 Thomas's
    level (1.1e-5 on all of c4; the fp32 composition reached 1.2e-4 there).
    Gate: 5e-5, half the north-star 1e-4."""
    arrs = gen(n, m, "f32", layout, "weak", eps=1e-2, seed=77)
    plan = tri.Plan(n, m, tri.F32, layout)
    plan.variant = getattr(tri, "VARIANT_" + variant)
    if lookback:
        plan.set_option(tri.OPT_SCAN_MC_LOOKBACK, lookback)
    x, _ = gpu_solve(n, m, arrs, "f32", layout, plan=plan)
    xo = oracle.solve_batch(n, m, *arrs, layout=layout)
    from tests._helpers import max_rel_err
    assert max_rel_err(x, xo) <= 5e-5


# ---------------------------------------------- interleaved SCAN split over the grid
def _grid_qr(plan):
    d = dict(kv.split("=") for kv in plan.describe().split() if "=" in kv)
    return int(d["grid_Q"]), int(d["grid_R"])


@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("n,m", [(1024, 1024), (1000, 36), (1, 8), (5, 12), (60, 40), (257, 64), (700, 300),
                                 (2048, 300), (2000, 32), (96, 4096), (1023, 100), (2048, 64)])
def test_scan_grid_parity(cuda_ok, dtype, n, m):
    """Interleaved SCAN through k_scan_grid (TRI_OPT_SCAN_GRID, the auto choice
    where 32-system blocks x Q row pieces fit one CTA per SM): every element vs
    the oracle for c2's shape, ragged last blocks (m % 32 != 0), rows past n in
    the last piece and warp, 1 to 4 TMA stages per warp (R = 4 .. 16), Q = 1 ..
    8 (thread-block clusters); repeated solves are bitwise identical; the
    chained kernel (option 0) agrees."""
    arrs = gen(n, m, dtype, 1, "weak", eps=1e-2)
    xo = oracle.solve_batch(n, m, *arrs, layout=1)
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, 1)
    plan.variant = tri.VARIANT_SCAN
    Q, R = _grid_qr(plan)
    assert Q > 0 and R in (4, 8, 12, 16)
    xs = [gpu_solve(n, m, arrs, dtype, 1, plan=plan)[0] for _ in range(3)]
    check_parity(n, m, arrs, xs[0], dtype, 1, x_oracle=xo)
    assert np.array_equal(xs[0], xs[1]) and np.array_equal(xs[0], xs[2])
    plan.set_option(tri.OPT_SCAN_GRID, 0)
    assert _grid_qr(plan) == (0, 0)
    x3, _ = gpu_solve(n, m, arrs, dtype, 1, plan=plan)
    check_parity(n, m, arrs, x3, dtype, 1, x_oracle=xo)
    plan.set_option(tri.OPT_SCAN_GRID, -1)
    x4, _ = gpu_solve(n, m, arrs, dtype, 1, plan=plan)
    assert np.array_equal(xs[0], x4)


def test_scan_grid_graph_replay_and_variant_switch(cuda_ok):
    """k_scan_grid under CUDA-graph replay (bench.py's timing) and after another
    variant has run on the same plan: every replay matches the oracle."""
    import torch
    n, m = 1024, 1024
    arrs = gen(n, m, "f64", 1)
    xo = oracle.solve_batch(n, m, *arrs, layout=1)
    plan = tri.Plan(n, m, tri.F64, 1)
    assert _grid_qr(plan)[0] > 0
    a, b, c, d = to_dev(*arrs)
    x = torch.empty_like(a)
    plan.solve(a, b, c, d, out=x)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s):
            plan.solve(a, b, c, d, out=x)
    for _ in range(5):
        x.fill_(float("nan"))
        g.replay()
        torch.cuda.synchronize()
        check_parity(n, m, arrs, x.cpu().numpy(), "f64", 1, x_oracle=xo)
    plan.variant = SPLIT
    plan.solve(a, b, c, d, out=x)
    plan.variant = tri.VARIANT_SCAN
    assert _grid_qr(plan)[0] > 0
    x.fill_(float("nan"))
    plan.solve(a, b, c, d, out=x)
    check_parity(n, m, arrs, x.cpu().numpy(), "f64", 1, x_oracle=xo)


@pytest.mark.parametrize("dtype,n,ms,nb", [("f64", 100, 64, 7), ("f32", 333, 36, 9), ("f64", 1000, 18, 5)])
def test_scan_grid_batched(cuda_ok, dtype, n, ms, nb):
    """k_scan_grid on BATCHED y-lines [nb][n][ms] (blocks per batch, batch stride)."""
    arrs, grid = _grid_lines(n, ms, nb, dtype, "weak")
    plan = tri.Plan.batched(n, ms, nb, tri.F64 if dtype == "f64" else tri.F32)
    assert _grid_qr(plan)[0] > 0
    xg = plan.solve(*to_dev(*grid)).cpu().numpy()
    x = np.ascontiguousarray(xg.reshape(nb, n, ms).transpose(0, 2, 1)).reshape(-1)
    check_parity(n, ms * nb, arrs, x, dtype, 0)


# ------------------------------------------ fp64 contiguous SCAN with 512-row windows
@pytest.mark.parametrize("n,m", [(16384, 40), (1024, 300), (1040, 64), (8192, 5), (4112, 7), (16384, 1),
                                 (528, 150), (65536, 3)])
@pytest.mark.parametrize("family", ["dd", "weak"])
def test_scan_w512_parity(cuda_ok, n, m, family):
    """k_scan_w512 (TRI_OPT_SCAN_W512, auto for fp64 contiguous n % 16 == 0 with
    >= 2 windows of 512 rows): every element vs the oracle; 2 .. 128 windows, a
    ragged last window (n % 512 != 0), one system (several windows per warp
    step), more systems than CTAs; repeated solves bitwise identical; the
    256-row-window kernel (option 0) agrees within the tolerance."""
    arrs = gen(n, m, "f64", 0, family, eps=1e-2)
    xo = oracle.solve_batch(n, m, *arrs)
    plan = tri.Plan(n, m, tri.F64, 0)
    plan.variant = tri.VARIANT_SCAN
    assert "w512=1" in plan.describe()
    x, _ = gpu_solve(n, m, arrs, "f64", 0, plan=plan)
    check_parity(n, m, arrs, x, "f64", 0, x_oracle=xo)
    x2, _ = gpu_solve(n, m, arrs, "f64", 0, plan=plan)
    assert np.array_equal(x, x2)
    plan.set_option(tri.OPT_SCAN_W512, 0)
    assert "w512=0" in plan.describe()
    x3, _ = gpu_solve(n, m, arrs, "f64", 0, plan=plan)
    check_parity(n, m, arrs, x3, "f64", 0, x_oracle=xo)


@pytest.mark.parametrize("dtype,n,m,layout,variant,opt", [
    ("f64", 1024, 40, 0, "SCAN", None),             # k_scan_w512, n a multiple of its 512-row window
    ("f64", 1024, 40, 0, "SCAN", ("W512", 0)),      # k_scan, n a multiple of its 256-row window
    ("f32", 768, 50, 0, "SCAN", None),              # k_scan fp32
    ("f32", 256, 64, 0, "SCAN", None),              # k_scan1_r16 (c4's kernel)
    ("f64", 256, 40, 0, "SCAN", None),              # one-window fp64
    ("f64", 65536, 1, 0, "SCAN_MC", None),          # SCAN_MC, n a multiple of 256
    ("f64", 65536, 1, 0, "SCAN_MC", ("LB", 32)),    # look-back SCAN_MC
    ("f64", 1024, 64, 1, "SCAN", None),             # k_scan_grid
    ("f64", 2048, 2048, 1, "SCAN", None),           # chained interleaved (beyond one wave)
    ("f64", 1024, 64, 1, "SCAN", ("CL", 1)),        # thread-block cluster option
    ("f64", 4800, 3, 0, "STREAM", None),            # STREAM, n a multiple of its 240-row window
    ("f64", 2048, 150, 0, "FUSED", None),           # FUSED
    ("f32", 1536, 200, 0, "FUSED", None),
])
def test_ignored_entries_nan_scan(cuda_ok, dtype, n, m, layout, variant, opt):
    """a[q][0] and c[q][n-1] lie outside A (Eq 1, reading X1): NaN there must not
    change x (bitwise) on the SCAN-family kernels, including systems whose length
    is a multiple of the kernel's window (the last window must still drop c_{n-1})."""
    import torch
    arrs = gen(n, m, dtype, layout)
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, layout)
    plan.variant = getattr(tri, "VARIANT_" + variant)
    if opt is not None:
        plan.set_option({"W512": tri.OPT_SCAN_W512, "LB": tri.OPT_SCAN_MC_LOOKBACK, "CL": tri.OPT_SCAN_CLUSTER}[opt[0]], opt[1])
    a, b, c, d = to_dev(*arrs)
    x1 = plan.solve(a, b, c, d).clone()
    a2, c2 = a.clone(), c.clone()
    if layout == 0:
        a2.view(m, n)[:, 0] = float("nan")
        c2.view(m, n)[:, -1] = float("nan")
    else:
        a2.view(n, m)[0, :] = float("nan")
        c2.view(n, m)[-1, :] = float("nan")
    x2 = plan.solve(a2, b, c2, d)
    assert torch.equal(x1, x2), plan.describe()


@pytest.mark.parametrize("dtype,n,m,layout,variant", [
    ("f64", 1024, 40, 0, "SCAN"), ("f64", 1032, 40, 0, "SCAN"), ("f32", 1024, 40, 0, "SCAN"),
    ("f32", 256, 64, 0, "SCAN"), ("f64", 65536, 1, 0, "SCAN_MC"), ("f64", 1024, 64, 1, "SCAN"),
    ("f64", 1024, 2048, 1, "SCAN")])
def test_scan_kernels_16_byte_offsets(cuda_ok, dtype, n, m, layout, variant):
    """Arrays that are 16-byte but not 32- / 128-byte aligned (views into larger
    buffers; the ABI's only alignment rule is 16 bytes): the TMA descriptors take
    any 16-byte base and the x stores fall back from 256-bit to narrower ones."""
    import torch
    arrs = gen(n, m, dtype, layout)
    xo = oracle.solve_batch(n, m, *arrs, layout=layout)
    tdt = torch.float64 if dtype == "f64" else torch.float32
    off = 16 // (8 if dtype == "f64" else 4)
    views = []
    for t in arrs:
        buf = torch.empty(n * m + 64, dtype=tdt, device="cuda")
        v = buf[off:off + n * m]
        v.copy_(torch.from_numpy(t))
        views.append(v)
    xbuf = torch.full((n * m + 64,), float("nan"), dtype=tdt, device="cuda")
    x = xbuf[off:off + n * m]
    assert x.data_ptr() % 32 == 16
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, layout)
    plan.variant = getattr(tri, "VARIANT_" + variant)
    plan.solve(*views, out=x)
    check_parity(n, m, arrs, x.cpu().numpy(), dtype, layout, x_oracle=xo)
    assert torch.isnan(xbuf[:off]).all() and torch.isnan(xbuf[off + n * m:]).all()


@pytest.mark.parametrize("dtype,n,m", [("f32", 256, 8192), ("f64", 256, 8192), ("f32", 100, 10000), ("f64", 64, 4800),
                                       ("f32", 600, 5000), ("f64", 37, 6000)])
def test_scan_interleaved_32_systems_per_window(cuda_ok, dtype, n, m):
    """Interleaved SCAN with one system per lane (32 systems x 8 rows per window,
    256-byte TMA rows, no lane scans) for many short systems: ragged rows and a
    ragged last group of 32 systems, every element vs the oracle."""
    arrs = gen(n, m, dtype, 1, "weak", eps=1e-2)
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, 1)
    plan.variant = tri.VARIANT_SCAN
    x, _ = gpu_solve(n, m, arrs, dtype, 1, plan=plan)
    check_parity(n, m, arrs, x, dtype, 1)


@pytest.mark.parametrize("dtype,n,m,layout,variant,opt,k", [
    ("f64", 1024, 1, 0, "SCAN", None, None),             # k_scan_w512, one system (lag 0)
    ("f64", 1000, 5, 0, "SCAN", ("W512", 1), None),      # k_scan_w512, ragged last window
    ("f64", 1536, 200, 0, "SCAN", None, None),           # k_scan_w512, more systems than SMs
    ("f64", 1032, 40, 0, "SCAN", ("W512", 0), None),     # k_scan
    ("f32", 1000, 7, 0, "SCAN", None, None),             # k_scan fp32, ragged
    ("f32", 224, 33, 0, "SCAN", None, None),             # k_scan1_r16
    ("f64", 200, 41, 0, "SCAN", None, None),             # one-window fp64
    ("f64", 65537, 1, 0, "SCAN_MC", None, None),         # SCAN_MC, ragged n
    ("f64", 65536, 1, 0, "SCAN_MC", ("LB", 32), None),   # look-back SCAN_MC
    ("f64", 700, 36, 1, "SCAN", None, None),             # k_scan_grid, ragged block and rows
    ("f32", 520, 24, 1, "SCAN", ("GRID", 0), None),      # chained interleaved, ragged window
    ("f64", 4800, 3, 0, "STREAM", None, None),
    ("f64", 2000, 3, 0, "FUSED", None, None),
    ("f64", 512, 16, 0, "WARP", None, None),
    ("f32", 1000, 3, 0, "ONCHIP", None, 4),
    ("f64", 5003, 3, 0, "SPLIT", None, 9),               # register-tile passes + p-Thomas
    ("f64", 1000, 37, 1, "SPLIT", None, 7),
    ("f64", 4096, 2, 0, "SPLIT", ("TMA", 0), 12),        # the paper's sliding window
])
def test_guard_bands_and_const_inputs(cuda_ok, dtype, n, m, layout, variant, opt, k):
    """Every kernel family writes x and nothing else a caller owns: each array
    sits between 4096-element guard bands of random bits; after the solve the
    guards of all five buffers and the whole of a, b, c, d (const in tri.h) are
    bitwise unchanged, and x matches the oracle.  (Our own out-of-bounds check:
    compute-sanitizer is closed on the GPU pool, profiles/r02_sanitize.)"""
    import torch
    arrs = gen(n, m, dtype, layout)
    xo = oracle.solve_batch(n, m, *arrs, layout=layout)
    tdt, idt = (torch.float64, torch.int64) if dtype == "f64" else (torch.float32, torch.int32)
    G, N = 4096, n * m
    g = torch.Generator().manual_seed(n * 131 + m)
    bufs, views = [], []
    for t in list(arrs) + [None]:
        bits = torch.randint(-2**31, 2**31 - 1, (N + 2 * G,), generator=g, dtype=torch.int64).to(idt)
        buf = bits.view(tdt).cuda()
        v = buf[G:G + N]
        if t is not None:
            v.copy_(torch.from_numpy(t))
        bufs.append(buf)
        views.append(v)
    before = [b_.view(idt).clone() for b_ in bufs]
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, layout)
    plan.variant = getattr(tri, "VARIANT_" + variant)
    if opt is not None:
        plan.set_option({"W512": tri.OPT_SCAN_W512, "LB": tri.OPT_SCAN_MC_LOOKBACK, "GRID": tri.OPT_SCAN_GRID,
                         "TMA": tri.OPT_TMA}[opt[0]], opt[1])
    if k is not None:
        plan.k = k
    plan.solve(*views[:4], out=views[4])
    torch.cuda.synchronize()
    for i in range(4):
        assert torch.equal(bufs[i].view(idt), before[i]), f"input {'abcd'[i]} modified [{plan.describe()}]"
    xb = bufs[4].view(idt)
    assert torch.equal(xb[:G], before[4][:G]), f"write below x [{plan.describe()}]"
    assert torch.equal(xb[G + N:], before[4][G + N:]), f"write past x [{plan.describe()}]"
    check_parity(n, m, arrs, views[4].cpu().numpy(), dtype, layout, x_oracle=xo)


@pytest.mark.parametrize("dtype,n,m,w512", [("f64", 65544, 2, 0), ("f64", 65536, 1, 1), ("f32", 1 << 17, 1, 0),
                                            ("f64", 30000, 150, 0), ("f64", 30208, 150, 1)])
def test_scan_spilled_slots_lag(cuda_ok, dtype, n, m, w512):
    """SCAN with more windows than on-chip slots (the spill to global scratch):
    one system per CTA (no back-substitution lag, the backward sweep reads the
    last window right after its store) and more systems than SMs (lag 8, slots
    reused by the CTA's next system) -- every element vs the oracle."""
    arrs = gen(n, m, dtype, 0, "weak", eps=1e-2)
    plan = tri.Plan(n, m, tri.F64 if dtype == "f64" else tri.F32, 0)
    plan.variant = tri.VARIANT_SCAN
    if dtype == "f64":
        plan.set_option(tri.OPT_SCAN_W512, w512)
    x, _ = gpu_solve(n, m, arrs, dtype, 0, plan=plan)
    check_parity(n, m, arrs, x, dtype, 0)
