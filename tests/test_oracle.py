"""Pins for the CPU oracle (oracle/) against things other than itself:
exact rational brute force, an independent dense GE cross-checked with numpy,
LAPACK dgtsv, the Poisson closed form, integer-manufactured exact solutions,
the residual invariant and the paper's PCR index structure (Figs 3, 4, 6).

Each test cites the PAPER.md passage (P:NNN) it follows."""
from fractions import Fraction

import numpy as np
import pytest
import scipy.linalg.lapack as lapack

import oracle
import trigen

U = np.finfo(np.float64).eps  # 2^-52


# ---------------------------------------------------------------- helpers
def exact_solve(a, b, c, d):
    """Exact rational Gauss-Jordan on the assembled Eq 1 matrix.
    Pure Python Fractions, tiny n only (brute force)."""
    n = len(b)
    M = [[Fraction(0)] * (n + 1) for _ in range(n)]
    for i in range(n):
        if i > 0:
            M[i][i - 1] = Fraction(a[i])
        M[i][i] = Fraction(b[i])
        if i < n - 1:
            M[i][i + 1] = Fraction(c[i])
        M[i][n] = Fraction(d[i])
    for col in range(n):
        piv = next(r for r in range(col, n) if M[r][col] != 0)
        M[col], M[piv] = M[piv], M[col]
        p = M[col][col]
        M[col] = [v / p for v in M[col]]
        for r in range(n):
            if r != col and M[r][col] != 0:
                f = M[r][col]
                M[r] = [vr - f * vc for vr, vc in zip(M[r], M[col])]
    return [M[i][n] for i in range(n)]


def dgtsv(a, b, c, d):
    """LAPACK tridiagonal GE with partial pivoting (third-party pin)."""
    n = len(b)
    dl = np.array(a[1:], dtype=np.float64)
    du = np.array(c[:-1], dtype=np.float64)
    _, _, _, x, info = lapack.dgtsv(dl, np.array(b, np.float64), du, np.array(d, np.float64))
    assert info == 0
    return x


def gen1(n, family="dd", seed=1, eps=1e-2, q=0):
    a, b, c, d, xs = trigen.generate(n, 1, "f64", family=family, seed=seed, eps=eps, q0=q, want_xstar=True)
    return a, b, c, d, xs


# ---------------------------------------------------------------- generator pins
def test_splitmix64_test_vectors():
    # SplitMix64 (Steele, Lea, Flood 2014; Vigna's reference) from state 0:
    # outputs 0xe220a8397b1dcdaf, 0x6e789e6aa1b965f4, 0x06c45d188009454f.
    g = 0x9E3779B97F4A7C15
    assert trigen.mix(0) == 0xE220A8397B1DCDAF
    assert trigen.mix(g) == 0x6E789E6AA1B965F4
    assert trigen.mix(2 * g % 2**64) == 0x06C45D188009454F


@pytest.mark.parametrize("family", ["dd", "weak", "integer", "poisson"])
def test_generator_layout_and_shard_invariance(family):
    n, m = 37, 11
    ac, bc, cc, dc = trigen.generate(n, m, "f64", trigen.CONTIGUOUS, family)
    ai, bi, ci, di = trigen.generate(n, m, "f64", trigen.INTERLEAVED, family)
    for u, v in ((ac, ai), (bc, bi), (cc, ci), (dc, di)):
        assert np.array_equal(u.reshape(m, n), v.reshape(n, m).T)
    # a rank that owns systems [4, 9) sees the same bytes
    a2, b2, c2, d2 = trigen.generate(n, 5, "f64", trigen.CONTIGUOUS, family, q0=4, nthreads=3)
    assert np.array_equal(a2, ac[4 * n:9 * n]) and np.array_equal(d2, dc[4 * n:9 * n])
    # edge entries outside A (Eq 1, reading X1) are 0
    assert np.all(ac.reshape(m, n)[:, 0] == 0) and np.all(cc.reshape(m, n)[:, -1] == 0)


def test_generator_families_properties():
    a, b, c, d = trigen.generate(1000, 3, "f64", family="dd")
    assert np.all(np.abs(b) >= np.abs(a) + np.abs(c) + 1.0)
    a, b, c, d = trigen.generate(1000, 3, "f64", family="weak", eps=1e-3)
    a2, c2 = a.reshape(3, -1), c.reshape(3, -1)
    assert np.all(a2[:, 1:] < 0) and np.all(c2[:, :-1] < 0)  # same-sign couplings
    assert np.all(np.abs(b) >= (np.abs(a) + np.abs(c)) * (1 + 1e-3) * (1 - 1e-15))
    a, b, c, d, xs = trigen.generate(500, 2, "f64", family="integer", want_xstar=True)
    for t in (a, b, c, d, xs):
        assert np.all(t == np.round(t))
    assert np.all(np.abs(b) >= np.abs(a) + np.abs(c) + 1)


# ---------------------------------------------------------------- Thomas pins
@pytest.mark.parametrize("n", [1, 2, 3, 5, 9, 12])
@pytest.mark.parametrize("seed", range(4))
def test_thomas_vs_exact_rational(n, seed):
    """Brute force: exact rational elimination (P:91 'special case of Gaussian
    elimination'); Thomas Eqs 2-4 must agree to a few ulp on integer systems."""
    a, b, c, d, xs = gen1(n, "integer", seed=seed)
    ex = exact_solve(a, b, c, d)
    assert [Fraction(v) for v in xs] == ex  # manufactured solution is exact
    x = oracle.thomas(a, b, c, d)
    for xi, ei in zip(x, ex):
        assert abs(Fraction(xi) - ei) <= 4 * U * abs(ei)


@pytest.mark.parametrize("n", [1, 2, 7, 33, 64])
@pytest.mark.parametrize("family", ["dd", "weak"])
def test_thomas_vs_dense_ge(n, family):
    """Dense GE with partial pivoting (independent code path, n <= 64), itself
    cross-checked with numpy.linalg.solve."""
    a, b, c, d, _ = gen1(n, family, seed=n)
    M = oracle.assemble(a, b, c)
    xg = oracle.dense_ge(M, d)
    xn = np.linalg.solve(M, d)
    assert np.max(np.abs(xg - xn) / np.abs(xn)) <= 1e-13
    x = oracle.thomas(a, b, c, d)
    assert np.max(np.abs(x - xg) / np.abs(xg)) <= 1e-13


def test_dense_ge_pivots():
    # a matrix that needs pivoting (zero leading entry): GE must still solve it
    M = np.array([[0.0, 1.0, 0.0], [2.0, 0.0, 1.0], [0.0, 3.0, 4.0]])
    r = np.array([1.0, 2.0, 3.0])
    assert np.allclose(oracle.dense_ge(M, r), np.linalg.solve(M, r), rtol=1e-15)


@pytest.mark.parametrize("n,family,tol", [(1024, "dd", 1e-13), (1 << 16, "dd", 1e-13),
                                          (1 << 20, "dd", 1e-13), (4096, "weak", 1e-12),
                                          (1 << 18, "weak", 1e-12)])
def test_thomas_vs_lapack_dgtsv(n, family, tol):
    a, b, c, d, _ = gen1(n, family, seed=7)
    x = oracle.thomas(a, b, c, d)
    xl = dgtsv(a, b, c, d)
    assert np.max(np.abs(x - xl) / np.abs(xl)) <= tol


@pytest.mark.parametrize("n", [8, 1024, 4096, 16384])
def test_thomas_poisson_closed_form(n):
    """Poisson [-1, 2, -1], d = 1: x_i = i(n+1-i)/2 (1-based), exact in fp64.
    Forward error bounded by kappa_inf * u with kappa_inf ~ (n+1)^2/2."""
    a, b, c, d, xs = gen1(n, "poisson")
    i = np.arange(1, n + 1, dtype=np.float64)
    assert np.array_equal(xs, i * (n + 1 - i) / 2)
    x = oracle.thomas(a, b, c, d)
    kappa = (n + 1) ** 2 / 2
    assert np.max(np.abs(x - xs)) / np.max(np.abs(xs)) <= 4 * kappa * U


@pytest.mark.parametrize("n", [3, 100, 5000])
def test_thomas_integer_manufactured(n):
    """|b| >= |a|+|c|+1 integer matrix, integer x*: d = A x* is exact, so the
    exact solution is x* itself."""
    a, b, c, d, xs = gen1(n, "integer", seed=3)
    x = oracle.thomas(a, b, c, d)
    assert np.max(np.abs(x - xs) / np.abs(xs)) <= 1e-14


def test_residual_helper_pinned():
    """Residual helper vs a numpy dense matvec of the assembled matrix; zero on
    an exact integer solution."""
    a, b, c, d, xs = gen1(40, "integer", seed=5)
    r, be = oracle.residual(a, b, c, d, xs)
    assert r == 0.0 and be == 0.0
    a, b, c, d, xs = gen1(40, "dd", seed=5)
    xp = xs * (1 + 1e-6 * np.sin(np.arange(40)))
    M = oracle.assemble(a, b, c)
    res = M @ xp - d
    r, be = oracle.residual(a, b, c, d, xp)
    assert r == pytest.approx(np.max(np.abs(res)) / np.max(np.abs(d)), rel=1e-9)
    s = np.abs(M) @ np.abs(xp) + np.abs(d)
    assert be == pytest.approx(np.max(np.abs(res)) / np.max(s), rel=1e-9)


@pytest.mark.parametrize("family,n", [("dd", 1024), ("dd", 1 << 18), ("weak", 16384)])
def test_residual_invariant(family, n):
    a, b, c, d, _ = gen1(n, family, seed=11, eps=1e-3)
    x = oracle.thomas(a, b, c, d)
    r, be = oracle.residual(a, b, c, d, x)
    assert r <= 1e-12 and be <= 1e-14


# ---------------------------------------------------------------- batch driver
@pytest.mark.parametrize("dtype", ["f64", "f32"])
def test_batch_layouts_threads_and_ignored_entries(dtype):
    n, m = 61, 23
    a, b, c, d = trigen.generate(n, m, dtype, trigen.CONTIGUOUS, "dd")
    x1 = oracle.solve_batch(n, m, a, b, c, d, layout=0, nthreads=1)
    x4 = oracle.solve_batch(n, m, a, b, c, d, layout=0, nthreads=4)
    assert np.array_equal(x1, x4)
    for q in (0, 7, 22):
        s = slice(q * n, (q + 1) * n)
        ref = oracle.thomas(a[s].astype(np.float64), b[s].astype(np.float64),
                            c[s].astype(np.float64), d[s].astype(np.float64))
        assert np.array_equal(x1[s], ref)
    ai, bi, ci, di = trigen.generate(n, m, dtype, trigen.INTERLEAVED, "dd")
    xi = oracle.solve_batch(n, m, ai, bi, ci, di, layout=1, nthreads=3)
    assert np.array_equal(xi.reshape(n, m).T.ravel(), x1)
    # a[0] and c[n-1] lie outside A (Eq 1, reading X1): NaN there changes nothing
    a2, c2 = a.copy(), c.copy()
    a2.reshape(m, n)[:, 0] = np.nan
    c2.reshape(m, n)[:, -1] = np.nan
    assert np.array_equal(oracle.solve_batch(n, m, a2, b, c2, d, nthreads=2), x1)


def test_batch_sample_range():
    n, m = 50, 10
    a, b, c, d = trigen.generate(n, m, "f64")
    full = oracle.solve_batch(n, m, a, b, c, d)
    part = oracle.solve_batch(n, m, a, b, c, d, q_begin=3, q_end=6)
    assert np.array_equal(part[3 * n:6 * n], full[3 * n:6 * n])
    assert np.all(part[:3 * n] == 0)


# ---------------------------------------------------------------- PCR pins
def _dense_from_stride(a, b, c, s):
    """Dense matrix of a stride-s tridiagonal system (row i couples i-s, i+s)."""
    n = len(b)
    M = np.zeros((n, n))
    for i in range(n):
        M[i, i] = b[i]
        if i - s >= 0:
            M[i, i - s] = a[i]
        if i + s < n:
            M[i, i + s] = c[i]
    return M


@pytest.mark.parametrize("n", [8, 13, 64])
@pytest.mark.parametrize("family", ["dd", "weak"])
def test_pcr_steps_preserve_solution(n, family):
    """PCR steps are row operations that preserve the solution:
    after k steps (strides 1..2^{k-1}, Eqs 5-6) the reduced stride-2^k system is
    satisfied by the exact solution, and row i couples only rows i -+ 2^k."""
    a, b, c, d, _ = gen1(n, family, seed=2)
    x = oracle.dense_ge(oracle.assemble(a, b, c), d)
    for k in range(0, int(np.log2(n)) + 2):
        ak, bk, ck, dk = oracle.pcr_k(a, b, c, d, k)
        s = 1 << k
        M = _dense_from_stride(ak, bk, ck, s)
        assert np.max(np.abs(M @ x - dk)) <= 1e-13 * np.max(np.abs(dk))
        # couplings to rows outside [0, n) vanish (reading X4)
        idx = np.arange(n)
        assert np.all(ak[idx < s] == 0) and np.all(ck[idx >= n - s] == 0)


def test_pcr_paper_figure_structure():
    """Figs 3/4/6: n = 8, one PCR step gives the subsystems
    {0,2,4,6} and {1,3,5,7}; two steps give {0,4},{1,5},{2,6},{3,7}; solving each
    subsystem independently (dense GE) reproduces x."""
    golden = open(__file__.replace("test_oracle.py", "golden/paper_fig4_subsystems_n8.txt")).read()
    expect = {}
    for line in golden.splitlines():
        if line and not line.startswith("#"):
            k, sets = line.split(":")
            expect[int(k)] = [sorted(int(v) for v in grp.split(",")) for grp in sets.split(";")]
    a, b, c, d, _ = gen1(8, "dd", seed=9)
    x = oracle.dense_ge(oracle.assemble(a, b, c), d)
    for k, groups in expect.items():
        ak, bk, ck, dk = oracle.pcr_k(a, b, c, d, k)
        s = 1 << k
        M = _dense_from_stride(ak, bk, ck, s)
        got = []
        for r in range(s):
            rows = list(range(r, 8, s))
            got.append(rows)
            sub = M[np.ix_(rows, rows)]
            # decoupled: no entries from this subsystem's rows into other rows
            others = [j for j in range(8) if j not in rows]
            assert np.all(M[np.ix_(rows, others)] == 0)
            xs = np.linalg.solve(sub, dk[rows])
            assert np.allclose(xs, x[rows], rtol=1e-13, atol=0)
        assert sorted(got) == sorted(groups)


@pytest.mark.parametrize("n", [1, 2, 5, 16, 100])
def test_full_pcr_gives_diagonal(n):
    """Reading X7 / P:253: once 2^k >= n every subsystem has one row, so
    x_i = d_i / b_i of the reduced system."""
    a, b, c, d, _ = gen1(n, "dd", seed=4)
    x = oracle.thomas(a, b, c, d)
    k = max(0, int(np.ceil(np.log2(n))))
    ak, bk, ck, dk = oracle.pcr_k(a, b, c, d, k)
    assert np.all(ak == 0) and np.all(ck == 0)
    assert np.max(np.abs(dk / bk - x) / np.abs(x)) <= 1e-13


def test_pcr_step_exact_rational():
    """One stride-s step (Eqs 5-6) equals the exact rational row operation
    row_i - k1 row_{i-s} - k2 row_{i+s} that zeroes columns i-s and i+s."""
    n, s = 9, 2
    a, b, c, d, _ = gen1(n, "integer", seed=8)
    a[0] = 0
    c[-1] = 0
    a2, b2, c2, d2 = oracle.pcr_step(a, b, c, d, s)
    F = Fraction
    rows = []
    for i in range(n):
        r = [F(0)] * (n + 1)
        r[i] = F(b[i])
        if i - s >= 0:
            r[i - s] = F(a[i])
        if i + s < n:
            r[i + s] = F(c[i])
        r[n] = F(d[i])
        rows.append(r)
    for i in range(n):
        new = list(rows[i])
        if i - s >= 0:
            k1 = F(a[i]) / F(b[i - s])
            new = [u - k1 * v for u, v in zip(new, rows[i - s])]
        if i + s < n:
            k2 = F(c[i]) / F(b[i + s])
            new = [u - k2 * v for u, v in zip(new, rows[i + s])]
        if i - s >= 0:
            assert new[i - s] == 0
        if i + s < n:
            assert new[i + s] == 0
        for val, ex in ((a2[i], new[i - 2 * s] if i - 2 * s >= 0 else F(0)),
                        (b2[i], new[i]),
                        (c2[i], new[i + 2 * s] if i + 2 * s < n else F(0)),
                        (d2[i], new[n])):
            assert abs(F(val) - ex) <= 4 * U * max(abs(ex), F(1))


def test_residual_batch_matches_single():
    n, m = 33, 9
    a, b, c, d = trigen.generate(n, m, "f32", trigen.INTERLEAVED, "dd")
    x = oracle.solve_batch(n, m, a, b, c, d, layout=1)
    xp = x * (1 + 1e-7 * np.cos(np.arange(n * m)))
    rb = oracle.residual_batch(n, m, a, b, c, d, xp, layout=1)
    for q in (0, 4, 8):
        sl = lambda t: t.reshape(n, m)[:, q].astype(np.float64)
        assert tuple(rb[q]) == oracle.residual(sl(a), sl(b), sl(c), sl(d), sl(xp))
