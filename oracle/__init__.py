"""CPU oracle -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct fp64 implementation of what the hot path
computes: the solution x of A x = d (Eq 1) for each of m
independent tridiagonal systems, via the Thomas algorithm exactly as Eqs 2-4
(P:91-127), plus dense Gaussian elimination with partial pivoting (brute force,
n <= 64), one PCR step (Eqs 5-6) and residuals.

May be imported ONLY by tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs.  Shares no code with the CUDA path
(paper_conf_icpp_kimwch11_b200/) and never imports it.  Pins:
tests/test_oracle.py.  Every function here is pinned (no "parity unpinned").
"""
import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-shared", "-fPIC"]


def build(force=False):
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", *CFLAGS, "-o", _LIB, _SRC, "-lm", "-lpthread"])
    return _LIB


_lib = None
_P = ctypes.c_void_p
_I64 = ctypes.c_int64


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.oracle_thomas.argtypes = [_I64, _P, _P, _P, _P, _P, _P, _P]
        lib.oracle_thomas.restype = None
        lib.oracle_dense_ge.argtypes = [_I64, _P, _P, _P]
        lib.oracle_dense_ge.restype = ctypes.c_int
        lib.oracle_assemble.argtypes = [_I64, _P, _P, _P, _P]
        lib.oracle_assemble.restype = None
        lib.oracle_pcr_step.argtypes = [_I64, _I64] + [_P] * 8
        lib.oracle_pcr_step.restype = None
        lib.oracle_pcr_k.argtypes = [_I64, ctypes.c_int] + [_P] * 9
        lib.oracle_pcr_k.restype = None
        lib.oracle_residual.argtypes = [_I64, _P, _P, _P, _P, _P, _P]
        lib.oracle_residual.restype = None
        lib.oracle_solve_batch.argtypes = [_I64, _I64, ctypes.c_int, ctypes.c_int, _P, _P, _P, _P, _P, _P,
                                           _I64, _I64, ctypes.c_int]
        lib.oracle_solve_batch.restype = ctypes.c_int
        lib.oracle_residual_batch.argtypes = [_I64, _I64, ctypes.c_int, ctypes.c_int, _P, _P, _P, _P, _P, _P,
                                              ctypes.c_int]
        lib.oracle_residual_batch.restype = ctypes.c_int
        _lib = lib
    return _lib


def _f64(x):
    return np.ascontiguousarray(x, dtype=np.float64)


def _p(x):
    return ctypes.c_void_p(x.ctypes.data)


def thomas(a, b, c, d):
    """Thomas algorithm, Eqs 2-4 on one system; a[0], c[n-1] must be
    the values to use (the batch driver zeroes them; this raw form does not)."""
    a, b, c, d = map(_f64, (a, b, c, d))
    n = b.size
    x = np.empty(n)
    cp = np.empty(n)
    dp = np.empty(n)
    _load().oracle_thomas(n, _p(a), _p(b), _p(c), _p(d), _p(x), _p(cp), _p(dp))
    return x


def assemble(a, b, c):
    a, b, c = map(_f64, (a, b, c))
    n = b.size
    M = np.empty((n, n))
    _load().oracle_assemble(n, _p(a), _p(b), _p(c), _p(M))
    return M


def dense_ge(M, r):
    """Textbook dense Gaussian elimination with partial pivoting."""
    M = np.array(M, dtype=np.float64, order="C")
    r = np.array(r, dtype=np.float64)
    n = r.size
    x = np.empty(n)
    if _load().oracle_dense_ge(n, _p(M), _p(r), _p(x)) != 0:
        raise ZeroDivisionError("singular matrix")
    return x


def pcr_step(a, b, c, d, s):
    """One PCR step at stride s, Eqs 5-6, identity rows outside."""
    a, b, c, d = map(_f64, (a, b, c, d))
    n = b.size
    out = [np.empty(n) for _ in range(4)]
    _load().oracle_pcr_step(n, int(s), _p(a), _p(b), _p(c), _p(d), *map(_p, out))
    return tuple(out)


def pcr_k(a, b, c, d, k):
    """k PCR steps (strides 1..2^{k-1}); a[0], c[n-1] treated as 0."""
    a, b, c, d = map(_f64, (a, b, c, d))
    n = b.size
    out = [np.empty(n) for _ in range(4)]
    work = np.empty(4 * n)
    _load().oracle_pcr_k(n, int(k), _p(a), _p(b), _p(c), _p(d), *map(_p, out), _p(work))
    return tuple(out)


def residual(a, b, c, d, x):
    """(relative residual ||Ax-d||/||d||, normwise backward error), inf-norms,
    long-double accumulation; a[0], c[n-1] not read."""
    a, b, c, d, x = map(_f64, (a, b, c, d, x))
    out = np.empty(2)
    _load().oracle_residual(b.size, _p(a), _p(b), _p(c), _p(d), _p(x), _p(out))
    return float(out[0]), float(out[1])


def solve_batch(n, m, a, b, c, d, layout=0, want_resid=False, q_begin=0, q_end=None, nthreads=None):
    """x (f64, same layout) for every system; a, b, c, d may be f32 or f64
    (f32 upcast exactly).  Threads over systems (P:747 policy)."""
    assert a.dtype == b.dtype == c.dtype == d.dtype
    dt = 1 if a.dtype == np.float64 else 0
    if nthreads is None:
        nthreads = len(os.sched_getaffinity(0))
    q_end = m if q_end is None else q_end
    x = np.zeros(n * m, np.float64)
    res = np.zeros(2 * m, np.float64) if want_resid else None
    arrs = [np.ascontiguousarray(t) for t in (a, b, c, d)]
    rc = _load().oracle_solve_batch(int(n), int(m), dt, int(layout), *map(_p, arrs), _p(x),
                                    _p(res) if res is not None else None, int(q_begin), int(q_end),
                                    int(nthreads))
    if rc != 0:
        raise ValueError("oracle_solve_batch: bad arguments")
    return (x, res.reshape(m, 2)) if want_resid else x


def residual_batch(n, m, a, b, c, d, x, layout=0, nthreads=None):
    """Per-system (relative residual, backward error) of a given solution x
    (any float dtype; upcast to f64) -> array of shape (m, 2)."""
    assert a.dtype == b.dtype == c.dtype == d.dtype
    dt = 1 if a.dtype == np.float64 else 0
    if nthreads is None:
        nthreads = len(os.sched_getaffinity(0))
    xx = np.ascontiguousarray(x, dtype=np.float64)
    out = np.zeros(2 * m, np.float64)
    arrs = [np.ascontiguousarray(t) for t in (a, b, c, d)]
    rc = _load().oracle_residual_batch(int(n), int(m), dt, int(layout), *map(_p, arrs), _p(xx), _p(out),
                                       int(nthreads))
    if rc != 0:
        raise ValueError("oracle_residual_batch: bad arguments")
    return out.reshape(m, 2)
