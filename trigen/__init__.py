"""Seeded, counter-based synthetic inputs for tridiagonal batches (shared by the
oracle side and the CUDA side of every parity test; holds none of the solve's
arithmetic).  See trigen.c for the recipe; DESIGN.md "Input recipe".

Arrays follow PAPER.md P:65-89 (Eq 1): a = sub-diagonal, b = diagonal,
c = super-diagonal, d = right-hand side; a[0] and c[n-1] lie outside A.
"""
import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "trigen.c")
_LIB = os.path.join(_HERE, "libtrigen.so")

DD, WEAK, INTEGER, POISSON = 0, 1, 2, 3
FAMILIES = {"dd": DD, "weak": WEAK, "integer": INTEGER, "poisson": POISSON}
CONTIGUOUS, INTERLEAVED = 0, 1
SEED_BASE = 0x7A1D0000  # seed = 0x7A1D0000 + config_id


def build(force=False):
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-o", _LIB, _SRC, "-lm"])
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.trigen_generate.restype = ctypes.c_int
        lib.trigen_generate.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
                                        ctypes.c_double, ctypes.c_uint64, ctypes.c_int, ctypes.c_int,
                                        ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                        ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int]
        lib.trigen_mix.restype = ctypes.c_uint64
        lib.trigen_mix.argtypes = [ctypes.c_uint64]
        _lib = lib
    return _lib


def _ptr(arr):
    return ctypes.c_void_p(arr.ctypes.data) if arr is not None else None


def generate(n, m, dtype="f64", layout=CONTIGUOUS, family="dd", eps=1e-2, seed=SEED_BASE,
             q0=0, m_total=None, want_xstar=False, nthreads=0, out=None):
    """Return (a, b, c, d[, xstar]) as flat numpy arrays of n*m elements.

    Systems are the GLOBAL systems [q0, q0+m); values do not depend on layout,
    q0 split or thread count.  `out` may pass preallocated (a, b, c, d) arrays
    (e.g. pinned host memory viewed as numpy)."""
    fam = FAMILIES[family] if isinstance(family, str) else int(family)
    npdt = np.float64 if dtype in ("f64", 1, np.float64) else np.float32
    dt = 1 if npdt is np.float64 else 0
    N = int(n) * int(m)
    if out is None:
        a, b, c, d = (np.empty(N, npdt) for _ in range(4))
    else:
        a, b, c, d = out
        for t in out:
            assert t.dtype == npdt and t.size == N and t.flags.c_contiguous
    xs = np.empty(N, np.float64) if want_xstar else None
    rc = _load().trigen_generate(int(n), int(q0), int(m), fam, float(eps), int(seed) & (2**64 - 1), dt,
                                 int(layout), _ptr(a), _ptr(b), _ptr(c), _ptr(d), _ptr(xs), int(nthreads))
    if rc != 0:
        raise ValueError("trigen_generate: bad arguments")
    return (a, b, c, d, xs) if want_xstar else (a, b, c, d)


def mix(z):
    return int(_load().trigen_mix(int(z) & (2**64 - 1)))
