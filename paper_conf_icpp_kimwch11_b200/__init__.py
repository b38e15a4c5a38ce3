"""B200-native hybrid tridiagonal solver (tiled PCR + p-Thomas; Kim, Wu, Chang,
Hwu, "A Scalable Tridiagonal Solver for GPUs", ICPP 2011).

Thin Python binding over the C ABI in include/tri.h (libtri.so, sm_100a).
Argument marshalling only: every step of the solve runs in the CUDA kernels.
There is no CPU fallback -- if libtri.so is missing or cannot load, importing
the binding raises.  PyTorch supplies device memory, streams and process
groups (plumbing only).
"""
import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TRI_LIB_PATH", os.path.join(HERE, "libtri.so"))  # override: experiments only

F32, F64 = 0, 1
CONTIGUOUS, INTERLEAVED, BATCHED, STRIDED = 0, 1, 2, 3
(VARIANT_AUTO, VARIANT_ONCHIP, VARIANT_SPLIT, VARIANT_FUSED, VARIANT_WARP, VARIANT_STREAM, VARIANT_SCAN,
 VARIANT_SCAN_MC) = 0, 1, 2, 3, 4, 5, 6, 7
VARIANT_NAMES = {1: "onchip", 2: "split", 3: "fused", 4: "warp", 5: "stream", 6: "scan", 7: "scan_mc"}
OPT_TMA, OPT_SCAN_MC_LOOKBACK, OPT_SCAN_CLUSTER, OPT_SCAN_GRID, OPT_SCAN_W512 = 1, 2, 3, 4, 5
STATUS = {0: "TRI_OK", 1: "TRI_ERR_INVALID_ARG", 2: "TRI_ERR_ALIGNMENT", 3: "TRI_ERR_ALIAS",
          4: "TRI_ERR_DEVICE", 5: "TRI_ERR_OOM", 6: "TRI_ERR_CUDA"}


class TriError(RuntimeError):
    def __init__(self, status, what=""):
        self.status = status
        super().__init__(f"{what}: {STATUS.get(status, status)}")


_lib = None
_P = ctypes.c_void_p
_I64 = ctypes.c_int64
_I = ctypes.c_int


def lib():
    """Load libtri.so (raises OSError if it is missing: no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise OSError(f"{LIB_PATH} not built; run __graft_entry__.build() "
                          "(python paper_conf_icpp_kimwch11_b200/_build.py)")
        L = ctypes.CDLL(LIB_PATH)
        sig = {
            "tri_plan": (_P, [_I64, _I64, _I, _I]),
            "tri_plan_batched": (_P, [_I64, _I64, _I64, _I]),
            "tri_plan_strided": (_P, [_I64, _I64, _I64, _I, _I64, _I64, _I64]),
            "tri_last_status": (_I, []),
            "tri_solve": (_I, [_P] * 7),
            "tri_solve_host": (_I, [_P] * 7),
            "tri_debug_pcr": (_I, [_P] * 9),
            "tri_destroy": (None, [_P]),
            "tri_plan_k": (_I, [_P]),
            "tri_plan_variant": (_I, [_P]),
            "tri_plan_launches": (_I, [_P]),
            "tri_plan_scratch_bytes": (_I64, [_P]),
            "tri_plan_set_k": (_I, [_P, _I]),
            "tri_plan_set_variant": (_I, [_P, _I]),
            "tri_plan_set_option": (_I, [_P, _I, _I]),
            "tri_plan_describe": (None, [_P, ctypes.c_char_p, _I]),
            "tri_status_str": (ctypes.c_char_p, [_I]),
            "tri_halo_f": (_I64, [_I]),
            "tri_halo_g": (_I64, [_I]),
            "tri_choose_k": (_I, [_I64, _I64, _I, _I, _I]),
            "tri_choose_variant": (_I, [_I64, _I64, _I, _I, _I]),
            "tri_shard_range": (None, [_I64, _I, _I, ctypes.POINTER(_I64), ctypes.POINTER(_I64)]),
            "tri_debug_set_profile": (None, [_P]),
            "tri_plan_autotune": (_I, [_P] * 7 + [_I, ctypes.POINTER(ctypes.c_float)]),
            "tri_slice_solve": (_I, [_P, _I, _I, _I] + [_P] * 7),
        }
        for name, (res, args) in sig.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def halo_f(k):
    """Eq 8."""
    return lib().tri_halo_f(k)


def halo_g(k):
    """Eq 9."""
    return lib().tri_halo_g(k)


def choose_k(n, m, dtype=F64, layout=CONTIGUOUS, sm_count=148):
    return lib().tri_choose_k(n, m, dtype, layout, sm_count)


def choose_variant(n, m, dtype=F64, layout=CONTIGUOUS, sm_count=148):
    return lib().tri_choose_variant(n, m, dtype, layout, sm_count)


def shard_range(m, G, r):
    """Contiguous system range (q0, m_r) of rank r among G (no collective in the solve)."""
    q0, mr = _I64(), _I64()
    lib().tri_shard_range(m, G, r, ctypes.byref(q0), ctypes.byref(mr))
    return q0.value, mr.value


def _dtype_code(dtype):
    import torch
    if dtype in (F64, "f64", torch.float64):
        return F64
    if dtype in (F32, "f32", torch.float32):
        return F32
    raise ValueError(f"unsupported dtype {dtype}")


class Plan:
    """Plan(n, m, dtype, layout) -> .solve(a, b, c, d, out=x) on CUDA tensors.

    Wraps tri_plan / tri_solve (include/tri.h).  The plan is bound to the CUDA
    device current at construction and owns its scratch."""

    def __init__(self, n, m, dtype=F64, layout=CONTIGUOUS, _batch=None, _strides=None):
        import torch
        self.n, self.m = int(n), int(m)
        self.dtype_code = _dtype_code(dtype)
        self.torch_dtype = torch.float64 if self.dtype_code == F64 else torch.float32
        self.layout = int(layout)
        self.strides = _strides
        if _strides is not None:
            ms, nb, es, ss, bs = _strides
            h = lib().tri_plan_strided(self.n, ms, nb, self.dtype_code, es, ss, bs)
        elif _batch is None:
            h = lib().tri_plan(self.n, self.m, self.dtype_code, self.layout)
        else:
            h = lib().tri_plan_batched(self.n, _batch[0], _batch[1], self.dtype_code)
        if not h:
            raise TriError(lib().tri_last_status(), "tri_plan")
        self._h = ctypes.c_void_p(h)
        self.device = torch.cuda.current_device()

    @classmethod
    def batched(cls, n, ms, nb, dtype=F64):
        """tri_plan_batched: nb batches of ms interleaved systems of size n (the
        y-lines of a row-major grid [nb][n][ms]; ADI)."""
        return cls(n, int(ms) * int(nb), dtype, BATCHED, _batch=(int(ms), int(nb)))

    @classmethod
    def strided(cls, n, ms, nb, es, ss, bs, dtype=F64):
        """tri_plan_strided: m = ms*nb systems of size n, element i of system
        q = b*ms + s at offset i*es + s*ss + b*bs of every array (lines of pitched /
        sub-grid views of a 3D array along any axis).  Solve
        with tensors whose data_ptr() is the view's origin (e.g. a sliced view
        of the parent array)."""
        strides = tuple(int(v) for v in (ms, nb, es, ss, bs))
        return cls(n, strides[0] * strides[1], dtype, STRIDED, _strides=strides)

    def footprint(self):
        """Elements from an array's base to its last element + 1."""
        if self.strides is None:
            return self.n * self.m
        ms, nb, es, ss, bs = self.strides
        return (self.n - 1) * es + (ms - 1) * ss + (nb - 1) * bs + 1

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and _lib is not None:
            _lib.tri_destroy(h)
            self._h = None

    @property
    def k(self):
        return lib().tri_plan_k(self._h)

    @k.setter
    def k(self, value):
        st = lib().tri_plan_set_k(self._h, int(value))
        if st != 0:
            raise TriError(st, f"tri_plan_set_k({value})")

    @property
    def variant(self):
        return lib().tri_plan_variant(self._h)

    @variant.setter
    def variant(self, v):
        st = lib().tri_plan_set_variant(self._h, int(v))
        if st != 0:
            raise TriError(st, f"tri_plan_set_variant({v})")

    @property
    def launches(self):
        return lib().tri_plan_launches(self._h)

    @property
    def scratch_bytes(self):
        return lib().tri_plan_scratch_bytes(self._h)

    def set_option(self, opt, value):
        """tri_plan_set_option: OPT_TMA (0 = SPLIT through the pre-TMA kernels),
        OPT_SCAN_MC_LOOKBACK (windows per look-back chunk, 0 = off),
        OPT_SCAN_CLUSTER (1 = interleaved SCAN through thread-block clusters),
        OPT_SCAN_GRID (0 = interleaved SCAN through the chained kernel, -1/1 = the
        grid-split kernel where it fits), OPT_SCAN_W512 (0 = fp64 contiguous SCAN
        with 256-row windows, -1/1 = 512-row windows where n % 16 == 0)."""
        st = lib().tri_plan_set_option(self._h, int(opt), int(value))
        if st != 0:
            raise TriError(st, f"tri_plan_set_option({opt}, {value})")

    def describe(self):
        buf = ctypes.create_string_buffer(512)
        lib().tri_plan_describe(self._h, buf, 512)
        return buf.value.decode()

    def _check(self, *ts):
        if self.strides is not None:  # views into larger arrays: the storage must hold the footprint
            need = self.footprint()
            for t in ts:
                avail = t.untyped_storage().nbytes() // t.element_size() - t.storage_offset()
                if not t.is_cuda or t.dtype != self.torch_dtype or avail < need:
                    raise ValueError(f"expected a CUDA {self.torch_dtype} view with >= {need} elements of storage "
                                     f"from its origin, got {t.dtype} on {t.device} ({avail} elements)")
            return
        for t in ts:
            if not t.is_cuda or t.dtype != self.torch_dtype or t.numel() != self.n * self.m \
                    or not t.is_contiguous():
                raise ValueError(f"expected contiguous CUDA {self.torch_dtype} tensor of {self.n * self.m} "
                                 f"elements, got {t.dtype} {tuple(t.shape)} on {t.device}")

    def solve(self, a, b, c, d, out=None, stream=None):
        import torch
        if out is None:
            if self.strides is not None:
                raise ValueError("strided plans need out= (a view with the plan's strides)")
            out = torch.empty_like(b)
        self._check(a, b, c, d, out)
        s = stream if stream is not None else torch.cuda.current_stream()
        st = lib().tri_solve(self._h, a.data_ptr(), b.data_ptr(), c.data_ptr(), d.data_ptr(),
                             out.data_ptr(), s.cuda_stream)
        if st != 0:
            raise TriError(st, "tri_solve")
        return out

    def solve_raw(self, a, b, c, d, x, stream=0):
        """tri_solve on raw device pointers (ints); returns the status code."""
        return lib().tri_solve(self._h, a, b, c, d, x, stream)

    def solve_host(self, a, b, c, d, out, stream=None):
        """End-to-end through host buffers (tri_solve_host): a..d, out are
        host tensors/arrays (pinned for bandwidth); copies are inside the call."""
        import numpy as np
        import torch
        np_dt = np.float64 if self.dtype_code == F64 else np.float32

        def ptr(t, what):
            # the C call reads / writes n*m elements of the plan's dtype through
            # raw host pointers: validate before handing them over
            if isinstance(t, torch.Tensor):
                ok = (t.device.type == "cpu" and t.dtype == self.torch_dtype and t.is_contiguous()
                      and t.numel() == self.n * self.m)
                p = t.data_ptr()
            elif isinstance(t, np.ndarray):
                ok = (t.dtype == np_dt and t.flags["C_CONTIGUOUS"] and t.size == self.n * self.m
                      and (what != "out" or t.flags["WRITEABLE"]))
                p = t.ctypes.data
            else:
                ok, p = False, 0
            if not ok:
                raise ValueError(f"solve_host {what}: expected a C-contiguous host tensor/array of "
                                 f"{self.n * self.m} {self.torch_dtype} elements, got {type(t).__name__} "
                                 f"{getattr(t, 'dtype', None)} {tuple(getattr(t, 'shape', ()))}")
            return p
        ps = [ptr(t, w) for t, w in zip((a, b, c, d, out), ("a", "b", "c", "d", "out"))]
        s = stream if stream is not None else torch.cuda.current_stream()
        st = lib().tri_solve_host(self._h, *ps, s.cuda_stream)
        if st != 0:
            raise TriError(st, "tri_solve_host")
        return out

    def autotune(self, a, b, c, d, out=None, reps=3, stream=None):
        """tri_plan_autotune: time every feasible (variant, k) on these device
        tensors and keep the fastest in the plan; returns its time in us."""
        import torch
        if out is None:
            out = torch.empty_like(b)
        self._check(a, b, c, d, out)
        s = stream if stream is not None else torch.cuda.current_stream()
        us = ctypes.c_float(0.0)
        st = lib().tri_plan_autotune(self._h, a.data_ptr(), b.data_ptr(), c.data_ptr(), d.data_ptr(),
                                     out.data_ptr(), s.cuda_stream, int(reps), ctypes.byref(us))
        if st != 0:
            raise TriError(st, "tri_plan_autotune")
        return us.value

    def slice_phase(self, phase, slice_, nslices, a=None, b=None, c=None, d=None, maps=None, out=None,
                    stream=None):
        """tri_slice_solve (NEXT-4): one phase of the solve of a system spread
        over devices; this plan (m = 1, SCAN_MC) holds one slice.  Phases 0 and
        1 return the slice's 8-value forward / backward map (device tensor),
        phase 2 writes and returns x of the slice."""
        import torch
        if phase < 2:
            self._check(a, b, c, d)
        if out is None:
            out = torch.empty(8 if phase < 2 else self.n, dtype=self.torch_dtype, device="cuda")
        s = stream if stream is not None else torch.cuda.current_stream()

        def ptr(t):
            return t.data_ptr() if t is not None else None
        st = lib().tri_slice_solve(self._h, int(phase), int(slice_), int(nslices), ptr(a), ptr(b), ptr(c), ptr(d),
                                   ptr(maps), out.data_ptr(), s.cuda_stream)
        if st != 0:
            raise TriError(st, f"tri_slice_solve(phase {phase})")
        return out

    def debug_pcr(self, a, b, c, d, stream=None):
        """Only the PCR stage: returns the k-step reduced system normalised to
        unit diagonal, (A, C, D) = (a'/b', c'/b', d'/b'), in the plan's layout."""
        import torch
        self._check(a, b, c, d)
        outs = [torch.empty_like(b) for _ in range(3)]
        s = stream if stream is not None else torch.cuda.current_stream()
        st = lib().tri_debug_pcr(self._h, a.data_ptr(), b.data_ptr(), c.data_ptr(), d.data_ptr(),
                                 *[o.data_ptr() for o in outs], s.cuda_stream)
        if st != 0:
            raise TriError(st, "tri_debug_pcr")
        return tuple(outs)


def solve(a, b, c, d, n, m, layout=CONTIGUOUS, out=None, k=None):
    """One-shot convenience: plan + solve on CUDA tensors."""
    p = Plan(n, m, b.dtype, layout)
    if k is not None:
        p.k = k
    return p.solve(a, b, c, d, out=out)
