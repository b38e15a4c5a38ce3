"""SURVEY 8(f) NEXT-3 (ADI / strided line solves; PAPER.md P:37 motivates the
solver with ADI and fluid simulation): tri_plan_strided on pitched and sub-grid
views of a 3D row-major array [NZ][NY][NX], lines along all three axes, fp64 and
fp32, on both paths -- the SCAN kernel through TMA tensor maps (pitches that are
16-byte multiples) and the packed fallback (odd pitches) -- against the oracle,
element by element.  Elements outside the view must be left untouched."""
import numpy as np
import pytest

import oracle
import trigen
from tests._helpers import TOL, max_rel_err

pytestmark = pytest.mark.gpu
tri = pytest.importorskip("paper_conf_icpp_kimwch11_b200")


def _lines(axis, nz, ny, nx, PZ, PY):
    """(n, ms, nb, es, ss, bs) of the lines along `axis` of a [nz][ny][nx] view
    with plane pitch PZ and row pitch PY (elements), and the index map
    (q, i) -> (z, y, x)."""
    if axis == "x":
        return (nx, ny, nz, 1, PY, PZ), lambda s, b, i: (b, s, i)
    if axis == "y":
        return (ny, nx, nz, PY, 1, PZ), lambda s, b, i: (b, i, s)
    return (nz, nx, ny, PZ, 1, PY), lambda s, b, i: (i, b, s)


CASES = [
    # (dtype, view (nz, ny, nx), parent (NZ, NY, NX), origin (z0, y0, x0)): NX / NY pitches
    ("f64", (5, 40, 64), (7, 44, 72), (1, 2, 4)),    # 16-byte multiples: TMA path on every axis
    ("f64", (6, 33, 48), (6, 33, 48), (0, 0, 0)),    # dense, ragged ny
    ("f32", (4, 64, 96), (5, 70, 100), (1, 3, 4)),   # fp32, pitch 100 (16-byte multiple)
    ("f64", (5, 24, 40), (6, 27, 43), (1, 1, 1)),    # odd pitches: packed fallback
    ("f32", (3, 40, 30), (4, 41, 31), (0, 1, 1)),    # odd pitches fp32
    ("f64", (3, 16, 1024), (3, 17, 1032), (0, 1, 8)),  # long x-lines (several SCAN windows)
    ("f64", (4, 32, 64), (5, 36, 72), (1, 2, 3)),    # 16-byte pitches, 8-byte-aligned origin: packed at solve
]


@pytest.mark.parametrize("axis", ["x", "y", "z"])
@pytest.mark.parametrize("dtype,view,parent,origin", CASES)
def test_strided_lines(cuda_ok, axis, dtype, view, parent, origin):
    import torch
    nz, ny, nx = view
    NZ, NY, NX = parent
    z0, y0, x0 = origin
    PZ, PY = NY * NX, NX
    (n, ms, nb, es, ss, bs), zyx = _lines(axis, nz, ny, nx, PZ, PY)
    m = ms * nb
    npdt = np.float64 if dtype == "f64" else np.float32
    arrs = trigen.generate(n, m, dtype, 0, "dd", seed=trigen.SEED_BASE + 31)  # system q = b ms + s, contiguous
    q = np.arange(m)
    s_, b_ = q % ms, q // ms
    i = np.arange(n)
    Z, Y, X = zyx(s_[:, None], b_[:, None], i[None, :])          # [m][n] coordinates in the view
    flat = ((Z + z0) * PZ + (Y + y0) * PY + (X + x0)).reshape(-1)  # parent element of (q, i)
    parents = []
    for t in arrs:
        P = np.full(NZ * NY * NX, np.nan, dtype=npdt)  # NaN outside the view: must never be read into x
        P[flat] = t
        parents.append(P)
    dev = [torch.from_numpy(P).cuda() for P in parents]
    xo_dev = torch.full((NZ * NY * NX,), -7.0, dtype=dev[0].dtype, device="cuda")
    off = z0 * PZ + y0 * PY + x0
    views = [t[off:] for t in dev]
    xv = xo_dev[off:]
    plan = tri.Plan.strided(n, ms, nb, es, ss, bs, tri.F64 if dtype == "f64" else tri.F32)
    plan.solve(*views, out=xv)
    torch.cuda.synchronize()
    xh = xo_dev.cpu().numpy()
    x = xh[flat]
    xo = oracle.solve_batch(n, m, *arrs, layout=0)
    assert max_rel_err(x, xo) <= TOL[dtype]["rel"], plan.describe()
    untouched = np.ones(xh.size, dtype=bool)
    untouched[flat] = False
    assert np.all(xh[untouched] == -7.0)  # only the view's elements are written


def test_strided_paths_and_rejects(cuda_ok):
    """The path each stride set takes (describe), and the calls a strided plan
    rejects."""
    import torch
    p = tri.Plan.strided(64, 40, 5, 1, 72, 44 * 72, tri.F64)
    assert "strided" in p.describe() and "packed" not in p.describe() and p.variant == tri.VARIANT_SCAN
    p = tri.Plan.strided(40, 24, 5, 1, 43, 27 * 43, tri.F64)
    assert "packed" in p.describe()
    p.k = 3  # the packed path's inner plan runs any k
    assert p.k == 3
    with pytest.raises(tri.TriError):
        tri.Plan.strided(64, 4, 2, 0, 1, 1, tri.F64)  # stride 0
    q = tri.Plan.strided(64, 40, 5, 1, 72, 44 * 72, tri.F64)
    small = torch.zeros(100, dtype=torch.float64, device="cuda")
    with pytest.raises(ValueError):
        q.solve(small, small, small, small, out=small)  # storage shorter than the footprint
