"""CPU tests of the C-ABI library: it loads without a GPU, exports every symbol
include/tri.h declares, and its pure host logic (halo formulas Eqs 8-9, the
transition heuristic, shard ranges, status strings) is right.  No compute calls."""
import ctypes
import os
import re

import pytest

import paper_conf_icpp_kimwch11_b200 as tri
from paper_conf_icpp_kimwch11_b200 import _build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    _build.build()
    return tri.lib()


def declared_symbols():
    hdr = open(os.path.join(ROOT, "include", "tri.h")).read()
    return sorted(set(re.findall(r"^TRI_API\s+[\w\s\*]+?\b(tri_\w+)\(", hdr, re.M)))


def test_header_declares_the_north_star_calls():
    syms = declared_symbols()
    for s in ("tri_plan", "tri_solve", "tri_destroy", "tri_plan_k", "tri_plan_set_k", "tri_status_str",
              "tri_last_status", "tri_solve_host"):
        assert s in syms


def test_library_exports_every_declared_symbol(L):
    for s in declared_symbols():
        assert hasattr(L, s), s
    # nothing else leaks (visibility=hidden): nm -D lists exactly the tri_ ABI
    import subprocess
    out = subprocess.run(["nm", "-D", "--defined-only", tri.LIB_PATH], capture_output=True, text=True).stdout
    exported = sorted(set(re.findall(r"\bT (tri_\w+)", out)))
    assert exported == declared_symbols()


def test_halo_formulas_match_paper_definitions(L):
    rows = [list(map(int, ln.split())) for ln in open(os.path.join(ROOT, "tests/golden/halo_eq8_eq9.txt"))
            if ln.strip() and not ln.startswith("#")]
    for k, f, g, cache in rows:
        assert tri.halo_f(k) == f          # Eq 8
        assert tri.halo_g(k) == g          # Eq 9
        assert 3 * tri.halo_f(k) == cache <= 3 * 2 ** k   # Table I
    # closed forms noted in SURVEY A7
    for k in range(0, 21):
        assert tri.halo_g(k) == (k - 2) * 2 ** k + 2


def test_status_strings(L):
    for code, name in tri.STATUS.items():
        assert L.tri_status_str(code).decode() == name


def test_plan_without_gpu_fails_cleanly(L):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    assert not L.tri_plan(1024, 4, tri.F64, tri.CONTIGUOUS)
    assert L.tri_last_status() == 4  # TRI_ERR_DEVICE
    assert not L.tri_plan(0, 4, tri.F64, tri.CONTIGUOUS)
    assert L.tri_last_status() == 1  # TRI_ERR_INVALID_ARG
    assert not L.tri_plan(16, 4, 7, tri.CONTIGUOUS)
    assert L.tri_last_status() == 1
    assert not L.tri_plan(16, 4, tri.F64, 9)
    assert L.tri_last_status() == 1
    assert not L.tri_plan_strided(64, 4, 2, tri.F64, 1, 64, 256)
    assert L.tri_last_status() == 4  # TRI_ERR_DEVICE (valid arguments, no GPU)
    for bad in [(64, 4, 2, tri.F64, 0, 64, 256), (64, 4, 2, tri.F64, 1, -1, 256), (0, 4, 2, tri.F64, 1, 64, 256),
                (64, 4, 2, 5, 1, 64, 256), (64, 4, 2, tri.F64, 1 << 50, 64, 256)]:
        assert not L.tri_plan_strided(*bad)
        assert L.tri_last_status() == 1, bad  # TRI_ERR_INVALID_ARG
    assert L.tri_plan_set_option(None, 1, 0) == 1
    assert L.tri_plan_set_option(None, 3, 1) == 1
    assert L.tri_plan_k(None) == -1
    L.tri_destroy(None)  # NULL-safe
    with pytest.raises(tri.TriError):
        tri.Plan(16, 4)


@pytest.mark.parametrize("dtype", [tri.F64, tri.F32])
@pytest.mark.parametrize("layout", [tri.CONTIGUOUS, tri.INTERLEAVED])
@pytest.mark.parametrize("n", [1, 2, 7, 256, 1024, 5000, 16384, 1 << 24])
def test_heuristic_k_valid_and_nonincreasing_in_m(L, dtype, layout, n):
    """Table III shape: k never grows as M grows; k <= floor(log2 n)."""
    prev = None
    for m in [1, 2, 16, 32, 100, 512, 1024, 4096, 16384, 1 << 20]:
        k = tri.choose_k(n, m, dtype, layout, 148)
        v = tri.choose_variant(n, m, dtype, layout, 148)
        assert v in (tri.VARIANT_ONCHIP, tri.VARIANT_SPLIT, tri.VARIANT_FUSED, tri.VARIANT_WARP, tri.VARIANT_STREAM,
                     tri.VARIANT_SCAN, tri.VARIANT_SCAN_MC)
        assert 0 <= k <= max(0, n.bit_length() - 1)
        if prev is not None:
            assert k <= prev[0], (n, m, k, prev)
        prev = (k, v)


def test_heuristic_paper_rule_extremes(L):
    """with M > P (plenty of systems) go straight to p-Thomas (k = 0);
    a single huge system gets deep PCR.  On B200 contiguous batches run p-Thomas
    as the SCAN kernel (k = 0, intermediates on chip: DESIGN.md planner table)."""
    assert tri.choose_k(16384, 16384, tri.F64, tri.INTERLEAVED, 148) == 0
    assert tri.choose_k(16384, 16384, tri.F32, tri.CONTIGUOUS, 148) == 0
    assert tri.choose_variant(16384, 16384, tri.F64, tri.CONTIGUOUS, 148) == tri.VARIANT_SCAN
    assert tri.choose_k(16384, 16384, tri.F64, tri.CONTIGUOUS, 148) == 0
    assert tri.choose_k(1 << 24, 1, tri.F64, tri.INTERLEAVED, 148) >= 8
    # one huge CONTIGUOUS system, any n: chunked SCAN (SCAN_MC) at k = 0; a ragged
    # n reads its last rows past the tensor map's 8-row groups directly
    assert tri.choose_variant((1 << 24) + 1, 1, tri.F64, tri.CONTIGUOUS, 148) == tri.VARIANT_SCAN_MC


@pytest.mark.parametrize("m,G", [(16384, 1), (16384, 8), (10, 4), (3, 8), (1, 2), (1000, 7)])
def test_shard_range_partitions(L, m, G):
    covered = []
    for r in range(G):
        q0, mr = tri.shard_range(m, G, r)
        assert mr >= 0
        covered += list(range(q0, q0 + mr))
    assert covered == list(range(m))


@pytest.mark.parametrize("cfg,n,m,dtype,layout,variant,k", [
    ("c1", 1024, 1, "F64", 0, "VARIANT_SCAN", 0),
    ("c2", 1024, 1024, "F64", 1, "VARIANT_SCAN", 0),
    ("c3", 1 << 24, 1, "F64", 0, "VARIANT_SCAN_MC", 0),
    ("c4", 256, 1 << 20, "F32", 0, "VARIANT_SCAN", 0),
    ("c5", 16384, 16384, "F64", 0, "VARIANT_SCAN", 0),
    ("c5/2", 16384, 8192, "F64", 0, "VARIANT_SCAN", 0),  # one of 2 ranks (strong scaling)
    ("c5/8", 16384, 2048, "F64", 0, "VARIANT_SCAN", 0),  # one of 8 ranks
    ("c5-il", 16384, 16384, "F64", 1, "VARIANT_SPLIT", 0),  # interleaved layout: k = 0 TMA p-Thomas
    ("c4-il", 256, 1 << 20, "F32", 1, "VARIANT_SCAN", 0),    # interleaved, one system per lane (S = 32)
    ("few-long", 65536, 37, "F64", 0, "VARIANT_SCAN_MC", 0),  # < 128 long systems: chunked SCAN
    ("few-long-il", 65536, 37, "F64", 1, "VARIANT_SPLIT", 8),  # interleaved: deep-k SPLIT
    ("odd-n", 1 << 20, 1, "F64", 0, "VARIANT_SCAN_MC", 0),
    ("ragged", (1 << 20) + 3, 1, "F64", 0, "VARIANT_SCAN_MC", 0),  # n % 8 != 0, one system: tail rows read directly
    ("ragged-batch", 1002, 4096, "F64", 0, "VARIANT_SCAN", 0),  # n % 8 != 0, 16-byte system pitch
    ("ragged-odd", 1001, 4096, "F64", 0, "VARIANT_WARP", 5),  # unaligned system starts: PCR in a warp + p-Thomas
])
def test_planner_picks_for_baseline_configs(L, cfg, n, m, dtype, layout, variant, k):
    """The planner's (variant, k) on a 148-SM B200 for BASELINE.json's configs,
    as calibrated by scripts/sweep_k.py, scripts/sweep_stream.py and
    scripts/sweep_scan.py (profiles/r01_sweep_*.jsonl)."""
    dt = getattr(tri, dtype)
    assert tri.choose_variant(n, m, dt, layout, 148) == getattr(tri, variant), cfg
    assert tri.choose_k(n, m, dt, layout, 148) == k, cfg


def test_planner_matches_sweeps(L):
    """The planner's (variant, k) against the committed B200 sweeps (SURVEY 8(f)
    NEXT-2; profiles/r02_sweep_scan*.jsonl: every whole-solve variant (SCAN_MC
included) timed on a
    grid of the paper's shapes): geometric-mean slowdown vs the fastest measured
    variant <= 5 %, no shape worse than 1.6x (the worst are few-microsecond
    solves)."""
    import glob
    import json
    import math
    ratios = []
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "r02_sweep_scan*.jsonl")))
    assert files
    skipped = 0
    for f in files:
        for line in open(f):
            r = json.loads(line)
            dt = tri.F64 if r["dtype"] == "f64" else tri.F32
            lay = r.get("layout", 0)
            v = tri.choose_variant(r["n"], r["m"], dt, lay, 148)
            k = tri.choose_k(r["n"], r["m"], dt, lay, 148)
            recs = r["all"] + [r["auto"]]
            mine = [x["us"] for x in recs if x["variant"] == v and (v != tri.VARIANT_SPLIT or x["k"] == k)]
            if not mine:
                skipped += 1
                continue
            ratios.append(min(mine) / min(x["us"] for x in recs))
    assert skipped == 0 and len(ratios) > 150
    geo = math.exp(sum(math.log(q) for q in ratios) / len(ratios))
    assert geo <= 1.05, geo
    assert max(ratios) <= 1.6, max(ratios)


def test_planner_grid_rule_matches_sweeps(L):
    """Interleaved SCAN through k_scan_grid (one wave of 32-system blocks x <= 8
    row pieces): on every swept shape with n > 256 where it fits
    (profiles/r02_sweep_grid_f64.jsonl, L2 flushed per replay) the planner picks
    SCAN and the grid kernel is no slower than the chained kernel (within the
    event timer's 2 us quantum); beyond one wave (r02_sweep_grid_multiwave_*) the
    chained kernel wins on the larger shapes, which is why the rule stops at one wave."""
    import json
    one = [json.loads(x) for x in open(os.path.join(ROOT, "profiles", "r02_sweep_grid_f64.jsonl"))]
    one = [r for r in one if r["n"] > 256]
    assert len(one) >= 10
    for r in one:
        assert tri.choose_variant(r["n"], r["m"], tri.F64, 1, 148) == tri.VARIANT_SCAN, r
        assert r["grid_us"] <= r["chained_us"] + 2.1, r
    multi = [json.loads(x) for x in open(os.path.join(ROOT, "profiles", "r02_sweep_grid_multiwave_f64.jsonl"))]
    big = [r for r in multi if (r["m"] + 31) // 32 * r["Q"] > 2 * 148]
    assert big and all(r["grid_us"] > r["chained_us"] for r in big)
