/*
 * tri.h -- C ABI of the B200 (sm_100a) hybrid tridiagonal solver.
 *
 * Operation (Sec. II.A, Eq 1): for each of m independent
 * systems q, solve A_q x_q = d_q where A_q is n x n tridiagonal with
 * sub-diagonal a (a_2..a_n), diagonal b (b_1..b_n) and super-diagonal c
 * (c_1..c_{n-1}).  Method (Sec. III): k steps of tiled parallel
 * cyclic reduction (Eqs 5-6 at stride 2^j) split every
 * system into 2^k interleaved independent subsystems, then thread-level
 * parallel Thomas (Eqs 2-4) solves each subsystem with one
 * thread.  The transition point k is chosen at plan time from n, m, the dtype
 * and the SM count; tri_plan_set_k overrides it.  At k = 0 (the
 * paper's rule for M > P) the planner's SCAN / SCAN_MC variants run
 * p-Thomas with each system spread over a warp's lanes (the forward sweep and
 * back substitution as scans of segment maps, reading X21).
 *
 * Conventions common to every call:
 *   - Element (system q, row i), 0 <= q < m, 0 <= i < n, lives at
 *       TRI_LAYOUT_CONTIGUOUS :  [q*n + i]   (system-major)
 *       TRI_LAYOUT_INTERLEAVED:  [i*m + q]   (the paper's interleave)
 *       TRI_LAYOUT_BATCHED    :  [(b*n + i)*ms + s] for q = b*ms + s (tri_plan_batched)
 *     in each of a, b, c, d, x; every array holds n*m elements of the dtype.
 *   - a[q][0] and c[q][n-1] lie outside A (Eq 1) and are IGNORED (read as 0,
 *     whatever they hold, including NaN) -- DESIGN.md reading X1.
 *   - No pivoting: the precondition is diagonal dominance (or SPD); numerical
 *     breakdown is not detected (reading X6).
 *   - No exceptions cross the ABI; every fallible call returns a tri_status.
 *   - All device pointers must be 16-byte aligned device allocations on the
 *     plan's device; x must not overlap a, b, c or d.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *     tri_solve is stream-ordered and asynchronous.
 *   - Determinism: a given (plan, inputs) gives bitwise-identical x every run.
 */
#ifndef TRI_H
#define TRI_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define TRI_API __attribute__((visibility("default")))
#else
#define TRI_API
#endif

typedef enum { TRI_F32 = 0, TRI_F64 = 1 } tri_dtype;

typedef enum {
    TRI_LAYOUT_CONTIGUOUS = 0,  /* element i of system q at [q*n + i] */
    TRI_LAYOUT_INTERLEAVED = 1, /* element i of system q at [i*m + q] */
    TRI_LAYOUT_BATCHED = 2,     /* nb batches of ms interleaved systems (only through tri_plan_batched):
                                   element i of system q = b*ms + s at [(b*n + i)*ms + s]; e.g. the
                                   y-lines of a row-major grid [nb][n][ms] (ADI) */
    TRI_LAYOUT_STRIDED = 3      /* caller's strides (only through tri_plan_strided): element i of system
                                   q = b*ms + s at [i*es + s*ss + b*bs] (elements); lines of pitched and
                                   sub-grid views of 3D arrays along any axis */
} tri_layout;

typedef enum {
    TRI_OK = 0,
    TRI_ERR_INVALID_ARG = 1, /* bad n, m, dtype, layout, k, variant, NULL pointer */
    TRI_ERR_ALIGNMENT = 2,   /* a device pointer not 16-byte aligned */
    TRI_ERR_ALIAS = 3,       /* x overlaps a, b, c or d */
    TRI_ERR_DEVICE = 4,      /* no CUDA device / not sm_100 / pointer not on the plan's device */
    TRI_ERR_OOM = 5,         /* scratch or staging allocation failed */
    TRI_ERR_CUDA = 6         /* a CUDA runtime call or kernel launch failed */
} tri_status;

/* Kernel variants; the planner picks one, tests may force. */
typedef enum {
    TRI_VARIANT_AUTO = 0,   /* only as an argument of tri_plan_set_variant */
    TRI_VARIANT_ONCHIP = 1, /* whole system(s) in one CTA's smem: PCR + Thomas (Fig 11a/c) */
    TRI_VARIANT_SPLIT = 2,  /* tiled-PCR pass (sliding window, Figs 8-10) -> scratch, then p-Thomas */
    TRI_VARIANT_FUSED = 3,  /* streaming tiled PCR feeding p-Thomas in one kernel (Sec. III.C) */
    TRI_VARIANT_WARP = 4,   /* 32 <= n <= 1024: one warp per system, k = 5 shuffle PCR steps + in-register
                               p-Thomas on the 32 subsystems (Sec. III) */
    TRI_VARIANT_STREAM = 5  /* CONTIGUOUS fp64, n % 8 == 0, n >= 512: tiled PCR (k = 3, TMA-staged 256-row
                               windows with 8-row halos, Eq 8 / Fig 7) streamed into p-Thomas in one
                               persistent kernel; c', d' stay in shared memory / L2, so HBM moves only
                               the compulsory 5 arrays (Sec. III.C) */,
    TRI_VARIANT_SCAN = 6    /* CONTIGUOUS (or m = 1), n % 8 == 0: p-Thomas at k = 0 (M > P) with the
                               forward sweep (Eqs 2-3) and back substitution (Eq 4) of each system spread
                               over the 32 lanes of a warp as segment maps combined by a shuffle scan
                               (X21); 256-row windows chained across warps, c', d' kept in
                               shared memory / L2: HBM moves only the compulsory 5 arrays */,
    TRI_VARIANT_SCAN_MC = 7 /* CONTIGUOUS (or m = 1), n % 8 == 0, few long systems: the SCAN solve with every
                               system cut into chunks over several CTAs; three streaming passes (chunk
                               forward maps; forward replay -> c', d'; back substitution) linked by two
                               scans over the chunk maps (X21): 13 arrays of HBM traffic */
} tri_variant;

typedef struct tri_plan_s* tri_plan_t;

/* Create a plan for m systems of size n on the CURRENT CUDA device.
 * n >= 1, m >= 1, n*m <= 2^40.  Chooses k and the variant, allocates the
 * plan-owned device scratch.  Returns NULL on failure; tri_last_status() says
 * why (TRI_ERR_INVALID_ARG, TRI_ERR_DEVICE, TRI_ERR_OOM, TRI_ERR_CUDA). */
TRI_API tri_plan_t tri_plan(int64_t n, int64_t m, tri_dtype dtype, tri_layout layout);

/* Thread-local status of the last tri_plan call on this thread. */
TRI_API tri_status tri_last_status(void);

/* Solve A x = d for the plan's m systems (Eq 1).  a, b, c, d: device
 * pointers (read-only) to n*m elements of the plan's dtype in the plan's layout
 * (CONTIGUOUS: system q row i at q*n + i; INTERLEAVED: at i*m + q); a of row 0
 * and c of row n-1 are ignored (never read into arithmetic).  x: device output,
 * same shape.  All five must be 16-byte aligned (TRI_ERR_ALIGNMENT), non-NULL
 * (TRI_ERR_INVALID_ARG), on the plan's device (TRI_ERR_DEVICE; verified when
 * the pointer set differs from the previous call's) and x must not overlap an
 * input (TRI_ERR_ALIAS).  On error nothing is launched.  Asynchronous on
 * `stream` (a cudaStream_t; NULL = legacy default stream); launch failures
 * return TRI_ERR_CUDA.  At most one tri_solve per plan may be in flight (the
 * plan's scratch is reused); use one plan per concurrent stream.  The caller
 * owns every buffer; the plan owns its scratch. */
TRI_API tri_status tri_solve(tri_plan_t plan, const void* a, const void* b, const void* c, const void* d,
                     void* x, void* stream);

/* End-to-end solve through HOST buffers: copies a, b, c, d host->device into
 * plan-owned staging, solves, copies x device->host, then synchronises
 * `stream`.  CONTIGUOUS batches of m >= 32 run as a pipeline of 16 chunks of
 * systems (H2D of chunk i+1, solve of chunk i and D2H of chunk i-1 overlap, on
 * plan-owned streams ordered after the caller's prior work on `stream`); other
 * shapes copy, solve and copy back on `stream`.  Host buffers should be pinned
 * for full bandwidth.  Returns after x is in host memory. */
TRI_API tri_status tri_solve_host(tri_plan_t plan, const void* a, const void* b, const void* c,
                          const void* d, void* x, void* stream);

/* Run only the tiled-PCR stage (k steps, Eqs 5-6 at strides 1..2^{k-1}) and
 * write the reduced system, rows normalised to unit diagonal (a/b, 1, c/b,
 * d/b; reading X17), into ao, co, do_ in the plan's layout.  For
 * tests of SURVEY 8(a) row A2.  Same pointer rules as tri_solve. */
TRI_API tri_status tri_debug_pcr(tri_plan_t plan, const void* a, const void* b, const void* c,
                         const void* d, void* ao, void* co, void* do_, void* stream);

/* Diagnostics: when dev_counters (device memory, 16 x uint64, zeroed by the
 * caller) is non-NULL, the fused kernel accumulates per-role clock64() cycle
 * counters into it (layout: scripts/prof_fused.py).  The environment variable
 * TRI_FUSED_DBG_MODE, read here, disables parts of the fused kernel for cost
 * attribution (results are then wrong).  Process-wide; NULL disables. */
TRI_API void tri_debug_set_profile(void* dev_counters);

/* Autotune the plan (the paper tunes its transition point once per machine,
 * P:743): time every feasible (variant, k) for the plan's
 * shape on the caller's device buffers (same rules as tri_solve; x is
 * overwritten) -- for SCAN also with TRI_OPT_SCAN_GRID / TRI_OPT_SCAN_W512 off
 * where the planner's geometry uses those kernels -- `reps` solves each after
 * one warm-up, CUDA events on `stream`, and keep the fastest in the plan.  Candidates whose scratch cannot be
 * allocated are skipped.  *best_us (may be NULL) receives the fastest mean
 * time per solve in microseconds.  Synchronises `stream`. */
TRI_API tri_status tri_plan_autotune(tri_plan_t plan, const void* a, const void* b, const void* c,
                                     const void* d, void* x, void* stream, int reps, float* best_us);

/* Plan for the BATCHED layout: nb batches, each an INTERLEAVED block of ms
 * systems of size n (m = ms * nb systems).  Lines of a 3D row-major grid
 * [nz][ny][nx] (ADI): along x is CONTIGUOUS (n = nx, m =
 * ny nz), along z is INTERLEAVED (n = nz, m = nx ny), along y is this layout
 * (n = ny, ms = nx, nb = nz).  ms = 1 and nb = 1 reduce to CONTIGUOUS /
 * INTERLEAVED plans.  Otherwise the plan runs the SCAN kernel (k = 0) and needs
 * ms * sizeof(dtype) to be a multiple of 16 bytes (TMA row stride) and n <=
 * 131072 (4096 windows of 32 rows); else NULL with TRI_ERR_INVALID_ARG.  The
 * solve semantics, pointer rules and ownership are those of tri_solve. */
TRI_API tri_plan_t tri_plan_batched(int64_t n, int64_t ms, int64_t nb, tri_dtype dtype);

/* Plan for arbitrary element / system / batch strides (ADI
 * line solves on pitched and sub-grid views of a 3D array).  m = ms * nb
 * systems of size n; element i of system q = b*ms + s (0 <= s < ms, 0 <= b < nb)
 * is at element offset i*es + s*ss + b*bs from each array's base pointer (a, b,
 * c, d and x alike; the base may point into a larger array).  All strides >= 1
 * and the caller guarantees distinct elements (no two (q, i) at one offset).
 * For lines of a row-major array [nz][ny][nx] with row pitch py and plane pitch
 * pz (elements): x-lines (n, ms, nb, es, ss, bs) = (nx, ny, nz, 1, py, pz);
 * y-lines (ny, nx, nz, py, 1, pz); z-lines (nz, nx, ny, pz, 1, py).
 * Runs the SCAN kernel (k = 0) directly on the caller's arrays when a TMA
 * tensor map can describe them -- es == 1 (n % 8 == 0) or ss == 1 (ms > 1), the
 * other strides 16-byte multiples; otherwise (odd pitches) a gather kernel packs
 * a, b, c, d into plan-owned dense arrays, an inner plan solves them and x is
 * scattered back (2 extra passes over the data); a TMA-path plan switches to the
 * packed path at the first solve whose view origins are not 16-byte aligned.
 * Pointers: element-aligned device pointers; x must not overlap the inputs'
 * footprint (TRI_ERR_ALIAS).
 * tri_solve_host, tri_debug_pcr and tri_plan_autotune return
 * TRI_ERR_INVALID_ARG for these plans; tri_plan_set_k runs k = 0 on the TMA path
 * and any k on the packed one.  NULL with TRI_ERR_INVALID_ARG for bad sizes or
 * strides < 1. */
TRI_API tri_plan_t tri_plan_strided(int64_t n, int64_t ms, int64_t nb, tri_dtype dtype, int64_t es, int64_t ss,
                                    int64_t bs);

/* One system spread over several devices.
 * Device r holds rows [r0, r0 + n) of the system -- a contiguous slice, n % 8
 * == 0, n > 256 -- in a plan made with tri_plan(n, 1, dtype, CONTIGUOUS) and
 * set to TRI_VARIANT_SCAN_MC.  The slice's forward sweep is a 3x3 map of the
 * incoming continuant state and its back substitution an affine map of the x
 * after it (X21), so the devices exchange only 8 values each, twice:
 *   phase 0: a, b, c, d (device, the slice) -> out = the slice's forward map
 *            (8 values of dtype, device);
 *   [all-gather the nslices forward maps, in slice order, into `maps`]
 *   phase 1: a, b, c, d, maps -> out = the slice's backward map (8 values);
 *   [all-gather the backward maps into `maps`]
 *   phase 2: maps -> out = x of the slice (n values, device).
 * The first row of slice r > 0 keeps its a (coupled to slice r - 1) and the
 * last row of slice r < nslices - 1 keeps its c.  Asynchronous on `stream`;
 * phases run in order on one plan; the plan's scratch carries c', d' from
 * phase 1 to phase 2.  TRI_ERR_INVALID_ARG for a plan that is not SCAN_MC with
 * m == 1 and TRI_OPT_SCAN_MC_LOOKBACK 0, a bad phase / slice, or a NULL pointer. */
TRI_API tri_status tri_slice_solve(tri_plan_t plan, int phase, int slice, int nslices, const void* a,
                                   const void* b, const void* c, const void* d, const void* maps, void* out,
                                   void* stream);

/* Release the plan and its scratch.  NULL-safe.  Must not race a solve. */
TRI_API void tri_destroy(tri_plan_t plan);

/* Plan introspection and overrides. */
TRI_API int tri_plan_k(tri_plan_t plan);                     /* chosen transition point k, -1 if NULL */
TRI_API int tri_plan_variant(tri_plan_t plan);               /* tri_variant in use, -1 if NULL */
TRI_API int tri_plan_launches(tri_plan_t plan);              /* kernels launched per tri_solve */
TRI_API int64_t tri_plan_scratch_bytes(tri_plan_t plan);     /* plan-owned device scratch */
/* Force the transition point k (Sec. III.D: k is the method's
 * knob), any 0 <= k <= floor(log2 n); else TRI_ERR_INVALID_ARG (so any k > 0
 * when n = 1).  When the plan's variant does not run this k (SCAN / SCAN_MC
 * run k = 0; STREAM k = 3, FUSED k = 4, WARP k = 5 only), the plan switches
 * to the first variant in the order SCAN, SCAN_MC, STREAM, FUSED, WARP,
 * ONCHIP (systems that fit a CTA, fewer than 48 x SMs of them), SPLIT that
 * runs it -- SPLIT runs every k (tiled-PCR passes of <= 10, then <= 5 steps).
 * TRI_LAYOUT_BATCHED plans run k = 0 only.  May reallocate scratch
 * (TRI_ERR_OOM, plan unchanged).  A forced k (or variant) is kept by the
 * chunk sub-plans of tri_solve_host. */
TRI_API tri_status tri_plan_set_k(tri_plan_t plan, int k);
/* Force a variant (TRI_VARIANT_AUTO re-runs the planner); re-plans k if the
 * current k is invalid for it; may reallocate scratch (TRI_ERR_OOM). */
TRI_API tri_status tri_plan_set_variant(tri_plan_t plan, tri_variant v);
/* Plan options (explicit per plan; nothing is read from the environment):
 *   TRI_OPT_TMA (default 1): 0 runs SPLIT through its pre-TMA kernels: the
 *     paper's shared-memory sliding-window tiled PCR (Figs 8-10) instead of the
 *     register-tile passes, and the non-TMA p-Thomas kernels (cp.async /
 *     ring-staged / thread-per-chain), which otherwise run only where a TMA
 *     descriptor cannot describe the arrays; for A/B measurement and tests.
 *   TRI_OPT_SCAN_MC_LOOKBACK (default -1 = auto): SCAN_MC passes 0 and 1 fused
 *     by a decoupled look-back over chunks of `value` windows (1 <= value <= 64;
 *     0 = the three-pass form; auto = the three-pass form, measured faster on
 *     B200).  tri_slice_solve needs it off (0 or auto).
 *   TRI_OPT_SCAN_CLUSTER (default 0): 1 solves INTERLEAVED SCAN batches of at
 *     most one 8-system group per SM (m <= 8 x SMs, n >= 512, n <= 16384) with
 *     one thread-block cluster of 2-8 CTAs per group, the group's windows
 *     spread over the cluster's warps and the forward state / x handed between
 *     its CTAs through distributed shared memory (P:687
 *     Fig 11b).  Off by default: measured slower than the chained kernel at c2
 *     (27.5 vs 21.0 us).
 *   TRI_OPT_SCAN_GRID (default -1 = auto = on where it fits): INTERLEAVED
 *     (and unit-system-stride BATCHED / STRIDED) SCAN batches whose 32-system
 *     blocks split into Q <= 8 row pieces of 16 warps x <= 16 rows with every
 *     block's thread-block cluster of Q CTAs resident at once (one wave) run
 *     k_scan_grid: each lane owns one system's run of rows, the whole batch is
 *     in flight at once, and the Q CTAs of a block exchange their forward /
 *     backward aggregate maps through distributed shared memory; 0 = the
 *     chained 8-system-window kernel; 1 = also batches of several waves
 *     (Q <= 8; measured slower than the chained kernel beyond one wave).
 *   TRI_OPT_SCAN_W512 (default -1 = auto = on): fp64 CONTIGUOUS SCAN batches
 *     with n % 16 == 0 and at least two 512-row windows run k_scan_w512 (16 rows
 *     per lane, 512-row windows: the per-window scans and handover paid once
 *     per 512 rows); 0 = the 256-row-window kernel; 1 = as auto.
 * TRI_ERR_INVALID_ARG for an unknown option or value; TRI_ERR_OOM if the new
 * geometry's scratch cannot be allocated (option unchanged). */
typedef enum {
    TRI_OPT_TMA = 1,
    TRI_OPT_SCAN_MC_LOOKBACK = 2,
    TRI_OPT_SCAN_CLUSTER = 3,
    TRI_OPT_SCAN_GRID = 4,
    TRI_OPT_SCAN_W512 = 5
} tri_option;
TRI_API tri_status tri_plan_set_option(tri_plan_t plan, tri_option opt, int value);
/* Human-readable one-line plan description into buf (NUL-terminated). */
TRI_API void tri_plan_describe(tri_plan_t plan, char* buf, int buflen);

TRI_API const char* tri_status_str(tri_status s);

/* ---- pure host helpers (no device needed; unit-testable on CPU) ---------- */
/* Eq 8: redundant loads per tile boundary f(k) = sum_{i<k} 2^i. */
TRI_API int64_t tri_halo_f(int k);
/* Eq 9: redundant eliminations g(k) = k f(k) - sum_{i<=k} f(i). */
TRI_API int64_t tri_halo_g(int k);
/* The planner's heuristic (Sec. III.D, re-derived for B200 in
 * DESIGN.md): transition point k for (n, m, dtype, layout) on sm_count SMs. */
TRI_API int tri_choose_k(int64_t n, int64_t m, tri_dtype dtype, tri_layout layout, int sm_count);
/* The planner's variant choice for the same arguments (a tri_variant). */
TRI_API int tri_choose_variant(int64_t n, int64_t m, tri_dtype dtype, tri_layout layout, int sm_count);
/* Contiguous shard of m systems for rank r of G (multi-GPU):
 * q0 = r*ceil(m/G) clipped to m, mr = min(ceil(m/G), m - q0). */
TRI_API void tri_shard_range(int64_t m, int G, int r, int64_t* q0, int64_t* mr);

#ifdef __cplusplus
}
#endif

#endif /* TRI_H */
