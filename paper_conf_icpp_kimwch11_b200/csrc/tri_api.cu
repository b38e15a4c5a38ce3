// tri_api.cu -- the C ABI of include/tri.h: planner (transition point k and
// variant, Sec. III.D, re-derived for B200 in DESIGN.md),
// argument validation, scratch ownership and dispatch to the per-family
// launchers (l_*.cu).  No kernel is instantiated here.
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -shared (see _build.py).
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "plan.cuh"
// constants and layouts only (no instantiation in this translation unit)
#include "common.cuh"
#include "k_fused.cuh"
#include "k_scan.cuh"
#include "k_scan_mc.cuh"
#include "k_scan_grid.cuh"
#include "k_scan_w512.cuh"
#include "k_stream.cuh"
#include "k_tiled_pcr.cuh"
#include "k_warp.cuh"

using namespace tri;
using namespace trih;

namespace {

thread_local tri_status g_last = TRI_OK;

constexpr int64_t MAX_ELEMS = int64_t(1) << 40;
// SCAN: back-substitution lag in steps (a window is read back >= delta + 1 steps
// after its store; 0..8 measured equal at c1 / c2 in round 1; 24 -- the lag at
// which the handover barrier chain alone would order every slot -- measured 3 %
// slower at c5 and 8 % at c2, so the slots keep their release / acquire table)
constexpr int SCAN_DELTA = 8;
#ifndef S32_F64_NMAX
#define S32_F64_NMAX 256           // fp64 interleaved: the longest systems the planner sends to S = 32
#endif
#ifndef S32_ENABLE
#define S32_ENABLE 1               // interleaved SCAN with 32 systems per window (A/B macro)
#endif
#ifndef S5_DELTA
#define S5_DELTA 8                 // k_scan_w512's lag (A/B macro)
#endif

// ---- pure host planner ------------------------------------------------------
// Rows of (normalised, 3-array) system data one ONCHIP CTA holds: sized for
// 3 resident CTAs per SM (72 KiB each) so loads of one CTA overlap compute of
// another.
int64_t onchip_rows_budget(tri_dtype t) { return t == TRI_F64 ? 3072 : 6144; }

int onchip_G(int64_t n, int64_t m, tri_dtype t, int sms) {
    int64_t G = std::max<int64_t>(1, std::min<int64_t>(onchip_rows_budget(t) / n, m));
    // keep >= 2 CTAs per SM when the batch allows it (wave balance, H6)
    if (cdiv(m, G) < 2 * (int64_t)sms) G = std::max<int64_t>(1, cdiv(m, 2 * (int64_t)sms));
    G = std::min<int64_t>(G, std::max<int64_t>(1, onchip_rows_budget(t) / n));
    return (int)G;
}

// FUSED needs the contiguous layout (or m = 1) and systems of >= 2 windows.
bool fused_ok(int64_t n, int64_t m, tri_layout layout) {
    return (layout == TRI_LAYOUT_CONTIGUOUS || m == 1) && n >= 2 * FU_W;
}

// WARP: 32 <= n <= 32 x WARP_RMAX rows, one system per warp (registers only).
constexpr int64_t WARP_RMAX = 32;
bool warp_ok(int64_t n, tri_layout layout) {
    return n >= 32 && n <= 32 * WARP_RMAX && layout != TRI_LAYOUT_BATCHED;
}

// STREAM: fp64, contiguous (or one system), n a multiple of 8 (the TMA tensor
// view [rows/8][8]), 8 .. 1024 windows of 240 rows (slot barriers, k_stream.cuh);
// tensor rows fit int32.
bool stream_ok(int64_t n, int64_t m, tri_dtype t, tri_layout layout) {
    return t == TRI_F64 && (layout == TRI_LAYOUT_CONTIGUOUS || m == 1) && n % 8 == 0 && n >= 2 * SK_W &&
           cdiv(n, SK_V) >= 8 && cdiv(n, SK_V) <= SK_NCMAX && (n / 8) * m < ((int64_t)1 << 31);
}

bool onchip_ok(int64_t n, tri_dtype t, tri_layout layout) {
    return n <= onchip_rows_budget(t) && layout != TRI_LAYOUT_BATCHED;
}

// SCAN: systems per window: 1 (contiguous), 8 (interleaved / batched: a window's
// row of 8 systems is 64 B fp64 / 32 B fp32, at least one whole DRAM sector per
// TMA row; S = 2 fp64 measured 2x slower: half sectors)
int scan_systems(tri_layout layout, int64_t m) {
    return (layout == TRI_LAYOUT_CONTIGUOUS || (layout == TRI_LAYOUT_INTERLEAVED && m == 1)) ? 1 : 8;
}
bool scan_ok(int64_t n, int64_t m, tri_dtype t, tri_layout layout, int64_t ms = -1) {
    if (layout == TRI_LAYOUT_BATCHED) {
        const int S = scan_systems(layout, m);
        return ms > 0 && (ms * (int64_t)esize(t)) % 16 == 0 && cdiv(n, SC_W / S) <= SC_NCMAX &&
               n < ((int64_t)1 << 31) && ms < ((int64_t)1 << 31) && m / ms < ((int64_t)1 << 31);
    }
    // CONTIGUOUS: n % 8 == 0, or ragged n of more than one window whose system
    // starts stay 16-byte aligned (one system, or n s % 16 == 0): the kernels read
    // the rows past the tensor map's last 8-row group directly (sc_patch_tail)
    if (layout == TRI_LAYOUT_CONTIGUOUS || m == 1)
        return (n % 8 == 0 || (n > SC_W && (m == 1 || (n * (int64_t)esize(t)) % 16 == 0))) &&
               cdiv(n, SC_W) <= SC_NCMAX && n / 8 < ((int64_t)1 << 31) && m < ((int64_t)1 << 31);
    // INTERLEAVED: TMA tensor [n][m], row stride m * s a multiple of 16 bytes
    const int S = scan_systems(layout, m);
    return (m * (int64_t)esize(t)) % 16 == 0 && cdiv(n, SC_W / S) <= SC_NCMAX && n < ((int64_t)1 << 31) &&
           m < ((int64_t)1 << 31);
}

// SCAN_MC: as SCAN, for systems of at least two windows.
bool scan_mc_ok(int64_t n, int64_t m, tri_dtype t, tri_layout layout) {
    return (layout == TRI_LAYOUT_CONTIGUOUS || m == 1) && (n % 8 == 0 || m == 1 || (n * (int64_t)esize(t)) % 16 == 0) &&
           n > SC_W && n / 8 < ((int64_t)1 << 31) && m < ((int64_t)1 << 31);
}

// STRIDED plans: the SCAN kernel through TMA maps when the caller's strides allow
// it -- unit element stride (x-lines: 4D view [nb][ms][n/8][8], n % 8 == 0) or unit
// system stride (y / z-lines: 3D view [nb][n][ms], 8 systems per window) -- with
// every other stride a 16-byte multiple; else the packed fallback (l_strided.cu)
bool strided_fast(int64_t n, int64_t ms, int64_t nb, tri_dtype t, int64_t es, int64_t ss, int64_t bs) {
    const int64_t sz = (int64_t)esize(t);
    const int64_t tma_stride = int64_t(1) << 40;  // a tensor map's byte strides must stay below 2^40
    if (es * sz >= tma_stride || ss * sz >= tma_stride || bs * sz >= tma_stride) return false;
    const bool bok = nb == 1 || (bs * sz) % 16 == 0;
    if (es == 1 && n % 8 == 0 && (ms == 1 || (ss * sz) % 16 == 0) && bok && cdiv(n, SC_W) <= SC_NCMAX &&
        n / 8 < ((int64_t)1 << 31) && ms < ((int64_t)1 << 31) && nb < ((int64_t)1 << 31))
        return true;
    if (ss == 1 && ms > 1 && (es * sz) % 16 == 0 && bok && cdiv(n, SC_W / 8) <= SC_NCMAX && n < ((int64_t)1 << 31) &&
        ms < ((int64_t)1 << 31) && nb < ((int64_t)1 << 31))
        return true;
    return false;
}

// Interleaved SCAN with one system per lane (32 systems x 8 rows per window,
// 256-byte TMA rows, no lane scans): a 32-system group's (c', d') slots
// (cdiv(n, 8) + delta windows) live in the CTA's shared memory, the overflow in an
// L2-resident spill of <= 24 MB over all CTAs, and there is a group for every SM.
bool s32_ok(int64_t n, int64_t m, tri_dtype t, int sms) {
    if (!S32_ENABLE) return false;
    const int64_t nc32 = cdiv(n, SC_W / 32), groups = cdiv(m, 32);
    if (nc32 > SC_NCMAX || groups < sms || n >= ((int64_t)1 << 31)) return false;
    // smem_optin is not known here: the B200's 227 KB per CTA
    const int64_t optin = 232448, slot = SC_W * 2 * (int64_t)esize(t);
    const int64_t fixed = t == TRI_F64 ? SCLayout<double>::smem_bytes((int)nc32, SCAN_DELTA, 0)
                                       : SCLayout<float>::smem_bytes((int)nc32, SCAN_DELTA, 0);
    const int64_t on_chip = std::max<int64_t>(0, (optin - fixed) / slot);
    const int64_t spill = std::max<int64_t>(0, nc32 + SCAN_DELTA - on_chip) * slot * std::min<int64_t>(groups, sms);
    return spill <= ((int64_t)24 << 20);
}

// the arithmetic part of k_scan_grid's feasibility (scan_grid_geometry adds the
// cluster occupancy check on the device)
bool grid_shape_ok(int64_t n, int64_t m, int sms) {
    const int64_t nblk = cdiv(m, 32), Q = cdiv(n, (int64_t)SG_NW * SG_RMAX);
    return m >= 8 && Q <= SG_QMAX && nblk * Q <= sms;
}

bool variant_ok(tri_variant v, const tri_plan_s* p) {
    if (p->layout == TRI_LAYOUT_STRIDED) return v == TRI_VARIANT_SCAN && !p->inner;
    switch (v) {
        case TRI_VARIANT_ONCHIP: return onchip_ok(p->n, p->dtype, p->layout);
        case TRI_VARIANT_SPLIT: return p->layout != TRI_LAYOUT_BATCHED;
        case TRI_VARIANT_FUSED: return fused_ok(p->n, p->m, p->layout);
        case TRI_VARIANT_WARP: return warp_ok(p->n, p->layout);
        case TRI_VARIANT_STREAM: return stream_ok(p->n, p->m, p->dtype, p->layout);
        case TRI_VARIANT_SCAN: return scan_ok(p->n, p->m, p->dtype, p->layout, p->ms);
        case TRI_VARIANT_SCAN_MC: return scan_mc_ok(p->n, p->m, p->dtype, p->layout);
        default: return false;
    }
}

// Variant choice, calibrated once on B200 (the paper tunes P once) from
// scripts/sweep_k.py / sweep_scan.py (profiles/r01_sweep_*.jsonl): every
// (variant, k) timed over the paper's shape grid (fixed n with m swept, fixed m
// with n swept).  See DESIGN.md §1 for the evidence behind each rule.
tri_variant choose_variant(int64_t n, int64_t m, tri_dtype t, tri_layout layout, int sms) {
    if (layout == TRI_LAYOUT_BATCHED) return TRI_VARIANT_SCAN;  // the only kernel for this layout
    // SCAN (profiles/r02_sweep_scan_*_0.jsonl): fastest, or within a few percent,
    // on every contiguous shape with n % 8 == 0 of the grid n = 256 .. 2^20 x
    // m = 1 .. 2^20 (fp64 and fp32), except fewer than 128 systems of 32 windows
    // or more, where one CTA per system leaves SMs idle; e.g. n = m = 16384 fp64:
    // 1.84 ms vs 2.92 ms (STREAM).  k = 0 throughout: the paper's M > P rule.
    // ... except fp32 batches of many systems of 2-4 windows, where the chained
    // fp32 windows (half the bytes of an fp64 step behind the same chain latency)
    // lose to the TMA p-Thomas at k = 0 (r02 sweep: n = 512, m = 151552: 395 vs
    // 539 us; n = 1024, m = 37888: 235 vs 268 us; equal from n = 2048)
    if (layout == TRI_LAYOUT_CONTIGUOUS && t == TRI_F32 && n > 256 && n <= 1024 && m >= 256 * (int64_t)sms)
        return TRI_VARIANT_SPLIT;
    if (layout == TRI_LAYOUT_CONTIGUOUS && scan_ok(n, m, t, layout) && (cdiv(n, SC_W) < 32 || m >= 128))
        return TRI_VARIANT_SCAN;
    // SCAN_MC: the remaining contiguous shapes (fewer than 128 systems of 32 windows
    // or more) -- every system split over several SMs (r02 sweep: n = 16384, m = 1:
    // 12.3 us vs 30.9 us SCAN; n = 8192, m = 16: 14.4 vs 18.5; n = 2^20, m = 1: 25 us
    // vs 1.6 ms; beats deep-k SPLIT on all of them: n = 2^24, m = 1: 0.29 ms vs 1.05 ms).
    if (layout == TRI_LAYOUT_CONTIGUOUS && scan_mc_ok(n, m, t, layout)) return TRI_VARIANT_SCAN_MC;
    // SCAN on the INTERLEAVED layout (8 adjacent systems per window;
    // profiles/r02_sweep_scan_*_1.jsonl): fastest from 256 systems of more than 256
    // rows (n = 256: WARP's in-register PCR is 1.2-1.6x faster) up to where the
    // 8-system groups' intermediates stop fitting on chip / in L2 (fp64 n m >= 2^27:
    // SPLIT k = 0 1.07x faster at 8192 x 16384) or, fp32, where many systems favour
    // one thread per system (m > 16384: SPLIT k = 0 1.06-1.11x faster); e.g. c2
    // 1024 x 1024: 23 us vs 28 us (WARP); 4096 x 4096: 170 us vs 879 us.
    // ... and from fewer systems where the whole batch fits the grid kernel (k_scan_grid:
    // 32-system blocks x <= 8 row pieces of <= 256 rows, one CTA per SM; r02
    // sweep_grid: n = 1024, m = 64: 14.4 us vs 18.4 us ONCHIP; n = 2048, m = 64: 16.4
    // vs 28.7; n <= 256 stays with WARP / ONCHIP, 1.2-1.5x faster there)
    if (layout == TRI_LAYOUT_INTERLEAVED && (n > 256 || (n >= 128 && m >= (t == TRI_F64 ? 1024 : 4096))) &&
        scan_ok(n, m, t, layout) && grid_shape_ok(n, m, sms))
        return TRI_VARIANT_SCAN;  // (n = 128 .. 256, larger m: fp64 n = 256, m = 4096: 14.4 vs 22.2 us WARP)
    if (layout == TRI_LAYOUT_INTERLEAVED && m >= 256 && n > 256 && scan_ok(n, m, t, layout)) {
        const int64_t N = n * m;
        const bool fits = t == TRI_F64 ? N < ((int64_t)1 << 27) : N < ((int64_t)1 << 28) && m <= 16384;
        if (fits) return TRI_VARIANT_SCAN;
    }
    // ... and many short interleaved systems, one system per lane (s32_ok;
    // profiles/r02_sweep_s32.jsonl, back-to-back replays): fp64 n <= 128 and fp32
    // 128 <= n <= 512 beat SPLIT k = 0 / WARP (fp64 n = 128, m = 2^20: 0.86 vs 1.22 ms;
    // fp32 n = 256, m = 2^20 (c4 interleaved): 1.35 vs 1.51 ms); fp32 n <= 64 does not
    if (layout == TRI_LAYOUT_INTERLEAVED && scan_ok(n, m, t, layout) && s32_ok(n, m, t, sms) &&
        (t == TRI_F64 ? n <= S32_F64_NMAX : n >= 128 && n <= 512))
        return TRI_VARIANT_SCAN;
    // STREAM (profiles/r01_sweep_stream_f64.jsonl): fp64 contiguous batches with
    // n % 8 == 0 are all taken by SCAN / SCAN_MC above; kept for completeness of
    // the rule list (the paper's fused PCR + p-Thomas, selectable).
    if (layout == TRI_LAYOUT_CONTIGUOUS && stream_ok(n, m, t, layout) && (m >= 64 || n <= 8192)) return TRI_VARIANT_STREAM;
    if (m >= 48 * (int64_t)sms) return TRI_VARIANT_SPLIT;
    const bool contig = layout == TRI_LAYOUT_CONTIGUOUS;
    if (contig && fused_ok(n, m, layout) && n >= 1024 && (n <= 2048 || m >= 128)) return TRI_VARIANT_FUSED;
    if (warp_ok(n, layout) && m >= (contig ? 1024 : (int64_t)sms)) return TRI_VARIANT_WARP;
    if (onchip_ok(n, t, layout)) return TRI_VARIANT_ONCHIP;
    return TRI_VARIANT_SPLIT;
}

// Transition point.  Paper rule: M > P => k = 0; otherwise the largest k
// with 2^k M <= P; B200 P = 64 chains per SM.  Measured refinement: below P the
// extra PCR steps stop paying once the subsystems are ~32 rows long (n = 8192,
// m = 1: k = 8 in 25 us vs k = 13 in 76 us), so k <= floor(log2 n) - 5.
int choose_k_for(tri_variant v, int64_t n, int64_t m, tri_dtype t, int sms) {
    const int kmax_n = floor_log2(n);
    if (v == TRI_VARIANT_ONCHIP) {
        const int G = onchip_G(n, m, t, sms);
        int k = ceil_log2(cdiv(64, G));
        return std::min(k, kmax_n);
    }
    if (v == TRI_VARIANT_FUSED) return FU_K;
    if (v == TRI_VARIANT_STREAM) return SK_K;
    if (v == TRI_VARIANT_WARP) return WARP_K;
    if (v == TRI_VARIANT_SCAN || v == TRI_VARIANT_SCAN_MC) return 0;
    const int64_t P = (int64_t)sms * 64;
    if (m >= 48 * (int64_t)sms) return 0;
    int k = m >= P ? 0 : ceil_log2(cdiv(P, m));
    k = std::min(k, std::max(0, kmax_n - 5));
    return std::min(std::min(k, kmax_n), 15);
}

// the k range a variant runs
int kmax_for(tri_variant v, int64_t n) {
    if (v == TRI_VARIANT_FUSED) return FU_K;
    if (v == TRI_VARIANT_STREAM) return SK_K;
    if (v == TRI_VARIANT_WARP) return WARP_K;
    if (v == TRI_VARIANT_SCAN || v == TRI_VARIANT_SCAN_MC) return 0;
    return floor_log2(n);  // ONCHIP, SPLIT: any k
}
int kmin_for(tri_variant v) {
    return v == TRI_VARIANT_FUSED ? FU_K : v == TRI_VARIANT_STREAM ? SK_K : v == TRI_VARIANT_WARP ? WARP_K : 0;
}

// ---- per-plan geometry -----------------------------------------------------
// SCAN on a unit-system-stride layout (8-system windows) through k_scan_grid when
// every 32-system block's rows split into Q <= 8 pieces of 16 warps x R rows (one
// thread-block cluster per block) and all the clusters are resident at once (one
// wave; cudaOccupancyMaxActiveClusters -- clusters of 8 need 8 free SMs of one
// GPC): R = 4 .. 16, the smallest that fits (the most SMs stream).  Off with
// TRI_OPT_SCAN_GRID 0.
void scan_grid_geometry(tri_plan_s* p) {
    p->sg_Q = p->sg_R = p->sg_bpb = 0;
    if (p->sk_S != 8 || p->opt_grid == 0 || p->n >= ((int64_t)1 << 30)) return;
    const int64_t bpb = cdiv(p->ms, 32), nblk = bpb * p->nb;
    for (int R = SG_SR; R <= SG_RMAX; R += SG_SR) {
        const int64_t Q = cdiv(p->n, (int64_t)SG_NW * R);
        if (Q <= SG_QMAX && nblk * Q <= p->sms && scan_grid_fits(p, (int)Q, R, nblk)) {
            p->sg_Q = (int)Q;
            p->sg_R = R;
            p->sg_bpb = (int)bpb;
            return;
        }
    }
    // TRI_OPT_SCAN_GRID 1: also batches of several waves (clusters are independent:
    // no co-residency needed), with the longest runs per warp (fewest CTAs)
    if (p->opt_grid == 1) {
        const int64_t Q = cdiv(p->n, (int64_t)SG_NW * SG_RMAX);
        if (Q <= SG_QMAX) {
            int R = SG_SR;
            while (cdiv(p->n, (int64_t)SG_NW * R) > Q) R += SG_SR;
            p->sg_Q = (int)Q;
            p->sg_R = R;
            p->sg_bpb = (int)bpb;
        }
    }
}

void plan_geometry(tri_plan_s* p) {
    const int64_t n = p->n, m = p->m;
    p->tmc.clear();
    p->s5 = 0;  // SCAN kernel choices: set again below when the variant is SCAN
    p->sg_Q = p->sg_R = p->sg_bpb = 0;
    if (p->variant == TRI_VARIANT_WARP) {
        int R = 1;
        while (32 * (int64_t)R < n) R *= 2;
        p->rpt = R;
        p->G = 0; p->P = 0; p->n_pad = 32 * (int64_t)R; p->L = R; p->C = m * 32;
        return;
    }
    if (p->variant == TRI_VARIANT_ONCHIP) {
        p->G = onchip_G(n, m, p->dtype, p->sms);
        // pad the per-system smem stride so the p-Thomas walk (lanes = chains,
        // chain r of system g at g*P + r + j 2^k) hits distinct banks
        const int S = 1 << p->k;
        const int mod = p->dtype == TRI_F64 ? 16 : 32;
        int P = (int)n;
        if (S < 32) while ((P % mod) != (S % mod)) ++P;
        p->P = P;
        const int64_t rows = (int64_t)p->G * n;
        int rpt = 1;
        while ((int64_t)rpt * 512 < rows) rpt *= 2;
        p->rpt = rpt;
        p->n_pad = n; p->L = 0; p->C = 0;
        return;
    }
    if (p->variant == TRI_VARIANT_SPLIT) {
        split_geometry(p);
        return;
    }
    if (p->variant == TRI_VARIANT_STREAM) {
        p->L = cdiv(n, SK_S);
        p->n_pad = p->L * SK_S;
        p->C = m * SK_S;
        p->sk_nc = (int)cdiv(n, SK_V);
        p->sk_grid = (int)std::min<int64_t>(m, p->sms);
        const int64_t avail = ((int64_t)p->smem_optin - SKLayout<double>::off_store - 1024) / SKLayout<double>::slot_bytes;
        p->sk_son = (int)std::max<int64_t>(0, std::min<int64_t>(p->sk_nc, avail));
    }
    if (p->variant == TRI_VARIANT_SCAN) {
        p->L = n; p->n_pad = n; p->C = m;
        p->sk_S = p->layout == TRI_LAYOUT_STRIDED ? (p->es == 1 ? 1 : 8) : scan_systems(p->layout, m);
        // many short interleaved systems: one system per lane (32 per window of 8 rows,
        // 256-byte TMA rows, no lane scans) when a group's (c', d') slots fit the CTA's
        // shared memory and there are groups for every SM
        if (p->sk_S == 8 && p->nb == 1 && p->layout == TRI_LAYOUT_INTERLEAVED && s32_ok(n, m, p->dtype, p->sms))
            p->sk_S = 32;
        p->sk_nc = (int)cdiv(n, SC_W / p->sk_S);
        const int64_t ms = p->ms;
        const int64_t groups = p->sk_S == 1 ? m : cdiv(ms, p->sk_S) * (m / ms);
        p->sk_grid = (int)std::min<int64_t>(groups, p->sms);
        // the back-substitution lag only matters when a CTA's slots are reused by a
        // later system: with one system (group) per CTA the backward sweep starts right
        // after the forward one (c1: no chain of idle steps)
        const bool one_per_cta = groups <= p->sms;
        p->sk_delta = one_per_cta ? 0 : SCAN_DELTA;
        const int fixed = SCLayout<double>::smem_bytes(p->sk_nc, p->sk_delta, 0);
        const int fixed32 = SCLayout<float>::smem_bytes(p->sk_nc, p->sk_delta, 0);
        const int slot = p->dtype == TRI_F64 ? SCLayout<double>::slot_bytes : SCLayout<float>::slot_bytes;
        const int64_t avail = ((int64_t)p->smem_optin - (p->dtype == TRI_F64 ? fixed : fixed32)) / slot;
        p->sk_son = (p->sk_nc == 1 && p->sk_S == 1) ? 0 : (int)std::max<int64_t>(0, std::min<int64_t>(p->sk_nc + p->sk_delta, avail));
        scan_grid_geometry(p);
        // fp64 contiguous batches of >= 2 windows of 512 rows (n % 16: the 128-byte
        // tensor rows): k_scan_w512, 16 rows per lane (the per-window scans, handover
        // and bookkeeping paid once per 512 rows)
        p->s5 = 0;
        if (p->opt_w512 != 0 && p->dtype == TRI_F64 && p->layout == TRI_LAYOUT_CONTIGUOUS && p->sk_S == 1 &&
            p->n % 16 == 0 && cdiv(n, S5_W) >= 2 && cdiv(n, S5_W) <= SC_NCMAX) {
            p->s5 = 1;
            p->sk_nc = (int)cdiv(n, S5_W);
            p->sk_delta = one_per_cta ? 0 : S5_DELTA;
            const int64_t av5 = ((int64_t)p->smem_optin - S5Layout::smem_bytes(p->sk_nc, p->sk_delta, 0)) / S5Layout::slot_bytes;
            p->sk_son = (int)std::max<int64_t>(0, std::min<int64_t>(p->sk_nc + p->sk_delta, av5));
        }
    }
    if (p->variant == TRI_VARIANT_SCAN_MC) {
        p->L = n; p->n_pad = n; p->C = m;
        const int64_t NC = cdiv(n, SC_W);
        p->sk_nc = (int)NC;
        int64_t P = std::max(cdiv(p->sms, m), cdiv(NC, SMC_WMAX));
        P = std::min(P, NC);
        int64_t NCW = cdiv(NC, P);
        p->mc_lb = 0; p->mc_NCWs = 0; p->mc_Ps = 0;
        // the look-back path (9 arrays) only when asked for: measured slower than the
        // three passes (13 arrays) at c3 -- 0.35 vs 0.29 ms; the look-back latency
        // (~15 us per chunk, waiting on the predecessors' phase A across CTAs) and
        // the latency-bound per-warp replay leave HBM idle; -1 = auto = off
        const int lbw = p->opt_lookback < 0 ? 0 : p->opt_lookback;
        if (lbw >= 1 && lbw <= LB_MAXW) {
            // pass 2's chunks are unions of the look-back's small chunks
            p->mc_lb = 1;
            p->mc_NCWs = lbw;
            p->mc_Ps = (int)cdiv(NC, p->mc_NCWs);
            NCW = std::min<int64_t>(SMC_WMAX / p->mc_NCWs * p->mc_NCWs, cdiv(NCW, p->mc_NCWs) * p->mc_NCWs);
        }
        p->mc_NCW = (int)NCW;
        p->mc_P = (int)cdiv(NC, NCW);
        p->sk_grid = (int)(m * p->mc_P);
    }
    if (p->variant == TRI_VARIANT_FUSED) {
        const size_t s = esize(p->dtype);
        p->L = cdiv(n, FU_S);
        p->n_pad = p->L * FU_S;
        p->C = m * FU_S;
        p->fu_nc = cdiv(p->n_pad, FU_V);
        p->fu_grid = (int)std::min<int64_t>(m, p->sms);
        const bool vec = (n % 8) == 0;  // the staged (cp.async) path; pointers checked at launch
        p->fu_vec = vec;
        const int fixed = p->dtype == TRI_F64
                              ? fused_fixed_smem<double>() + (vec ? fused_stage_smem<double>() : 0)
                              : fused_fixed_smem<float>() + (vec ? fused_stage_smem<float>() : 0);
        const int64_t avail = ((int64_t)p->smem_optin - fixed) / (int64_t)(FU_S * 2 * s);
        p->fu_son = (int)std::max<int64_t>(0, std::min<int64_t>(p->L, avail));
    }
}

size_t scratch_need(const tri_plan_s* p) {
    const size_t es = esize(p->dtype);
    if (p->variant == TRI_VARIANT_SCAN_MC)  // c', d' per window, the fp64 chunk maps, 16 slice values (+ the
                                            // fp64 look-back records and their flags)
        return (size_t)p->m * (size_t)p->sk_nc * (size_t)sc_slot_elems<double>() * es +
               (size_t)p->m * (size_t)p->mc_P * 16 * 8 + 16 * es +
               (p->mc_lb ? (size_t)p->m * (size_t)p->mc_Ps * (SMC_REC * 8 + 4) +
                               (size_t)p->m * (size_t)((p->mc_Ps + 31) / 32) * (8 * 8 + 4) + 256 : 0);
    if (p->variant == TRI_VARIANT_SCAN && p->sg_Q > 0) return 0;  // k_scan_grid: no global scratch
    if (p->variant == TRI_VARIANT_SCAN && p->s5)  // k_scan_w512: spilled 8 KB slots per CTA
        return (size_t)p->sk_grid * (size_t)std::max(0, p->sk_nc + p->sk_delta - p->sk_son) * S5Layout::slot_bytes;
    if (p->variant == TRI_VARIANT_SCAN)
        return (p->sk_nc == 1 && p->sk_S == 1) ? 0
                             : (size_t)p->sk_grid * (size_t)std::max(0, p->sk_nc + p->sk_delta - p->sk_son) *
                                   (size_t)sc_slot_elems<double>() * es;
    if (p->variant == TRI_VARIANT_STREAM)
        return (size_t)p->sk_grid * (size_t)std::max(0, p->sk_nc - p->sk_son) * SK_SLOT * es;
    if (p->variant == TRI_VARIANT_FUSED)
        return (size_t)p->fu_grid * 2 * (size_t)std::max<int64_t>(0, p->L - p->fu_son) * FU_S * 2 * es;
    if (p->variant == TRI_VARIANT_SPLIT) return split_scratch(p);
    return 0;
}

tri_status ensure_scratch(tri_plan_s* p) {
    const size_t need = scratch_need(p);
    if (need <= p->scratch_bytes) return TRI_OK;
    if (p->scratch) cudaFree(p->scratch);
    p->scratch = nullptr;
    p->scratch_bytes = 0;
    if (cudaMalloc(&p->scratch, need) != cudaSuccess) {
        cudaGetLastError();
        return TRI_ERR_OOM;
    }
    // defined contents once per allocation: padding columns of storage slots are
    // copied (never used) by whole-slot bulk prefetches (compute-sanitizer initcheck)
    if (cudaMemset(p->scratch, 0, need) != cudaSuccess) {
        cudaGetLastError();
        cudaFree(p->scratch);
        p->scratch = nullptr;
        return TRI_ERR_CUDA;
    }
    p->scratch_bytes = need;
    return TRI_OK;
}

// switch to (v, k) with rollback on failure
tri_status set_plan(tri_plan_s* p, tri_variant v, int k) {
    const tri_variant ov = p->variant;
    const int ok = p->k;
    p->variant = v;
    p->k = k;
    plan_geometry(p);
    const tri_status st = ensure_scratch(p);
    if (st != TRI_OK) { p->variant = ov; p->k = ok; plan_geometry(p); }
    return st;
}

// STRIDED packed fallback: gather into the dense layout whose order follows the
// source's unit stride (rows -> CONTIGUOUS, systems -> INTERLEAVED), solve with an
// inner plan, scatter x (l_strided.cu)
tri_status make_packed(tri_plan_s* p);

tri_status check_ptrs(tri_plan_s* p, const void* const* in, int nin, const void* const* out, int nout) {
    // footprint of an array: its last element's offset + 1 (n m for the dense layouts)
    const size_t bytes = (size_t)((p->n - 1) * p->es + (p->ms - 1) * p->ss + (p->nb - 1) * p->bs + 1) * esize(p->dtype);
    bool same = nin + nout <= 8;
    for (int i = 0; i < nin + nout && same; ++i) same = p->seen[i] == (i < nin ? in[i] : out[i - nin]);
    for (int i = 0; i < nin + nout; ++i) {
        const void* q = i < nin ? in[i] : out[i - nin];
        if (!q) return TRI_ERR_INVALID_ARG;
        // STRIDED views may start anywhere (element-aligned); tri_solve picks the path
        if (((uintptr_t)q & (p->layout == TRI_LAYOUT_STRIDED ? esize(p->dtype) - 1 : 15)) != 0) return TRI_ERR_ALIGNMENT;
        if (same) continue;  // residency verified on the previous call with these pointers
        cudaPointerAttributes at;
        if (cudaPointerGetAttributes(&at, q) != cudaSuccess) { cudaGetLastError(); return TRI_ERR_DEVICE; }
        if ((at.type != cudaMemoryTypeDevice && at.type != cudaMemoryTypeManaged) || at.device != p->device)
            return TRI_ERR_DEVICE;
    }
    for (int o = 0; o < nout; ++o) {
        const uintptr_t x0 = (uintptr_t)out[o], x1 = x0 + bytes;
        for (int i = 0; i < nin; ++i) {
            const uintptr_t a0 = (uintptr_t)in[i], a1 = a0 + bytes;
            if (x0 < a1 && a0 < x1) return TRI_ERR_ALIAS;
        }
        for (int o2 = 0; o2 < o; ++o2) {
            const uintptr_t y0 = (uintptr_t)out[o2], y1 = y0 + bytes;
            if (x0 < y1 && y0 < x1) return TRI_ERR_ALIAS;
        }
    }
    if (!same && nin + nout <= 8) {
        for (int i = 0; i < 8; ++i) p->seen[i] = i < nin + nout ? (i < nin ? in[i] : out[i - nin]) : nullptr;
    }
    return TRI_OK;
}

tri_status current_device_ok(int* dev, int* sms) {
    int count = 0;
    if (cudaGetDeviceCount(&count) != cudaSuccess || count == 0) { cudaGetLastError(); return TRI_ERR_DEVICE; }
    if (cudaGetDevice(dev) != cudaSuccess) { cudaGetLastError(); return TRI_ERR_DEVICE; }
    int major = 0, minor = 0;
    cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, *dev);
    cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, *dev);
    cudaDeviceGetAttribute(sms, cudaDevAttrMultiProcessorCount, *dev);
    if (major != 10 || minor != 0) return TRI_ERR_DEVICE;  // kernels are sm_100a only
    return TRI_OK;
}

tri_plan_s* new_plan(int64_t n, int64_t m, int64_t ms, tri_dtype dtype, tri_layout layout, tri_status* st);

tri_status make_packed(tri_plan_s* p) {
    const tri_layout il = (p->ss == 1 && p->es != 1) ? TRI_LAYOUT_INTERLEAVED : TRI_LAYOUT_CONTIGUOUS;
    tri_status st;
    p->inner = new_plan(p->n, p->m, p->m, p->dtype, il, &st);
    if (!p->inner) return st;
    p->variant = p->inner->variant;
    p->k = p->inner->k;
    const size_t bytes = 5 * ((size_t)p->n * (size_t)p->m * esize(p->dtype) / 256 * 256 + 256);
    if (cudaMalloc(&p->packbuf, bytes) != cudaSuccess) { cudaGetLastError(); return TRI_ERR_OOM; }
    p->packbuf_bytes = bytes;
    return TRI_OK;
}

tri_plan_s* new_plan(int64_t n, int64_t m, int64_t ms, tri_dtype dtype, tri_layout layout, tri_status* st) {
    int dev = 0, sms = 0;
    *st = current_device_ok(&dev, &sms);
    if (*st != TRI_OK) return nullptr;
    tri_plan_s* p = new tri_plan_s();
    p->n = n; p->m = m; p->ms = ms; p->dtype = dtype; p->layout = layout; p->device = dev; p->sms = sms;
    p->nb = m / ms;
    if (layout == TRI_LAYOUT_CONTIGUOUS) { p->es = 1; p->ss = n; p->bs = n * m; }
    else if (layout == TRI_LAYOUT_INTERLEAVED) { p->es = m; p->ss = 1; p->bs = n * m; }
    else { p->es = ms; p->ss = 1; p->bs = n * ms; }  // BATCHED
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    p->smem_optin = (size_t)optin;
    p->variant = choose_variant(n, m, dtype, layout, sms);
    p->k = choose_k_for(p->variant, n, m, dtype, sms);
    plan_geometry(p);
    *st = ensure_scratch(p);
    if (*st != TRI_OK) { delete p; return nullptr; }
    return p;
}

}  // namespace

extern "C" {

int64_t tri_halo_f(int k) { return k < 0 || k > 62 ? -1 : halo_f(k); }

int64_t tri_halo_g(int k) {
    if (k < 0 || k > 40) return -1;
    int64_t s = 0;
    for (int i = 0; i <= k; ++i) s += halo_f(i);
    return (int64_t)k * halo_f(k) - s;
}

int tri_choose_variant(int64_t n, int64_t m, tri_dtype dtype, tri_layout layout, int sm_count) {
    if (n < 1 || m < 1 || sm_count < 1) return -1;
    return (int)choose_variant(n, m, dtype, layout, sm_count);
}

int tri_choose_k(int64_t n, int64_t m, tri_dtype dtype, tri_layout layout, int sm_count) {
    if (n < 1 || m < 1 || sm_count < 1) return -1;
    return choose_k_for(choose_variant(n, m, dtype, layout, sm_count), n, m, dtype, sm_count);
}

void tri_shard_range(int64_t m, int G, int r, int64_t* q0, int64_t* mr) {
    if (G < 1 || r < 0 || r >= G || m < 0) { if (q0) *q0 = 0; if (mr) *mr = 0; return; }
    const int64_t per = cdiv(m, G);
    const int64_t s = std::min<int64_t>((int64_t)r * per, m);
    if (q0) *q0 = s;
    if (mr) *mr = std::min<int64_t>(per, m - s);
}

const char* tri_status_str(tri_status s) {
    switch (s) {
        case TRI_OK: return "TRI_OK";
        case TRI_ERR_INVALID_ARG: return "TRI_ERR_INVALID_ARG";
        case TRI_ERR_ALIGNMENT: return "TRI_ERR_ALIGNMENT";
        case TRI_ERR_ALIAS: return "TRI_ERR_ALIAS";
        case TRI_ERR_DEVICE: return "TRI_ERR_DEVICE";
        case TRI_ERR_OOM: return "TRI_ERR_OOM";
        case TRI_ERR_CUDA: return "TRI_ERR_CUDA";
    }
    return "TRI_ERR_UNKNOWN";
}

tri_status tri_last_status(void) { return g_last; }

void tri_debug_set_profile(void* dev_counters) {
    g_fused_prof = dev_counters;
    const char* e = getenv("TRI_FUSED_DBG_MODE");  // diagnostics only, read here (not at load, not per solve)
    g_fused_dbg_mode = e ? atoi(e) : 0;
}

tri_plan_t tri_plan(int64_t n, int64_t m, tri_dtype dtype, tri_layout layout) {
    if (n < 1 || m < 1 || (dtype != TRI_F32 && dtype != TRI_F64) ||
        (layout != TRI_LAYOUT_CONTIGUOUS && layout != TRI_LAYOUT_INTERLEAVED) || n > MAX_ELEMS / m) {
        g_last = TRI_ERR_INVALID_ARG;
        return nullptr;
    }
    tri_status st;
    tri_plan_s* p = new_plan(n, m, m, dtype, layout, &st);
    g_last = st;
    return p;
}

tri_plan_t tri_plan_batched(int64_t n, int64_t ms, int64_t nb, tri_dtype dtype) {
    if (n < 1 || ms < 1 || nb < 1 || (dtype != TRI_F32 && dtype != TRI_F64) || ms > MAX_ELEMS / nb ||
        n > MAX_ELEMS / (ms * nb)) {
        g_last = TRI_ERR_INVALID_ARG;
        return nullptr;
    }
    if (ms == 1) return tri_plan(n, nb, dtype, TRI_LAYOUT_CONTIGUOUS);  // [(b n + i)]: contiguous systems
    if (nb == 1) return tri_plan(n, ms, dtype, TRI_LAYOUT_INTERLEAVED);
    if (!scan_ok(n, ms * nb, dtype, TRI_LAYOUT_BATCHED, ms)) {
        g_last = TRI_ERR_INVALID_ARG;
        return nullptr;
    }
    tri_status st;
    tri_plan_s* p = new_plan(n, ms * nb, ms, dtype, TRI_LAYOUT_BATCHED, &st);
    g_last = st;
    return p;
}

tri_plan_t tri_plan_strided(int64_t n, int64_t ms, int64_t nb, tri_dtype dtype, int64_t es, int64_t ss,
                            int64_t bs) {
    // strides >= 1 and every offset (n-1) es + (ms-1) ss + (nb-1) bs below 2^52 elements
    // (no int64 overflow anywhere in the index arithmetic); that the (q, i) map to
    // distinct elements is the caller's contract
    constexpr int64_t LIM = int64_t(1) << 50;
    if (n < 1 || ms < 1 || nb < 1 || (dtype != TRI_F32 && dtype != TRI_F64) || ms > MAX_ELEMS / nb ||
        n > MAX_ELEMS / (ms * nb) || es < 1 || ss < 1 || bs < 1 || es > LIM / n || ss > LIM / ms || bs > LIM / nb) {
        g_last = TRI_ERR_INVALID_ARG;
        return nullptr;
    }
    int dev = 0, sms = 0;
    tri_status st = current_device_ok(&dev, &sms);
    if (st != TRI_OK) { g_last = st; return nullptr; }
    tri_plan_s* p = new tri_plan_s();
    p->n = n; p->m = ms * nb; p->ms = ms; p->nb = nb; p->dtype = dtype; p->layout = TRI_LAYOUT_STRIDED;
    p->device = dev; p->sms = sms; p->es = es; p->ss = ss; p->bs = bs;
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    p->smem_optin = (size_t)optin;
    if (strided_fast(n, ms, nb, dtype, es, ss, bs)) {
        p->variant = TRI_VARIANT_SCAN;
        p->k = 0;
        plan_geometry(p);
        st = ensure_scratch(p);
    } else {
        st = make_packed(p);
    }
    if (st != TRI_OK) { tri_destroy(p); g_last = st; return nullptr; }
    g_last = TRI_OK;
    return p;
}

void tri_destroy(tri_plan_t p) {
    if (!p) return;
    tri_destroy(p->inner);
    if (p->packbuf) cudaFree(p->packbuf);
    for (int i = 0; i < 2; ++i) tri_destroy(p->sub[i]);
    for (int i = 0; i < 3; ++i)
        if (p->hs[i]) cudaStreamDestroy(p->hs[i]);
    for (auto& e : p->ev)
        if (e) cudaEventDestroy(e);
    if (p->scratch) cudaFree(p->scratch);
    if (p->stage) cudaFree(p->stage);
    delete p;
}

int tri_plan_k(tri_plan_t p) { return p ? p->k : -1; }
int tri_plan_variant(tri_plan_t p) { return p ? (int)p->variant : -1; }
int64_t tri_plan_scratch_bytes(tri_plan_t p) { return p ? (int64_t)p->scratch_bytes : -1; }

int tri_plan_launches(tri_plan_t p) {
    if (!p) return -1;
    if (p->inner) return tri_plan_launches(p->inner) + 2;  // gather, inner solve, scatter
    if (p->variant == TRI_VARIANT_SPLIT) return p->k == 0 ? 1 : p->npass + 1;
    if (p->variant == TRI_VARIANT_SCAN_MC) return p->mc_lb ? 2 : 3;  // three passes, or look-back kernel + pass 2
    return 1;
}

tri_status tri_plan_set_k(tri_plan_t p, int k) {
    if (!p || k < 0 || k > floor_log2(p->n)) return TRI_ERR_INVALID_ARG;
    if (p->layout == TRI_LAYOUT_STRIDED) {  // the packed fallback's inner plan runs any k
        if (!p->inner) return k == 0 ? TRI_OK : TRI_ERR_INVALID_ARG;
        const tri_status st = tri_plan_set_k(p->inner, k);
        if (st == TRI_OK) { p->k = p->inner->k; p->variant = p->inner->variant; }
        return st;
    }
    tri_variant v = p->variant;
    if (k < kmin_for(v) || k > kmax_for(v, p->n)) {
        // the current variant does not run this k: the fastest variant that does
        // (the fixed-k fused kernels at their own k, the k = 0 SCAN kernels, then
        // ONCHIP for systems that fit a CTA, else SPLIT, which runs any k)
        const tri_variant cand[] = {TRI_VARIANT_SCAN, TRI_VARIANT_SCAN_MC, TRI_VARIANT_STREAM, TRI_VARIANT_FUSED,
                                    TRI_VARIANT_WARP, TRI_VARIANT_ONCHIP, TRI_VARIANT_SPLIT};
        v = TRI_VARIANT_AUTO;
        for (tri_variant c : cand) {
            if (!variant_ok(c, p) || k < kmin_for(c) || k > kmax_for(c, p->n)) continue;
            if (c == TRI_VARIANT_ONCHIP && p->m >= 48 * (int64_t)p->sms) continue;  // many systems: SPLIT streams them
            v = c;
            break;
        }
        if (v == TRI_VARIANT_AUTO) return TRI_ERR_INVALID_ARG;  // BATCHED layout: k = 0 only
    }
    const tri_status st = set_plan(p, v, k);
    if (st == TRI_OK) p->forced = true;
    return st;
}

tri_status tri_plan_set_variant(tri_plan_t p, tri_variant v) {
    if (!p) return TRI_ERR_INVALID_ARG;
    if (p->layout == TRI_LAYOUT_STRIDED) {
        if (!p->inner) return (v == TRI_VARIANT_AUTO || v == TRI_VARIANT_SCAN) ? TRI_OK : TRI_ERR_INVALID_ARG;
        const tri_status st = tri_plan_set_variant(p->inner, v);
        if (st == TRI_OK) { p->k = p->inner->k; p->variant = p->inner->variant; }
        return st;
    }
    const bool autov = v == TRI_VARIANT_AUTO;
    if (autov) v = choose_variant(p->n, p->m, p->dtype, p->layout, p->sms);
    if (!variant_ok(v, p)) return TRI_ERR_INVALID_ARG;
    const tri_status st = set_plan(p, v, choose_k_for(v, p->n, p->m, p->dtype, p->sms));
    if (st == TRI_OK) p->forced = !autov;
    return st;
}

tri_status tri_plan_set_option(tri_plan_t p, tri_option opt, int value) {
    if (!p) return TRI_ERR_INVALID_ARG;
    if (p->layout == TRI_LAYOUT_STRIDED) return p->inner ? tri_plan_set_option(p->inner, opt, value) : TRI_ERR_INVALID_ARG;
    if (opt == TRI_OPT_TMA) {
        if (value != 0 && value != 1) return TRI_ERR_INVALID_ARG;
        const int old = p->opt_tma;
        p->opt_tma = value;
        // the SPLIT pass structure (and so its scratch) depends on the TMA kernels
        const tri_status st = set_plan(p, p->variant, p->k);
        if (st != TRI_OK) { p->opt_tma = old; plan_geometry(p); }
        return st;
    }
    if (opt == TRI_OPT_SCAN_CLUSTER) {
        if (value != 0 && value != 1) return TRI_ERR_INVALID_ARG;
        p->opt_cluster = value;
        p->tmc.clear();
        return TRI_OK;
    }
    if (opt == TRI_OPT_SCAN_W512) {
        if (value < -1 || value > 1) return TRI_ERR_INVALID_ARG;
        const int old = p->opt_w512;
        p->opt_w512 = value;
        const tri_status st = set_plan(p, p->variant, p->k);
        if (st != TRI_OK) { p->opt_w512 = old; plan_geometry(p); }
        return st;
    }
    if (opt == TRI_OPT_SCAN_GRID) {
        if (value < -1 || value > 1) return TRI_ERR_INVALID_ARG;
        const int old = p->opt_grid;
        p->opt_grid = value;
        const tri_status st = set_plan(p, p->variant, p->k);
        if (st != TRI_OK) { p->opt_grid = old; plan_geometry(p); }
        return st;
    }
    if (opt == TRI_OPT_SCAN_MC_LOOKBACK) {
        if (value < -1 || value > LB_MAXW) return TRI_ERR_INVALID_ARG;
        const int old = p->opt_lookback;
        p->opt_lookback = value;
        const tri_status st = set_plan(p, p->variant, p->k);
        if (st != TRI_OK) { p->opt_lookback = old; plan_geometry(p); }
        return st;
    }
    return TRI_ERR_INVALID_ARG;
}

tri_status tri_slice_solve(tri_plan_t p, int phase, int slice, int nslices, const void* a, const void* b,
                           const void* c, const void* d, const void* maps, void* out, void* stream) {
    if (!p || p->variant != TRI_VARIANT_SCAN_MC || p->m != 1 || p->mc_lb || nslices < 1 || slice < 0 ||
        slice >= nslices || phase < 0 || phase > 2 || !out || (phase > 0 && !maps))
        return TRI_ERR_INVALID_ARG;
    if (phase < 2) {  // the slice's rows; `out` is an 8-value map
        const void* in[4] = {a, b, c, d};
        tri_status st = check_ptrs(p, in, 4, nullptr, 0);
        if (st != TRI_OK) return st;
    }
    if ((uintptr_t)out % 16 || (maps && (uintptr_t)maps % 16)) return TRI_ERR_ALIGNMENT;
    const cudaError_t e = launch_scan_mc_slice(p, phase, slice, nslices, a, b, c, d, maps, out, (cudaStream_t)stream);
    return e == cudaSuccess ? TRI_OK : TRI_ERR_CUDA;
}

tri_status tri_plan_autotune(tri_plan_t p, const void* a, const void* b, const void* c, const void* d, void* x,
                             void* stream, int reps, float* best_us) {
    if (!p || reps < 1 || p->layout == TRI_LAYOUT_STRIDED) return TRI_ERR_INVALID_ARG;
    const void* in[4] = {a, b, c, d};
    const void* out[1] = {x};
    tri_status st = check_ptrs(p, in, 4, out, 1);
    if (st != TRI_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    cudaEvent_t e0, e1;
    if (cudaEventCreate(&e0) != cudaSuccess) return TRI_ERR_CUDA;
    if (cudaEventCreate(&e1) != cudaSuccess) { cudaEventDestroy(e0); return TRI_ERR_CUDA; }
    const tri_variant vs[] = {TRI_VARIANT_SCAN, TRI_VARIANT_SCAN_MC, TRI_VARIANT_STREAM, TRI_VARIANT_FUSED,
                              TRI_VARIANT_WARP, TRI_VARIANT_ONCHIP, TRI_VARIANT_SPLIT};
    float best = -1.f;
    tri_variant bv = p->variant;
    int bk = p->k;
    const int og = p->opt_grid, ow = p->opt_w512;
    int bg = og, bw = ow;
    auto time_it = [&](tri_variant v, int k) {
        if (set_plan(p, v, k) != TRI_OK) { cudaGetLastError(); return; }
        if (tri_solve(p, a, b, c, d, x, stream) != TRI_OK) { cudaGetLastError(); return; }  // warm-up
        cudaEventRecord(e0, s);
        bool ok = true;
        for (int r = 0; r < reps && ok; ++r) ok = tri_solve(p, a, b, c, d, x, stream) == TRI_OK;
        cudaEventRecord(e1, s);
        if (!ok || cudaEventSynchronize(e1) != cudaSuccess) { cudaGetLastError(); return; }
        float ms = 0.f;
        cudaEventElapsedTime(&ms, e0, e1);
        const float us = ms * 1e3f / reps;
        if (best < 0.f || us < best) { best = us; bv = v; bk = k; bg = p->opt_grid; bw = p->opt_w512; }
    };
    for (tri_variant v : vs) {
        if (!variant_ok(v, p)) continue;
        // SPLIT / ONCHIP run any k; the sweep stops at 15 (deeper k only shortens
        // chains below 2^(log2 n - 15) rows, never faster on the sweep grid)
        const int k0 = kmin_for(v), k1 = std::min(kmax_for(v, p->n), 15);
        for (int k = k0; k <= k1; ++k) {
            p->opt_grid = og; p->opt_w512 = ow;
            time_it(v, k);
            if (v == TRI_VARIANT_SCAN) {  // SCAN's kernel choices: the cluster / 512-row kernels or not
                const bool grid = p->sg_Q > 0, w512 = p->s5 != 0;
                if (grid) { p->opt_grid = 0; time_it(v, k); p->opt_grid = og; }
                if (w512) { p->opt_w512 = 0; time_it(v, k); p->opt_w512 = ow; }
            }
        }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    if (best < 0.f) return TRI_ERR_CUDA;
    p->opt_grid = bg;
    p->opt_w512 = bw;
    st = set_plan(p, bv, bk);
    if (best_us) *best_us = best;
    return st;
}

void tri_plan_describe(tri_plan_t p, char* buf, int len) {
    if (!buf || len <= 0) return;
    if (!p) { snprintf(buf, len, "null plan"); return; }
    static const char* vn[] = {"auto", "onchip", "split", "fused", "warp", "stream", "scan", "scan_mc"};
    char passes[64] = "";
    if (p->variant == TRI_VARIANT_SPLIT && p->npass > 0) {
        int o = snprintf(passes, sizeof passes, " passes=");
        for (int i = 0; i < p->npass && o < (int)sizeof passes; ++i)
            o += snprintf(passes + o, sizeof passes - o, i ? "+%d" : "%d", p->kp[i]);
    }
    snprintf(buf, len,
             "n=%lld m=%lld dtype=%s layout=%s variant=%s k=%d%s G=%d P=%d rpt=%d L=%lld C=%lld "
             "fu_grid=%d fu_son=%d fu_nc=%lld sk_grid=%d sk_nc=%d sk_son=%d mc_P=%d lookback=%d tma=%d scratch=%zu "
             "sms=%d grid_Q=%d grid_R=%d w512=%d",
             (long long)p->n, (long long)p->m, p->dtype == TRI_F64 ? "f64" : "f32",
             p->layout == TRI_LAYOUT_CONTIGUOUS ? "contiguous" : p->layout == TRI_LAYOUT_INTERLEAVED ? "interleaved"
             : p->layout == TRI_LAYOUT_BATCHED ? "batched" : (p->inner ? "strided(packed)" : "strided"),
             vn[p->variant], p->k, passes, p->G, p->P, p->rpt, (long long)p->L, (long long)p->C, p->fu_grid,
             p->fu_son, (long long)p->fu_nc, p->sk_grid, p->sk_nc, p->sk_son, p->mc_P, p->mc_lb ? p->mc_NCWs : 0,
             p->opt_tma, p->scratch_bytes, p->sms, p->sg_Q, p->sg_R, p->s5);
}

tri_status tri_solve(tri_plan_t p, const void* a, const void* b, const void* c, const void* d, void* x,
                     void* stream) {
    if (!p) return TRI_ERR_INVALID_ARG;
    const void* in[4] = {a, b, c, d};
    const void* out[1] = {x};
    tri_status st = check_ptrs(p, in, 4, out, 1);
    if (st != TRI_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    if (p->layout == TRI_LAYOUT_STRIDED && !p->inner) {
        // the TMA path needs 16-byte aligned view origins; a view that starts
        // elsewhere (odd x0 of a sub-grid) switches the plan to the packed path
        bool al = ((uintptr_t)x & 15) == 0;
        for (int i = 0; i < 4; ++i) al = al && ((uintptr_t)in[i] & 15) == 0;
        if (!al && (st = make_packed(p)) != TRI_OK) return st;
    }
    if (p->inner) {  // STRIDED, packed fallback: gather, solve the dense copy, scatter x
        const size_t slot = (size_t)p->n * (size_t)p->m * esize(p->dtype) / 256 * 256 + 256;
        char* pb = (char*)p->packbuf;
        void* const dv[4] = {pb, pb + slot, pb + 2 * slot, pb + 3 * slot};
        e = launch_pack(p, in, dv, s);
        if (e != cudaSuccess) return TRI_ERR_CUDA;
        st = tri_solve(p->inner, dv[0], dv[1], dv[2], dv[3], pb + 4 * slot, stream);
        if (st != TRI_OK) return st;
        e = launch_unpack(p, pb + 4 * slot, x, s);
        return e == cudaSuccess ? TRI_OK : TRI_ERR_CUDA;
    }
    switch (p->variant) {
        case TRI_VARIANT_WARP: e = launch_warp(p, a, b, c, d, x, nullptr, nullptr, nullptr, 0, s); break;
        case TRI_VARIANT_ONCHIP: e = launch_onchip(p, a, b, c, d, x, nullptr, nullptr, nullptr, 0, s); break;
        case TRI_VARIANT_STREAM: e = launch_stream(p, a, b, c, d, x, s, nullptr, nullptr, nullptr); break;
        case TRI_VARIANT_SCAN: e = launch_scan(p, a, b, c, d, x, s); break;
        case TRI_VARIANT_SCAN_MC: e = launch_scan_mc(p, a, b, c, d, x, s); break;
        case TRI_VARIANT_FUSED: e = launch_fused(p, a, b, c, d, x, s, nullptr, nullptr, nullptr); break;
        default: e = launch_split(p, a, b, c, d, x, s); break;
    }
    return e == cudaSuccess ? TRI_OK : TRI_ERR_CUDA;
}

tri_status tri_debug_pcr(tri_plan_t p, const void* a, const void* b, const void* c, const void* d, void* ao,
                         void* co, void* do_, void* stream) {
    if (!p || p->layout == TRI_LAYOUT_STRIDED) return TRI_ERR_INVALID_ARG;
    const void* in[4] = {a, b, c, d};
    const void* out[3] = {ao, co, do_};
    tri_status st = check_ptrs(p, in, 4, out, 3);
    if (st != TRI_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    switch (p->variant) {
        case TRI_VARIANT_WARP: e = launch_warp(p, a, b, c, d, nullptr, ao, co, do_, 1, s); break;
        case TRI_VARIANT_ONCHIP: e = launch_onchip(p, a, b, c, d, nullptr, ao, co, do_, 1, s); break;
        case TRI_VARIANT_STREAM: e = launch_stream(p, a, b, c, d, nullptr, s, ao, co, do_); break;
        case TRI_VARIANT_SCAN:
        case TRI_VARIANT_SCAN_MC: return TRI_ERR_INVALID_ARG;  // k = 0: no PCR stage to show
        case TRI_VARIANT_FUSED: e = launch_fused(p, a, b, c, d, nullptr, s, ao, co, do_); break;
        default:
            if (p->k == 0) return TRI_ERR_INVALID_ARG;  // no PCR stage to show
            e = launch_split_pcr(p, a, b, c, d, ao, co, do_, s);
            break;
    }
    return e == cudaSuccess ? TRI_OK : TRI_ERR_CUDA;
}

}  // extern "C"

namespace {

inline size_t align256(size_t v) { return (v + 255) / 256 * 256; }

// chunk i of the pipelined host solve: systems [q0, q0 + mi)
struct HostChunks {
    int nch = 0;
    int64_t mc = 0, mlast = 0;
    size_t slot = 0;  // device bytes per array (sum of the chunks' 256-aligned regions)
};
HostChunks host_chunks(const tri_plan_s* p) {
    HostChunks h;
    const size_t es = esize(p->dtype);
    h.mc = cdiv(p->m, HOST_CHUNKS);
    h.nch = (int)cdiv(p->m, h.mc);
    h.mlast = p->m - (int64_t)(h.nch - 1) * h.mc;
    h.slot = (size_t)(h.nch - 1) * align256((size_t)(h.mc * p->n) * es) + align256((size_t)(h.mlast * p->n) * es);
    return h;
}

// a sub-plan for a chunk: the parent's variant, k and options when the caller
// forced them (tri_plan_set_variant / tri_plan_set_k / tri_plan_set_option)
tri_status make_sub(tri_plan_s* p, int i, int64_t mi) {
    if (p->sub[i] && p->sub_m[i] == mi && p->sub[i]->variant == (p->forced ? p->variant : p->sub[i]->variant) &&
        (!p->forced || p->sub[i]->k == p->k) && p->sub[i]->opt_tma == p->opt_tma &&
        p->sub[i]->opt_lookback == p->opt_lookback && p->sub[i]->opt_cluster == p->opt_cluster &&
        p->sub[i]->opt_grid == p->opt_grid && p->sub[i]->opt_w512 == p->opt_w512)
        return TRI_OK;
    tri_destroy(p->sub[i]);
    p->sub[i] = nullptr;
    tri_status st;
    tri_plan_s* s = new_plan(p->n, mi, mi, p->dtype, p->layout, &st);
    if (!s) return st;
    s->opt_tma = p->opt_tma;
    s->opt_lookback = p->opt_lookback;
    s->opt_cluster = p->opt_cluster;
    s->opt_grid = p->opt_grid;
    s->opt_w512 = p->opt_w512;
    if (p->forced) {
        if (!variant_ok(p->variant, s)) { tri_destroy(s); return TRI_ERR_INVALID_ARG; }
        st = set_plan(s, p->variant, p->k);
    } else {
        st = set_plan(s, s->variant, s->k);  // applies the options
    }
    if (st != TRI_OK) { tri_destroy(s); return st; }
    s->forced = p->forced;
    p->sub[i] = s;
    p->sub_m[i] = mi;
    return TRI_OK;
}

void drain(tri_plan_s* p) {
    for (int i = 0; i < 3; ++i)
        if (p->hs[i]) cudaStreamSynchronize(p->hs[i]);
    cudaGetLastError();
}

// Pipelined end-to-end solve for a CONTIGUOUS batch: HOST_CHUNKS ranges of
// systems; chunk i's H2D copies (stream 0), solve (stream 1, sub-plan for the
// chunk size) and x D2H copy (stream 2) overlap the other chunks' (PCIe is full
// duplex; each chunk's staging region is its own, 256-byte aligned, so no
// buffer is reused and every chunk's device pointers meet tri_solve's rules).
tri_status solve_host_pipelined(tri_plan_s* p, const void* const hv[4], void* x, char* const dv[5], cudaStream_t us) {
    const size_t es = esize(p->dtype);
    const int64_t n = p->n;
    const HostChunks h = host_chunks(p);
    for (int i = 0; i < 3; ++i)
        if (!p->hs[i] && cudaStreamCreateWithFlags(&p->hs[i], cudaStreamNonBlocking) != cudaSuccess) return TRI_ERR_CUDA;
    for (auto& e : p->ev)
        if (!e && cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return TRI_ERR_CUDA;
    tri_status st = make_sub(p, 0, h.mc);
    if (st == TRI_OK) st = make_sub(p, 1, h.mlast);
    if (st != TRI_OK) return st;
    cudaEvent_t* evH = p->ev;
    cudaEvent_t* evC = p->ev + HOST_CHUNKS;
    cudaEvent_t* evD = p->ev + 2 * HOST_CHUNKS;
    cudaEvent_t evU = p->ev[3 * HOST_CHUNKS];
    if (cudaEventRecord(evU, us) != cudaSuccess) return TRI_ERR_CUDA;  // after the caller's prior work
    if (cudaStreamWaitEvent(p->hs[0], evU, 0) != cudaSuccess) return TRI_ERR_CUDA;
    size_t doff = 0;
    for (int i = 0; i < h.nch; ++i) {
        const int64_t q0 = (int64_t)i * h.mc, mi = i + 1 < h.nch ? h.mc : h.mlast;
        const size_t hoff = (size_t)(q0 * n) * es, bytes = (size_t)(mi * n) * es;
        bool ok = true;
        for (int k = 0; k < 4 && ok; ++k)
            ok = cudaMemcpyAsync(dv[k] + doff, (const char*)hv[k] + hoff, bytes, cudaMemcpyHostToDevice, p->hs[0]) ==
                 cudaSuccess;
        ok = ok && cudaEventRecord(evH[i], p->hs[0]) == cudaSuccess &&
             cudaStreamWaitEvent(p->hs[1], evH[i], 0) == cudaSuccess;
        if (!ok) { drain(p); return TRI_ERR_CUDA; }
        st = tri_solve(p->sub[i + 1 < h.nch ? 0 : 1], dv[0] + doff, dv[1] + doff, dv[2] + doff, dv[3] + doff,
                       dv[4] + doff, p->hs[1]);
        if (st != TRI_OK) { drain(p); return st; }
        ok = cudaEventRecord(evC[i], p->hs[1]) == cudaSuccess && cudaStreamWaitEvent(p->hs[2], evC[i], 0) == cudaSuccess &&
             cudaMemcpyAsync((char*)x + hoff, dv[4] + doff, bytes, cudaMemcpyDeviceToHost, p->hs[2]) == cudaSuccess &&
             cudaEventRecord(evD[i], p->hs[2]) == cudaSuccess;
        if (!ok) { drain(p); return TRI_ERR_CUDA; }
        doff += align256(bytes);
    }
    if (cudaStreamWaitEvent(us, evD[h.nch - 1], 0) != cudaSuccess) { drain(p); return TRI_ERR_CUDA; }
    if (cudaStreamSynchronize(us) != cudaSuccess) { drain(p); return TRI_ERR_CUDA; }
    return TRI_OK;
}

}  // namespace

extern "C" {

tri_status tri_solve_host(tri_plan_t p, const void* a, const void* b, const void* c, const void* d, void* x,
                          void* stream) {
    if (!p || !a || !b || !c || !d || !x || p->layout == TRI_LAYOUT_STRIDED) return TRI_ERR_INVALID_ARG;
    const size_t bytes = (size_t)p->n * (size_t)p->m * esize(p->dtype);
    const bool pipe = p->layout == TRI_LAYOUT_CONTIGUOUS && p->m >= 2 * HOST_CHUNKS;
    const size_t slot = pipe ? host_chunks(p).slot : align256(bytes);
    const size_t need = 5 * slot;
    if (p->stage_bytes < need) {
        if (p->stage) cudaFree(p->stage);
        p->stage = nullptr;
        p->stage_bytes = 0;
        if (cudaMalloc(&p->stage, need) != cudaSuccess) { cudaGetLastError(); return TRI_ERR_OOM; }
        p->stage_bytes = need;
    }
    char* base = (char*)p->stage;
    char* const dv[5] = {base, base + slot, base + 2 * slot, base + 3 * slot, base + 4 * slot};
    const void* hv[4] = {a, b, c, d};
    cudaStream_t s = (cudaStream_t)stream;
    if (pipe) return solve_host_pipelined(p, hv, x, dv, s);
    for (int i = 0; i < 4; ++i)
        if (cudaMemcpyAsync(dv[i], hv[i], bytes, cudaMemcpyHostToDevice, s) != cudaSuccess) {
            cudaStreamSynchronize(s);
            cudaGetLastError();
            return TRI_ERR_CUDA;
        }
    tri_status st = tri_solve(p, dv[0], dv[1], dv[2], dv[3], dv[4], stream);
    if (st == TRI_OK && cudaMemcpyAsync(x, dv[4], bytes, cudaMemcpyDeviceToHost, s) != cudaSuccess) st = TRI_ERR_CUDA;
    if (cudaStreamSynchronize(s) != cudaSuccess && st == TRI_OK) st = TRI_ERR_CUDA;
    if (st != TRI_OK) cudaGetLastError();
    return st;
}

}  // extern "C"
