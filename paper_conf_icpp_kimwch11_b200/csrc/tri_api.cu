// tri_api.cu -- the C ABI of include/tri.h: planner (transition point k and
// variant, Sec. III.D, re-derived for B200 in DESIGN.md),
// argument validation, scratch ownership and kernel dispatch.
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -shared (see _build.py).
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "tri.h"
#include "common.cuh"
#include "k_onchip.cuh"
#include "k_tiled_pcr.cuh"
#include "k_pthomas.cuh"
#include "k_fused.cuh"
#include "k_stream.cuh"
#include "k_scan.cuh"
#include "k_scan_mc.cuh"
#include "k_scan_rs.cuh"
#include "k_warp.cuh"
#include "k_pthomas_tma.cuh"

using namespace tri;

namespace {

thread_local tri_status g_last = TRI_OK;
void* g_fused_prof = nullptr;  // tri_debug_set_profile: device counters for the fused kernel
int g_fused_dbg_mode = 0;     // TRI_FUSED_DBG_MODE (diagnostics only)
// waves of regions per tiled-PCR pass (TRI_TILED_WAVES1/2 override, for tuning)
int env_int(const char* name, int dflt) {
    const char* e = getenv(name);
    return e ? std::max(1, atoi(e)) : dflt;
}
int g_tiled_waves1 = env_int("TRI_TILED_WAVES1", 1);
int g_split_k1max = std::min(10, env_int("TRI_SPLIT_K1MAX", 10));  // steps kept in pass 1 (tuning)
int g_tiled_waves2 = env_int("TRI_TILED_WAVES2", 3);  // measured best at c3 (1 / 3 waves)
int g_scan_mc_lb = env_int("TRI_SCAN_MC_LB", 0);     // SCAN_MC: passes 0 + 1 fused by a look-back (tuning)
int g_scan_mc_lbw = env_int("TRI_SCAN_MC_LBW", 64);   // SCAN_MC look-back: windows per small chunk (64 measured best at c3)
int g_scan_delta = env_int("TRI_SCAN_DELTA", 8);      // SCAN: back-substitution lag in steps (tuning)
int g_scan1 = getenv("TRI_SCAN1_OFF") ? 0 : 1;        // SCAN, one-window systems: chain-free kernel (A/B)
int g_scan_rs = getenv("TRI_SCAN_RS") ? atoi(getenv("TRI_SCAN_RS")) : 0;  // SCAN: role-split kernel (A/B)
int g_scan_w128 = getenv("TRI_SCAN_W128") ? atoi(getenv("TRI_SCAN_W128")) : 3;  // 128-byte TMA rows: bit 0 fp32, bit 1 fp64

constexpr int ONCHIP_THREADS = 512;
constexpr int SPLIT_K1MAX = 10;  // deepest k one sliding-window pass holds in smem (T = 256)
constexpr int SPLIT_K2MAX = 5;   // steps of the second (interleaved-batch) pass
constexpr int SPLIT_KMAX = SPLIT_K1MAX + SPLIT_K2MAX;
constexpr int64_t MAX_ELEMS = int64_t(1) << 40;

int floor_log2(int64_t v) {
    int r = -1;
    while (v > 0) { v >>= 1; ++r; }
    return r;
}
int ceil_log2(int64_t v) {
    int r = 0;
    while ((int64_t(1) << r) < v) ++r;
    return r;
}
int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }
size_t esize(tri_dtype t) { return t == TRI_F64 ? 8 : 4; }

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
bool warp_ok(int64_t n) { return n >= 32 && n <= 32 * WARP_RMAX; }

// STREAM: fp64, contiguous (or one system), n a multiple of 8 (the TMA tensor
// view [rows/8][8]), 8 .. 1024 windows of 240 rows (slot barriers, k_stream.cuh);
// tensor rows fit int32.
bool stream_ok(int64_t n, int64_t m, tri_dtype t, tri_layout layout) {
    return t == TRI_F64 && (layout == TRI_LAYOUT_CONTIGUOUS || m == 1) && n % 8 == 0 && n >= 2 * SK_W &&
           cdiv(n, SK_V) >= 8 && cdiv(n, SK_V) <= SK_NCMAX && (n / 8) * m < ((int64_t)1 << 31);
}

// SCAN: contiguous (or one system), n a multiple of 8 (the TMA tensor view
// [m][n/8][8]), at most SC_NCMAX windows of 256 rows.
int g_scan_s_il = env_int("TRI_SCAN_S", 0);  // SCAN, interleaved: systems per window (tuning; 0 = planner)
// systems per window of the SCAN kernel: 1 (contiguous), 2 / 4 / 8 (interleaved:
// the TMA box's inner extent S * s must be >= 16 bytes)
int scan_systems(int64_t n, int64_t m, tri_dtype t, tri_layout layout) {
    (void)n; (void)m;
    if (layout == TRI_LAYOUT_CONTIGUOUS) return 1;  // (BATCHED: like INTERLEAVED)
    // 8: a window's row of S systems is 64 B (fp64) / 32 B (fp32), at least one
    // whole DRAM sector per TMA row (S = 2 fp64 measured 2x slower: half sectors)
    const int smin = t == TRI_F64 ? 2 : 4;
    if (g_scan_s_il == 2 || g_scan_s_il == 4 || g_scan_s_il == 8 || g_scan_s_il == 16) return std::max(smin, g_scan_s_il);
    return 8;
}
bool scan_ok(int64_t n, int64_t m, tri_dtype t, tri_layout layout, int64_t ms = -1) {
    if (layout == TRI_LAYOUT_BATCHED) {
        const int S = scan_systems(n, m, t, layout);
        return ms > 0 && (ms * (int64_t)esize(t)) % 16 == 0 && cdiv(n, SC_W / S) <= SC_NCMAX &&
               n < ((int64_t)1 << 31) && ms < ((int64_t)1 << 31) && m / ms < ((int64_t)1 << 31);
    }
    if (layout == TRI_LAYOUT_CONTIGUOUS || m == 1)
        return n % 8 == 0 && cdiv(n, SC_W) <= SC_NCMAX && n / 8 < ((int64_t)1 << 31) && m < ((int64_t)1 << 31);
    // INTERLEAVED: TMA tensor [n][m], row stride m * s a multiple of 16 bytes
    const int S = scan_systems(n, m, t, layout);
    return (m * (int64_t)esize(t)) % 16 == 0 && cdiv(n, SC_W / S) <= SC_NCMAX && n < ((int64_t)1 << 31) &&
           m < ((int64_t)1 << 31);
}

// SCAN_MC: as SCAN, for systems of at least two windows.
bool scan_mc_ok(int64_t n, int64_t m, tri_dtype t, tri_layout layout) {
    (void)t;
    return (layout == TRI_LAYOUT_CONTIGUOUS || m == 1) && n % 8 == 0 && n > SC_W && n / 8 < ((int64_t)1 << 31) &&
           m < ((int64_t)1 << 31);
}

// Variant choice, calibrated once on B200 (the paper tunes P once) from
// scripts/sweep_k.py (profiles/r01_sweep_k_*.jsonl): every (variant, k) timed
// over the paper's shape grid (fixed n with m swept, fixed m with n swept).
//   * m >= 48 x SMs: straight to p-Thomas (paper rule M > P) -- the TMA
//     k = 0 kernel moves 9 arrays at ~86 % of the copy bandwidth and beats every
//     PCR variant there (n = 256..16384; e.g. n = 2048, m = 16384: 438 us vs
//     1266 us ONCHIP; n = 16384: FUSED wins at m = 4096, k = 0 from m = 8192);
//   * contiguous, n >= 1024 and (n <= 2048 or m >= 128): FUSED (n = 1024..16384,
//     m = 1..2048: 1.0-1.65x faster than ONCHIP/WARP/SPLIT);
//   * 32 <= n <= 1024 with many systems: WARP (contiguous from m = 1024, where
//     it overtakes ONCHIP; interleaved from one system per SM);
//   * whole systems that fit a CTA's smem: ONCHIP;
//   * otherwise (few large systems): SPLIT with k from choose_k_for.
tri_variant choose_variant(int64_t n, int64_t m, tri_dtype t, tri_layout layout, int sms) {
    if (layout == TRI_LAYOUT_BATCHED) return TRI_VARIANT_SCAN;  // the only kernel for this layout
    // SCAN (profiles/r01_sweep_scan_*.jsonl): fastest of all variants on every
    // contiguous shape with n % 8 == 0 of the grid n = 256 .. 2^20 x m = 1 .. 2^20
    // (fp64 and fp32), except a few (< 128) systems of more than 64 windows, where
    // SPLIT's deep k keeps more SMs busy (n = 65536, m = 16: 86 us vs 100 us);
    // e.g. n = m = 16384 fp64: 1.84 ms vs 2.92 ms (STREAM), n = 256, m = 2^20 fp32:
    // 1.01 ms vs 1.12 ms (SPLIT k = 0).  k = 0 throughout: the paper's M > P rule.
    if (layout == TRI_LAYOUT_CONTIGUOUS && scan_ok(n, m, t, layout) && (cdiv(n, SC_W) <= 64 || m >= 128))
        return TRI_VARIANT_SCAN;
    // SCAN_MC: the remaining contiguous shapes (fewer than 128 systems of more than
    // 64 windows) -- every system split over several SMs; beats deep-k SPLIT on all
    // of them (n = 2^24, m = 1: 354 us vs 1052 us; n = 65536, m = 16: 41 us vs 87 us;
    // n = 2^20, m = 1: 75 us vs 103 us; fp32 n = 2^24: 219 us vs 671 us).
    if (layout == TRI_LAYOUT_CONTIGUOUS && scan_mc_ok(n, m, t, layout)) return TRI_VARIANT_SCAN_MC;
    // SCAN on the INTERLEAVED layout (8 adjacent systems per window;
    // profiles/r01_sweep_scan_il_*.jsonl): fastest from 256 systems of >= 256 rows
    // up to where the 8-system groups' intermediates stop fitting on chip / in L2
    // (fp64 n m >= 2^27: SPLIT k = 0 1.07x faster at 8192 x 16384) or, fp32, where
    // many short systems favour one thread per system (n < 1024, m > 16384);
    // e.g. c2 1024 x 1024: 18 us vs 28 us (WARP); 4096 x 4096: 170 us vs 879 us.
    if (layout == TRI_LAYOUT_INTERLEAVED && m >= 256 && n >= 256 && scan_ok(n, m, t, layout)) {
        const int64_t N = n * m;
        const bool fits = t == TRI_F64 ? N < ((int64_t)1 << 27) : N < ((int64_t)1 << 28) && (n >= 1024 || m <= 16384);
        if (fits) return TRI_VARIANT_SCAN;
    }
    // STREAM (profiles/r01_sweep_stream_f64.jsonl): fastest of all variants for
    // fp64 contiguous batches with n % 8 == 0 from 8 windows up, except a few
    // (< 64) very long systems, where SPLIT's deep k keeps more SMs busy
    // (n = 65536, m = 37: 136 us vs 166 us); e.g. n = m = 16384: 2.92 ms vs
    // 3.41 ms (k = 0 TMA), n = 2048, m = 2368: 63 us vs 111 us (FUSED).
    if (layout == TRI_LAYOUT_CONTIGUOUS && stream_ok(n, m, t, layout) && (m >= 64 || n <= 8192)) return TRI_VARIANT_STREAM;
    if (m >= 48 * (int64_t)sms) return TRI_VARIANT_SPLIT;
    const bool contig = layout == TRI_LAYOUT_CONTIGUOUS;
    if (contig && fused_ok(n, m, layout) && n >= 1024 && (n <= 2048 || m >= 128)) return TRI_VARIANT_FUSED;
    if (warp_ok(n) && m >= (contig ? 1024 : (int64_t)sms)) return TRI_VARIANT_WARP;
    if (n <= onchip_rows_budget(t)) return TRI_VARIANT_ONCHIP;
    return TRI_VARIANT_SPLIT;
}

// Transition point.  Paper rule: M > P => k = 0; otherwise the largest k
// with 2^k M <= P; B200 P = 64 chains per SM.  Measured refinement: below P the
// extra PCR steps stop paying once the subsystems are ~32 rows long (n = 8192,
// m = 1: k = 8 in 25 us vs k = 13 in 76 us), so k <= floor(log2 n) - 5.
int choose_k_for(tri_variant v, int64_t n, int64_t m, tri_dtype t, tri_layout layout, int sms) {
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
    return std::min(std::min(k, kmax_n), SPLIT_KMAX);
}

int kmax_for(tri_variant v, int64_t n) {
    const int kn = floor_log2(n);
    if (v == TRI_VARIANT_FUSED) return FU_K;
    if (v == TRI_VARIANT_STREAM) return SK_K;
    if (v == TRI_VARIANT_WARP) return WARP_K;
    if (v == TRI_VARIANT_SCAN || v == TRI_VARIANT_SCAN_MC) return 0;
    return v == TRI_VARIANT_SPLIT ? std::min(kn, SPLIT_KMAX) : kn;
}
int kmin_for(tri_variant v) {
    return v == TRI_VARIANT_FUSED ? FU_K : v == TRI_VARIANT_STREAM ? SK_K : v == TRI_VARIANT_WARP ? WARP_K : 0;
}

}  // namespace

struct tri_plan_s {
    int64_t n, m;
    tri_dtype dtype;
    tri_layout layout;
    int device, sms;
    int k;
    tri_variant variant;
    int G, P, rpt;            // ONCHIP geometry
    int64_t n_pad, L, C;      // SPLIT: chain length, chains
    int64_t region, nreg;     // SPLIT: tiled-PCR regions per system (pass 1)
    int k1;                   // SPLIT: steps of pass 1 (k - k1 in pass 2)
    int64_t L1, C1;           // SPLIT: pass-1 positions per chain, chains
    int64_t region2, nreg2, nblk2;  // SPLIT pass 2: positions per region, regions, chain blocks
    int fu_grid, fu_son;      // FUSED: persistent CTAs, on-chip positions per chain
    bool fu_vec;              // FUSED: staged 8-row-aligned path
    int64_t fu_nc;            // FUSED: windows per system
    int sk_grid, sk_nc, sk_son;  // STREAM / SCAN: persistent CTAs, windows per system, resident storage slots
    int sk_delta;                // SCAN: back-substitution lag (steps)
    int sk_S;                    // SCAN: systems per window (1 contiguous; 2 / 4 / 8 interleaved)
    int64_t ms;                  // systems per batch (BATCHED; m otherwise)
    int mc_P, mc_NCW;            // SCAN_MC: chunks per system, windows per chunk
    int mc_lb, mc_NCWs, mc_Ps;   // SCAN_MC look-back path: on, windows per small chunk, small chunks per system
    size_t smem_optin;
    void* scratch;
    size_t scratch_bytes;
    void* stage;              // tri_solve_host staging (5 arrays), lazily allocated
    size_t stage_bytes;
    // tri_solve_host pipeline (CONTIGUOUS, m >= 2): chunks of systems flow
    // H2D -> solve -> D2H on three streams; sub-plans for the chunk sizes
    tri_plan_s* sub[2];
    int64_t sub_m[2];
    cudaStream_t hs[3];
    cudaEvent_t ev[3 * 16 + 1];
    const void* seen[8];      // pointers whose device residency was last verified
};

namespace {

// resident CTAs per SM of the tiled-PCR passes (one full wave of regions)
template <typename T, int K>
int tiled_occ_k() {
    const int smem = 3 * TPCRRing<K>::total() * (int)sizeof(T);
    if (cudaFuncSetAttribute(k_tiled_pcr<T, K>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess) {
        cudaGetLastError();
        return 1;
    }
    int occ = 1;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_tiled_pcr<T, K>, TPCR_T, smem) != cudaSuccess) {
        cudaGetLastError();
        occ = 1;
    }
    return std::max(1, occ);
}
template <typename T>
int tiled_occ(int k1) {
    switch (k1) {
        case 1: return tiled_occ_k<T, 1>();
        case 2: return tiled_occ_k<T, 2>();
        case 3: return tiled_occ_k<T, 3>();
        case 4: return tiled_occ_k<T, 4>();
        case 5: return tiled_occ_k<T, 5>();
        case 6: return tiled_occ_k<T, 6>();
        case 7: return tiled_occ_k<T, 7>();
        case 8: return tiled_occ_k<T, 8>();
        case 9: return tiled_occ_k<T, 9>();
        default: return tiled_occ_k<T, 10>();
    }
}
template <typename T, int K2>
int tiled_il_occ_k() {
    const int smem = 3 * TPCRILRing<K2>::total() * TPCR_IL_CB * (int)sizeof(T);
    if (cudaFuncSetAttribute(k_tiled_pcr_il<T, K2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess) {
        cudaGetLastError();
        return 1;
    }
    int occ = 1;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_tiled_pcr_il<T, K2>, TPCR_T, smem) != cudaSuccess) {
        cudaGetLastError();
        occ = 1;
    }
    return std::max(1, occ);
}
template <typename T>
int tiled_il_occ(int k2) {
    switch (k2) {
        case 1: return tiled_il_occ_k<T, 1>();
        case 2: return tiled_il_occ_k<T, 2>();
        case 3: return tiled_il_occ_k<T, 3>();
        case 4: return tiled_il_occ_k<T, 4>();
        default: return tiled_il_occ_k<T, 5>();
    }
}

// ---- per-plan geometry -----------------------------------------------------
void plan_geometry(tri_plan_s* p) {
    const int64_t n = p->n, m = p->m;
    if (p->variant == TRI_VARIANT_WARP) {
        int R = 1;
        while (32 * (int64_t)R < n) R *= 2;
        p->rpt = R;
        p->G = 0; p->P = 0; p->n_pad = 32 * (int64_t)R; p->L = R; p->C = m * 32; p->region = 0; p->nreg = 0;
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
        while ((int64_t)rpt * ONCHIP_THREADS < rows) rpt *= 2;
        p->rpt = rpt;
        p->n_pad = n; p->L = 0; p->C = 0; p->region = 0; p->nreg = 0;
    } else {
        const int S = 1 << p->k;
        p->L = cdiv(n, S);
        p->n_pad = p->L * S;
        p->C = m * S;
        p->k1 = std::min(p->k, g_split_k1max);
        if (p->k - p->k1 > SPLIT_K2MAX) p->k1 = p->k - SPLIT_K2MAX;
        const int S1 = 1 << p->k1;
        p->L1 = cdiv(n, S1);
        p->C1 = m * S1;
        p->region2 = p->nreg2 = p->nblk2 = 0;
        if (p->k > 0) {
            const int occ = p->dtype == TRI_F64 ? tiled_occ<double>(p->k1) : tiled_occ<float>(p->k1);
            const int64_t target = (int64_t)occ * p->sms * g_tiled_waves1;
            const int64_t n_pad1 = p->L1 * S1;
            int64_t nreg = std::max<int64_t>(1, cdiv(target, m));
            // regions no shorter than 4 f(k1) + T so halos stay a small fraction
            const int64_t minreg = 4 * halo_f(p->k1) + TPCR_T;
            nreg = std::max<int64_t>(1, std::min<int64_t>(nreg, n_pad1 / minreg));
            p->region = cdiv(n_pad1, nreg);
            p->nreg = cdiv(n_pad1, p->region);
        } else {
            p->region = 0; p->nreg = 0;
        }
        if (p->k > p->k1) {  // pass 2 over the C1 chains, TPCR_IL_CB per CTA
            const int k2 = p->k - p->k1;
            p->nblk2 = cdiv(p->C1, TPCR_IL_CB);
            const int occ2 = p->dtype == TRI_F64 ? tiled_il_occ<double>(k2) : tiled_il_occ<float>(k2);
            int64_t nreg2 = std::max<int64_t>(1, cdiv((int64_t)occ2 * p->sms * g_tiled_waves2, p->nblk2));
            const int64_t minreg2 = 4 * halo_f(k2) + TPCR_IL_TP;
            nreg2 = std::max<int64_t>(1, std::min<int64_t>(nreg2, p->L1 / minreg2));
            p->region2 = cdiv(p->L1, nreg2);
            p->nreg2 = cdiv(p->L1, p->region2);
        }
        p->G = 0; p->P = 0; p->rpt = 0;
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
        const bool il = (p->layout == TRI_LAYOUT_INTERLEAVED && m > 1) || p->layout == TRI_LAYOUT_BATCHED;
        p->sk_S = il ? scan_systems(n, m, p->dtype, p->layout) : 1;
        p->sk_nc = (int)cdiv(n, SC_W / p->sk_S);
        const int64_t ms = p->layout == TRI_LAYOUT_BATCHED ? p->ms : m;
        const int64_t groups = p->sk_S == 1 ? m : cdiv(ms, p->sk_S) * (m / ms);
        p->sk_grid = (int)std::min<int64_t>(groups, p->sms);
        p->sk_delta = g_scan_delta;
        const int fixed = p->dtype == TRI_F64 ? SCLayout<double>::smem_bytes(p->sk_nc, p->sk_delta, 0)
                                              : SCLayout<float>::smem_bytes(p->sk_nc, p->sk_delta, 0);
        const int slot = p->dtype == TRI_F64 ? SCLayout<double>::slot_bytes : SCLayout<float>::slot_bytes;
        const int64_t avail = ((int64_t)p->smem_optin - fixed) / slot;
        p->sk_son = (p->sk_nc == 1 && p->sk_S == 1) ? 0 : (int)std::max<int64_t>(0, std::min<int64_t>(p->sk_nc + p->sk_delta, avail));
    }
    if (p->variant == TRI_VARIANT_SCAN_MC) {
        p->L = n; p->n_pad = n; p->C = m;
        const int64_t NC = cdiv(n, SC_W);
        p->sk_nc = (int)NC;
        int64_t P = std::max(cdiv(p->sms, m), cdiv(NC, SMC_WMAX));
        P = std::min(P, NC);
        int64_t NCW = cdiv(NC, P);
        p->mc_lb = 0; p->mc_NCWs = 0; p->mc_Ps = 0;
        if (g_scan_mc_lb && g_scan_mc_lbw >= 1 && 2 * g_scan_mc_lbw <= SMC_WMAX) {
            // pass 2's chunks are unions of the look-back's small chunks
            p->mc_lb = 1;
            p->mc_NCWs = g_scan_mc_lbw;
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
        const int fixed = (p->dtype == TRI_F64 ? fused_fixed_smem<double>() : fused_fixed_smem<float>()) +
                          (vec ? (p->dtype == TRI_F64 ? fused_stage_smem<double>() : fused_stage_smem<float>()) : 0);
        const int64_t avail = ((int64_t)p->smem_optin - fixed) / (int64_t)(FU_S * 2 * s);
        p->fu_son = (int)std::max<int64_t>(0, std::min<int64_t>(p->L, avail));
    }
}

size_t scratch_need(const tri_plan_s* p) {
    if (p->variant == TRI_VARIANT_SCAN_MC)  // c', d' per window + the chunk maps (+ the look-back records and flags)
        return ((size_t)p->m * (size_t)p->sk_nc * (size_t)sc_slot_elems<double>() +
                (size_t)p->m * (size_t)p->mc_P * 16 + 16) * esize(p->dtype) +
               (p->mc_lb ? (size_t)p->m * (size_t)p->mc_Ps * (SMC_REC * esize(p->dtype) + 4) + 256 : 0);
    if (p->variant == TRI_VARIANT_SCAN)
        return (p->sk_nc == 1 && p->sk_S == 1) ? 0
                             : (size_t)p->sk_grid * (size_t)std::max(0, p->sk_nc + p->sk_delta - p->sk_son) *
                                   (size_t)sc_slot_elems<double>() * esize(p->dtype);
    if (p->variant == TRI_VARIANT_STREAM)
        return (size_t)p->sk_grid * (size_t)std::max(0, p->sk_nc - p->sk_son) * SK_SLOT * esize(p->dtype);
    if (p->variant == TRI_VARIANT_FUSED)
        return (size_t)p->fu_grid * 2 * (size_t)std::max<int64_t>(0, p->L - p->fu_son) * FU_S * 2 * esize(p->dtype);
    if (p->variant != TRI_VARIANT_SPLIT) return 0;
    const size_t s = esize(p->dtype);
    const size_t chain_elems = (size_t)p->C * (size_t)p->L;
    // k > 0: normalised reduced rows (3 arrays) + c', d' (2 arrays); k = 0: c', d';
    // two passes: + the pass-1 rows (3 arrays of C1 x L1)
    const size_t pass1 = p->k > p->k1 ? 3 * (size_t)p->C1 * (size_t)p->L1 : 0;
    return ((p->k > 0 ? 5 : 2) * chain_elems + pass1) * s;
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
    p->scratch_bytes = need;
    return TRI_OK;
}


// ---- launches ---------------------------------------------------------------
template <typename T, int RPT>
cudaError_t launch_onchip_rpt(const tri_plan_s* p, OnchipArgs<T> a, cudaStream_t st) {
    const size_t smem = (size_t)3 * p->G * p->P * sizeof(T);
    cudaError_t e = cudaFuncSetAttribute(k_onchip<T, RPT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    const int64_t grid = cdiv(p->m, p->G);
    k_onchip<T, RPT><<<(unsigned)grid, ONCHIP_THREADS, smem, st>>>(a);
    return cudaGetLastError();
}

template <typename T>
cudaError_t launch_onchip(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d,
                          void* x, void* ao, void* co, void* do_, int mode, cudaStream_t st) {
    OnchipArgs<T> A;
    A.a = (const T*)a; A.b = (const T*)b; A.c = (const T*)c; A.d = (const T*)d;
    A.x = (T*)x; A.ao = (T*)ao; A.co = (T*)co; A.do_ = (T*)do_;
    A.n = p->n; A.m = p->m; A.layout = p->layout; A.k = p->k; A.G = p->G; A.P = p->P; A.mode = mode;
    switch (p->rpt) {
        case 1: return launch_onchip_rpt<T, 1>(p, A, st);
        case 2: return launch_onchip_rpt<T, 2>(p, A, st);
        case 4: return launch_onchip_rpt<T, 4>(p, A, st);
        case 8: return launch_onchip_rpt<T, 8>(p, A, st);
        case 16: return launch_onchip_rpt<T, 16>(p, A, st);
        default: return cudaErrorInvalidValue;
    }
}

template <typename T>
cudaError_t launch_warp(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                        void* ao, void* co, void* do_, int mode, cudaStream_t st) {
    WarpArgs<T> A;
    A.a = (const T*)a; A.b = (const T*)b; A.c = (const T*)c; A.d = (const T*)d;
    A.x = (T*)x; A.ao = (T*)ao; A.co = (T*)co; A.do_ = (T*)do_;
    A.n = p->n; A.m = p->m; A.layout = p->layout; A.mode = mode;
    const bool il = p->layout == TRI_LAYOUT_INTERLEAVED && p->m > 1;
    const int wpb = il ? WARP_WPB_IL : WARP_WPB;
    const int64_t need = cdiv(p->m, wpb);
    // contiguous: persistent warps (one resident wave), each walking systems
    // q, q + grid*WPB, ... with the next system's loads in flight
    auto contig_grid = [&](auto kern) {
        int occ = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, wpb * 32, 0) != cudaSuccess || occ < 1) {
            cudaGetLastError();
            occ = 1;
        }
        return (unsigned)std::min<int64_t>(need, (int64_t)occ * p->sms);
    };
#define TRI_WARP_CASE(R)                                                                  \
    case R:                                                                               \
        if (il) k_warp<T, R, true><<<(unsigned)need, wpb * 32, 0, st>>>(A);               \
        else k_warp<T, R, false><<<warp_persistent<T, R>() ? contig_grid(k_warp<T, R, false>) : (unsigned)need, \
                                   wpb * 32, 0, st>>>(A);                                 \
        break;
    switch (p->rpt) {
        TRI_WARP_CASE(1) TRI_WARP_CASE(2) TRI_WARP_CASE(4) TRI_WARP_CASE(8) TRI_WARP_CASE(16) TRI_WARP_CASE(32)
        default: return cudaErrorInvalidValue;
    }
#undef TRI_WARP_CASE
    return cudaGetLastError();
}

template <typename T, int K>
cudaError_t launch_tiled_k(const TiledArgs<T>& A, int64_t grid, cudaStream_t st) {
    const size_t smem = (size_t)3 * TPCRRing<K>::total() * sizeof(T);
    cudaError_t e = cudaFuncSetAttribute(k_tiled_pcr<T, K>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    k_tiled_pcr<T, K><<<(unsigned)grid, TPCR_T, smem, st>>>(A);
    return cudaGetLastError();
}

template <typename T>
cudaError_t launch_tiled(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d,
                         void* oA, void* oC, void* oD, int mode, cudaStream_t st) {
    TiledArgs<T> A;
    A.a = (const T*)a; A.b = (const T*)b; A.c = (const T*)c; A.d = (const T*)d;
    A.oA = (T*)oA; A.oC = (T*)oC; A.oD = (T*)oD;
    A.n = p->n; A.m = p->m; A.n_pad = p->L1 << p->k1; A.region = p->region; A.nreg = p->nreg; A.C = p->C1;
    A.layout = p->layout; A.k = p->k1; A.mode = mode;
    const int64_t grid = p->m * p->nreg;
    switch (p->k1) {
        case 1: return launch_tiled_k<T, 1>(A, grid, st);
        case 2: return launch_tiled_k<T, 2>(A, grid, st);
        case 3: return launch_tiled_k<T, 3>(A, grid, st);
        case 4: return launch_tiled_k<T, 4>(A, grid, st);
        case 5: return launch_tiled_k<T, 5>(A, grid, st);
        case 6: return launch_tiled_k<T, 6>(A, grid, st);
        case 7: return launch_tiled_k<T, 7>(A, grid, st);
        case 8: return launch_tiled_k<T, 8>(A, grid, st);
        case 9: return launch_tiled_k<T, 9>(A, grid, st);
        case 10: return launch_tiled_k<T, 10>(A, grid, st);
        default: return cudaErrorInvalidValue;
    }
}

template <typename T, int K2>
cudaError_t launch_tiled_il_k(const TiledILArgs<T>& A, int64_t grid, cudaStream_t st) {
    const size_t smem = (size_t)3 * TPCRILRing<K2>::total() * TPCR_IL_CB * sizeof(T);
    cudaError_t e = cudaFuncSetAttribute(k_tiled_pcr_il<T, K2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    k_tiled_pcr_il<T, K2><<<(unsigned)grid, TPCR_T, smem, st>>>(A);
    return cudaGetLastError();
}

template <typename T>
cudaError_t launch_tiled_il(const tri_plan_s* p, const void* iA, const void* iC, const void* iD, void* oA, void* oC,
                            void* oD, int mode, cudaStream_t st) {
    TiledILArgs<T> A;
    A.iA = (const T*)iA; A.iC = (const T*)iC; A.iD = (const T*)iD;
    A.oA = (T*)oA; A.oC = (T*)oC; A.oD = (T*)oD;
    A.n = p->n; A.m = p->m; A.L1 = p->L1; A.C1 = p->C1; A.C = p->C;
    A.region = p->region2; A.nreg = p->nreg2; A.nblk = p->nblk2;
    A.layout = p->layout; A.k1 = p->k1; A.mode = mode;
    const int64_t grid = p->nblk2 * p->nreg2;
    switch (p->k - p->k1) {
        case 1: return launch_tiled_il_k<T, 1>(A, grid, st);
        case 2: return launch_tiled_il_k<T, 2>(A, grid, st);
        case 3: return launch_tiled_il_k<T, 3>(A, grid, st);
        case 4: return launch_tiled_il_k<T, 4>(A, grid, st);
        case 5: return launch_tiled_il_k<T, 5>(A, grid, st);
        default: return cudaErrorInvalidValue;
    }
}

template <typename T>
cudaError_t launch_fused(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                         cudaStream_t st, void* dA = nullptr, void* dC = nullptr, void* dD = nullptr) {
    FusedArgs<T> A;
    A.dA = (T*)dA; A.dC = (T*)dC; A.dD = (T*)dD;
    A.prof = (unsigned long long*)g_fused_prof;
    A.dbg_mode = g_fused_dbg_mode;
    A.a = (const T*)a; A.b = (const T*)b; A.c = (const T*)c; A.d = (const T*)d; A.x = (T*)x;
    A.spill = (T*)p->scratch;
    A.n = p->n; A.m = p->m; A.L = p->L; A.NC = p->fu_nc; A.S_on = p->fu_son;
    const bool vec = p->fu_vec && ((uintptr_t)a | (uintptr_t)b | (uintptr_t)c | (uintptr_t)d) % 16 == 0;
    const size_t smem = (size_t)fused_fixed_smem<T>() + (vec ? (size_t)fused_stage_smem<T>() : 0) +
                        (size_t)p->fu_son * FU_S * 2 * sizeof(T);
    auto kern = vec ? k_fused<T, true> : k_fused<T, false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    kern<<<p->fu_grid, FU_THREADS, smem, st>>>(A);
    return cudaGetLastError();
}

// ---- TMA tensor maps (cuTensorMapEncodeTiled through the runtime's driver
// entry point: no link-time dependency on libcuda)
PFN_cuTensorMapEncodeTiled_v12000 tma_encoder() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static bool tried = false;
    if (!tried) {
        tried = true;
        void* f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (PFN_cuTensorMapEncodeTiled_v12000)f;
        else
            cudaGetLastError();
    }
    return fn;
}

template <typename T>
bool tma_map_2d(CUtensorMap* tm, const void* base, uint64_t d0, uint64_t d1, uint32_t b0, uint32_t b1, bool swz) {
    auto enc = tma_encoder();
    if (!enc) return false;
    cuuint64_t dims[2] = {d0, d1};
    cuuint64_t strides[1] = {d0 * sizeof(T)};
    cuuint32_t box[2] = {b0, b1};
    cuuint32_t es[2] = {1, 1};
    return enc(tm, sizeof(T) == 8 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2,
               const_cast<void*>(base), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
               swz ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// ---- STREAM launch: tensor maps [n m / 8][8] (64-byte rows, 64B swizzle, box 8 x 32)
bool tma_map_rows8(CUtensorMap* tm, const void* base, uint64_t rows8) {
    auto enc = tma_encoder();
    if (!enc) return false;
    cuuint64_t dims[2] = {8, rows8};
    cuuint64_t strides[1] = {8 * sizeof(double)};
    cuuint32_t box[2] = {8, 32};
    cuuint32_t es[2] = {1, 1};
    return enc(tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, const_cast<void*>(base), dims, strides, box, es,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

cudaError_t launch_stream(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                          cudaStream_t st, void* ao = nullptr, void* co = nullptr, void* do_ = nullptr) {
    StreamMaps tm;
    const uint64_t rows8 = (uint64_t)(p->n / 8) * (uint64_t)p->m;
    if (!tma_map_rows8(&tm.a, a, rows8) || !tma_map_rows8(&tm.b, b, rows8) || !tma_map_rows8(&tm.c, c, rows8) ||
        !tma_map_rows8(&tm.d, d, rows8))
        return cudaErrorNotSupported;
    StreamArgs<double> A;
    A.x = (double*)x;
    A.spill = (double*)p->scratch;
    A.n = p->n; A.m = p->m; A.NC = p->sk_nc; A.S_on = p->sk_son;
    A.dA = (double*)ao; A.dC = (double*)co; A.dD = (double*)do_;
    A.prof = (unsigned long long*)g_fused_prof;
    A.dbg = g_fused_dbg_mode;
    const size_t smem = (size_t)SKLayout<double>::off_store + (size_t)p->sk_son * SKLayout<double>::slot_bytes + 1024;
    auto kern = A.prof ? k_stream<double, true> : k_stream<double, false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    kern<<<p->sk_grid, SK_THREADS, smem, st>>>(tm, A);
    return cudaGetLastError();
}

// ---- SCAN / SCAN_MC launch: tensor maps [m][n/8][8] (fp64: 64-byte rows, 64B
// swizzle; fp32: 32-byte rows, 32B swizzle), box [1][32][8] = one 256-row window
// of one system per array; every coordinate fits int32 for any n, m of the API
template <typename T>
bool tma_map_sys_rows8(CUtensorMap* tm, const void* base, int64_t n, int64_t m, int sys_per_box = 1,
                       bool w128 = false) {
    auto enc = tma_encoder();
    if (!enc) return false;
    const int rw = w128 ? 128 / (int)sizeof(T) : 8;  // elements per tensor row (w128: 128-byte rows)
    cuuint64_t dims[3] = {(cuuint64_t)rw, (cuuint64_t)(n / rw), (cuuint64_t)m};
    cuuint64_t strides[2] = {(cuuint64_t)rw * sizeof(T), (cuuint64_t)n * sizeof(T)};
    cuuint32_t box[3] = {(cuuint32_t)rw, (cuuint32_t)(SC_W / rw), (cuuint32_t)sys_per_box};
    cuuint32_t es[3] = {1, 1, 1};
    return enc(tm, sizeof(T) == 8 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3,
               const_cast<void*>(base), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
               w128 ? CU_TENSOR_MAP_SWIZZLE_128B : sizeof(T) == 8 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B,
               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// INTERLEAVED / BATCHED: tensor [nb][n][ms] (row stride ms elements, batch stride
// n ms), box [1][256 / S rows][S systems]
template <typename T>
bool tma_map_il(CUtensorMap* tm, const void* base, int64_t n, int64_t ms, int64_t nb, int S) {
    auto enc = tma_encoder();
    if (!enc) return false;
    cuuint64_t dims[3] = {(cuuint64_t)ms, (cuuint64_t)n, (cuuint64_t)nb};
    cuuint64_t strides[2] = {(cuuint64_t)ms * sizeof(T), (cuuint64_t)(n * ms) * sizeof(T)};
    cuuint32_t box[3] = {(cuuint32_t)S, (cuuint32_t)(SC_W / S), 1};
    cuuint32_t es[3] = {1, 1, 1};
    return enc(tm, sizeof(T) == 8 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3,
               const_cast<void*>(base), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
               CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

template <typename T, int S>
void* scan_kernel(bool prof) {
    return prof ? (void*)k_scan<T, S, true> : (void*)k_scan<T, S, false>;
}

template <typename T>
cudaError_t launch_scan(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                        cudaStream_t st) {
    StreamMaps tm;
    const int64_t n = p->n, m = p->m;
    const int S = p->sk_S;
    // 128-byte TMA rows (n % 32 fp32 / n % 16 fp64; the k_scan chain and one-window
    // paths): one TMA request per 128 bytes (fp32 c4: 0.99 -> 0.84 ms)
    const bool w128 = S == 1 && n % (128 / (int)sizeof(T)) == 0 && (g_scan_w128 & (sizeof(T) == 4 ? 1 : 2)) &&
                      !(p->sk_nc == 1 && g_scan1 && p->n <= 3 * SC_W / 4) && !(p->sk_nc >= 2 && g_scan_rs);
    if (S == 1) {
        if (!tma_map_sys_rows8<T>(&tm.a, a, n, m, 1, w128) || !tma_map_sys_rows8<T>(&tm.b, b, n, m, 1, w128) ||
            !tma_map_sys_rows8<T>(&tm.c, c, n, m, 1, w128) || !tma_map_sys_rows8<T>(&tm.d, d, n, m, 1, w128))
            return cudaErrorNotSupported;
    } else {
        const int64_t ms = p->ms, nb = m / p->ms;
        if (!tma_map_il<T>(&tm.a, a, n, ms, nb, S) || !tma_map_il<T>(&tm.b, b, n, ms, nb, S) ||
            !tma_map_il<T>(&tm.c, c, n, ms, nb, S) || !tma_map_il<T>(&tm.d, d, n, ms, nb, S))
            return cudaErrorNotSupported;
    }
    ScanArgs<T> A;
    A.x = (T*)x;
    A.spill = (T*)p->scratch;
    A.n = p->n; A.m = p->m; A.ms = p->ms; A.NC = p->sk_nc; A.S_on = p->sk_son; A.delta = p->sk_delta;
    A.w128 = w128 ? 1 : 0;
    A.prof = (unsigned long long*)g_fused_prof;
    A.dbg = g_fused_dbg_mode;
    if (S == 1 && p->sk_nc >= 2 && g_scan_rs) {  // role-split warps (k_scan_rs.cuh)
        const int NS = p->sk_nc + p->sk_delta;
        const int fixed = RSLayout<T>::smem_bytes(p->sk_nc, p->sk_delta, 0);
        const int son = (int)std::min<int64_t>(NS, std::max<int64_t>(0, ((int64_t)p->smem_optin - fixed) /
                                                                             RSLayout<T>::slot_bytes));
        if (son >= p->sk_son) {  // the plan's spill scratch covers NS - son slots
            ScanArgs<T> B = A;
            B.S_on = son;
            const int smem = RSLayout<T>::smem_bytes(p->sk_nc, p->sk_delta, son);
            cudaError_t e = cudaFuncSetAttribute(k_scan_rs<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            if (e != cudaSuccess) return e;
            k_scan_rs<T><<<p->sk_grid, RS_THREADS, smem, st>>>(tm, B);
            return cudaGetLastError();
        }
    }
    // one-window systems shorter than 3/4 of a window (many idle rows: compute-heavy)
    // run the chain-free kernel with more warps (fp32 n = 128: 1.19 ms vs 1.50 ms
    // per 2^28 rows); at n = 256 the 12-warp kernel is faster (c4: 0.99 vs 1.02 ms)
    if (S == 1 && p->sk_nc == 1 && g_scan1 && p->n <= 3 * SC_W / 4) {
        cudaError_t e = cudaFuncSetAttribute(k_scan1<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, SC1<T>::smem_bytes);
        if (e != cudaSuccess) return e;
        k_scan1<T><<<p->sk_grid, SC1<T>::NW * 32, SC1<T>::smem_bytes, st>>>(tm, A);
        return cudaGetLastError();
    }
    // one-window systems (S = 1): the slot area holds the warps' second staging buffers
    const int son_or_buf = (p->sk_S == 1 && p->sk_nc == 1)
                               ? (SC_NW * SCLayout<T>::in_stride + SCLayout<T>::slot_bytes - 1) / SCLayout<T>::slot_bytes
                               : p->sk_son;
    const size_t smem = (size_t)SCLayout<T>::smem_bytes(p->sk_nc, p->sk_delta, son_or_buf);
    const bool pr = A.prof != nullptr;
    void* kern = S == 1 ? scan_kernel<T, 1>(pr) : S == 2 ? scan_kernel<T, 2>(pr) : S == 4 ? scan_kernel<T, 4>(pr)
                 : S == 8 ? scan_kernel<T, 8>(pr) : scan_kernel<T, 16>(pr);
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    void* args[] = {(void*)&tm, (void*)&A};
    return cudaLaunchKernel(kern, dim3(p->sk_grid), dim3(SC_THREADS), args, smem, st);
}

template <typename T>
cudaError_t scan_mc_setup(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                          StreamMaps& tm, ScanMCArgs<T>& A, int& smem) {
    const int64_t n = p->n, m = p->m;
    const bool w = n % (128 / (int)sizeof(T)) == 0 && (g_scan_w128 & (sizeof(T) == 4 ? 1 : 2));
    if (a && (!tma_map_sys_rows8<T>(&tm.a, a, n, m, 1, w) || !tma_map_sys_rows8<T>(&tm.b, b, n, m, 1, w) ||
              !tma_map_sys_rows8<T>(&tm.c, c, n, m, 1, w) || !tma_map_sys_rows8<T>(&tm.d, d, n, m, 1, w)))
        return cudaErrorNotSupported;
    A = ScanMCArgs<T>{};
    A.w128 = w ? 1 : 0;
    A.x = (T*)x;
    A.cd = (T*)p->scratch;
    const int64_t mp = p->m * (int64_t)p->mc_P;
    A.cmap = A.cd + p->m * (int64_t)p->sk_nc * sc_slot_elems<T>();
    A.cbm = A.cmap + 8 * mp;
    A.n = p->n; A.m = p->m; A.NC = p->sk_nc; A.NCW = p->mc_NCW; A.P = p->mc_P;
    smem = SMCLayout<T>::smem_bytes(p->mc_NCW);
    for (auto k : {k_scan_mc<T, 0>, k_scan_mc<T, 1>, k_scan_mc<T, 2>}) {
        cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}
// the 16 values after the chunk maps: the slice's incoming state (3) and x after it (1)
template <typename T>
T* scan_mc_slice_vals(const tri_plan_s* p) {
    return (T*)p->scratch + p->m * (int64_t)p->sk_nc * sc_slot_elems<T>() + 16 * p->m * (int64_t)p->mc_P;
}

template <typename T>
cudaError_t launch_scan_mc(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                           cudaStream_t st) {
    StreamMaps tm;
    ScanMCArgs<T> A;
    int smem = 0;
    cudaError_t e = scan_mc_setup<T>(p, a, b, c, d, x, tm, A, smem);
    if (e != cudaSuccess) return e;
    if (p->mc_lb) {
        ScanMCLB<T> lb;
        lb.rec = scan_mc_slice_vals<T>(p) + 16;
        const int64_t nrec = p->m * (int64_t)p->mc_Ps;
        lb.flag = (unsigned*)(lb.rec + nrec * SMC_REC);
        lb.NCWs = p->mc_NCWs;
        lb.Ps = p->mc_Ps;
        const int smem_lb = SMCLayout<T>::smem_bytes(4 * p->mc_NCWs);
        e = cudaFuncSetAttribute(k_scan_mc_lb<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_lb);
        if (e != cudaSuccess) return e;
        e = cudaMemsetAsync(lb.flag, 0, (size_t)(nrec + 1) * sizeof(unsigned), st);
        if (e != cudaSuccess) return e;
        const int grid = (int)std::min<int64_t>(p->sms, nrec);
        k_scan_mc_lb<T><<<grid, SC_THREADS, smem_lb, st>>>(tm, A, lb);
        k_scan_mc_lb_fin<T><<<(unsigned)p->m, 1024, 0, st>>>(lb);
        A.xafter = lb.rec;
        A.NCWs = p->mc_NCWs;
        A.Ps = p->mc_Ps;
        k_scan_mc<T, 2><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
        return cudaGetLastError();
    }
    k_scan_mc<T, 0><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
    k_scan_mc<T, 1><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
    k_scan_mc<T, 2><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
    return cudaGetLastError();
}

// sliced solve of one system over devices (NEXT-4): phase 0 = pass 0 + the
// slice's forward map; 1 = incoming state from every slice's map, pass 1, the
// slice's backward map; 2 = x after the slice from every backward map, pass 2
template <typename T>
cudaError_t launch_scan_mc_slice(const tri_plan_s* p, int phase, int slice, int nslices, const void* a, const void* b,
                                 const void* c, const void* d, const void* maps, void* out, cudaStream_t st) {
    StreamMaps tm;
    ScanMCArgs<T> A;
    int smem = 0;
    cudaError_t e = scan_mc_setup<T>(p, phase < 2 ? a : nullptr, b, c, d, phase == 2 ? out : nullptr, tm, A, smem);
    if (e != cudaSuccess) return e;
    A.keep_a0 = slice > 0;
    A.keep_cn = slice < nslices - 1;
    T* vals = scan_mc_slice_vals<T>(p);
    if (phase == 0) {
        k_scan_mc<T, 0><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
        k_scan_mc_slice_map<T, 0><<<1, 32, 0, st>>>(A, (T*)out);
    } else if (phase == 1) {
        k_scan_mc_slice_link<T, 0><<<1, 32, 0, st>>>((const T*)maps, nslices, slice, vals);
        A.s0 = vals;
        k_scan_mc<T, 1><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
        k_scan_mc_slice_map<T, 1><<<1, 32, 0, st>>>(A, (T*)out);
    } else {
        k_scan_mc_slice_link<T, 1><<<1, 32, 0, st>>>((const T*)maps, nslices, slice, vals + 4);
        A.xe = vals + 4;
        k_scan_mc<T, 2><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
    }
    return cudaGetLastError();
}

// k = 0, CONTIGUOUS: the TMA kernel when both row strides (n and m elements)
// are 16-byte multiples; returns cudaErrorNotSupported to request the fallback.
template <typename T>
cudaError_t launch_contig_tma(const tri_plan_s* p, const PThomasArgs<T>& A, cudaStream_t st) {
    constexpr int R = PTTCfg<T>::R;
    if ((p->n * (int64_t)sizeof(T)) % 16 || (p->m * (int64_t)sizeof(T)) % 16) return cudaErrorNotSupported;
    if (p->n > INT32_MAX || p->m > INT32_MAX) return cudaErrorNotSupported;
    PTTMaps tm;
    const uint64_t n = (uint64_t)p->n, m = (uint64_t)p->m;
    bool ok = tma_map_2d<T>(&tm.a, A.a, n, m, R, PTT_CH, true) && tma_map_2d<T>(&tm.b, A.b, n, m, R, PTT_CH, true) &&
              tma_map_2d<T>(&tm.c, A.c, n, m, R, PTT_CH, true) && tma_map_2d<T>(&tm.d, A.d, n, m, R, PTT_CH, true) &&
              tma_map_2d<T>(&tm.x, A.x, n, m, R, PTT_CH, true) &&
              tma_map_2d<T>(&tm.cp, A.cps, m, n, PTT_CH, R, false) && tma_map_2d<T>(&tm.dp, A.dps, m, n, PTT_CH, R, false);
    if (!ok) return cudaErrorNotSupported;
    constexpr int smem = ptt_smem_bytes<T>();
    cudaError_t e = cudaFuncSetAttribute(k_pthomas_tma<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    k_pthomas_tma<T><<<(unsigned)cdiv(p->m, PTT_CH), PTT_CH, smem, st>>>(tm, A);
    return cudaGetLastError();
}

template <typename T, int CH>
cudaError_t launch_contig(const tri_plan_s* p, const PThomasArgs<T>& A, bool vec, cudaStream_t st) {
    constexpr int smem = pt2_smem_bytes<T, CH>();
    auto kern = vec ? k_pthomas_contig<T, CH, true> : k_pthomas_contig<T, CH, false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    kern<<<(unsigned)cdiv(p->m, CH), CH, smem, st>>>(A);
    return cudaGetLastError();
}

// p-Thomas over chain-interleaved input (MODE 0 scratch, MODE 1 user
// INTERLEAVED).  Few chains (< 8 warps' worth per SM): the ring-staged kernel
// with CW chains per CTA, CW the largest of 32/16/8 that still gives every SM
// a CTA; many chains: one thread per chain with a register prefetch window.
template <typename T, int CW, int MODE>
cudaError_t launch_ring(const tri_plan_s* p, const PThomasArgs<T>& A, bool vec, cudaStream_t st) {
    const int smem = ptr_smem_bytes<T, CW>(MODE == 1);
    auto kern = vec ? k_pthomas_ring<T, CW, MODE, true> : k_pthomas_ring<T, CW, MODE, false>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    kern<<<(unsigned)cdiv(p->C, CW), CW, smem, st>>>(A);
    return cudaGetLastError();
}

// chain-interleaved p-Thomas through TMA (C >= 32 x SMs); cudaErrorNotSupported
// asks for the fallback kernels
template <typename T, int MODE>
cudaError_t launch_pthomas_il_tma(const tri_plan_s* p, const PThomasArgs<T>& A, cudaStream_t st) {
    constexpr int R = PTICfg<T>::R;
    const int64_t C = p->C, L = p->L;
    if ((C * (int64_t)sizeof(T)) % 16 || C > INT32_MAX || L > INT32_MAX) return cudaErrorNotSupported;
    PTIMaps tm;
    const void* in[4] = {MODE == 1 ? (const void*)A.a : (const void*)A.iA, MODE == 1 ? (const void*)A.b : (const void*)A.iC,
                         MODE == 1 ? (const void*)A.c : (const void*)A.iD, MODE == 1 ? (const void*)A.d : (const void*)A.iD};
    bool ok = true;
    for (int i = 0; i < 4 && ok; ++i) ok = tma_map_2d<T>(&tm.a + i, in[i], C, L, PTT_CH, R, false);
    ok = ok && tma_map_2d<T>(&tm.cp, A.cps, C, L, PTT_CH, R, false) && tma_map_2d<T>(&tm.dp, A.dps, C, L, PTT_CH, R, false);
    // x as a [L][C] view: INTERLEAVED user layout (MODE 1), or one system whose
    // rows pos * 2^k + r are exactly [pos * C + r] (m = 1, n = L * 2^k)
    const bool x_view = MODE == 1 || (p->m == 1 && p->n == L * C);
    int x_tma = 0;
    if (ok && x_view) x_tma = tma_map_2d<T>(&tm.x, A.x, C, L, PTT_CH, R, false) ? 1 : 0;
    if (!ok) return cudaErrorNotSupported;
    constexpr int smem = pti_smem_bytes<T, MODE>();
    cudaError_t e = cudaFuncSetAttribute(k_pthomas_il_tma<T, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    k_pthomas_il_tma<T, MODE><<<(unsigned)cdiv(C, PTT_CH), PTT_CH, smem, st>>>(tm, A, x_tma);
    return cudaGetLastError();
}

template <typename T, int MODE>
cudaError_t launch_pthomas_il(const tri_plan_s* p, const PThomasArgs<T>& A, cudaStream_t st) {
    const int64_t C = p->C, sms = p->sms;
    if (C >= 32 * sms && !getenv("TRI_NO_TMA")) {
        const cudaError_t et = launch_pthomas_il_tma<T, MODE>(p, A, st);
        if (et != cudaErrorNotSupported) return et;
    }
    if (C >= 32 * 8 * sms) {
        k_pthomas<T, MODE><<<(unsigned)cdiv(C, 128), 128, 0, st>>>(A);
        return cudaGetLastError();
    }
    const T* in0 = MODE == 1 ? A.a : A.iA;
    const bool vec = ((C * (int64_t)sizeof(T)) % 16) == 0 && ((uintptr_t)in0 % 16) == 0;
    if (C >= 32 * sms) return launch_ring<T, 32, MODE>(p, A, vec, st);
    if (C >= 16 * sms) return launch_ring<T, 16, MODE>(p, A, vec, st);
    return launch_ring<T, 8, MODE>(p, A, vec, st);
}

template <typename T>
cudaError_t launch_split(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d,
                         void* x, cudaStream_t st) {
    const size_t ce = (size_t)p->C * (size_t)p->L;
    T* base = (T*)p->scratch;
    PThomasArgs<T> A;
    A.a = (const T*)a; A.b = (const T*)b; A.c = (const T*)c; A.d = (const T*)d;
    A.x = (T*)x;
    A.n = p->n; A.m = p->m; A.C = p->C; A.L = p->L; A.layout = p->layout; A.k = p->k;
    // 32 chains x s bytes per scratch row segment start on 128-byte lines when
    // the row pitch C s is a multiple of 128 (and the scratch base is 256-aligned)
    A.discard = ((p->C * (int64_t)sizeof(T)) % 128 == 0 && !getenv("TRI_NO_DISCARD")) ? 1 : 0;
    if (p->k > 0) {
        T *rA = base, *rC = base + ce, *rD = base + 2 * ce;
        cudaError_t e;
        if (p->k > p->k1) {  // two passes: pass-1 rows after the 5 chain arrays
            const size_t ce1 = (size_t)p->C1 * (size_t)p->L1;
            T *pA = base + 5 * ce, *pC = pA + ce1, *pD = pA + 2 * ce1;
            e = launch_tiled<T>(p, a, b, c, d, pA, pC, pD, 0, st);
            if (e != cudaSuccess) return e;
            e = launch_tiled_il<T>(p, pA, pC, pD, rA, rC, rD, 0, st);
        } else {
            e = launch_tiled<T>(p, a, b, c, d, rA, rC, rD, 0, st);
        }
        if (e != cudaSuccess) return e;
        A.iA = rA; A.iC = rC; A.iD = rD;
        A.cps = base + 3 * ce; A.dps = base + 4 * ce;
        return launch_pthomas_il<T, 0>(p, A, st);
    } else {
        A.iA = A.iC = A.iD = nullptr;
        A.cps = base; A.dps = base + ce;
        if (p->layout == TRI_LAYOUT_INTERLEAVED) {
            return launch_pthomas_il<T, 1>(p, A, st);
        } else {
            if (!getenv("TRI_NO_TMA")) {
                const cudaError_t et = launch_contig_tma<T>(p, A, st);
                if (et != cudaErrorNotSupported) return et;
            }
            const bool vec = ((p->n * (int64_t)sizeof(T)) % 16) == 0 && ((uintptr_t)a % 16) == 0;
            // 16 systems per CTA when the batch is thin (finer balance over the SMs)
            const bool thin = cdiv(p->m, 32) < 6 * (int64_t)p->sms;
            return thin ? launch_contig<T, 16>(p, A, vec, st) : launch_contig<T, 32>(p, A, vec, st);
        }
    }
    return cudaGetLastError();
}

tri_status check_ptrs(tri_plan_s* p, const void* const* in, int nin, const void* const* out, int nout) {
    const size_t bytes = (size_t)p->n * (size_t)p->m * esize(p->dtype);
    bool same = nin + nout <= 8;
    for (int i = 0; i < nin + nout && same; ++i) same = p->seen[i] == (i < nin ? in[i] : out[i - nin]);
    for (int i = 0; i < nin + nout; ++i) {
        const void* q = i < nin ? in[i] : out[i - nin];
        if (!q) return TRI_ERR_INVALID_ARG;
        if (((uintptr_t)q & 15) != 0) return TRI_ERR_ALIGNMENT;
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
    return choose_k_for(choose_variant(n, m, dtype, layout, sm_count), n, m, dtype, layout, sm_count);
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
    const char* e = getenv("TRI_FUSED_DBG_MODE");
    g_fused_dbg_mode = e ? atoi(e) : 0;
}

tri_plan_t tri_plan(int64_t n, int64_t m, tri_dtype dtype, tri_layout layout) {
    if (n < 1 || m < 1 || (dtype != TRI_F32 && dtype != TRI_F64) ||
        (layout != TRI_LAYOUT_CONTIGUOUS && layout != TRI_LAYOUT_INTERLEAVED) || n > MAX_ELEMS / m) {
        g_last = TRI_ERR_INVALID_ARG;
        return nullptr;
    }
    int dev = 0, sms = 0;
    tri_status st = current_device_ok(&dev, &sms);
    if (st != TRI_OK) { g_last = st; return nullptr; }
    tri_plan_s* p = new tri_plan_s();
    p->n = n; p->m = m; p->dtype = dtype; p->layout = layout; p->device = dev; p->sms = sms;
    p->ms = m;
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    p->smem_optin = (size_t)optin;
    p->variant = choose_variant(n, m, dtype, layout, sms);
    p->k = choose_k_for(p->variant, n, m, dtype, layout, sms);
    plan_geometry(p);
    st = ensure_scratch(p);
    if (st != TRI_OK) { delete p; g_last = st; return nullptr; }
    g_last = TRI_OK;
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
    int dev = 0, sms = 0;
    tri_status st = current_device_ok(&dev, &sms);
    if (st != TRI_OK) { g_last = st; return nullptr; }
    tri_plan_s* p = new tri_plan_s();
    p->n = n; p->m = ms * nb; p->dtype = dtype; p->layout = TRI_LAYOUT_BATCHED; p->device = dev; p->sms = sms;
    p->ms = ms;
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    p->smem_optin = (size_t)optin;
    p->variant = TRI_VARIANT_SCAN;
    p->k = 0;
    plan_geometry(p);
    st = ensure_scratch(p);
    if (st != TRI_OK) { delete p; g_last = st; return nullptr; }
    g_last = TRI_OK;
    return p;
}

void tri_destroy(tri_plan_t p) {
    if (!p) return;
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
    if (p->variant == TRI_VARIANT_SPLIT) return p->k == 0 ? 1 : p->k > p->k1 ? 3 : 2;
    if (p->variant == TRI_VARIANT_SCAN_MC) return 3;
    return 1;  // ONCHIP, FUSED
}

tri_status tri_plan_set_k(tri_plan_t p, int k) {
    if (!p || k < kmin_for(p->variant) || k > kmax_for(p->variant, p->n)) return TRI_ERR_INVALID_ARG;
    const int old = p->k;
    p->k = k;
    plan_geometry(p);
    tri_status st = ensure_scratch(p);
    if (st != TRI_OK) { p->k = old; plan_geometry(p); }
    return st;
}

tri_status tri_plan_set_variant(tri_plan_t p, tri_variant v) {
    if (!p) return TRI_ERR_INVALID_ARG;
    if (p->layout == TRI_LAYOUT_BATCHED)  // one kernel for this layout
        return (v == TRI_VARIANT_AUTO || v == TRI_VARIANT_SCAN) ? TRI_OK : TRI_ERR_INVALID_ARG;
    if (v == TRI_VARIANT_AUTO) v = choose_variant(p->n, p->m, p->dtype, p->layout, p->sms);
    if (v == TRI_VARIANT_ONCHIP && p->n > onchip_rows_budget(p->dtype)) return TRI_ERR_INVALID_ARG;
    if (v == TRI_VARIANT_FUSED && !fused_ok(p->n, p->m, p->layout)) return TRI_ERR_INVALID_ARG;
    if (v == TRI_VARIANT_WARP && !warp_ok(p->n)) return TRI_ERR_INVALID_ARG;
    if (v == TRI_VARIANT_STREAM && !stream_ok(p->n, p->m, p->dtype, p->layout)) return TRI_ERR_INVALID_ARG;
    if (v == TRI_VARIANT_SCAN && !scan_ok(p->n, p->m, p->dtype, p->layout)) return TRI_ERR_INVALID_ARG;
    if (v == TRI_VARIANT_SCAN_MC && !scan_mc_ok(p->n, p->m, p->dtype, p->layout)) return TRI_ERR_INVALID_ARG;
    if (v != TRI_VARIANT_ONCHIP && v != TRI_VARIANT_SPLIT && v != TRI_VARIANT_FUSED && v != TRI_VARIANT_WARP &&
        v != TRI_VARIANT_STREAM && v != TRI_VARIANT_SCAN && v != TRI_VARIANT_SCAN_MC)
        return TRI_ERR_INVALID_ARG;
    const tri_variant ov = p->variant;
    const int ok = p->k;
    p->variant = v;
    p->k = choose_k_for(v, p->n, p->m, p->dtype, p->layout, p->sms);
    plan_geometry(p);
    tri_status st = ensure_scratch(p);
    if (st != TRI_OK) { p->variant = ov; p->k = ok; plan_geometry(p); }
    return st;
}

tri_status tri_slice_solve(tri_plan_t p, int phase, int slice, int nslices, const void* a, const void* b,
                           const void* c, const void* d, const void* maps, void* out, void* stream) {
    if (!p || p->variant != TRI_VARIANT_SCAN_MC || p->m != 1 || nslices < 1 || slice < 0 || slice >= nslices ||
        phase < 0 || phase > 2 || !out || (phase > 0 && !maps))
        return TRI_ERR_INVALID_ARG;
    if (phase < 2) {  // the slice's rows; `out` is an 8-value map
        const void* in[4] = {a, b, c, d};
        tri_status st = check_ptrs(p, in, 4, nullptr, 0);
        if (st != TRI_OK) return st;
    }
    if ((uintptr_t)out % 16 || (maps && (uintptr_t)maps % 16)) return TRI_ERR_ALIGNMENT;
    cudaStream_t s = (cudaStream_t)stream;
    const cudaError_t e = p->dtype == TRI_F64
                              ? launch_scan_mc_slice<double>(p, phase, slice, nslices, a, b, c, d, maps, out, s)
                              : launch_scan_mc_slice<float>(p, phase, slice, nslices, a, b, c, d, maps, out, s);
    return e == cudaSuccess ? TRI_OK : TRI_ERR_CUDA;
}

tri_status tri_plan_autotune(tri_plan_t p, const void* a, const void* b, const void* c, const void* d, void* x,
                             void* stream, int reps, float* best_us) {
    if (!p || reps < 1) return TRI_ERR_INVALID_ARG;
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
    for (tri_variant v : vs) {
        if (tri_plan_set_variant(p, v) != TRI_OK) { cudaGetLastError(); continue; }
        const int k0 = kmin_for(v), k1 = kmax_for(v, p->n);
        for (int k = k0; k <= k1; ++k) {
            if (tri_plan_set_k(p, k) != TRI_OK) { cudaGetLastError(); continue; }
            if (tri_solve(p, a, b, c, d, x, stream) != TRI_OK) { cudaGetLastError(); continue; }  // warm-up
            cudaEventRecord(e0, s);
            bool ok = true;
            for (int r = 0; r < reps && ok; ++r) ok = tri_solve(p, a, b, c, d, x, stream) == TRI_OK;
            cudaEventRecord(e1, s);
            if (!ok || cudaEventSynchronize(e1) != cudaSuccess) { cudaGetLastError(); continue; }
            float ms = 0.f;
            cudaEventElapsedTime(&ms, e0, e1);
            const float us = ms * 1e3f / reps;
            if (best < 0.f || us < best) { best = us; bv = v; bk = k; }
        }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    if (best < 0.f) return TRI_ERR_CUDA;
    st = tri_plan_set_variant(p, bv);
    if (st == TRI_OK) st = tri_plan_set_k(p, bk);
    if (best_us) *best_us = best;
    return st;
}

void tri_plan_describe(tri_plan_t p, char* buf, int len) {
    if (!buf || len <= 0) return;
    if (!p) { snprintf(buf, len, "null plan"); return; }
    static const char* vn[] = {"auto", "onchip", "split", "fused", "warp", "stream", "scan", "scan_mc"};
    snprintf(buf, len,
             "n=%lld m=%lld dtype=%s layout=%s variant=%s k=%d G=%d P=%d rpt=%d L=%lld C=%lld region=%lld nreg=%lld "
             "fu_grid=%d fu_son=%d fu_nc=%lld sk_grid=%d sk_nc=%d sk_son=%d scratch=%zu sms=%d",
             (long long)p->n, (long long)p->m, p->dtype == TRI_F64 ? "f64" : "f32",
             p->layout == TRI_LAYOUT_CONTIGUOUS ? "contiguous" : p->layout == TRI_LAYOUT_INTERLEAVED ? "interleaved" : "batched",
             vn[p->variant], p->k, p->G, p->P,
             p->rpt, (long long)p->L, (long long)p->C, (long long)p->region, (long long)p->nreg, p->fu_grid, p->fu_son,
             (long long)p->fu_nc, p->sk_grid, p->sk_nc, p->sk_son, p->scratch_bytes, p->sms);
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
    if (p->variant == TRI_VARIANT_WARP) {
        e = p->dtype == TRI_F64 ? launch_warp<double>(p, a, b, c, d, x, nullptr, nullptr, nullptr, 0, s)
                                : launch_warp<float>(p, a, b, c, d, x, nullptr, nullptr, nullptr, 0, s);
    } else if (p->variant == TRI_VARIANT_ONCHIP) {
        e = p->dtype == TRI_F64 ? launch_onchip<double>(p, a, b, c, d, x, nullptr, nullptr, nullptr, 0, s)
                                : launch_onchip<float>(p, a, b, c, d, x, nullptr, nullptr, nullptr, 0, s);
    } else if (p->variant == TRI_VARIANT_STREAM) {
        e = launch_stream(p, a, b, c, d, x, s);
    } else if (p->variant == TRI_VARIANT_SCAN) {
        e = p->dtype == TRI_F64 ? launch_scan<double>(p, a, b, c, d, x, s) : launch_scan<float>(p, a, b, c, d, x, s);
    } else if (p->variant == TRI_VARIANT_SCAN_MC) {
        e = p->dtype == TRI_F64 ? launch_scan_mc<double>(p, a, b, c, d, x, s)
                                : launch_scan_mc<float>(p, a, b, c, d, x, s);
    } else if (p->variant == TRI_VARIANT_FUSED) {
        e = p->dtype == TRI_F64 ? launch_fused<double>(p, a, b, c, d, x, s) : launch_fused<float>(p, a, b, c, d, x, s);
    } else {
        e = p->dtype == TRI_F64 ? launch_split<double>(p, a, b, c, d, x, s) : launch_split<float>(p, a, b, c, d, x, s);
    }
    return e == cudaSuccess ? TRI_OK : TRI_ERR_CUDA;
}

tri_status tri_debug_pcr(tri_plan_t p, const void* a, const void* b, const void* c, const void* d, void* ao,
                         void* co, void* do_, void* stream) {
    if (!p) return TRI_ERR_INVALID_ARG;
    const void* in[4] = {a, b, c, d};
    const void* out[3] = {ao, co, do_};
    tri_status st = check_ptrs(p, in, 4, out, 3);
    if (st != TRI_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    if (p->variant == TRI_VARIANT_WARP) {
        e = p->dtype == TRI_F64 ? launch_warp<double>(p, a, b, c, d, nullptr, ao, co, do_, 1, s)
                                : launch_warp<float>(p, a, b, c, d, nullptr, ao, co, do_, 1, s);
    } else if (p->variant == TRI_VARIANT_ONCHIP) {
        e = p->dtype == TRI_F64 ? launch_onchip<double>(p, a, b, c, d, nullptr, ao, co, do_, 1, s)
                                : launch_onchip<float>(p, a, b, c, d, nullptr, ao, co, do_, 1, s);
    } else if (p->variant == TRI_VARIANT_STREAM) {
        e = launch_stream(p, a, b, c, d, nullptr, s, ao, co, do_);
    } else if (p->variant == TRI_VARIANT_SCAN || p->variant == TRI_VARIANT_SCAN_MC) {
        return TRI_ERR_INVALID_ARG;  // k = 0: no PCR stage to show
    } else if (p->variant == TRI_VARIANT_FUSED) {
        e = p->dtype == TRI_F64 ? launch_fused<double>(p, a, b, c, d, nullptr, s, ao, co, do_)
                                : launch_fused<float>(p, a, b, c, d, nullptr, s, ao, co, do_);
    } else {
        if (p->k == 0) return TRI_ERR_INVALID_ARG;  // no PCR stage to show
        if (p->k > p->k1) {
            const size_t ce = (size_t)p->C * (size_t)p->L, ce1 = (size_t)p->C1 * (size_t)p->L1;
            char* pA = (char*)p->scratch + 5 * ce * esize(p->dtype);
            char* pC = pA + ce1 * esize(p->dtype);
            char* pD = pC + ce1 * esize(p->dtype);
            e = p->dtype == TRI_F64 ? launch_tiled<double>(p, a, b, c, d, pA, pC, pD, 0, s)
                                    : launch_tiled<float>(p, a, b, c, d, pA, pC, pD, 0, s);
            if (e == cudaSuccess)
                e = p->dtype == TRI_F64 ? launch_tiled_il<double>(p, pA, pC, pD, ao, co, do_, 1, s)
                                        : launch_tiled_il<float>(p, pA, pC, pD, ao, co, do_, 1, s);
        } else {
            e = p->dtype == TRI_F64 ? launch_tiled<double>(p, a, b, c, d, ao, co, do_, 1, s)
                                    : launch_tiled<float>(p, a, b, c, d, ao, co, do_, 1, s);
        }
    }
    return e == cudaSuccess ? TRI_OK : TRI_ERR_CUDA;
}

}  // extern "C"

namespace {

constexpr int HOST_CHUNKS = 16;

// Pipelined end-to-end solve for a CONTIGUOUS batch: HOST_CHUNKS ranges of
// systems; chunk i's H2D copies (stream 0), solve (stream 1, sub-plan for the
// chunk size) and x D2H copy (stream 2) overlap the other chunks' (PCIe is full
// duplex; each chunk's staging region is its own, so no buffer is reused).
tri_status solve_host_pipelined(tri_plan_s* p, const void* const hv[4], void* x, char* const dv[5],
                                cudaStream_t us) {
    const size_t es = esize(p->dtype);
    const int64_t n = p->n, m = p->m;
    const int64_t mc = cdiv(m, HOST_CHUNKS);
    const int nch = (int)cdiv(m, mc);
    for (int i = 0; i < 3; ++i)
        if (!p->hs[i] && cudaStreamCreateWithFlags(&p->hs[i], cudaStreamNonBlocking) != cudaSuccess) return TRI_ERR_CUDA;
    for (auto& e : p->ev)
        if (!e && cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return TRI_ERR_CUDA;
    const int64_t sizes[2] = {mc, m - (int64_t)(nch - 1) * mc};
    for (int i = 0; i < 2; ++i) {
        if (p->sub[i] && p->sub_m[i] == sizes[i]) continue;
        tri_destroy(p->sub[i]);
        p->sub[i] = tri_plan(n, sizes[i], p->dtype, p->layout);
        p->sub_m[i] = sizes[i];
        if (!p->sub[i]) return tri_last_status();
    }
    cudaEvent_t* evH = p->ev;
    cudaEvent_t* evC = p->ev + HOST_CHUNKS;
    cudaEvent_t* evD = p->ev + 2 * HOST_CHUNKS;
    cudaEvent_t evU = p->ev[3 * HOST_CHUNKS];
    if (cudaEventRecord(evU, us) != cudaSuccess) return TRI_ERR_CUDA;  // after the caller's prior work
    if (cudaStreamWaitEvent(p->hs[0], evU, 0) != cudaSuccess) return TRI_ERR_CUDA;
    for (int i = 0; i < nch; ++i) {
        const int64_t q0 = (int64_t)i * mc, mi = i + 1 < nch ? mc : sizes[1];
        const size_t off = (size_t)(q0 * n) * es, bytes = (size_t)(mi * n) * es;
        for (int k = 0; k < 4; ++k)
            if (cudaMemcpyAsync(dv[k] + off, (const char*)hv[k] + off, bytes, cudaMemcpyHostToDevice, p->hs[0]) !=
                cudaSuccess)
                return TRI_ERR_CUDA;
        cudaEventRecord(evH[i], p->hs[0]);
        cudaStreamWaitEvent(p->hs[1], evH[i], 0);
        const tri_status st = tri_solve(p->sub[i + 1 < nch ? 0 : 1], dv[0] + off, dv[1] + off, dv[2] + off,
                                        dv[3] + off, dv[4] + off, p->hs[1]);
        if (st != TRI_OK) return st;
        cudaEventRecord(evC[i], p->hs[1]);
        cudaStreamWaitEvent(p->hs[2], evC[i], 0);
        if (cudaMemcpyAsync((char*)x + off, dv[4] + off, bytes, cudaMemcpyDeviceToHost, p->hs[2]) != cudaSuccess)
            return TRI_ERR_CUDA;
        cudaEventRecord(evD[i], p->hs[2]);
    }
    if (cudaStreamWaitEvent(us, evD[nch - 1], 0) != cudaSuccess) return TRI_ERR_CUDA;
    if (cudaStreamSynchronize(us) != cudaSuccess) return TRI_ERR_CUDA;
    return TRI_OK;
}

}  // namespace

extern "C" {

tri_status tri_solve_host(tri_plan_t p, const void* a, const void* b, const void* c, const void* d, void* x,
                          void* stream) {
    if (!p || !a || !b || !c || !d || !x) return TRI_ERR_INVALID_ARG;
    const size_t bytes = (size_t)p->n * (size_t)p->m * esize(p->dtype);
    const size_t need = 5 * ((bytes + 255) / 256 * 256);
    if (p->stage_bytes < need) {
        if (p->stage) cudaFree(p->stage);
        p->stage = nullptr;
        p->stage_bytes = 0;
        if (cudaMalloc(&p->stage, need) != cudaSuccess) { cudaGetLastError(); return TRI_ERR_OOM; }
        p->stage_bytes = need;
    }
    const size_t slot = need / 5;
    char* base = (char*)p->stage;
    void* dv[5] = {base, base + slot, base + 2 * slot, base + 3 * slot, base + 4 * slot};
    const void* hv[4] = {a, b, c, d};
    cudaStream_t s = (cudaStream_t)stream;
    if (p->layout == TRI_LAYOUT_CONTIGUOUS && p->m >= 2 * HOST_CHUNKS) {
        char* const dc[5] = {(char*)dv[0], (char*)dv[1], (char*)dv[2], (char*)dv[3], (char*)dv[4]};
        return solve_host_pipelined(p, hv, x, dc, s);
    }
    for (int i = 0; i < 4; ++i)
        if (cudaMemcpyAsync(dv[i], hv[i], bytes, cudaMemcpyHostToDevice, s) != cudaSuccess) return TRI_ERR_CUDA;
    tri_status st = tri_solve(p, dv[0], dv[1], dv[2], dv[3], dv[4], stream);
    if (st != TRI_OK) return st;
    if (cudaMemcpyAsync(x, dv[4], bytes, cudaMemcpyDeviceToHost, s) != cudaSuccess) return TRI_ERR_CUDA;
    if (cudaStreamSynchronize(s) != cudaSuccess) return TRI_ERR_CUDA;
    return TRI_OK;
}

}  // extern "C"
