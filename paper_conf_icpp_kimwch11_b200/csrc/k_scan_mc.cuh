// k_scan_mc.cuh -- TRI_VARIANT_SCAN_MC: p-Thomas at k = 0 for FEW LONG systems
// (one huge system, config c3), each system cut into P chunks of consecutive
// 256-row windows, one CTA per chunk, so that every SM works on every system.
//
// Paper: Thomas Eqs 2-4 (reading X2), p-Thomas; the
// continuant form of the forward sweep and its segment maps are DESIGN.md X21
// (k_scan.cuh); this file adds one level above the windows: chunks.  The
// forward sweep of a chunk is a 3x3 linear map of the incoming state and the
// back substitution an affine map of the x after the chunk, so the solve runs
// as three streaming passes:
//   pass 0 (k_scan_mc<0>): read a, b, c, d; every window's forward map (lane
//     segment maps reduced over the warp); the chunk's map = their product;
//   pass 1 (k_scan_mc<1>): the chunk's incoming state = product of the maps of
//     the chunks before it (read by warp 0 while the first tiles load); read
//     a, b, c, d again; windows chained across the CTA's warps (state handed
//     over through named barriers, as in k_scan), replay -> c', d' to scratch;
//     every window's back-substitution map; the chunk's backward map;
//   pass 2 (k_scan_mc<2>): x after the chunk = the backward maps of the chunks
//     after it applied to 0; read c', d' (TMA bulk copies); windows in reverse
//     order chained across warps (x handed over), replay Eq 4 -> x.
// HBM traffic: 4 + 4 + 2 + 2 + 1 = 13 arrays (the deep-k SPLIT path moves 21).
#pragma once
#include "k_scan.cuh"

namespace tri {

constexpr int SMC_WMAX = 1024;  // windows per chunk (per-window maps live in smem)

template <typename T>
struct ScanMCArgs {
    T* x;
    T* cd;        // c', d' of every window (q, w): sc_slot_elems<T>() elements at (q NC + w)
    double* cmap; // [m P][8] chunk forward maps (SKMat a..g; fp64 for both dtypes, k_scan.cuh SCM)
    double* cbm;  // [m P][8] chunk back-substitution maps (al, be, -): x_first = al + be x_after
    int64_t n, m;
    int NC;       // windows per system
    int NCW;      // windows per chunk
    int P;        // chunks per system
    // sliced solve of one system spread over devices (m == 1; NEXT-4): the rows
    // here are a slice of a larger system; keep_a0 / keep_cn keep the coupling
    // of its first / last row; s0 = incoming forward state (theta, psi, delta)
    // of the slice (null: the system's start, (1, 0, 0)); xe = x after the slice
    // (null: 0, the system's end)
    int keep_a0, keep_cn;
    // L2 reuse between the passes: pass 0 loads the last `keep0` windows it reads of
    // its chunk (the chunk start, which pass 1 reads first) with evict_last; pass 1
    // stores c', d' of the last `keep1` windows it writes (the chunk end, which pass 2
    // reads first) with evict_last; 0 = plain policies
    int keep0, keep1;
    int discard;  // pass 2 discards each window's (c', d') L2 lines after reading them
    int w128;     // tensor view with 128-byte rows (k_scan.cuh)
    int x32;      // fp64: x rows 32-byte aligned (256-bit stores)
    const T* s0;
    const T* xe;
    // look-back path (k_scan_mc_lb): small-chunk records (x after each at [14]);
    // null otherwise
    const double* xafter;
    int NCWs, Ps;
    // ragged n (k_scan.cuh sc_patch_tail): rows >= n_al of system q from the arrays
    // (q n); n_al == n otherwise
    const T *ga, *gb, *gc, *gd;
    int64_t n_al;
};

template <typename T>
struct SMCLayout {
    static constexpr int in_bytes = 4 * SC_W * (int)sizeof(T);        // one window: a, b, c, d (or c', d')
    static constexpr int in_stride = (in_bytes + 1023) / 1024 * 1024;
    static constexpr int off_in = 0;
    static constexpr int off_hv = off_in + SC_NW * in_stride;          // [NW][4] handover
    static constexpr int off_bar = off_hv + SC_NW * 4 * (int)sizeof(T);
    static constexpr int off_wm = (off_bar + SC_NW * 8 + 15) / 16 * 16;  // [NCW][8] per-window maps (fp64)
    static __host__ __device__ constexpr int smem_bytes(int NCW) { return off_wm + NCW * 8 * 8 + 1024; }
};

__device__ __forceinline__ void smc_bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            (unsigned)__cvta_generic_to_shared(dst)),
        "l"(src), "r"(bytes), "r"((unsigned)__cvta_generic_to_shared(bar))
        : "memory");
}

template <typename T>
__device__ __forceinline__ SKMat<T> sk_shfl_down(const SKMat<T>& m, int d) {
    SKMat<T> r;
    r.a = __shfl_down_sync(0xffffffffu, m.a, d);
    r.b = __shfl_down_sync(0xffffffffu, m.b, d);
    r.c = __shfl_down_sync(0xffffffffu, m.c, d);
    r.d = __shfl_down_sync(0xffffffffu, m.d, d);
    r.e = __shfl_down_sync(0xffffffffu, m.e, d);
    r.f = __shfl_down_sync(0xffffffffu, m.f, d);
    r.g = __shfl_down_sync(0xffffffffu, m.g, d);
    return r;
}

template <typename T>
__device__ __forceinline__ void smc_rescale(SKMat<T>& M) {
    const T s = sc_scale2(M.a, M.b);
    M.a *= s; M.b *= s; M.c *= s; M.d *= s; M.e *= s; M.f *= s; M.g *= s;
}

// product of the maps of `cnt` consecutive windows / chunks (8 values apart, in
// shared or global memory; warp-wide, order-preserving): forward maps compose later-after-earlier; backward maps
// (al, be) compose earlier-after-later (x_first(window i) depends on window i+1)
__device__ __forceinline__ SCM smc_reduce_fwd(const double* wm, int cnt, int lane) {
    const int per = (cnt + 31) / 32, lo = lane * per, hi = min(cnt, lo + per);
    SCM R{1.0, 0.0, 0.0, 1.0, 0.0, 0.0, 1.0};
    for (int i = lo; i < hi; ++i) {
        const double* s = wm + 8 * i;
        R = sk_compose(SCM{s[0], s[1], s[2], s[3], s[4], s[5], s[6]}, R);
        smc_rescale(R);
    }
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {  // lane l combines with lane l + d (later windows)
        const SCM o = sk_shfl_down(R, d);
        if ((lane & (2 * d - 1)) == 0) { R = sk_compose(o, R); smc_rescale(R); }
    }
    return R;  // lane 0
}
__device__ __forceinline__ void smc_reduce_bwd(const double* wm, int cnt, int lane, double& al, double& be) {
    const int per = (cnt + 31) / 32, lo = lane * per, hi = min(cnt, lo + per);
    al = 0.0; be = 1.0;
    for (int i = hi - 1; i >= lo; --i) {  // R = B_i o R
        const double a2 = wm[8 * i], b2 = wm[8 * i + 1];
        al = fma(b2, al, a2);
        be = b2 * be;
    }
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {  // (lane l) o (lane l + d)
        const double oa = __shfl_down_sync(0xffffffffu, al, d), ob = __shfl_down_sync(0xffffffffu, be, d);
        if ((lane & (2 * d - 1)) == 0) { al = fma(be, oa, al); be = be * ob; }
    }
}

template <typename T, int MODE>
__global__ void __launch_bounds__(SC_THREADS, 1) k_scan_mc(const __grid_constant__ StreamMaps tm, ScanMCArgs<T> p) {
    using L = SMCLayout<T>;
    extern __shared__ __align__(16) unsigned char smc_smem_raw[];
    unsigned char* sbase = smc_smem_raw + ((1024 - ((unsigned)__cvta_generic_to_shared(smc_smem_raw) & 1023)) & 1023);
    uint64_t* in_full = reinterpret_cast<uint64_t*>(sbase + L::off_bar);
    T* hv = reinterpret_cast<T*>(sbase + L::off_hv);
    double* wm = reinterpret_cast<double*>(sbase + L::off_wm);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, pw = warp;
    if (threadIdx.x == 0) {
        for (int i = 0; i < SC_NW; ++i) sk_bar_init(&in_full[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    __syncthreads();

    const int64_t n = p.n;
    const int NC = p.NC;
    const int64_t q = blockIdx.x / p.P;
    const int ch = (int)(blockIdx.x - q * p.P);
    const int w0 = ch * p.NCW;
    const int nwin = min(NC, w0 + p.NCW) - w0;
    T* ib = reinterpret_cast<T*>(sbase + L::off_in + pw * L::in_stride);
    // pass 0 keeps its lines (evict_normal): the chunk starts it reads last are
    // what pass 1 reads first; pass 1 is the inputs' last use (evict_first)
    const uint64_t pol_in = MODE == 0 ? sk_policy_evict_normal() : sk_policy_evict_first();
    const uint64_t pol_keep = sk_policy_evict_last();
    // pass 0 and pass 2 walk their chunk backwards, pass 1 forwards: each pass
    // starts where the previous one ended, so the windows still in L2 (the last
    // ~100 MB a pass touched, at the same end of every chunk) are read first
    auto win_of = [&](int g) { return MODE != 1 ? w0 + nwin - 1 - g : w0 + g; };
    auto issue = [&](int g) {
        const int w = win_of(g);
        if (MODE < 2) {
            const int y = w * (p.w128 ? SC_W * (int)sizeof(T) / 128 : SC_W / 8);
            const uint64_t pl = (MODE == 0 && g >= nwin - p.keep0) ? pol_keep : pol_in;
            sk_expect(&in_full[pw], (unsigned)(4 * SC_W * sizeof(T)));
            sc_tma3d(ib + 0 * SC_W, &tm.a, y, (int)q, &in_full[pw], pl);
            sc_tma3d(ib + 1 * SC_W, &tm.b, y, (int)q, &in_full[pw], pl);
            sc_tma3d(ib + 2 * SC_W, &tm.c, y, (int)q, &in_full[pw], pl);
            sc_tma3d(ib + 3 * SC_W, &tm.d, y, (int)q, &in_full[pw], pl);
        } else {
            const unsigned bytes = (unsigned)(sc_slot_elems<T>() * sizeof(T));
            sk_expect(&in_full[pw], bytes);
            smc_bulk_g2s(ib, p.cd + (q * NC + w) * (int64_t)sc_slot_elems<T>(), bytes, &in_full[pw]);
        }
    };
    if (lane == 0 && pw < nwin) issue(pw);
    unsigned ph = 0;
    const int pi = (pw + SC_NW - 1) % SC_NW;
    // the chunk's boundary value from the maps of pass 0 / pass 1 (warp 0 runs step 0)
    T st0 = T(1), ps0 = T(0), de0 = T(0), xa0 = T(0);
    if (MODE == 1 && warp == 0) {  // incoming state = (M_{ch-1} ... M_0) S0, S0 = (1, 0, 0) or the slice's
        const SCM R = smc_reduce_fwd(p.cmap + 8 * (q * p.P), ch, lane);
        double t0 = 1.0, q0 = 0.0, e0 = 0.0;
        if (p.s0) { t0 = p.s0[0]; q0 = p.s0[1]; e0 = p.s0[2]; }
        double a0 = fma(R.a, t0, R.b * q0), b0 = fma(R.c, t0, R.d * q0), c0 = fma(R.e, t0, fma(R.f, q0, R.g * e0));
        const double sc0 = sk_exp2_scale(a0);
        st0 = (T)__shfl_sync(0xffffffffu, a0 * sc0, 0);
        ps0 = (T)__shfl_sync(0xffffffffu, b0 * sc0, 0);
        de0 = (T)__shfl_sync(0xffffffffu, c0 * sc0, 0);
    }
    if (MODE == 2 && p.xafter && warp == 0) {
        // look-back path: x after this chunk = the backward maps of the small chunks
        // after it (records [12..13], written by k_scan_mc_lb) applied to x_end = 0
        const int s1 = (w0 + nwin + p.NCWs - 1) / p.NCWs;  // first small chunk after this chunk
        const double* r0 = p.xafter + (int64_t)(q * p.Ps + s1) * 16;
        const int cnt = p.Ps - s1, per = (cnt + 31) / 32, lo = lane * per, hi = min(cnt, lo + per);
        double al = 0.0, be = 1.0;
        for (int k = hi - 1; k >= lo; --k) {
            const double a2 = __ldcg(r0 + 16 * k + 12), b2 = __ldcg(r0 + 16 * k + 13);
            al = fma(b2, al, a2);
            be = b2 * be;
        }
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const double oa = __shfl_down_sync(0xffffffffu, al, d), ob = __shfl_down_sync(0xffffffffu, be, d);
            if ((lane & (2 * d - 1)) == 0) { al = fma(be, oa, al); be = be * ob; }
        }
        xa0 = (T)__shfl_sync(0xffffffffu, al, 0);
    } else if (MODE == 2 && warp == 0) {  // x after the chunk = (B_{ch+1} ... B_{P-1})(x_end), x_end = 0 or the slice's
        double al, be;
        smc_reduce_bwd(p.cbm + 8 * (q * p.P + ch + 1), p.P - 1 - ch, lane, al, be);
        const double xend = p.xe ? (double)p.xe[0] : 0.0;
        xa0 = (T)__shfl_sync(0xffffffffu, fma(be, xend, al), 0);
    }
    const unsigned ib_s = (unsigned)__cvta_generic_to_shared(ib);

    for (int g = pw; g < nwin; g += SC_NW) {
        const int w = win_of(g);
        const int64_t i0 = (int64_t)w * SC_W + lane * SC_R;
        const bool edge = w == 0 || (int64_t)(w + 1) * SC_W >= n;  // holds row 0 or row n - 1
        sk_wait(&in_full[pw], ph);
        ph ^= 1u;
        if (MODE == 0) {
            // ---- the window's forward map (product of the lane segment maps)
            T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
            sc_ld_rows_any(ib, lane, p.w128 != 0, ra, rb, rc, rd);
            sc_release_buf();  // this warp's reads of the buffer before the TMA refill
            if (lane == 0 && g + SC_NW < nwin) issue(g + SC_NW);
            if (edge) {
                if (p.n_al < n)
                    sc_patch_tail<T>(i0, p.n_al, n, p.ga + q * n, p.gb + q * n, p.gc + q * n, p.gd + q * n, ra, rb, rc, rd);
                sc_fix_rows<T>(i0, n, ra, rb, rc, rd, p.keep_a0, p.keep_cn);
            }
            sc_range(ra, rb, rc, rd);
            const int nvalid = (int)(n - i0 < 0 ? 0 : n - i0 < SC_R ? n - i0 : SC_R);
            SCM M = sc_wide((p.keep_cn && nvalid < SC_R) ? sc_fwd_map_n(ra, rb, rc, rd, nvalid) : sc_fwd_map(ra, rb, rc, rd));
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {  // lane l: lanes l .. l + 2d - 1 (later after earlier)
                const SCM o = sk_shfl_down(M, d);
                if ((lane & (2 * d - 1)) == 0) { M = sk_compose(o, M); smc_rescale(M); }
            }
            if (lane == 0) {
                double* s = wm + 8 * (w - w0);  // by window (pass 0 walks backwards)
                s[0] = M.a; s[1] = M.b; s[2] = M.c; s[3] = M.d; s[4] = M.e; s[5] = M.f; s[6] = M.g;
            }
        } else if (MODE == 1) {
            // ---- forward replay from the chunk's / previous window's state
            T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
            sc_ld_rows_any(ib, lane, p.w128 != 0, ra, rb, rc, rd);
            if (edge) {
                if (p.n_al < n)
                    sc_patch_tail<T>(i0, p.n_al, n, p.ga + q * n, p.gb + q * n, p.gc + q * n, p.gd + q * n, ra, rb, rc, rd);
                sc_fix_rows<T>(i0, n, ra, rb, rc, rd, p.keep_a0, p.keep_cn);
            }
            sc_range(ra, rb, rc, rd);
            const int nvalid = (int)(n - i0 < 0 ? 0 : n - i0 < SC_R ? n - i0 : SC_R);
            const bool tr = p.keep_cn && nvalid < SC_R;  // transparent padding rows (slice of a larger system)
            SCM M = sc_wide(tr ? sc_fwd_map_n(ra, rb, rc, rd, nvalid) : sc_fwd_map(ra, rb, rc, rd));
            sc_fwd_scan(M, lane);
            if (g > 0) asm volatile("bar.sync %0, 64;" ::"r"(1 + pi) : "memory");
            T th, ps, de;
            if (g == 0) {
                th = st0; ps = ps0; de = de0;
            } else {
                th = hv[4 * pi + 0]; ps = hv[4 * pi + 1]; de = hv[4 * pi + 2];
            }
            const double ot = fma(M.a, (double)th, M.b * (double)ps);
            const double op = fma(M.c, (double)th, M.d * (double)ps);
            const double od = fma(M.e, (double)th, fma(M.f, (double)ps, M.g * (double)de));
            if (lane == 31) {
                const double sc = sk_exp2_scale(ot);
                hv[4 * pw + 0] = (T)(ot * sc); hv[4 * pw + 1] = (T)(op * sc); hv[4 * pw + 2] = (T)(od * sc);
            }
            if (g + 1 < nwin) asm volatile("bar.arrive %0, 64;" ::"r"(1 + pw) : "memory");
            {
                const T it_ = (T)__shfl_up_sync(0xffffffffu, ot, 1);
                const T ip = (T)__shfl_up_sync(0xffffffffu, op, 1);
                const T id = (T)__shfl_up_sync(0xffffffffu, od, 1);
                if (lane > 0) { th = it_; ps = ip; de = id; }
            }
            sc_release_buf();  // this warp's reads of the buffer before the TMA refill
            if (lane == 0 && g + SC_NW < nwin) issue(g + SC_NW);  // rows are in registers
            T cp[SC_R], dp[SC_R];
            if (tr) sc_fwd_replay_n(ra, rb, rc, rd, th, ps, de, cp, dp, nvalid);
            else sc_fwd_replay(ra, rb, rc, rd, th, ps, de, cp, dp);
            T* dst = p.cd + (q * NC + w) * (int64_t)sc_slot_elems<T>();
            if (g >= nwin - p.keep1) {  // read first by pass 2: keep in L2
                if constexpr (sizeof(T) == 8) {
#pragma unroll
                    for (int t = 0; t < SC_R; ++t) sk_st_global_last(dst + 2 * sc_chunk<T>(lane, t), cp[t], dp[t], pol_keep);
                } else {
#pragma unroll
                    for (int t = 0; t < SC_R / 2; ++t)
                        sc_stg4_last(dst + 4 * sc_chunk<T>(lane, t), cp[2 * t], dp[2 * t], cp[2 * t + 1], dp[2 * t + 1],
                                     pol_keep);
                }
            } else if constexpr (sizeof(T) == 8) {
#pragma unroll
                for (int t = 0; t < SC_R; ++t)
                    __stcg(reinterpret_cast<double2*>(dst + 2 * sc_chunk<T>(lane, t)), make_double2(cp[t], dp[t]));
            } else {
#pragma unroll
                for (int t = 0; t < SC_R / 2; ++t)
                    __stcg(reinterpret_cast<float4*>(dst + 4 * sc_chunk<T>(lane, t)),
                           make_float4(cp[2 * t], dp[2 * t], cp[2 * t + 1], dp[2 * t + 1]));
            }
            // the window's back-substitution map
            T al, be;
            sc_bwd_map(cp, dp, al, be);
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {  // lane l: lanes l .. l + 2d - 1
                const T oa = __shfl_down_sync(0xffffffffu, al, d), ob = __shfl_down_sync(0xffffffffu, be, d);
                if ((lane & (2 * d - 1)) == 0) { al = fma(be, oa, al); be = be * ob; }
            }
            if (lane == 0) { wm[8 * g] = (double)al; wm[8 * g + 1] = (double)be; }
        } else {
            // ---- back substitution in reverse window order, x handed over
            T cp[SC_R], dp[SC_R];
            sc_load_slot_s(ib_s, lane, cp, dp);
            if (p.discard) {
                // the scratch copy of (c', d') is dead after this read: drop its L2 lines
                // without a write-back (pass 1 leaves the chunk ends dirty in L2)
                constexpr int lines = (int)(sc_slot_elems<T>() * sizeof(T) / 128);
                if (lane < lines) {
                    const T* src = p.cd + (q * NC + w) * (int64_t)sc_slot_elems<T>() + lane * (128 / (int)sizeof(T));
                    asm volatile("discard.global.L2 [%0], 128;" ::"l"(src) : "memory");
                }
            }
            sc_release_buf();  // this warp's reads of the buffer before the TMA refill
            if (lane == 0 && g + SC_NW < nwin) issue(g + SC_NW);
            T al, be;
            sc_bwd_map(cp, dp, al, be);
            sc_bwd_scan(al, be, lane);
            if (g > 0) asm volatile("bar.sync %0, 64;" ::"r"(1 + pi) : "memory");
            const T xw = g == 0 ? xa0 : hv[4 * pi];
            const T xs = fma(be, xw, al);
            if (lane == 0) hv[4 * pw] = xs;
            if (g + 1 < nwin) asm volatile("bar.arrive %0, 64;" ::"r"(1 + pw) : "memory");
            T x = __shfl_down_sync(0xffffffffu, xs, 1);
            if (lane == 31) x = xw;
            T xv[SC_R];
#pragma unroll
            for (int t = SC_R - 1; t >= 0; --t) {
                x = fma(-cp[t], x, dp[t]);
                xv[t] = x;
            }
            sc_store_x(p.x + q * n + i0, n - i0, xv, p.x32 != 0);
        }
    }
    if (MODE == 2) return;
    __syncthreads();
    if (warp == 0) {
        if (MODE == 0) {
            const SCM R = smc_reduce_fwd(wm, nwin, lane);
            if (lane == 0) {
                double* s = p.cmap + 8 * (int64_t)blockIdx.x;
                s[0] = R.a; s[1] = R.b; s[2] = R.c; s[3] = R.d; s[4] = R.e; s[5] = R.f; s[6] = R.g;
            }
        } else {
            double al, be;
            smc_reduce_bwd(wm, nwin, lane, al, be);
            if (lane == 0) { p.cbm[8 * (int64_t)blockIdx.x] = al; p.cbm[8 * (int64_t)blockIdx.x + 1] = be; }
        }
    }
}

// ---- SCAN_MC with passes 0 and 1 fused by a decoupled look-back over small
// chunks: HBM traffic 4 (+ an L2 re-read of each chunk) + 2 + 2
// + 1 = 9 arrays instead of 13.  Persistent CTAs take chunks of NCWs windows in
// ticket order (an atomic counter, so a CTA only ever waits on chunks that
// started before it).  The CTA's warps are split by role, so that the HBM
// stream of forward maps never waits for a look-back or for the replay chain:
//   * LB_NA "A" warps: phase A of chunk i -- every window's forward map (lane
//     segment maps composed over the warp, fp64), stored to shared memory
//     (double-buffered by chunk parity); windows streamed from HBM by TMA, two
//     in flight per warp, L2 evict_normal so phase B finds them in L2;
//   * one "L" warp: the chunk's aggregate map (flag 1), the look-back with a
//     FIXED structure (bitwise reproducible: the inclusive state of the chunk at
//     the largest multiple of 32 below, plus the aggregates after it, one round
//     of 32 flags), the chunk's inclusive state (flag 2), and the incoming state
//     handed to the B warps;
//   * LB_NB "B" warps: phase B of chunk i - 1 or earlier -- the forward replay of
//     the chunk (re-read from L2) from every window's incoming state (the L warp
//     scans the chunk's window maps from the chunk's incoming state, so the
//     windows need no chain), c', d' to scratch, every window's back-substitution
//     map and the chunk's (record [12..13]).
// Roles hand chunks over through mbarriers in shared memory (ticket ring,
// maps full / free, state full / free), at most a few chunks apart.
// Pass 2 (k_scan_mc<2>, big chunks that are unions of small ones) then reduces
// the backward maps of the small chunks after its chunk into the x after it.
// record per small chunk (16 values): [0..6] aggregate map, [8..10] inclusive
// state, [12..13] backward map (al, be)
constexpr int SMC_REC = 16;
constexpr int LB_NA = 5;                           // phase-A warps
constexpr int LB_NB = 10;                          // phase-B warps (chain barriers 1 .. LB_NB)
constexpr int LB_WARPS = LB_NA + LB_NB + 1;        // + the look-back warp
constexpr int LB_THREADS = 32 * LB_WARPS;
constexpr int LB_MAXW = 64;                        // windows per small chunk
constexpr int LB_RING = 8;                         // ticket ring (roles are at most ~4 chunks apart)
static_assert(LB_NB + 1 <= 15, "named barriers 1 .. LB_NB + 1");

template <typename T>
struct LBLayout {
    static constexpr int in_stride = SMCLayout<T>::in_stride;
    static constexpr int off_a = 0;                                  // [NA][2] staging
    static constexpr int off_b = off_a + LB_NA * 2 * in_stride;      // [NB] staging
    static constexpr int off_wm = off_b + LB_NB * in_stride;         // [2][MAXW][8] fwd window maps (fp64)
    static constexpr int off_wb = off_wm + 2 * LB_MAXW * 8 * 8;      // [2][MAXW][2] bwd window maps (fp64)
    static constexpr int off_st = off_wb + 2 * LB_MAXW * 2 * 8;      // [2][MAXW][4] windows' incoming states (fp64)
    static constexpr int off_tk = off_st + 2 * LB_MAXW * 4 * 8;      // [RING] tickets
    static constexpr int off_bar = (off_tk + LB_RING * 4 + 15) / 16 * 16;
    // mbarriers: a_full[NA][2], b_full[NB], tkfull[RING], mapsfull[2], wmfree[2], statefull[2], stfree[2], bdone[2]
    static constexpr int nbar = 2 * LB_NA + LB_NB + LB_RING + 10;
    static constexpr int smem_bytes = off_bar + nbar * 8 + 1024;
};

__device__ __forceinline__ unsigned smc_ld_acquire_gpu(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void smc_st_release_gpu(unsigned* p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

template <typename T>
struct ScanMCLB {
    double* rec;       // [m Ps][SMC_REC] (fp64 for both dtypes)
    double* brec;      // [m Pb][8] block aggregates (32 chunks each)
    unsigned* flag;    // [m Ps] chunk flags (1 aggregate, 2 + incoming state), the ticket counter at [m Ps],
                       // then [m Pb] block flags (1 aggregate); all zeroed before the launch
    int NCWs, Ps, Pb;  // windows per small chunk (<= LB_MAXW), small chunks per system, blocks per system
    unsigned long long* prof;  // diagnostics (tri_debug_set_profile): [m Ps][8] %globaltimer stamps per chunk, or null
};
__device__ __forceinline__ unsigned long long lb_now() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

// Look-back step of the L warp (warp-wide): the product M_{j0} M_{j0-1} ... M_{j0-cnt+1}
// of cnt <= 32 published aggregate maps (map i at rec + i * stride, flag fl[i] >= 1;
// lane l polls and reads map j0 - l, so each lane reads only what it acquired),
// applied to a base state (3 values at base, flag *bfl >= 2, polled and read by
// lane 0), or to `s` when base is null.  Fixed composition order: bitwise
// reproducible.  Returns the state on every lane.
__device__ __forceinline__ void lb_lookback(const double* rec, int stride, const unsigned* fl, int j0, int cnt,
                                            const double* base, const unsigned* bfl, int lane, double (&s)[3]) {
    const unsigned want = lane < cnt ? 1u : 0u;
    const bool wb = base != nullptr && lane == 0;
    while (true) {
        const unsigned v = want ? smc_ld_acquire_gpu(fl + (j0 - lane)) : 0u;
        const unsigned vb = wb ? smc_ld_acquire_gpu(bfl) : 2u;
        if (!__any_sync(0xffffffffu, v < want || vb < 2u)) break;
        __nanosleep(32);
    }
    SCM A{1.0, 0.0, 0.0, 1.0, 0.0, 0.0, 1.0};
    if (lane < cnt) {
        const double* r = rec + (int64_t)(j0 - lane) * stride;
        A = SCM{__ldcg(r + 0), __ldcg(r + 1), __ldcg(r + 2), __ldcg(r + 3), __ldcg(r + 4), __ldcg(r + 5), __ldcg(r + 6)};
    }
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {  // lane l: maps j0-l .. j0-l-2d+1 (lane l latest)
        const SCM o = sk_shfl_down(A, d);
        if ((lane & (2 * d - 1)) == 0) { A = sk_compose(A, o); smc_rescale(A); }
    }
    double th = s[0], ps = s[1], de = s[2];
    if (wb) { th = __ldcg(base + 0); ps = __ldcg(base + 1); de = __ldcg(base + 2); }
    const double ot = fma(A.a, th, A.b * ps), op = fma(A.c, th, A.d * ps), od = fma(A.e, th, fma(A.f, ps, A.g * de));
    const double sc = sk_exp2_scale(ot);
    s[0] = __shfl_sync(0xffffffffu, ot * sc, 0);
    s[1] = __shfl_sync(0xffffffffu, op * sc, 0);
    s[2] = __shfl_sync(0xffffffffu, od * sc, 0);
}

template <typename T>
__global__ void __launch_bounds__(LB_THREADS, 1) k_scan_mc_lb(const __grid_constant__ StreamMaps tm, ScanMCArgs<T> p,
                                                               ScanMCLB<T> lb) {
    using L = LBLayout<T>;
    extern __shared__ __align__(16) unsigned char smc_smem_raw[];
    unsigned char* sbase = smc_smem_raw + ((1024 - ((unsigned)__cvta_generic_to_shared(smc_smem_raw) & 1023)) & 1023);
    uint64_t* bars = reinterpret_cast<uint64_t*>(sbase + L::off_bar);
    uint64_t* a_full = bars;                          // [NA][2]
    uint64_t* b_full = a_full + 2 * LB_NA;            // [NB]
    uint64_t* tkfull = b_full + LB_NB;                // [RING]
    uint64_t* mapsfull = tkfull + LB_RING;            // [2]
    uint64_t* wmfree = mapsfull + 2;                  // [2]
    uint64_t* statefull = wmfree + 2;                 // [2]
    uint64_t* stfree = statefull + 2;                 // [2]
    uint64_t* bdone = stfree + 2;                     // [2] B finished a chunk (throttles A: L2 reuse)
    double* wm0 = reinterpret_cast<double*>(sbase + L::off_wm);
    double* wb0 = reinterpret_cast<double*>(sbase + L::off_wb);
    double* st0 = reinterpret_cast<double*>(sbase + L::off_st);
    int* tk = reinterpret_cast<int*>(sbase + L::off_tk);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int k = 0; k < 2 * LB_NA + LB_NB; ++k) sk_bar_init(&bars[k], 1);
        for (int k = 0; k < LB_RING; ++k) sk_bar_init(&tkfull[k], 1);
        for (int k = 0; k < 2; ++k) {
            // every lane of the arriving warp(s) arrives: each releases its own
            // shared-memory accesses (no reliance on __syncwarp cumulativity)
            sk_bar_init(&mapsfull[k], LB_NA * 32);
            sk_bar_init(&wmfree[k], 32);
            sk_bar_init(&statefull[k], 32);
            sk_bar_init(&stfree[k], 32);
            sk_bar_init(&bdone[k], 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    __syncthreads();
    const int64_t n = p.n;
    const int NC = p.NC, NCW = lb.NCWs;
    const int total = (int)(p.m * lb.Ps);
    unsigned* counter = &lb.flag[total];
    auto nwin_of = [&](int t) {
        const int ch = t % lb.Ps;
        return min(NC, ch * NCW + NCW) - ch * NCW;
    };
    auto issue = [&](T* buf, uint64_t* bar, int t, int g, uint64_t pol) {
        const int q = t / lb.Ps, w = (t - q * lb.Ps) * NCW + g;
        const int y = w * (p.w128 ? SC_W * (int)sizeof(T) / 128 : SC_W / 8);
        sk_expect(bar, (unsigned)(4 * SC_W * sizeof(T)));
        sc_tma3d(buf + 0 * SC_W, &tm.a, y, q, bar, pol);
        sc_tma3d(buf + 1 * SC_W, &tm.b, y, q, bar, pol);
        sc_tma3d(buf + 2 * SC_W, &tm.c, y, q, bar, pol);
        sc_tma3d(buf + 3 * SC_W, &tm.d, y, q, bar, pol);
    };
    auto load_rows = [&](const T* buf, int t, int g, T (&ra)[SC_R], T (&rb)[SC_R], T (&rc)[SC_R], T (&rd)[SC_R]) {
        const int q = t / lb.Ps, w = (t - q * lb.Ps) * NCW + g;
        const int64_t i0 = (int64_t)w * SC_W + lane * SC_R;
        sc_ld_rows_any(buf, lane, p.w128 != 0, ra, rb, rc, rd);
        if (w == 0 || (int64_t)(w + 1) * SC_W >= n) {  // holds row 0 or row n - 1
            if (p.n_al < n)
                sc_patch_tail<T>(i0, p.n_al, n, p.ga + q * n, p.gb + q * n, p.gc + q * n, p.gd + q * n, ra, rb, rc, rd);
            sc_fix_rows<T>(i0, n, ra, rb, rc, rd, 0, 0);
        }
        sc_range(ra, rb, rc, rd);
    };

    if (warp < LB_NA) {
        // ======================= A: forward window maps =======================
        const int aw = warp;
        auto buf = [&](int b) { return reinterpret_cast<T*>(sbase + L::off_a + (2 * aw + b) * L::in_stride); };
        const uint64_t pol = sk_policy_evict_normal();  // phase B re-reads the chunk from L2
        unsigned ph2 = 0;                                // bit b: phase of buffer b
        int nb = 0;                                      // loads issued by this warp (buffer = nb & 1)
        int nc = 0;                                      // loads consumed
        for (int i = 0;; ++i) {
            const int par = i & 1;
            if (aw == 0 && lane == 0) {  // the ticket of chunk i, just in time
                tk[i % LB_RING] = (int)atomicAdd(counter, 1u);
                sk_arrive(&tkfull[i % LB_RING]);
            }
            sk_wait(&tkfull[i % LB_RING], (unsigned)((i / LB_RING) & 1));
            const int t = tk[i % LB_RING];
            if (t >= total) {
                if (i >= 2) sk_wait(&wmfree[par], (unsigned)(((i >> 1) - 1) & 1));  // never two phases ahead of L
                sk_arrive(&mapsfull[par]);  // tells the L warp: no more chunks
                break;
            }
            const int nwin = nwin_of(t);
            if (lb.prof && aw == 0 && lane == 0) lb.prof[(int64_t)t * 8 + 0] = lb_now();
            double* wm = wm0 + par * LB_MAXW * 8;
            // at most one chunk ahead of the B warps: the chunk phase B re-reads must
            // still be in L2 (148 CTAs x 2 chunks x 256 KB = 76 MB of the 126 MB)
            if (i >= 2) sk_wait(&bdone[par], (unsigned)(((i >> 1) - 1) & 1));
            // first two windows of this warp (before waiting for the map buffer)
            if (lane == 0) {
                for (int g = aw; g < nwin && g < aw + 2 * LB_NA; g += LB_NA, ++nb) issue(buf(nb & 1), &a_full[2 * aw + (nb & 1)], t, g, pol);
            } else {
                for (int g = aw; g < nwin && g < aw + 2 * LB_NA; g += LB_NA) ++nb;
            }
            if (i >= 2) sk_wait(&wmfree[par], (unsigned)(((i >> 1) - 1) & 1));  // L has read chunk i - 2's maps
            for (int g = aw; g < nwin; g += LB_NA, ++nc) {
                const int bsel = nc & 1;
                sk_wait(&a_full[2 * aw + bsel], (ph2 >> bsel) & 1u);
                ph2 ^= 1u << bsel;
                T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
                load_rows(buf(bsel), t, g, ra, rb, rc, rd);
                sc_release_buf();  // this warp's reads of the buffer before the TMA refill
                if (g + 2 * LB_NA < nwin) {
                    if (lane == 0) issue(buf(bsel), &a_full[2 * aw + bsel], t, g + 2 * LB_NA, pol);
                    ++nb;
                }
                SCM M = sc_wide(sc_fwd_map(ra, rb, rc, rd));
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {  // lane l: lanes l .. l + 2d - 1 (later after earlier)
                    const SCM o = sk_shfl_down(M, d);
                    if ((lane & (2 * d - 1)) == 0) { M = sk_compose(o, M); smc_rescale(M); }
                }
                if (lane == 0) {
                    double* s = wm + 8 * g;
                    s[0] = M.a; s[1] = M.b; s[2] = M.c; s[3] = M.d; s[4] = M.e; s[5] = M.f; s[6] = M.g;
                }
            }
            __syncwarp();
            if (lb.prof && aw == 0 && lane == 0) lb.prof[(int64_t)t * 8 + 1] = lb_now();
            sk_arrive(&mapsfull[par]);  // release: this warp's maps are in shared memory
        }
    } else if (warp == LB_NA) {
        // ======================= L: aggregate, look-back, incoming state =======================
        unsigned* fl = lb.flag;
        for (int i = 0;; ++i) {
            const int par = i & 1;
            sk_wait(&mapsfull[par], (unsigned)((i >> 1) & 1));
            const int t = tk[i % LB_RING];
            if (i >= 2) sk_wait(&stfree[par], (unsigned)(((i >> 1) - 1) & 1));  // B has read chunk i - 2's state
            if (t >= total) {
                if (lane == 0) st0[4 * par + 3] = (double)t;
                sk_arrive(&statefull[par]);
                break;
            }
            const int nwin = nwin_of(t);
            const int q = t / lb.Ps, ch = t - q * lb.Ps;
            if (lb.prof && lane == 0) lb.prof[(int64_t)t * 8 + 2] = lb_now();
            const SCM R = smc_reduce_fwd(wm0 + par * LB_MAXW * 8, nwin, lane);  // lane 0
            double* rec = lb.rec + (int64_t)t * SMC_REC;
            if (lane == 0) {  // the aggregate, published with flag 1
                __stcg(rec + 0, R.a); __stcg(rec + 1, R.b); __stcg(rec + 2, R.c); __stcg(rec + 3, R.d);
                __stcg(rec + 4, R.e); __stcg(rec + 5, R.f); __stcg(rec + 6, R.g);
                smc_st_release_gpu(fl + t, 1u);  // release: the stores above are visible first
            }
            // Look-back with a FIXED two-level structure (bitwise reproducible, and no
            // serial chain through every 32nd chunk): blocks of 32 chunks; the last chunk
            // of a block publishes the block's aggregate; the first chunk of block K
            // publishes its incoming state E_32K = BA_{K-1} ... BA_{32J} E_1024J (J =
            // K / 32, the block aggregates since the last 1024-chunk boundary; at that
            // boundary the 32 block aggregates before it and E of the previous one);
            // any other chunk: E_t = A_{t-1} ... A_{32K} E_32K.
            const int tfirst = q * lb.Ps, K = ch / 32;
            unsigned* bfl = fl + total + 1;
            if (ch % 32 == 31) {  // the block aggregate BA_K = A_t ... A_32K
                SCM BA{1.0, 0.0, 0.0, 1.0, 0.0, 0.0, 1.0};
                {
                    const int cnt = 32;
                    while (true) {
                        const unsigned v = lane < cnt ? smc_ld_acquire_gpu(fl + (t - lane)) : 1u;
                        if (!__any_sync(0xffffffffu, v < 1u)) break;
                        __nanosleep(32);
                    }
                    const double* r = lb.rec + (int64_t)(t - lane) * SMC_REC;
                    BA = SCM{__ldcg(r + 0), __ldcg(r + 1), __ldcg(r + 2), __ldcg(r + 3), __ldcg(r + 4), __ldcg(r + 5),
                             __ldcg(r + 6)};
#pragma unroll
                    for (int d = 1; d < 32; d <<= 1) {
                        const SCM o = sk_shfl_down(BA, d);
                        if ((lane & (2 * d - 1)) == 0) { BA = sk_compose(BA, o); smc_rescale(BA); }
                    }
                }
                if (lane == 0) {
                    double* br = lb.brec + (int64_t)(q * lb.Pb + K) * 8;
                    __stcg(br + 0, BA.a); __stcg(br + 1, BA.b); __stcg(br + 2, BA.c); __stcg(br + 3, BA.d);
                    __stcg(br + 4, BA.e); __stcg(br + 5, BA.f); __stcg(br + 6, BA.g);
                    smc_st_release_gpu(bfl + q * lb.Pb + K, 1u);
                }
            }
            double E[3] = {1.0, 0.0, 0.0};  // the system's start
            if (ch % 32 != 0) {
                lb_lookback(lb.rec, SMC_REC, fl, t - 1, ch % 32, lb.rec + (int64_t)(tfirst + 32 * K) * SMC_REC + 8,
                            fl + tfirst + 32 * K, lane, E);
            } else if (K > 0) {
                const int J = K / 32;
                const int kb = K % 32 != 0 ? 32 * J : K - 32;  // blocks kb .. K-1, base chunk 32 kb
                lb_lookback(lb.brec + (int64_t)(q * lb.Pb) * 8, 8, bfl + q * lb.Pb, K - 1, K - kb,
                            kb > 0 ? lb.rec + (int64_t)(tfirst + 32 * kb) * SMC_REC + 8 : nullptr,
                            kb > 0 ? fl + tfirst + 32 * kb : nullptr, lane, E);
            }
            if (lane == 0 && ch % 32 == 0) {  // block start: publish the incoming state with flag 2
                __stcg(rec + 8, E[0]); __stcg(rec + 9, E[1]); __stcg(rec + 10, E[2]);
                smc_st_release_gpu(fl + t, 2u);
            }
            // every window's incoming state: the window maps scanned over the lanes
            // (two windows per lane when NCWs > 32), applied to E -- the B warps then
            // need no chain between windows
            {
                const double* wm = wm0 + par * LB_MAXW * 8;
                double* ws = st0 + par * LB_MAXW * 4;
                double s[3] = {E[0], E[1], E[2]};
                for (int base = 0; base < nwin; base += 32) {
                    const int g = base + lane;
                    SCM W{1.0, 0.0, 0.0, 1.0, 0.0, 0.0, 1.0};
                    if (g < nwin) { const double* m = wm + 8 * g; W = SCM{m[0], m[1], m[2], m[3], m[4], m[5], m[6]}; }
                    sc_fwd_scan(W, lane);  // lane l: W_{base+l} ... W_base
                    // state entering window g = (W_{g-1} ... W_base) s
                    SCM X = sk_shfl_up(W, 1);
                    if (lane == 0) X = SCM{1.0, 0.0, 0.0, 1.0, 0.0, 0.0, 1.0};
                    const double xt = fma(X.a, s[0], X.b * s[1]), xp = fma(X.c, s[0], X.d * s[1]),
                                 xd = fma(X.e, s[0], fma(X.f, s[1], X.g * s[2]));
                    const double sc = sk_exp2_scale(xt);
                    if (g < nwin) { ws[4 * g + 0] = xt * sc; ws[4 * g + 1] = xp * sc; ws[4 * g + 2] = xd * sc; }
                    // the state after this group of 32 windows, for the next group
                    const double yt = fma(W.a, s[0], W.b * s[1]), yp = fma(W.c, s[0], W.d * s[1]),
                                 yd = fma(W.e, s[0], fma(W.f, s[1], W.g * s[2]));
                    const double sy = sk_exp2_scale(yt);
                    s[0] = __shfl_sync(0xffffffffu, yt * sy, 31);
                    s[1] = __shfl_sync(0xffffffffu, yp * sy, 31);
                    s[2] = __shfl_sync(0xffffffffu, yd * sy, 31);
                }
            }
            if (lb.prof && lane == 0) lb.prof[(int64_t)t * 8 + 3] = lb_now();
            sk_arrive(&wmfree[par]);     // the window maps are consumed
            sk_arrive(&statefull[par]);  // release: the window states are in shared memory
        }
    } else {
        // ======================= B: forward replay, c', d', backward maps =======================
        const int bw = warp - LB_NA - 1;
        T* buf = reinterpret_cast<T*>(sbase + L::off_b + bw * L::in_stride);
        const uint64_t pol = sk_policy_evict_first();  // last use of the chunk's rows
        unsigned ph = 0;
        for (int i = 0;; ++i) {
            const int par = i & 1;
            sk_wait(&tkfull[i % LB_RING], (unsigned)((i / LB_RING) & 1));
            const int t = tk[i % LB_RING];
            if (t >= total) break;
            const int nwin = nwin_of(t);
            const int q = t / lb.Ps, w0 = (t - q * lb.Ps) * NCW;
            if (lane == 0 && bw < nwin) issue(buf, &b_full[bw], t, bw, pol);  // prefetch before the state is known
            if (lb.prof && bw == 0 && lane == 0) lb.prof[(int64_t)t * 8 + 4] = lb_now();
            sk_wait(&statefull[par], (unsigned)((i >> 1) & 1));
            if (lb.prof && bw == 0 && lane == 0) lb.prof[(int64_t)t * 8 + 5] = lb_now();
            double* wb = wb0 + par * LB_MAXW * 2;
            for (int g = bw; g < nwin; g += LB_NB) {
                const int w = w0 + g;
                sk_wait(&b_full[bw], ph);
                ph ^= 1u;
                T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
                load_rows(buf, t, g, ra, rb, rc, rd);
                sc_release_buf();
                if (lane == 0 && g + LB_NB < nwin) issue(buf, &b_full[bw], t, g + LB_NB, pol);  // rows are in registers
                SCM M = sc_wide(sc_fwd_map(ra, rb, rc, rd));
                sc_fwd_scan(M, lane);
                const double* ws = st0 + par * LB_MAXW * 4 + 4 * g;  // the window's incoming state (L warp)
                const double th = ws[0], ps = ws[1], de = ws[2];
                const double ot = fma(M.a, th, M.b * ps);
                const double op = fma(M.c, th, M.d * ps);
                const double od = fma(M.e, th, fma(M.f, ps, M.g * de));
                T lt, lp, ld;
                {
                    const double it_ = __shfl_up_sync(0xffffffffu, ot, 1);
                    const double ip = __shfl_up_sync(0xffffffffu, op, 1);
                    const double id = __shfl_up_sync(0xffffffffu, od, 1);
                    const double sc = sk_exp2_scale(lane > 0 ? it_ : th);
                    lt = (T)((lane > 0 ? it_ : th) * sc);
                    lp = (T)((lane > 0 ? ip : ps) * sc);
                    ld = (T)((lane > 0 ? id : de) * sc);
                }
                T cp[SC_R], dp[SC_R];
                sc_fwd_replay(ra, rb, rc, rd, lt, lp, ld, cp, dp);
                T* dst = p.cd + (q * NC + w) * (int64_t)sc_slot_elems<T>();
                if constexpr (sizeof(T) == 8) {
#pragma unroll
                    for (int u = 0; u < SC_R; ++u)
                        __stcg(reinterpret_cast<double2*>(dst + 2 * sc_chunk<T>(lane, u)), make_double2(cp[u], dp[u]));
                } else {
#pragma unroll
                    for (int u = 0; u < SC_R / 2; ++u)
                        __stcg(reinterpret_cast<float4*>(dst + 4 * sc_chunk<T>(lane, u)),
                               make_float4(cp[2 * u], dp[2 * u], cp[2 * u + 1], dp[2 * u + 1]));
                }
                T al, be;
                sc_bwd_map(cp, dp, al, be);
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const T oa = __shfl_down_sync(0xffffffffu, al, d), ob = __shfl_down_sync(0xffffffffu, be, d);
                    if ((lane & (2 * d - 1)) == 0) { al = fma(be, oa, al); be = be * ob; }
                }
                if (lane == 0) { wb[2 * g] = (double)al; wb[2 * g + 1] = (double)be; }
            }
            // the chunk's backward map, once every B warp has stored its windows'
            asm volatile("bar.sync %0, %1;" ::"r"(LB_NB + 1), "r"(LB_NB * 32) : "memory");
            if (bw == 0) {
                const int per = (nwin + 31) / 32, lo = lane * per, hi = min(nwin, lo + per);
                double al = 0.0, be = 1.0;
                for (int k = hi - 1; k >= lo; --k) { al = fma(wb[2 * k + 1], al, wb[2 * k]); be = wb[2 * k + 1] * be; }
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const double oa = __shfl_down_sync(0xffffffffu, al, d), ob = __shfl_down_sync(0xffffffffu, be, d);
                    if ((lane & (2 * d - 1)) == 0) { al = fma(be, oa, al); be = be * ob; }
                }
                if (lane == 0) { lb.rec[(int64_t)t * SMC_REC + 12] = al; lb.rec[(int64_t)t * SMC_REC + 13] = be; }
                __syncwarp();
                if (lb.prof && lane == 0) { lb.prof[(int64_t)t * 8 + 6] = lb_now(); lb.prof[(int64_t)t * 8 + 7] = blockIdx.x; }
                sk_arrive(&bdone[par]);
                sk_arrive(&stfree[par]);
            }
        }
    }
}

// ---- sliced solve of one system over devices (NEXT-4): the products of all P
// chunk maps of this device's slice (warp 0; MODE 0: forward 3x3 map, MODE 1:
// backward affine map), written as 8 values to `out`
template <typename T, int MODE>
__global__ void k_scan_mc_slice_map(ScanMCArgs<T> p, T* out) {
    const int lane = threadIdx.x & 31;
    if (MODE == 0) {
        const SCM R = smc_reduce_fwd(p.cmap, p.P, lane);
        if (lane == 0) {
            out[0] = (T)R.a; out[1] = (T)R.b; out[2] = (T)R.c; out[3] = (T)R.d; out[4] = (T)R.e; out[5] = (T)R.f;
            out[6] = (T)R.g; out[7] = T(0);
        }
    } else {
        double al, be;
        smc_reduce_bwd(p.cbm, p.P, lane, al, be);
        if (lane == 0) { out[0] = (T)al; out[1] = (T)be; for (int i = 2; i < 8; ++i) out[i] = T(0); }
    }
}

// the slice boundary values from every device's slice maps (G x 8 values, in
// slice order; one thread): MODE 0: incoming forward state of slice r =
// (M_{r-1} ... M_0)(1, 0, 0), rescaled; MODE 1: x after slice r =
// (B_{r+1} ... B_{G-1})(0)
template <typename T, int MODE>
__global__ void k_scan_mc_slice_link(const T* maps, int G, int r, T* out) {
    if (threadIdx.x != 0) return;
    if (MODE == 0) {
        T th = T(1), ps = T(0), de = T(0);
        for (int s = 0; s < r; ++s) {
            const T* M = maps + 8 * s;
            const T ot = fma(M[0], th, M[1] * ps);
            const T op = fma(M[2], th, M[3] * ps);
            const T od = fma(M[4], th, fma(M[5], ps, M[6] * de));
            const T sc = sk_exp2_scale(ot);
            th = ot * sc; ps = op * sc; de = od * sc;
        }
        out[0] = th; out[1] = ps; out[2] = de;
    } else {
        T x = T(0);
        for (int s = G - 1; s > r; --s) x = fma(maps[8 * s + 1], x, maps[8 * s]);
        out[0] = x;
    }
}

}  // namespace tri
