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
    int w128;     // tensor view with 128-byte rows (k_scan.cuh)
    const T* s0;
    const T* xe;
    // look-back path (k_scan_mc_lb): small-chunk records (x after each at [14]);
    // null otherwise
    const double* xafter;
    int NCWs, Ps;
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
    const uint64_t pol_in = sk_policy_evict_first();
    auto win_of = [&](int g) { return MODE == 2 ? w0 + nwin - 1 - g : w0 + g; };
    auto issue = [&](int g) {
        const int w = win_of(g);
        if (MODE < 2) {
            const int y = w * (p.w128 ? SC_W * (int)sizeof(T) / 128 : SC_W / 8);
            sk_expect(&in_full[pw], (unsigned)(4 * SC_W * sizeof(T)));
            sc_tma3d(ib + 0 * SC_W, &tm.a, y, (int)q, &in_full[pw], pol_in);
            sc_tma3d(ib + 1 * SC_W, &tm.b, y, (int)q, &in_full[pw], pol_in);
            sc_tma3d(ib + 2 * SC_W, &tm.c, y, (int)q, &in_full[pw], pol_in);
            sc_tma3d(ib + 3 * SC_W, &tm.d, y, (int)q, &in_full[pw], pol_in);
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
    if (MODE == 2 && p.xafter) {  // look-back path: x after the small chunk that ends this chunk
        xa0 = (T)p.xafter[(int64_t)((q * p.Ps + (w0 + nwin + p.NCWs - 1) / p.NCWs - 1)) * 16 + 14];
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
        const bool edge = w == 0 || (int64_t)(w + 1) * SC_W > n;
        sk_wait(&in_full[pw], ph);
        ph ^= 1u;
        if (MODE == 0) {
            // ---- the window's forward map (product of the lane segment maps)
            T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
            sc_ld_rows_any(ib, lane, p.w128 != 0, ra, rb, rc, rd);
            sc_release_buf();  // this warp's reads of the buffer before the TMA refill
            if (lane == 0 && g + SC_NW < nwin) issue(g + SC_NW);
            if (edge) sc_fix_rows<T>(i0, n, ra, rb, rc, rd, p.keep_a0, p.keep_cn);
            sc_range(ra, rb, rc, rd);
            const int nvalid = (int)(n - i0 < 0 ? 0 : n - i0 < SC_R ? n - i0 : SC_R);
            SCM M = sc_wide((p.keep_cn && nvalid < SC_R) ? sc_fwd_map_n(ra, rb, rc, rd, nvalid) : sc_fwd_map(ra, rb, rc, rd));
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {  // lane l: lanes l .. l + 2d - 1 (later after earlier)
                const SCM o = sk_shfl_down(M, d);
                if ((lane & (2 * d - 1)) == 0) { M = sk_compose(o, M); smc_rescale(M); }
            }
            if (lane == 0) {
                double* s = wm + 8 * g;
                s[0] = M.a; s[1] = M.b; s[2] = M.c; s[3] = M.d; s[4] = M.e; s[5] = M.f; s[6] = M.g;
            }
        } else if (MODE == 1) {
            // ---- forward replay from the chunk's / previous window's state
            T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
            sc_ld_rows_any(ib, lane, p.w128 != 0, ra, rb, rc, rd);
            if (edge) sc_fix_rows<T>(i0, n, ra, rb, rc, rd, p.keep_a0, p.keep_cn);
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
            if constexpr (sizeof(T) == 8) {
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
            sc_store_x(p.x + q * n + i0, n - i0, xv);
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
// chunks (TRI_SCAN_MC_LB): HBM traffic 4 + 2 (+ the
// L2 re-read of each chunk) + 2 + 1 = 9 arrays instead of 13.
// Persistent CTAs take chunks of NCWs windows in ticket order (an atomic
// counter, so a CTA only ever waits on chunks that started before it).  Per
// chunk: phase A = every window's forward map (as pass 0) and the chunk's
// aggregate map, published with flag 1; warp 0 looks back over the earlier
// chunks of the system (32 flags per round: the nearest inclusive state and
// the aggregates after it) and publishes the chunk's inclusive state with flag
// 2; phase B = pass 1 on the chunk (re-read from L2, prefetched during the
// look-back).  k_scan_mc_lb_fin then turns the chunks' backward maps into the x
// after every chunk, which pass 2 (k_scan_mc<2>, big chunks that are unions of
// small ones) reads instead of reducing chunk maps.
// Measured (c3, fp64 n = 2^24, B200; profiles/r01_ncu_c3_scanmc_lb.txt): correct
// and bitwise reproducible, DRAM traffic as designed (586 MB read + 219 MB
// written by the look-back kernel: the L2 re-read hits), but the kernel runs at
// 3.3 TB/s -- 36 % of stall samples at __syncthreads while warp 0 reduces the
// chunk and looks back -- so the solve takes 0.30-0.33 ms against 0.29 ms for
// the three-pass path (small chunks of 24 / 32 / 48 / 64 / 80 windows: 0.39 /
// 0.35 / 0.31-0.34 / 0.30-0.32 / 0.32 ms).  Now only warp 0 waits at the end
// of phase A (the other warps arrive and start phase B; the next ticket, claimed
// just in time after the look-back, travels with the state hand-over):
// 0.380 / 0.342 / 0.307 / 0.301 ms at 24 / 32 / 48 / 64 windows.  Kept off by default
// (TRI_SCAN_MC_LB=0); the lever is to overlap the look-back of chunk t with
// phase A of chunk t + 1 (a dedicated look-back warp, two chunks per CTA in L2).
// Tried and measured slower (not kept): a lag-1 pipeline in which warp 0 looks
// back on chunk t - 1 after phase A of chunk t (so predecessors have had a phase
// longer to publish): correct, but 0.33-0.41 ms -- barrier stalls rose to 43 %
// and two chunks per CTA pushed the L2 re-read out (778 MB DRAM read;
// profiles/r01_ncu_c3_scanmc_lb_lag1.txt): the bubble is warp 0's serial
// reduce + publish, not waiting on flags.  Also measured and not kept: the
// other warps only ARRIVE at the post-phase-A barrier (warp 0 alone waits) with
// tickets claimed two chunks ahead: correct, but 2.3-2.7 ms -- a ticket
// claimed before its CTA can start it stalls every later chunk's look-back on
// its aggregate, so tickets must stay just-in-time.
// record per small chunk (16 values): [0..6] aggregate map, [8..10] inclusive
// state, [12..13] backward map (al, be), [14] x after the chunk
constexpr int SMC_REC = 16;

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
    unsigned* flag;    // [m Ps] (zeroed before the launch), then the ticket counter at [m Ps]
    int NCWs, Ps;      // windows per small chunk, small chunks per system
};

template <typename T>
__global__ void __launch_bounds__(SC_THREADS, 1) k_scan_mc_lb(const __grid_constant__ StreamMaps tm, ScanMCArgs<T> p,
                                                               ScanMCLB<T> lb) {
    using L = SMCLayout<T>;
    extern __shared__ __align__(16) unsigned char smc_smem_raw[];
    __shared__ int s_tk[2];
    __shared__ T s_st[4];
    unsigned char* sbase = smc_smem_raw + ((1024 - ((unsigned)__cvta_generic_to_shared(smc_smem_raw) & 1023)) & 1023);
    uint64_t* in_full = reinterpret_cast<uint64_t*>(sbase + L::off_bar);
    T* hv = reinterpret_cast<T*>(sbase + L::off_hv);
    double* wm0 = reinterpret_cast<double*>(sbase + L::off_wm);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, pw = warp;
    if (threadIdx.x == 0) {
        for (int i = 0; i < SC_NW; ++i) sk_bar_init(&in_full[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        s_tk[0] = (int)atomicAdd(&lb.flag[p.m * (int64_t)lb.Ps], 1u);
    }
    __syncthreads();
    const int64_t n = p.n;
    const int NC = p.NC, NCW = lb.NCWs;
    const int total = (int)(p.m * lb.Ps);
    T* ib = reinterpret_cast<T*>(sbase + L::off_in + pw * L::in_stride);
    const unsigned ib_s = (unsigned)__cvta_generic_to_shared(ib);
    (void)ib_s;
    const uint64_t pol_a = sk_policy_evict_normal();  // phase A: keep the chunk in L2 for phase B
    const uint64_t pol_b = sk_policy_evict_first();   // phase B: last use
    auto issue = [&](int q, int w, uint64_t pol) {
        const int y = w * (p.w128 ? SC_W * (int)sizeof(T) / 128 : SC_W / 8);
        sk_expect(&in_full[pw], (unsigned)(4 * SC_W * sizeof(T)));
        sc_tma3d(ib + 0 * SC_W, &tm.a, y, q, &in_full[pw], pol);
        sc_tma3d(ib + 1 * SC_W, &tm.b, y, q, &in_full[pw], pol);
        sc_tma3d(ib + 2 * SC_W, &tm.c, y, q, &in_full[pw], pol);
        sc_tma3d(ib + 3 * SC_W, &tm.d, y, q, &in_full[pw], pol);
    };
    unsigned ph = 0;
    int par = 0;
    int t = s_tk[0];
    const int pi = (pw + SC_NW - 1) % SC_NW;
    if (t < total && lane == 0) {
        const int q = t / lb.Ps, ch = t - q * lb.Ps;
        if (pw < min(NC, ch * NCW + NCW) - ch * NCW) issue(q, ch * NCW + pw, pol_a);
    }
    while (t < total) {
        const int q = t / lb.Ps, ch = t - q * lb.Ps;
        const int w0 = ch * NCW;
        const int nwin = min(NC, w0 + NCW) - w0;
        double* wm = wm0 + par * 8 * NCW;          // forward window maps (phase A)
        double* wmb = wm0 + (2 + par) * 8 * NCW;   // backward window maps (phase B)
        // ---- phase A: window forward maps
        for (int g = pw; g < nwin; g += SC_NW) {
            const int w = w0 + g;
            const int64_t i0 = (int64_t)w * SC_W + lane * SC_R;
            const bool edge = w == 0 || (int64_t)(w + 1) * SC_W > n;
            sk_wait(&in_full[pw], ph);
            ph ^= 1u;
            T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
            sc_ld_rows_any(ib, lane, p.w128 != 0, ra, rb, rc, rd);
            sc_release_buf();
            if (lane == 0) {
                if (g + SC_NW < nwin) issue((int)q, w + SC_NW, pol_a);
                else issue((int)q, w0 + pw, pol_b);  // phase B's first window, during the look-back
            }
            if (edge) sc_fix_rows<T>(i0, n, ra, rb, rc, rd, 0, 0);
            sc_range(ra, rb, rc, rd);
            SCM M = sc_wide(sc_fwd_map(ra, rb, rc, rd));
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const SCM o = sk_shfl_down(M, d);
                if ((lane & (2 * d - 1)) == 0) { M = sk_compose(o, M); smc_rescale(M); }
            }
            if (lane == 0) {
                double* s = wm + 8 * g;
                s[0] = M.a; s[1] = M.b; s[2] = M.c; s[3] = M.d; s[4] = M.e; s[5] = M.f; s[6] = M.g;
            }
        }
        // warp 0 waits for every warp's window maps; the others go straight on to
        // phase B (their chain waits for warp 0's first window anyway)
        if (warp == 0) asm volatile("bar.sync 13, %0;" ::"r"(SC_THREADS) : "memory");
        else asm volatile("bar.arrive 13, %0;" ::"r"(SC_THREADS) : "memory");
        if (warp == 0) {
            // aggregate of the chunk, published with flag 1
            const SCM R = smc_reduce_fwd(wm, nwin, lane);  // lane 0
            double* rec = lb.rec + (int64_t)t * SMC_REC;
            unsigned* fl = lb.flag;
            if (lane == 0 && ch > 0) {
                __stcg(rec + 0, R.a); __stcg(rec + 1, R.b); __stcg(rec + 2, R.c); __stcg(rec + 3, R.d);
                __stcg(rec + 4, R.e); __stcg(rec + 5, R.f); __stcg(rec + 6, R.g);
                smc_st_release_gpu(fl + t, 1u);  // release: the stores above are visible first
            }
            // look-back with a FIXED structure (bitwise reproducible): incoming state =
            // A_{t-1} ... A_{b+1} S_b, b = the chunk of the system at the largest multiple
            // of 32 below ch (S_b inclusive, published with flag 2), so one round of 32
            // flags; ch <= 32 starts from the system start when b = 0 ... and b's own
            // inclusive state is built the same way from its base
            SCM acc{1.0, 0.0, 0.0, 1.0, 0.0, 0.0, 1.0};
            double th = 1.0, ps = 0.0, de = 0.0;
            if (ch > 0) {
                const int tfirst = (int)(q * lb.Ps);
                const int b = tfirst + ((ch - 1) / 32) * 32;  // base chunk (inclusive state)
                const int nag = t - 1 - b;                     // aggregates after it, lanes 0 .. nag - 1
                const int j = t - 1 - lane;
                const unsigned want = lane < nag ? 1u : (lane == nag ? 2u : 0u);
                while (true) {
                    const unsigned v = want ? smc_ld_acquire_gpu(fl + j) : 0u;
                    if (!__any_sync(0xffffffffu, v < want)) break;
                    __nanosleep(32);
                }
                SCM A{1.0, 0.0, 0.0, 1.0, 0.0, 0.0, 1.0};
                if (lane < nag) {
                    const double* r = lb.rec + (int64_t)j * SMC_REC;
                    A = SCM{__ldcg(r + 0), __ldcg(r + 1), __ldcg(r + 2), __ldcg(r + 3), __ldcg(r + 4),
                            __ldcg(r + 5), __ldcg(r + 6)};
                }
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {  // lane l: A_{j_l} ... A_{j_{l+2d-1}} (lane l latest)
                    const SCM o = sk_shfl_down(A, d);
                    if ((lane & (2 * d - 1)) == 0) { A = sk_compose(A, o); smc_rescale(A); }
                }
                acc.a = __shfl_sync(0xffffffffu, A.a, 0); acc.b = __shfl_sync(0xffffffffu, A.b, 0);
                acc.c = __shfl_sync(0xffffffffu, A.c, 0); acc.d = __shfl_sync(0xffffffffu, A.d, 0);
                acc.e = __shfl_sync(0xffffffffu, A.e, 0); acc.f = __shfl_sync(0xffffffffu, A.f, 0);
                acc.g = __shfl_sync(0xffffffffu, A.g, 0);
                const double* r = lb.rec + (int64_t)b * SMC_REC;
                th = __ldcg(r + 8); ps = __ldcg(r + 9); de = __ldcg(r + 10);
            }
            const double it = fma(acc.a, th, acc.b * ps);
            const double ip = fma(acc.c, th, acc.d * ps);
            const double id = fma(acc.e, th, fma(acc.f, ps, acc.g * de));
            // inclusive state of this chunk, published with flag 2
            double ot = fma(R.a, it, R.b * ip), op = fma(R.c, it, R.d * ip), od = fma(R.e, it, fma(R.f, ip, R.g * id));
            if (lane == 0) {
                const double sc = sk_exp2_scale(ot);
                ot *= sc; op *= sc; od *= sc;
                __stcg(rec + 8, ot); __stcg(rec + 9, op); __stcg(rec + 10, od);
                smc_st_release_gpu(fl + t, 2u);
                const double si = sk_exp2_scale(it);
                s_st[0] = (T)(it * si); s_st[1] = (T)(ip * si); s_st[2] = (T)(id * si);
                s_tk[par ^ 1] = (int)atomicAdd(&lb.flag[total], 1u);  // the next chunk, just in time
            }
        }
        __syncwarp();
        // the next ticket: warp 0 from shared memory; the others through the chain
        // (hv[4 w + 3], handed over with the state); warps with no window here after
        // the end-of-chunk barrier
        int tn = warp == 0 ? s_tk[par ^ 1] : total;
        // ---- phase B: forward replay (pass 1) from the chunk's incoming state
        for (int g = pw; g < nwin; g += SC_NW) {
            const int w = w0 + g;
            const int64_t i0 = (int64_t)w * SC_W + lane * SC_R;
            const bool edge = w == 0 || (int64_t)(w + 1) * SC_W > n;
            sk_wait(&in_full[pw], ph);
            ph ^= 1u;
            T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
            sc_ld_rows_any(ib, lane, p.w128 != 0, ra, rb, rc, rd);
            if (edge) sc_fix_rows<T>(i0, n, ra, rb, rc, rd, 0, 0);
            sc_range(ra, rb, rc, rd);
            SCM M = sc_wide(sc_fwd_map(ra, rb, rc, rd));
            sc_fwd_scan(M, lane);
            if (g > 0) asm volatile("bar.sync %0, 64;" ::"r"(1 + pi) : "memory");
            T th, ps, de;
            if (g == 0) {
                th = s_st[0]; ps = s_st[1]; de = s_st[2];
            } else {
                th = hv[4 * pi + 0]; ps = hv[4 * pi + 1]; de = hv[4 * pi + 2];
                tn = (int)hv[4 * pi + 3];
            }
            const double ot = fma(M.a, (double)th, M.b * (double)ps);
            const double op = fma(M.c, (double)th, M.d * (double)ps);
            const double od = fma(M.e, (double)th, fma(M.f, (double)ps, M.g * (double)de));
            if (lane == 31) {
                const double sc = sk_exp2_scale(ot);
                hv[4 * pw + 0] = (T)(ot * sc); hv[4 * pw + 1] = (T)(op * sc); hv[4 * pw + 2] = (T)(od * sc);
                hv[4 * pw + 3] = (T)tn;
            }
            if (g + 1 < nwin) asm volatile("bar.arrive %0, 64;" ::"r"(1 + pw) : "memory");
            {
                const T it_ = (T)__shfl_up_sync(0xffffffffu, ot, 1);
                const T ip = (T)__shfl_up_sync(0xffffffffu, op, 1);
                const T id = (T)__shfl_up_sync(0xffffffffu, od, 1);
                if (lane > 0) { th = it_; ps = ip; de = id; }
            }
            sc_release_buf();
            if (lane == 0) {
                if (g + SC_NW < nwin) {
                    issue((int)q, w + SC_NW, pol_b);
                } else if (tn < total) {  // the next chunk's first window for this warp
                    const int qn = tn / lb.Ps, chn = tn - qn * lb.Ps;
                    if (pw < min(NC, chn * NCW + NCW) - chn * NCW) issue(qn, chn * NCW + pw, pol_a);
                }
            }
            T cp[SC_R], dp[SC_R];
            sc_fwd_replay(ra, rb, rc, rd, th, ps, de, cp, dp);
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
            if (lane == 0) { wmb[8 * g] = (double)al; wmb[8 * g + 1] = (double)be; }
        }
        __syncthreads();
        if (pw >= nwin) tn = s_tk[par ^ 1];
        // warps with no window in this chunk still prefetch the next one
        if (pw >= nwin && lane == 0 && tn < total) {
            const int qn = tn / lb.Ps, chn = tn - qn * lb.Ps;
            if (pw < min(NC, chn * NCW + NCW) - chn * NCW) issue(qn, chn * NCW + pw, pol_a);
        }
        if (warp == 0) {
            double al, be;
            smc_reduce_bwd(wmb, nwin, lane, al, be);
            if (lane == 0) { lb.rec[(int64_t)t * SMC_REC + 12] = al; lb.rec[(int64_t)t * SMC_REC + 13] = be; }
        }
        t = tn;
        par ^= 1;
    }
}

// x after every small chunk from the chunks' backward maps (one CTA per system):
// x_after(ch) = B_{ch+1}(... B_{Ps-1}(0)); written to rec[14]
template <typename T>
__global__ void __launch_bounds__(1024) k_scan_mc_lb_fin(ScanMCLB<T> lb) {
    __shared__ double sa[32], sb[32];
    const int64_t q = blockIdx.x;
    const int Ps = lb.Ps, tid = threadIdx.x, lane = tid & 31, wp = tid >> 5;
    double* rec = lb.rec + q * Ps * SMC_REC;
    const int per = (Ps + 1023) / 1024, lo = min(Ps, tid * per), hi = min(Ps, lo + per);
    double al = 0.0, be = 1.0;  // this thread's chunks composed: x_first(lo) = al + be x_after(hi - 1)
    for (int i = hi - 1; i >= lo; --i) {
        const double a2 = rec[(int64_t)i * SMC_REC + 12], b2 = rec[(int64_t)i * SMC_REC + 13];
        al = fma(b2, al, a2);
        be = b2 * be;
    }
    // exclusive suffix over threads: the map of all chunks after this thread's range
    double sal = al, sbe = be;  // inclusive suffix within the warp (lane l: lanes l..31)
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const double oa = __shfl_down_sync(0xffffffffu, sal, d), ob = __shfl_down_sync(0xffffffffu, sbe, d);
        if (lane + d < 32) { sal = fma(sbe, oa, sal); sbe = sbe * ob; }
    }
    if (lane == 0) { sa[wp] = sal; sb[wp] = sbe; }
    __syncthreads();
    // x after warp wp's range: the warps after it applied to 0
    double xw = 0.0;
    for (int v = 31; v > wp; --v) xw = fma(sb[v], xw, sa[v]);
    // x after this thread's range: lanes after it in the warp, then xw
    double ea = __shfl_down_sync(0xffffffffu, sal, 1), eb = __shfl_down_sync(0xffffffffu, sbe, 1);
    if (lane == 31) { ea = 0.0; eb = 1.0; }
    double x = fma(eb, xw, ea);
    for (int i = hi - 1; i >= lo; --i) {
        rec[(int64_t)i * SMC_REC + 14] = x;
        x = fma(rec[(int64_t)i * SMC_REC + 13], x, rec[(int64_t)i * SMC_REC + 12]);
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
