// k_scan_w512.cuh -- TRI_VARIANT_SCAN for fp64 CONTIGUOUS batches of chained
// windows (BASELINE c5): the k_scan chain (k_scan.cuh) with 512-row windows,
// 16 rows per lane instead of 8.
//
// Paper: Thomas, Eqs 2-4 (reading X2); p-Thomas at k = 0 for M > P
// (Sec. III.B / III.D); the segment-map form of the sweeps is
// DESIGN.md X21.
//
// Why: k_scan at c5 issues ~1070 warp instructions per 256-row window step and
// runs at ~0.5 IPC per SMSP with 3 warps per SMSP (latency-bound, not HBM-bound:
// its memory-only pipeline takes 1.70 ms of the 1.90 ms).  A third of those
// instructions are the per-window work that does not scale with the rows of a
// lane: the 5-level shuffle scans of the 3x3 forward maps and affine backward
// maps (fp64 SHFL = two 32-bit shuffles at one warp instruction per clock per
// SM), the handover between warps, the slot table and the TMA issue.  With 16
// rows per lane a window holds 512 rows, so that work is paid once per 512 rows
// (ncu at c5: 740 M warp instructions instead of 1104 M).  The rows are streamed
// from the staging buffer 8 at a time (they do not all fit in registers; 8-row
// groups measured 0.8 % faster than 4-row ones), the
// lane's forward map is rescaled by an exact power of two every 8 rows (raw fp64
// rows with pivots in 2^+-64, X21), and 8-row groups whose live pivots leave
// 2^+-64 are renormalised by 2^-exponent(b) (warp-uniform test per group;
// scaling a row by a power of two leaves c', d' unchanged and is exact, so the
// two passes over a window need not take the same decisions).
//
// Measured (c5, same box, alternating runs): 1.87-1.91 ms vs 1.92-1.95 ms for the
// 256-row kernel with 8 warps per CTA; 12 warps (16 KB staging each leaves 4
// on-chip 8 KB slots, so 90 % of the slots spill to L2 and 0.77 GB per solve
// leaks to DRAM): 1.98-2.01 ms; 10 warps 1.93-1.94; 6 warps 2.15.  The lag delta
// (2, 4, 8) is within the noise.
//
// Structure (as k_scan, S = 1): persistent CTAs, S5_NW warps; step g = (system j,
// window w) on warp g % S5_NW: TMA load of the window (4 arrays x 4 KB, tensor view
// [m][n/16][16], 128-byte box rows, 128B swizzle: lane l's 16 rows are box row l),
// forward map, back-substitution map of the window delta steps behind (c', d'
// from its storage slot, held in registers, loads issued before the TMA wait),
// both scans, the handover through named barrier 1 + warp, forward replay (c', d'
// into the slot the backward part just read), back substitution, 256-bit x
// stores.  Slots of 8 KB: the first S_on in shared memory (12 at c5), the rest
// in a per-CTA L2-resident spill region.
#pragma once
#include "k_scan.cuh"

namespace tri {

constexpr int S5_R = 16;             // rows per lane
constexpr int S5_W = 32 * S5_R;      // rows per window (512)
#ifndef S5_G_DEF
#define S5_G_DEF 8
#endif
constexpr int S5_G = S5_G_DEF;       // rows per streamed group
#ifndef S5_NW_DEF
#define S5_NW_DEF 8
#endif
constexpr int S5_NW = S5_NW_DEF;     // warps per CTA (staging 16 KB per warp: fewer warps leave smem for slots)
constexpr int S5_THREADS = 32 * S5_NW;

struct S5Layout {
    static constexpr int in_bytes = 4 * S5_W * 8;                        // one window, 4 arrays (16 KB)
    static constexpr int in_stride = in_bytes;                           // 1 KB multiple (swizzle atoms)
    static constexpr int off_in = 0;
    static constexpr int off_st = off_in + S5_NW * in_stride;            // [NW][theta|psi|delta|-]
    static constexpr int off_xh = off_st + S5_NW * 4 * 8;                // [NW] x handover
    static constexpr int off_bar = (off_xh + S5_NW * 8 + 7) / 8 * 8;     // [NW] in_full
    static constexpr int off_tab = off_bar + S5_NW * 8;                  // [K][NC] slot table (u32)
    static constexpr int slot_bytes = S5_W * 16;                         // (c', d') per row
    static __host__ __device__ constexpr int off_store(int NC, int D) {
        return (off_tab + 4 * (3 * NC + D) + 1023) / 1024 * 1024;
    }
    static __host__ __device__ constexpr int smem_bytes(int NC, int D, int S_on) {
        return off_store(NC, D) + S_on * slot_bytes + 1024;
    }
};

// rows G h .. G h + G - 1 of lane `lane` from the window's staging buffer: box row
// `lane` of each array (128 bytes = 16 fp64), 16-byte chunk c at c ^ (lane & 7)
__device__ __forceinline__ void s5_ld_group(const double* ib, int lane, int h, double (&a)[S5_G], double (&b)[S5_G],
                                            double (&c)[S5_G], double (&d)[S5_G]) {
    const int sw = lane & 7;
#pragma unroll
    for (int k = 0; k < S5_G / 2; ++k) {
        const int o = lane * 16 + ((((S5_G / 2) * h + k) ^ sw) * 2);
        const double2 va = *reinterpret_cast<const double2*>(ib + 0 * S5_W + o);
        const double2 vb = *reinterpret_cast<const double2*>(ib + 1 * S5_W + o);
        const double2 vc = *reinterpret_cast<const double2*>(ib + 2 * S5_W + o);
        const double2 vd = *reinterpret_cast<const double2*>(ib + 3 * S5_W + o);
        a[2 * k] = va.x; a[2 * k + 1] = va.y;
        b[2 * k] = vb.x; b[2 * k + 1] = vb.y;
        c[2 * k] = vc.x; c[2 * k + 1] = vc.y;
        d[2 * k] = vd.x; d[2 * k + 1] = vd.y;
    }
}

// group fix-ups: a_0, c_{n-1} outside A; identity rows past n (edge windows only).
// Then the range decision (fp64 raw rows, X21): `scl` bit h set = renormalise
// group h by 2^-exponent(b) because a live pivot leaves 2^+-64; the map pass
// takes the decision (warp-uniform), the replay pass reuses it (bit known).
__device__ __forceinline__ void s5_fix_group(bool edge, int64_t i0, int64_t n, int h, unsigned& scl, bool decide,
                                             double (&a)[S5_G], double (&b)[S5_G], double (&c)[S5_G],
                                             double (&d)[S5_G]) {
    if (__builtin_expect(edge, 0)) {
#pragma unroll
        for (int u = 0; u < S5_G; ++u) {
            const int64_t i = i0 + u;
            if (i == 0) a[u] = 0.0;
            if (i == n - 1) c[u] = 0.0;
            if (i >= n) { a[u] = 0.0; b[u] = 1.0; c[u] = 0.0; d[u] = 0.0; }
        }
    }
    if (decide) {
        unsigned mx = 0u, mn = 0xffffffffu;
#pragma unroll
        for (int u = 0; u < S5_G; ++u) {
            const unsigned hb = (unsigned)__double2hiint(b[u]) & 0x7ff00000u;
            mx = max(mx, hb);
            mn = min(mn, hb);
        }
        if (__any_sync(0xffffffffu, mx > ((1023u + 64u) << 20) || mn < ((1023u - 64u) << 20))) scl |= 1u << h;
    }
    if (scl & (1u << h)) {
#pragma unroll
        for (int u = 0; u < S5_G; ++u) {
            const double s = sk_exp2_scale(b[u]);
            a[u] *= s; b[u] *= s; c[u] *= s; d[u] *= s;
        }
    }
}

template <typename T>
__global__ void __launch_bounds__(S5_THREADS, 1) k_scan_w512(const __grid_constant__ StreamMaps tm, ScanArgs<T> p) {
    static_assert(sizeof(T) == 8, "fp64 only");
    using L = S5Layout;
    extern __shared__ __align__(16) unsigned char s5_smem_raw[];
    unsigned char* sbase = s5_smem_raw + ((1024 - ((unsigned)__cvta_generic_to_shared(s5_smem_raw) & 1023)) & 1023);
    uint64_t* in_full = reinterpret_cast<uint64_t*>(sbase + L::off_bar);
    unsigned* tab = reinterpret_cast<unsigned*>(sbase + L::off_tab);
    double* stt = reinterpret_cast<double*>(sbase + L::off_st);
    double* xh = reinterpret_cast<double*>(sbase + L::off_xh);
    const int NC = p.NC;
    const unsigned store_s = (unsigned)__cvta_generic_to_shared(sbase + L::off_store(NC, p.delta));
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, pw = warp;
    if (threadIdx.x == 0) {
        for (int i = 0; i < S5_NW; ++i) sk_bar_init(&in_full[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    for (int i = threadIdx.x; i < 3 * NC + p.delta; i += blockDim.x) tab[i] = 0u;
    __syncthreads();

    const int64_t n = p.n;
    const int nsys = (int)((p.m - blockIdx.x + gridDim.x - 1) / gridDim.x);
    double* ib = reinterpret_cast<double*>(sbase + L::off_in + pw * L::in_stride);
    const uint64_t pol_in = SC_POL_IN, pol_sp = SC_POL_SP;
    auto issue = [&](int jj, int ww) {
        const int q = (int)(blockIdx.x + (int64_t)jj * gridDim.x);
        sk_expect(&in_full[pw], (unsigned)L::in_bytes);
        const int y = ww * (S5_W / 16);  // 128-byte rows of the [m][n/16][16] view
        sc_tma3d(ib + 0 * S5_W, &tm.a, y, q, &in_full[pw], pol_in);
        sc_tma3d(ib + 1 * S5_W, &tm.b, y, q, &in_full[pw], pol_in);
        sc_tma3d(ib + 2 * S5_W, &tm.c, y, q, &in_full[pw], pol_in);
        sc_tma3d(ib + 3 * S5_W, &tm.d, y, q, &in_full[pw], pol_in);
    };
    unsigned ph = 0;
    const int D = p.delta;
    const int NS = NC + D;
    const int K = 3 + (D - 1) / NC;
    const int nfwd = nsys * NC;
    const int total = nfwd + NC + D;
    const int nspill = NS - p.S_on;
    double* spill_cta = p.spill + (int64_t)blockIdx.x * (int64_t)(nspill > 0 ? nspill : 0) * (S5_W * 2);
    int j = 0, w = pw;
    while (w >= NC) { w -= NC; ++j; }
    if (lane == 0 && pw < nfwd) issue(j, w);
    const int pi = (pw + S5_NW - 1) % S5_NW;
    // incremental bookkeeping (k_scan): forward (j, jk = j % K, jt = j % 65535 + 1),
    // backward index g - NC - D = bjv NC + br
    int jk = j % K, jt = j % 65535 + 1;
    int bjv, br;
    {
        const int b0 = pw - NC - D;
        bjv = b0 >= 0 ? b0 / NC : -((-b0 + NC - 1) / NC);
        br = b0 - bjv * NC;
    }
    int bk = ((bjv % K) + K) % K, bt = ((bjv % 65535) + 65535) % 65535 + 1;

    for (int g = pw; g < total; g += S5_NW) {
        const int cj = j, cw = w, cjk = jk, cjt = jt;
        w += S5_NW;
        while (w >= NC) {
            w -= NC; ++j;
            jk = jk + 1 == K ? 0 : jk + 1;
            jt = jt == 65535 ? 1 : jt + 1;
        }
        const int bj = bjv, bjk = bk, bjt = bt, wb = NC - 1 - br;
        br += S5_NW;
        while (br >= NC) {
            br -= NC; ++bjv;
            bk = bk + 1 == K ? 0 : bk + 1;
            bt = bt == 65535 ? 1 : bt + 1;
        }
        const bool fwd = cj < nsys, bwd = bj >= 0;
        int slot = g;
        if (bwd) {  // window (bj, wb) stored >= delta + 1 steps ago (release / acquire, k_scan)
            const int* e = reinterpret_cast<const int*>(&tab[bjk * NC + wb]);
            unsigned v = (unsigned)sk_ld_acquire(e);
            while ((v >> 16) != (unsigned)bjt) {
                __nanosleep(64);
                v = (unsigned)sk_ld_acquire(e);
            }
            slot = (int)(v & 0xffffu);
        }
        const bool res = slot < p.S_on;
        const unsigned sp_s = store_s + (unsigned)(slot * L::slot_bytes);
        double* sp_g = spill_cta + (size_t)(res ? 0 : slot - p.S_on) * (S5_W * 2);

        // ---- backward: (c', d') of window (bj, wb), held in registers
        double cpb[S5_R], dpb[S5_R];
        if (bwd) {
            if (res) {
#pragma unroll
                for (int t = 0; t < S5_R; ++t) sc_lds2(sp_s + 16u * (t * 32 + lane), cpb[t], dpb[t]);
            } else {
#pragma unroll
                for (int t = 0; t < S5_R; ++t) {
                    const double2 v = __ldcg(reinterpret_cast<const double2*>(sp_g + 2 * (t * 32 + lane)));
                    cpb[t] = v.x; dpb[t] = v.y;
                }
            }
        } else {
#pragma unroll
            for (int t = 0; t < S5_R; ++t) { cpb[t] = 0.0; dpb[t] = 0.0; }
        }

        // ---- forward: the lane's 16-row map, rows streamed from the staging buffer
        const int64_t i0 = (int64_t)cw * S5_W + lane * S5_R;
        const bool edge = cw == 0 || (int64_t)(cw + 1) * S5_W >= n;  // holds row 0 or row n - 1
        SCM M{1.0, 0.0, 0.0, 1.0, 0.0, 0.0, 1.0};
        unsigned scl = 0u;  // per 4-row group: renormalised (decided by the map pass)
        if (fwd) {
            sk_wait(&in_full[pw], ph);
            ph ^= 1u;
            double t1 = 1.0, p1 = 0.0, d1 = 0.0, t2 = 0.0, p2 = 1.0, d2 = 0.0, d3 = 1.0;
#pragma unroll
            for (int h = 0; h < S5_R / S5_G; ++h) {
                double ra[S5_G], rb[S5_G], rc[S5_G], rd[S5_G];
                s5_ld_group(ib, lane, h, ra, rb, rc, rd);
                s5_fix_group(edge, i0 + h * S5_G, n, h, scl, true, ra, rb, rc, rd);
#pragma unroll
                for (int u = 0; u < S5_G; ++u) {
                    const double au = ra[u], bu = rb[u], cu = rc[u], du = rd[u];
                    const double nt1 = fma(bu, t1, -au * p1), np1 = cu * t1, nd1 = fma(du, t1, -au * d1);
                    const double nt2 = fma(bu, t2, -au * p2), np2 = cu * t2, nd2 = fma(du, t2, -au * d2);
                    d3 = -au * d3;
                    t1 = nt1; p1 = np1; d1 = nd1;
                    t2 = nt2; p2 = np2; d2 = nd2;
                }
                if (((h + 1) * S5_G) % 8 == 0) {  // every 8 rows: exact power-of-two rescale
                    const double s = sc_scale2(t1, t2);
                    t1 *= s; p1 *= s; d1 *= s; t2 *= s; p2 *= s; d2 *= s; d3 *= s;
                }
            }
            M = SCM{t1, t2, p1, p2, d1, d2, d3};
        }
        // the backward map after the forward one: the slot loads (L2 when spilled)
        // were issued before the TMA wait and the forward map
        double al = dpb[S5_R - 1], be = -cpb[S5_R - 1];
#pragma unroll
        for (int t = S5_R - 2; t >= 0; --t) {
            al = fma(-cpb[t], al, dpb[t]);
            be = -cpb[t] * be;
        }
        if (bwd && !fwd && !res) {
            // draining steps: this spilled slot is never written again in this solve;
            // its (c', d') are in registers (used above), so drop its dirty L2 lines
            // instead of letting them be written back during the next solve
            __syncwarp();
#pragma unroll
            for (int k = 0; k < L::slot_bytes / 128 / 32; ++k)
                asm volatile("discard.global.L2 [%0], 128;" ::"l"(sp_g + (k * 32 + lane) * 16) : "memory");
        }
        sc_scans<1>(M, al, be, lane);

        // ---- the serial steps: the forward state and x of step g - 1 (named barrier 1 + pi)
        if (g > 0) asm volatile("bar.sync %0, 64;" ::"r"(1 + pi) : "memory");
        const double xw = (bwd && wb < NC - 1) ? xh[pi] : 0.0;
        double th = 1.0, ps = 0.0, de = 0.0;
        if (fwd && cw > 0) {
            th = stt[pi * 4 + 0];
            ps = stt[pi * 4 + 1];
            de = stt[pi * 4 + 2];
        }
        const double xs = fma(be, xw, al);
        const double ot = fma(M.a, th, M.b * ps);
        const double op = fma(M.c, th, M.d * ps);
        const double od = fma(M.e, th, fma(M.f, ps, M.g * de));
        if (lane == 0) xh[pw] = xs;
        if (lane == 31) {
            const double sc = sk_exp2_scale(ot);
            stt[pw * 4 + 0] = ot * sc;
            stt[pw * 4 + 1] = op * sc;
            stt[pw * 4 + 2] = od * sc;
        }
        if (g + 1 < total) asm volatile("bar.arrive %0, 64;" ::"r"(1 + pw) : "memory");
        double x = __shfl_down_sync(0xffffffffu, xs, 1);
        if (lane == 31) x = xw;
        {
            const double it_ = __shfl_up_sync(0xffffffffu, ot, 1);
            const double ip = __shfl_up_sync(0xffffffffu, op, 1);
            const double id = __shfl_up_sync(0xffffffffu, od, 1);
            if (lane > 0) { th = it_; ps = ip; de = id; }
        }

        // ---- forward replay: c', d' (Eqs 2-3) into the slot, rows streamed again
        if (fwd) {
#pragma unroll
            for (int h = 0; h < S5_R / S5_G; ++h) {
                double ra[S5_G], rb[S5_G], rc[S5_G], rd[S5_G];
                s5_ld_group(ib, lane, h, ra, rb, rc, rd);
                s5_fix_group(edge, i0 + h * S5_G, n, h, scl, false, ra, rb, rc, rd);
                if (h == S5_R / S5_G - 1) {  // the buffer's last read: refill it
                    sc_release_buf();
                    if (lane == 0 && g + S5_NW < nfwd) issue(j, w);
                }
#pragma unroll
                for (int u = 0; u < S5_G; ++u) {
                    const double nt = fma(rb[u], th, -ra[u] * ps);
                    const double np = rc[u] * th;
                    const double nd = fma(rd[u], th, -ra[u] * de);
                    const double inv = rcp(nt);
                    const double c_ = np * inv, d_ = nd * inv;
                    const int t = h * S5_G + u;
                    if (res) sc_sts2(sp_s + 16u * (t * 32 + lane), c_, d_);
                    else sk_st_global_last(sp_g + 2 * (t * 32 + lane), c_, d_, pol_sp);
                    th = nt; ps = np; de = nd;
                }
                if (((h + 1) * S5_G) % 8 == 0) {
                    const double s = sk_exp2_scale(th);
                    th *= s; ps *= s; de *= s;
                }
            }
            __syncwarp();
            if (lane == 0)
                sk_st_release(reinterpret_cast<int*>(&tab[cjk * NC + cw]), (int)(((unsigned)cjt << 16) | (unsigned)slot));
        }
        // ---- backward replay: x (Eq 4) of window (bj, wb), 256-bit stores
        if (bwd) {
            double xv[S5_R];
#pragma unroll
            for (int t = S5_R - 1; t >= 0; --t) {
                x = fma(-cpb[t], x, dpb[t]);
                xv[t] = x;
            }
            const int64_t qb = blockIdx.x + (int64_t)bj * gridDim.x;
            const int64_t xr = (int64_t)wb * S5_W + lane * S5_R;
            double* xo = p.x + qb * p.xsys + xr;
            const int64_t rmax = n - xr;
            if (rmax >= S5_R && p.x32) {
#pragma unroll
                for (int t = 0; t < S5_R; t += 4)
                    asm volatile(SC_XST ".v4.f64 [%0], {%1, %2, %3, %4};" ::"l"(xo + t), "d"(xv[t]), "d"(xv[t + 1]),
                                 "d"(xv[t + 2]), "d"(xv[t + 3])
                                 : "memory");
            } else {
#pragma unroll
                for (int t = 0; t < S5_R; ++t)
                    if (t < rmax) __stcs(xo + t, xv[t]);
            }
        }
    }
}

}  // namespace tri
