// k_scan_cl.cuh -- TRI_VARIANT_SCAN for INTERLEAVED batches of few system groups
// (c2-class: m = 1024 systems = 128 groups of 8, n ~ 10^3): one thread-block
// CLUSTER per group of 8 adjacent systems, the group's windows spread over all
// the warps of the cluster, the forward state and x handed between the CTAs of
// the cluster through distributed shared memory (multi-CTA
// per system with DSMEM exchange, Fig 11b, here for the k = 0 sweep).
//
// Paper: Thomas Eqs 2-4 as p-Thomas at k = 0,
// parallelised within a system as in k_scan.cuh (X21): every window of
// 32 rows x 8 systems is a 3x3 map of the forward state (theta, psi, delta) and
// an affine map of x for the back substitution; the chained kernel (k_scan<T, 8>)
// walks the windows of a group one after another across the 12 warps of one CTA
// (72 chained steps at c2: latency-bound, one group per SM).  Here the windows
// are independent until two short chains:
//   A  every warp: maps of its windows (loaded by TMA from HBM, kept in L2:
//      evict_last), composed into one warp map per system;
//   B  warp 0: the CTA's map; the incoming state arrives from CTA r - 1 of the
//      cluster (remote stores into this CTA's shared memory + a remote mbarrier
//      arrive, release/acquire at cluster scope), the outgoing state goes to
//      CTA r + 1 the same way, then every warp's incoming state;
//   C  every warp: windows again (L2), forward replay from the true incoming
//      states (c', d' in registers), the window's back-substitution map,
//      composed into one affine map per warp; every window's incoming state is
//      kept in shared memory;
//   D  warp 0: the CTA's backward map; x after the CTA's rows arrives from CTA
//      r + 1, x at its first row goes to CTA r - 1; x after every warp;
//   E  every warp, windows in reverse: replay again (L2, evict_first), back
//      substitution, x stores.
// HBM moves the compulsory 5 arrays (inputs once, x once); the second and third
// reads of the inputs hit L2.  Maps and states in fp64 (X22), exact power-of-two
// rescaling of every composed map and handed state.
#pragma once
#include "k_scan.cuh"

namespace tri {

constexpr int SCL_NW = 8;  // warps per CTA
constexpr int SCL_S = 8;   // systems per window (the interleaved window of k_scan<T, 8>)
constexpr int SCL_WR = SC_W / SCL_S;  // rows per window (32)
constexpr int SCL_WMAX = 8;           // windows per warp (shared-memory state table)

template <typename T>
struct SCLArgs {  // dynamic shared memory: SCL_NW staging buffers of SCLayout<T>::in_stride bytes + 1 KB slack
    T* x;
    int64_t n, m;  // rows, systems (one batch: row i of system q at i m + q)
    int wpw;       // windows per warp
};

struct SCLShared {
    double wmap[SCL_NW][SCL_S][8];              // phase A: warp forward maps
    double wst[SCL_NW][SCL_S][4];               // phase B: warp incoming states
    double winst[SCL_NW][SCL_WMAX][SCL_S][4];   // phase C: window incoming states
    double wbk[SCL_NW][SCL_S][2];               // phase C: warp backward maps (x_first = A + B x_after)
    double wxa[SCL_NW][SCL_S];                  // phase D: x after each warp's rows
    double cl_in[SCL_S][4];                     // written by CTA r - 1 (DSMEM)
    double cl_x[SCL_S];                         // written by CTA r + 1 (DSMEM)
    uint64_t full[SCL_NW];                      // TMA -> warp
    uint64_t bar_in, bar_x;                     // remote arrivals (8 each: one per system lane)
};

__device__ __forceinline__ unsigned scl_rank() {
    unsigned r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void scl_cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// address of `p` (this CTA's shared memory) in CTA `rank` of the cluster
__device__ __forceinline__ unsigned scl_remote(const void* p, unsigned rank) {
    unsigned r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"((unsigned)__cvta_generic_to_shared(p)), "r"(rank));
    return r;
}
__device__ __forceinline__ void scl_st_remote(unsigned addr, double v) {
    asm volatile("st.shared::cluster.f64 [%0], %1;" ::"r"(addr), "d"(v) : "memory");
}
__device__ __forceinline__ void scl_arrive_remote(unsigned bar_addr) {
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(bar_addr) : "memory");
}
__device__ __forceinline__ void scl_wait_cluster(uint64_t* bar, unsigned parity) {
    const unsigned a = (unsigned)__cvta_generic_to_shared(bar);
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "SCLW_%=:\n"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra SCLW_%=;\n"
        "}\n" ::"r"(a),
        "r"(parity)
        : "memory");
}

__device__ __forceinline__ void scl_rescale(SCM& M) {
    const double s = sc_scale2(M.a, M.b);
    M.a *= s; M.b *= s; M.c *= s; M.d *= s; M.e *= s; M.f *= s; M.g *= s;
}
__device__ __forceinline__ void scl_apply(const SCM& M, double& th, double& ps, double& de) {
    const double t = fma(M.a, th, M.b * ps), p = fma(M.c, th, M.d * ps), d = fma(M.e, th, fma(M.f, ps, M.g * de));
    const double s = sk_exp2_scale(t);
    th = t * s; ps = p * s; de = d * s;
}

template <typename T, int CL>
__global__ void __launch_bounds__(32 * SCL_NW) k_scan_cl(const __grid_constant__ StreamMaps tm, SCLArgs<T> p) {
    constexpr int NSEG = 32 / SCL_S;  // lane segments per system (4 x 8 rows)
    extern __shared__ __align__(16) unsigned char scl_smem_raw[];
    unsigned char* scl_smem =
        scl_smem_raw + ((1024 - ((unsigned)__cvta_generic_to_shared(scl_smem_raw) & 1023)) & 1023);
    __shared__ SCLShared sh;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int ls = lane % SCL_S, seg = lane / SCL_S;
    const unsigned rank = scl_rank();
    const int64_t grp = blockIdx.x / CL;
    const int64_t n = p.n, m = p.m;
    const int64_t qf = grp * SCL_S + ls;  // this lane's system
    const int nwin = (int)((n + SCL_WR - 1) / SCL_WR);
    const int w0 = ((int)rank * SCL_NW + warp) * p.wpw;                  // first window of the warp
    const int nw = max(0, min(p.wpw, nwin - w0));                       // windows of the warp
    T* buf = reinterpret_cast<T*>(scl_smem + warp * SCLayout<T>::in_stride);

    if (threadIdx.x == 0) {
        for (int i = 0; i < SCL_NW; ++i) sk_bar_init(&sh.full[i], 1);
        sk_bar_init(&sh.bar_in, SCL_S);
        sk_bar_init(&sh.bar_x, SCL_S);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    scl_cluster_sync();  // every CTA's barriers exist before any remote arrival

    // loads l = 0 .. 3 nw - 1: windows forward (A), forward (C), backward (E)
    const uint64_t pol_keep = sk_policy_evict_last(), pol_last = sk_policy_evict_first();
    auto win_of = [&](int l) { return l < 2 * nw ? w0 + (l < nw ? l : l - nw) : w0 + (3 * nw - 1 - l); };
    auto issue = [&](int l) {
        if (l >= 3 * nw) return;
        const int y = win_of(l) * SCL_WR, xq = (int)(grp * SCL_S);
        const uint64_t pol = l < 2 * nw ? pol_keep : pol_last;
        sk_expect(&sh.full[warp], (unsigned)(4 * SC_W * sizeof(T)));
        sc_tma3d(buf + 0 * SC_W, &tm.a, y, 0, &sh.full[warp], pol, xq);
        sc_tma3d(buf + 1 * SC_W, &tm.b, y, 0, &sh.full[warp], pol, xq);
        sc_tma3d(buf + 2 * SC_W, &tm.c, y, 0, &sh.full[warp], pol, xq);
        sc_tma3d(buf + 3 * SC_W, &tm.d, y, 0, &sh.full[warp], pol, xq);
    };
    // rows of load l in registers (identity rows outside the system / batch),
    // then the next load into the freed buffer
    auto rows = [&](int l, T (&ra)[SC_R], T (&rb)[SC_R], T (&rc)[SC_R], T (&rd)[SC_R]) {
        sk_wait(&sh.full[warp], (unsigned)(l & 1));
        sc_ld_rows_il<SCL_S>(buf, ls, seg, ra, rb, rc, rd);
        sc_release_buf();
        if (lane == 0) issue(l + 1);
        const int wi = win_of(l);
        sc_fix_rows<T>((int64_t)wi * SCL_WR + seg * SC_R, n, ra, rb, rc, rd);
        if (qf >= m) {
#pragma unroll
            for (int u = 0; u < SC_R; ++u) { ra[u] = T(0); rb[u] = T(1); rc[u] = T(0); rd[u] = T(0); }
        }
        sc_range(ra, rb, rc, rd);
    };
    // window map, inclusive over the lane segments of each system
    auto wmap = [&](const T (&ra)[SC_R], const T (&rb)[SC_R], const T (&rc)[SC_R], const T (&rd)[SC_R]) {
        SCM M = sc_wide(sc_fwd_map(ra, rb, rc, rd));
#pragma unroll
        for (int dd = SCL_S; dd < 32; dd <<= 1) {
            const SCM o = sk_shfl_up(M, dd);
            if (lane >= dd) M = sk_compose(M, o);
        }
        return M;
    };
    // lane incoming state from the window's incoming state (th, ps, de) and the
    // inclusive lane maps; returns the window's outgoing state in (th, ps, de)
    auto lane_state = [&](const SCM& M, double& th, double& ps, double& de, T& lt, T& lp, T& ld) {
        const double ot = fma(M.a, th, M.b * ps), op = fma(M.c, th, M.d * ps),
                     od = fma(M.e, th, fma(M.f, ps, M.g * de));
        const double it = __shfl_up_sync(0xffffffffu, ot, SCL_S), ip = __shfl_up_sync(0xffffffffu, op, SCL_S),
                     id = __shfl_up_sync(0xffffffffu, od, SCL_S);
        const double s0 = sk_exp2_scale(seg > 0 ? it : th);
        lt = (T)((seg > 0 ? it : th) * s0); lp = (T)((seg > 0 ? ip : ps) * s0); ld = (T)((seg > 0 ? id : de) * s0);
        // outgoing state of the window: the last segment's
        th = __shfl_sync(0xffffffffu, ot, (NSEG - 1) * SCL_S + ls);
        ps = __shfl_sync(0xffffffffu, op, (NSEG - 1) * SCL_S + ls);
        de = __shfl_sync(0xffffffffu, od, (NSEG - 1) * SCL_S + ls);
        const double s = sk_exp2_scale(th);
        th *= s; ps *= s; de *= s;
    };
    // suffix scan of the lanes' back-substitution maps over the segments:
    // x at the lane's first row = al + be x_after_window
    auto bwd_scan = [&](T& al, T& be) {
#pragma unroll
        for (int dd = SCL_S; dd < 32; dd <<= 1) {
            const T oa = __shfl_down_sync(0xffffffffu, al, dd), ob = __shfl_down_sync(0xffffffffu, be, dd);
            if (lane + dd < 32) { al = fma(be, oa, al); be = be * ob; }
        }
    };

    if (lane == 0) issue(0);
    // ---- A: warp map (later windows after earlier ones)
    {
        SCM W{1.0, 0.0, 0.0, 1.0, 0.0, 0.0, 1.0};
        for (int i = 0; i < nw; ++i) {
            T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
            rows(i, ra, rb, rc, rd);
            const SCM M = wmap(ra, rb, rc, rd);
            W = sk_compose(M, W);
            scl_rescale(W);
        }
        if (seg == NSEG - 1) {
            double* o = sh.wmap[warp][ls];
            o[0] = W.a; o[1] = W.b; o[2] = W.c; o[3] = W.d; o[4] = W.e; o[5] = W.f; o[6] = W.g;
        }
    }
    __syncthreads();
    // ---- B: the cluster's forward chain (warp 0, one lane per system)
    if (warp == 0 && lane < SCL_S) {
        auto ld = [&](int w) {
            const double* o = sh.wmap[w][lane];
            return SCM{o[0], o[1], o[2], o[3], o[4], o[5], o[6]};
        };
        SCM Tm{1.0, 0.0, 0.0, 1.0, 0.0, 0.0, 1.0};
        for (int w = 0; w < SCL_NW; ++w) { Tm = sk_compose(ld(w), Tm); scl_rescale(Tm); }
        double th = 1.0, ps = 0.0, de = 0.0;  // theta_{-1} = 1, psi_0 = 0, delta_{-1} = 0
        if (rank > 0) {
            scl_wait_cluster(&sh.bar_in, 0);
            th = sh.cl_in[lane][0]; ps = sh.cl_in[lane][1]; de = sh.cl_in[lane][2];
        }
        if (rank + 1 < CL) {
            double t = th, q = ps, d = de;
            scl_apply(Tm, t, q, d);
            scl_st_remote(scl_remote(&sh.cl_in[lane][0], rank + 1), t);
            scl_st_remote(scl_remote(&sh.cl_in[lane][1], rank + 1), q);
            scl_st_remote(scl_remote(&sh.cl_in[lane][2], rank + 1), d);
            scl_arrive_remote(scl_remote(&sh.bar_in, rank + 1));
        }
        for (int w = 0; w < SCL_NW; ++w) {
            sh.wst[w][lane][0] = th; sh.wst[w][lane][1] = ps; sh.wst[w][lane][2] = de;
            scl_apply(ld(w), th, ps, de);
        }
    }
    __syncthreads();
    // ---- C: forward replay per window, back-substitution maps composed per warp
    {
        double th = sh.wst[warp][ls][0], ps = sh.wst[warp][ls][1], de = sh.wst[warp][ls][2];
        T A = T(0), B = T(1);  // x at the warp's first row = A + B x_after(window i)
        for (int i = 0; i < nw; ++i) {
            T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
            rows(nw + i, ra, rb, rc, rd);
            const SCM M = wmap(ra, rb, rc, rd);
            if (seg == 0) {
                double* o = sh.winst[warp][i][ls];
                o[0] = th; o[1] = ps; o[2] = de;
            }
            T lt, lp, lq;
            lane_state(M, th, ps, de, lt, lp, lq);
            T cp[SC_R], dp[SC_R];
            sc_fwd_replay(ra, rb, rc, rd, lt, lp, lq, cp, dp);
            T al, be;
            sc_bwd_map(cp, dp, al, be);
            bwd_scan(al, be);
            A = fma(B, al, A);
            B = B * be;
        }
        if (seg == 0) { sh.wbk[warp][ls][0] = (double)A; sh.wbk[warp][ls][1] = (double)B; }
    }
    __syncthreads();
    // ---- D: the cluster's backward chain
    if (warp == 0 && lane < SCL_S) {
        double A = 0.0, B = 1.0;
        for (int w = 0; w < SCL_NW; ++w) { A = fma(B, sh.wbk[w][lane][0], A); B *= sh.wbk[w][lane][1]; }
        double xa = 0.0;  // x after the last row of the system
        if (rank + 1 < CL) {
            scl_wait_cluster(&sh.bar_x, 0);
            xa = sh.cl_x[lane];
        }
        if (rank > 0) {
            scl_st_remote(scl_remote(&sh.cl_x[lane], rank - 1), fma(B, xa, A));
            scl_arrive_remote(scl_remote(&sh.bar_x, rank - 1));
        }
        for (int w = SCL_NW - 1; w >= 0; --w) {
            sh.wxa[w][lane] = xa;
            xa = fma(sh.wbk[w][lane][1], xa, sh.wbk[w][lane][0]);
        }
    }
    __syncthreads();
    // ---- E: windows in reverse: replay, back substitution, x
    {
        T xa = (T)sh.wxa[warp][ls];  // x after the warp's current (last unsolved) window
        for (int i = nw - 1; i >= 0; --i) {
            T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
            rows(2 * nw + (nw - 1 - i), ra, rb, rc, rd);
            const SCM M = wmap(ra, rb, rc, rd);
            double th = sh.winst[warp][i][ls][0], ps = sh.winst[warp][i][ls][1], de = sh.winst[warp][i][ls][2];
            T lt, lp, lq;
            lane_state(M, th, ps, de, lt, lp, lq);
            T cp[SC_R], dp[SC_R];
            sc_fwd_replay(ra, rb, rc, rd, lt, lp, lq, cp, dp);
            T al, be;
            sc_bwd_map(cp, dp, al, be);
            bwd_scan(al, be);
            const T xf = fma(be, xa, al);                     // x at the lane's first row
            T x = __shfl_down_sync(0xffffffffu, xf, SCL_S);   // x after the lane's rows
            if (seg == NSEG - 1) x = xa;
            T xv[SC_R];
#pragma unroll
            for (int t = SC_R - 1; t >= 0; --t) {
                x = fma(-cp[t], x, dp[t]);
                xv[t] = x;
            }
            const int64_t r0 = (int64_t)win_of(2 * nw + (nw - 1 - i)) * SCL_WR + seg * SC_R;
            if (qf < m) {
#pragma unroll
                for (int t = 0; t < SC_R; ++t)
                    if (r0 + t < n) __stcs(p.x + (r0 + t) * m + qf, xv[t]);
            }
            xa = __shfl_sync(0xffffffffu, xf, ls);  // x at the window's first row
        }
    }
    scl_cluster_sync();  // no CTA leaves while a peer may still write its shared memory
}

}  // namespace tri
