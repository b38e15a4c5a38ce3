// k_scan_grid.cuh -- TRI_VARIANT_SCAN on the INTERLEAVED layout (and unit-system-
// stride STRIDED / BATCHED views) when the batch is small enough that every SM
// holds a piece of it at once: p-Thomas at k = 0 (M > P) with the
// sweeps of each system split over the rows of Q CTAs.
//
// Paper: Thomas, Eqs 2-4; p-Thomas, one thread per (sub)system
// (Sec. III.B) -- here lane l of a warp owns system l of a 32-system
// block for a run of R consecutive rows (a 256-byte row of the interleaved
// layout per array and row: coalesced, P:647-653's access pattern).
//
// Why not the chained SCAN kernel (k_scan<T, 8>): at BASELINE c2 (1024 systems of
// 1024 rows) it has 128 8-system groups, one per SM, each a chain of 72 window
// steps -- latency-bound at 28 % of the HBM roofline (profiles/r02_ncu_c2_scanil.txt).
// Here the whole batch is in flight at once:
//
//   The Q CTAs of a 32-system block form one thread-block cluster; CTA q (its
//   cluster rank) owns rows [q RC, (q+1) RC) of the block's 32 systems, RC = 16
//   warps x R rows (R <= 16, a multiple of 4).
//   phase A  every warp streams its R rows (TMA boxes [4 rows][32 systems], three
//            in flight per warp, L2 evict_last) and composes the forward state
//            map of its rows (the continuant recurrence on raw rows, DESIGN.md
//            X21: a 3x3 map of (theta, psi, delta), fp64, power-of-two rescaled).
//            Warps 0-3 compose the 16 warp maps into exclusive prefixes and the
//            CTA's aggregate (shared memory); after a cluster barrier, warp 3
//            folds the aggregates of CTAs 0 .. q-1 (read through distributed
//            shared memory) into the CTA's incoming state.
//   phase C  every warp applies its prefix to the incoming state, re-reads its
//            rows (from L2: prefetched by TMA during phase A) and replays them:
//            c', d' (Eqs 2-3) in registers; then the affine back-substitution
//            map of its rows (x_first = al + be x_after).  Warps 0-3 compose the
//            suffixes and the CTA's aggregate; after a second cluster barrier
//            warp 0 folds those of CTAs q+1 .. Q-1 into x after the CTA.
//   phase D  every warp back-substitutes (Eq 4) from x after its rows and
//            stores x (one 256-byte row per warp store).
//
// HBM traffic: the compulsory 5 arrays (a, b, c, d read once; the phase C re-read
// hits L2; x written once).  No global scratch, no flags: the only exchange is
// 9 x 32 fp64 values per CTA through DSMEM.  Requirements (checked by the
// planner): Q <= 8 (a portable cluster), blocks x Q <= SMs (one wave, one CTA
// per SM); the tensor [nb][n][ms] with 16-byte row / batch strides (TMA).
#pragma once
#include <utility>

#include "k_scan.cuh"  // sc_* TMA helpers, SKMat / sk_compose, sk_exp2_scale, rcp

namespace tri {

constexpr int SG_NW = 16;            // warps per CTA
constexpr int SG_THREADS = 32 * SG_NW;
constexpr int SG_SR = 4;             // rows per TMA stage
constexpr int SG_RMAX = 16;          // rows per warp (c', d' kept in registers)
constexpr int SG_NBUF = 3;          // TMA stage buffers per warp
constexpr int SG_QMAX = 8;          // CTAs per block = cluster size (portable)

template <typename T>
struct SGLayout {
    static constexpr int stage_bytes = 4 * SG_SR * 32 * (int)sizeof(T);   // 4 arrays x [4 rows][32 systems]
    static constexpr int off_buf = 0;                                      // [NW][3] stages
    // [7][32 systems][16 warps] fp64 (warp index XOR-swizzled by the system: lane
    // accesses of one warp column hit distinct bank pairs): the warp maps, then
    // the warp prefixes; then the warps' backward maps [2][32][16], then their suffixes
    static constexpr int off_x = off_buf + SG_NW * SG_NBUF * stage_bytes;
    static constexpr int off_in = off_x + 7 * 32 * 16 * 8;                 // [3][32] CTA state, [32] x after
    static constexpr int off_agg = off_in + 4 * 32 * 8;                    // [7][32] forward, [2][32] backward aggregate
    static constexpr int off_bar = off_agg + 9 * 32 * 8;                   // [NW][3] mbarriers
    static constexpr int smem_bytes = off_bar + SG_NW * SG_NBUF * 8 + 1024;  // + alignment slack
};

template <typename T>
struct SGArgs {
    T* x;
    int64_t n, ms;      // rows, systems per batch
    int64_t xel, xbat;  // x: row i of system s of batch b at b xbat + i xel + s
    int bpb;            // 32-system blocks per batch
    int Q;              // CTAs per block
    unsigned long long* prof;  // diagnostics (scripts/prof_grid.py): [CTAs][16 warps][16] %globaltimer stamps
    int dbg;                   // diagnostics: 3 = skip everything after the prologue (launch cost; x not written)
};
__device__ __forceinline__ unsigned long long sg_gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)::"memory");
    return t;
}

// the load sequence after whose consumption sequence h can be issued (-1: at the
// start): buffer h % 3 free (h - 3 consumed) and, for a phase C re-read (h >= NST),
// its phase A load consumed (h - NST)
__host__ __device__ constexpr int sg_ready_after(int h, int NST) {
    return h - SG_NBUF > (h >= NST ? h - NST : -1) ? h - SG_NBUF : (h >= NST ? h - NST : -1);
}

// thread-block cluster of the Q CTAs of a block: barrier (release / acquire) and
// fp64 loads from another CTA's shared memory (DSMEM)
__device__ __forceinline__ void sg_cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ void sg_cluster_arrive() {
    asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
}
__device__ __forceinline__ void sg_cluster_wait() {
    asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ double sg_ld_remote(const double* local, unsigned rank) {
    unsigned a;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(a) : "r"((unsigned)__cvta_generic_to_shared(local)), "r"(rank));
    double v;
    asm volatile("ld.shared::cluster.f64 %0, [%1];" : "=d"(v) : "r"(a) : "memory");
    return v;
}

// apply the forward map M to the state (th, ps, de), then rescale by an exact
// power of two (the state is projective: c', d' are ratios)
__device__ __forceinline__ void sg_apply(const SCM& M, double& th, double& ps, double& de) {
    const double ot = fma(M.a, th, M.b * ps);
    const double op = fma(M.c, th, M.d * ps);
    const double od = fma(M.e, th, fma(M.f, ps, M.g * de));
    const double s = sk_exp2_scale(ot);
    th = ot * s; ps = op * s; de = od * s;
}
__device__ __forceinline__ SCM sg_rescale(const SCM& M) {
    const double s = sk_exp2_scale(fmax(fabs(M.a), fabs(M.b)));
    return SCM{M.a * s, M.b * s, M.c * s, M.d * s, M.e * s, M.f * s, M.g * s};
}

// f(integral_constant<0>), ..., f(integral_constant<N - 1>)
template <int I, int N>
struct SGFor {
    template <typename F>
    __device__ __forceinline__ static void run(F& f) {
        f(std::integral_constant<int, I>{});
        SGFor<I + 1, N>::run(f);
    }
};
template <int N>
struct SGFor<N, N> {
    template <typename F>
    __device__ __forceinline__ static void run(F&) {}
};
template <int N, typename F>
__device__ __forceinline__ void sg_static_for(F&& f) {
    SGFor<0, N>::run(f);
}

// NST = R / 4 TMA stages per warp (1 .. 4): every loop, the load schedule and the
// edge tests are resolved at compile time
template <typename T, int NST>
__global__ void __launch_bounds__(SG_THREADS, 1) k_scan_grid(const __grid_constant__ StreamMaps tm, SGArgs<T> p) {
    constexpr int R = NST * SG_SR;
    using L = SGLayout<T>;
    extern __shared__ __align__(16) unsigned char sg_smem_raw[];
    unsigned char* sbase = sg_smem_raw + ((1024 - ((unsigned)__cvta_generic_to_shared(sg_smem_raw) & 1023)) & 1023);
    uint64_t* bar = reinterpret_cast<uint64_t*>(sbase + L::off_bar);  // [NW][3]
    double* xch = reinterpret_cast<double*>(sbase + L::off_x);        // the transposed exchange area
    double* cst = reinterpret_cast<double*>(sbase + L::off_in);
    double* agg = reinterpret_cast<double*>(sbase + L::off_agg);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    auto X = [&](int k, int s, int w) -> double& { return xch[(k * 32 + s) * 16 + (w ^ (s & 15))]; };
    // diagnostics: [CTA][warp][8] %globaltimer stamps taken by lane 0 of every warp
    unsigned long long* const prof = p.prof ? p.prof + 16 * (SG_NW * blockIdx.x + warp) : nullptr;
#define SG_T(k) do { if (prof && lane == 0) prof[k] = sg_gtime(); } while (0)
    SG_T(0);
    if (threadIdx.x == 0) {
        for (int i = 0; i < SG_NBUF * SG_NW; ++i) sk_bar_init(&bar[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    __syncthreads();
    if (p.dbg == 3) {  // every CTA of the cluster still meets the cluster barriers
        sg_cluster_sync(); sg_cluster_sync(); sg_cluster_arrive(); sg_cluster_wait();
        return;
    }

    const int n = (int)p.n;  // < 2^30 (planner)
    const int cta = blockIdx.x, blk = cta / p.Q, q = cta - blk * p.Q;
    const int bt = blk / p.bpb, sb = blk - bt * p.bpb;
    const int64_t sys = (int64_t)sb * 32 + lane;           // this lane's system within the batch
    const bool live_sys = sys < p.ms;
    const int r0 = (q * SG_NW + warp) * R;                 // the warp's first row
    const bool live_w = r0 < n;
    T* buf0 = reinterpret_cast<T*>(sbase + L::off_buf + (SG_NBUF * warp) * L::stage_bytes);
    constexpr int AS = SG_SR * 32;                         // elements per array in a stage
    // load sequence g = 0 .. 2 NST - 1: phase A's stages, then phase C's re-read of
    // the same rows (L2); sequence g lands in buffer g % 3
    const uint64_t pol_keep = sk_policy_evict_last(), pol_once = sk_policy_evict_first();
    auto issue = [&](int g) {  // TMA zero-fills rows past n and systems past ms
        const int s = g < NST ? g : g - NST, bi = g % SG_NBUF;
        uint64_t* b = &bar[SG_NBUF * warp + bi];
        T* d = buf0 + bi * (L::stage_bytes / (int)sizeof(T));
        sk_expect(b, (unsigned)L::stage_bytes);
        const int y = (int)(r0 + s * SG_SR), x0 = sb * 32;
        const uint64_t pol = g < NST ? pol_keep : pol_once;
        sc_tma3d(d + 0 * AS, &tm.a, y, bt, b, pol, x0);
        sc_tma3d(d + 1 * AS, &tm.b, y, bt, b, pol, x0);
        sc_tma3d(d + 2 * AS, &tm.c, y, bt, b, pol, x0);
        sc_tma3d(d + 3 * AS, &tm.d, y, bt, b, pol, x0);
    };
    unsigned ph = 0;  // bit b: parity of buffer b
    // wait for sequence g and read its rows as fp64.  Stages holding row 0, row
    // n - 1 or rows past n (warp-uniform) apply a_0 = 0, c_{n-1} = 0 (outside A)
    // and identity rows past n; the padding systems of the last block (lanes past
    // ms) are never stored and stay in their own lane.  fp64 rows are renormalised
    // by 2^-exponent(b) (exact, X21) only when a live pivot of the stage leaves
    // 2^+-64 (warp-uniform test).  Then the freed buffer is refilled with
    // sequence g + 3 (at most 3 loads in flight per warp; a phase C re-read is
    // issued only after its phase A load landed, so it hits L2).
    auto consume = [&](auto gc, double (&ra)[SG_SR], double (&rb)[SG_SR], double (&rc)[SG_SR], double (&rd)[SG_SR]) {
        constexpr int g = decltype(gc)::value;
        constexpr int bi = g % SG_NBUF, s = g < NST ? g : g - NST;
        sk_wait(&bar[SG_NBUF * warp + bi], (ph >> bi) & 1u);
        ph ^= 1u << bi;
        const T* st = buf0 + bi * (L::stage_bytes / (int)sizeof(T));
#pragma unroll
        for (int u = 0; u < SG_SR; ++u) {
            ra[u] = (double)st[0 * AS + u * 32 + lane];
            rb[u] = (double)st[1 * AS + u * 32 + lane];
            rc[u] = (double)st[2 * AS + u * 32 + lane];
            rd[u] = (double)st[3 * AS + u * 32 + lane];
        }
        const int i0 = r0 + s * SG_SR;
        if (i0 == 0 || i0 + SG_SR > n - 1) {
#pragma unroll
            for (int u = 0; u < SG_SR; ++u) {
                const int i = i0 + u;
                if (i == 0) ra[u] = 0.0;
                if (i == n - 1) rc[u] = 0.0;
                if (i >= n) { ra[u] = 0.0; rb[u] = 1.0; rc[u] = 0.0; rd[u] = 0.0; }
            }
        }
        if constexpr (sizeof(T) == 8) {
            bool out = false;
#pragma unroll
            for (int u = 0; u < SG_SR; ++u) {
                const unsigned hb = (unsigned)__double2hiint(rb[u]) & 0x7ff00000u;
                out |= hb - ((1023u - 64u) << 20) > (128u << 20);
            }
            if (__any_sync(0xffffffffu, out && live_sys)) {
#pragma unroll
                for (int u = 0; u < SG_SR; ++u) {
                    const double sc = sk_exp2_scale(rb[u]);
                    ra[u] *= sc; rb[u] *= sc; rc[u] *= sc; rd[u] *= sc;
                }
            }
        }
        sc_release_buf();
        // issue every sequence h whose last prerequisite is g: its buffer's previous
        // load (h - 3) consumed and, for a phase C re-read, its phase A load (h - NST)
#pragma unroll
        for (int h = g + 1; h <= g + SG_NBUF; ++h)
            if (h < 2 * NST && sg_ready_after(h, NST) == g && lane == 0) issue(h);
    };

    // ---- phase A: the warp's forward map
    if (live_w && lane == 0) {
#pragma unroll
        for (int h = 0; h < SG_NBUF; ++h)
            if (h < 2 * NST && sg_ready_after(h, NST) < 0) issue(h);
    }
    SCM M{1.0, 0.0, 0.0, 1.0, 0.0, 0.0, 1.0};
    if (live_w) {
        sg_static_for<NST>([&](auto sc) {
            double ra[SG_SR], rb[SG_SR], rc[SG_SR], rd[SG_SR];
            consume(sc, ra, rb, rc, rd);
#pragma unroll
            for (int u = 0; u < SG_SR; ++u) {  // columns of M through row u (X21)
                const double au = ra[u], bu = rb[u], cu = rc[u], du = rd[u];
                const double t1 = fma(bu, M.a, -au * M.c), p1 = cu * M.a, d1 = fma(du, M.a, -au * M.e);
                const double t2 = fma(bu, M.b, -au * M.d), p2 = cu * M.b, d2 = fma(du, M.b, -au * M.f);
                M = SCM{t1, t2, p1, p2, d1, d2, -au * M.g};
            }
            M = sg_rescale(M);
        });
    }
    SG_T(6);
    X(0, lane, warp) = M.a; X(1, lane, warp) = M.b; X(2, lane, warp) = M.c; X(3, lane, warp) = M.d;
    X(4, lane, warp) = M.e; X(5, lane, warp) = M.f; X(6, lane, warp) = M.g;
    __syncthreads();
    SG_T(1);
    // Warp prefixes P_w = M_{w-1} .. M_0 by warps 0-3 (lane = system; warp k owns
    // the quarter of warps 4k .. 4k+3): local compositions, the quarter aggregates
    // exchanged through shared memory (two 128-thread named barriers), so no
    // shuffles (fp64 SHFL is 2 x 32-bit at one warp instruction per clock per SM).
    // Warp 3 then holds the CTA aggregate (shared memory, read by the later CTAs of
    // the cluster).
    if (warp < 4) {
        const int k = warp, w0 = 4 * k;
        auto ldM = [&](int w) { return SCM{X(0, lane, w), X(1, lane, w), X(2, lane, w), X(3, lane, w), X(4, lane, w),
                                           X(5, lane, w), X(6, lane, w)}; };
        auto stM = [&](int w, const SCM& m) {
            X(0, lane, w) = m.a; X(1, lane, w) = m.b; X(2, lane, w) = m.c; X(3, lane, w) = m.d;
            X(4, lane, w) = m.e; X(5, lane, w) = m.f; X(6, lane, w) = m.g;
        };
        const SCM L1 = ldM(w0), m1 = ldM(w0 + 1), m2 = ldM(w0 + 2), m3 = ldM(w0 + 3);
        const SCM L2 = sk_compose(m1, L1), L3 = sk_compose(m2, L2);
        const SCM Lq = sg_rescale(sk_compose(m3, L3));  // the quarter's aggregate
        stM(w0, Lq);
        asm volatile("bar.sync 1, 128;" ::: "memory");
        SCM E{1.0, 0.0, 0.0, 1.0, 0.0, 0.0, 1.0};       // quarters 0 .. k-1
        for (int j = 0; j < k; ++j) E = sk_compose(ldM(4 * j), E);
        asm volatile("bar.sync 1, 128;" ::: "memory");
        stM(w0, E);
        stM(w0 + 1, sk_compose(L1, E));
        stM(w0 + 2, sk_compose(L2, E));
        stM(w0 + 3, sk_compose(L3, E));
        SG_T(15);
        if (k == 3) {  // the CTA's aggregate, for the later CTAs of the cluster
            const SCM A = sg_rescale(sk_compose(Lq, E));
            agg[lane] = A.a; agg[32 + lane] = A.b; agg[64 + lane] = A.c; agg[96 + lane] = A.d;
            agg[128 + lane] = A.e; agg[160 + lane] = A.f; agg[192 + lane] = A.g;
        }
    }
    sg_cluster_sync();  // every CTA's aggregate written (release / acquire across the cluster)
    SG_T(13);
    if (warp == 3) {
        // incoming state of the CTA: the aggregates of CTAs 0 .. q-1 applied to (1, 0, 0)
        double th = 1.0, ps = 0.0, de = 0.0;
        for (int qq = 0; qq < q; ++qq) {
            const SCM A{sg_ld_remote(agg + lane, qq), sg_ld_remote(agg + 32 + lane, qq),
                        sg_ld_remote(agg + 64 + lane, qq), sg_ld_remote(agg + 96 + lane, qq),
                        sg_ld_remote(agg + 128 + lane, qq), sg_ld_remote(agg + 160 + lane, qq),
                        sg_ld_remote(agg + 192 + lane, qq)};
            sg_apply(A, th, ps, de);
        }
        cst[lane] = th; cst[32 + lane] = ps; cst[64 + lane] = de;
        SG_T(14);
    }
    __syncthreads();
    SG_T(2);

    // ---- phase C: replay the warp's rows from its incoming state
    double cp[R], dp[R];
    double al = 0.0, be = 1.0;  // x_first = al + be x_after (identity for a warp past n)
    double th = cst[lane], ps = cst[32 + lane], de = cst[64 + lane];
    {
        const SCM Pw{X(0, lane, warp), X(1, lane, warp), X(2, lane, warp), X(3, lane, warp), X(4, lane, warp),
                     X(5, lane, warp), X(6, lane, warp)};
        sg_apply(Pw, th, ps, de);
    }
    __syncthreads();  // every warp has its state: the exchange area takes the backward maps next

    if (live_w) {
        sg_static_for<NST>([&](auto sc) {
            constexpr int st = decltype(sc)::value;
            double ra[SG_SR], rb[SG_SR], rc[SG_SR], rd[SG_SR];
            consume(std::integral_constant<int, NST + st>{}, ra, rb, rc, rd);
            SG_T(8 + st);
#pragma unroll
            for (int u = 0; u < SG_SR; ++u) {
                const double nt = fma(rb[u], th, -ra[u] * ps);
                const double np = rc[u] * th;
                const double nd = fma(rd[u], th, -ra[u] * de);
                const double inv = rcp(nt);
                cp[st * SG_SR + u] = np * inv;
                dp[st * SG_SR + u] = nd * inv;
                th = nt; ps = np; de = nd;
            }
            const double h = sk_exp2_scale(th);
            th *= h; ps *= h; de *= h;
        });
        SG_T(7);
        // backward map of the warp's rows (rows past n: c' = d' = 0 -> x = 0)
#pragma unroll
        for (int t = R - 1; t >= 0; --t) {
            al = fma(-cp[t], al, dp[t]);
            be = -cp[t] * be;
        }
    }
    X(0, lane, warp) = al; X(1, lane, warp) = be;
    __syncthreads();
    SG_T(3);
    // Warp suffixes F_w = B_{w+1} .. B_15 (x after warp w = F_w(x after the CTA);
    // affine maps x_first = al + be x_after, composed (al, be) o (al', be') =
    // (al + be al', be be')) by warps 0-3 as above; warp 0 then holds the CTA
    // aggregate, publishes it and folds the later CTAs' aggregates into x after
    // the CTA.
    if (warp < 4) {
        const int k = warp, w0 = 4 * k;
        const double a0 = X(0, lane, w0), b0 = X(1, lane, w0), a1 = X(0, lane, w0 + 1), b1 = X(1, lane, w0 + 1);
        const double a2 = X(0, lane, w0 + 2), b2 = X(1, lane, w0 + 2), a3 = X(0, lane, w0 + 3), b3 = X(1, lane, w0 + 3);
        // quarter-local exclusive suffixes G (warp w0+3: identity), aggregate Gq
        const double g2a = a3, g2b = b3;
        const double g1a = fma(b2, g2a, a2), g1b = b2 * g2b;
        const double g0a = fma(b1, g1a, a1), g0b = b1 * g1b;
        const double qa = fma(b0, g0a, a0), qb = b0 * g0b;
        X(0, lane, w0) = qa; X(1, lane, w0) = qb;
        asm volatile("bar.sync 1, 128;" ::: "memory");
        double ha = 0.0, hb = 1.0;                    // quarters k+1 .. 3
        for (int j = 3; j > k; --j) { ha = fma(X(1, lane, 4 * j), ha, X(0, lane, 4 * j)); hb *= X(1, lane, 4 * j); }
        asm volatile("bar.sync 1, 128;" ::: "memory");
        X(0, lane, w0) = fma(g0b, ha, g0a); X(1, lane, w0) = g0b * hb;
        X(0, lane, w0 + 1) = fma(g1b, ha, g1a); X(1, lane, w0 + 1) = g1b * hb;
        X(0, lane, w0 + 2) = fma(g2b, ha, g2a); X(1, lane, w0 + 2) = g2b * hb;
        X(0, lane, w0 + 3) = ha; X(1, lane, w0 + 3) = hb;
        if (k == 0) {  // the CTA's aggregate, for the earlier CTAs of the cluster
            agg[224 + lane] = fma(qb, ha, qa);
            agg[256 + lane] = qb * hb;
        }
    }
    sg_cluster_sync();
    if (warp == 0) {
        // x after the CTA: the later CTAs' aggregates folded from the block's end
        double x = 0.0;
        for (int qq = p.Q - 1; qq > q; --qq)
            x = fma(sg_ld_remote(agg + 256 + lane, qq), x, sg_ld_remote(agg + 224 + lane, qq));
        cst[96 + lane] = x;
    }
    // the remote reads of this CTA's shared memory are over once every CTA has
    // arrived here; the matching wait is the last instruction (a CTA's shared
    // memory must outlive its peers' reads)
    sg_cluster_arrive();
    __syncthreads();
    SG_T(4);

    // ---- phase D: back substitution (Eq 4) and the x stores
    if (live_w) {
        double x = fma(X(1, lane, warp), cst[96 + lane], X(0, lane, warp));  // x after the warp's rows
        const int64_t xel = p.xel;
        // the warp's last row; walked backwards one row stride at a time
        T* xp = p.x + (int64_t)bt * p.xbat + sys + (int64_t)(r0 + R - 1) * xel;
        if (r0 + R <= n) {  // warp-uniform: no row past n
#pragma unroll
            for (int t = R - 1; t >= 0; --t) {
                x = fma(-cp[t], x, dp[t]);
                if (live_sys) __stcs(xp, (T)x);
                xp -= xel;
            }
        } else {
#pragma unroll
            for (int t = R - 1; t >= 0; --t) {
                x = fma(-cp[t], x, dp[t]);
                if (live_sys && r0 + t < n) __stcs(xp, (T)x);
                xp -= xel;
            }
        }
    }

    SG_T(5);
#undef SG_T
    sg_cluster_wait();
}

}  // namespace tri
