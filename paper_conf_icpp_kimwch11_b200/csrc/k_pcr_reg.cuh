// k_pcr_reg.cuh -- tiled PCR passes with the rows in registers (TRI_VARIANT_SPLIT
// frontend, round 2).
//
// Paper: Sec. III.A: PCR steps (Eqs 5-6) applied tile by tile, with
// tiles overlapping by the f(k) = 2^k - 1 rows a k-step reduction depends on
// (Eq 8, "overlapping tiles in the boundary of regions", Fig 11b).  The
// paper keeps the levels of a sub-tile in shared memory and slides a window
// (Figs 8-10); on sm_100a that window is bound by shared-memory bandwidth
// (k_tiled_pcr.cuh: 12 shared-memory accesses per row per level).  Here every
// warp owns whole tiles: a tile plus its f(k) halo is read once (straight into
// registers, or by TMA / cp.async through a per-warp shared-memory ring), and
// all k levels run in registers -- in-lane neighbours directly, cross-lane
// neighbours by warp shuffle -- so shared memory is touched at most once per
// row, not once per row per level.  The halo rows are recomputed by the neighbouring tile (redundant
// arithmetic instead of the paper's cached dependency rows: the ALU and shuffle
// pipes have headroom, HBM does not).
//
// Two kernels:
//   k_pcr_rows   -- the user's CONTIGUOUS layout.  A tile = 256 consecutive rows
//                   of one system (8 per lane, lane l rows 8l..8l+7, loaded as
//                   32-byte vectors straight into registers); k <= 5 steps
//                   (strides 1..16: in-lane for s < 8, shuffles by s/8 lanes
//                   above); the centre 256 - 2 H rows are written.
//   k_pcr_chains -- a chain-interleaved batch ([pos * C1 + ch], C1 chains of L1
//                   positions: the previous pass's output, or the user's
//                   INTERLEAVED layout with RAW rows): lane = chain, a warp = 32
//                   adjacent chains, PO positions per lane per tile plus f(K)
//                   halo positions on each side read from the neighbouring
//                   tiles of the ring; K <= 3 steps per pass.
// Both write the output of the cumulative k steps chain-interleaved (row i of
// system q -> [ (i >> k) * C + q 2^k + (i mod 2^k) ], the interleave transform
// fused into the store), or the user layout (mode 1,
// tri_debug_pcr).
#pragma once
#include "common.cuh"
#include "k_pthomas.cuh"
#include "k_pthomas_tma.cuh"  // ptt_bar_init / ptt_expect / ptt_wait / ptt_load

namespace tri {

template <typename T>
__device__ __forceinline__ NRow<T> pr_shfl_up(const NRow<T>& r, int d) {
    return NRow<T>{__shfl_up_sync(0xffffffffu, r.A, d), __shfl_up_sync(0xffffffffu, r.C, d),
                   __shfl_up_sync(0xffffffffu, r.D, d)};
}
template <typename T>
__device__ __forceinline__ NRow<T> pr_shfl_down(const NRow<T>& r, int d) {
    return NRow<T>{__shfl_down_sync(0xffffffffu, r.A, d), __shfl_down_sync(0xffffffffu, r.C, d),
                   __shfl_down_sync(0xffffffffu, r.D, d)};
}

// Raw row (a, b, c, d) of row i of an n-row system -> normalised row, with the
// boundary conventions of X1 (a_0 = c_{n-1} = 0) and identity rows outside [0, n).
template <typename T>
__device__ __forceinline__ NRow<T> pr_norm(int64_t i, int64_t n, T a, T b, T c, T d) {
    if (i <= 0) a = T(0);
    if (i >= n - 1) c = T(0);
    if (i < 0 || i >= n) return identity_row<T>();
    return normalise(a, b, c, d);
}

// 8 consecutive chain-interleaved elements (idx a multiple of 8: 64-byte aligned)
__device__ __forceinline__ void pr_st8(double* p, const double (&v)[8]) {
    asm volatile("st.global.v4.f64 [%0], {%1, %2, %3, %4};" ::"l"(p), "d"(v[0]), "d"(v[1]), "d"(v[2]), "d"(v[3])
                 : "memory");
    asm volatile("st.global.v4.f64 [%0], {%1, %2, %3, %4};" ::"l"(p + 4), "d"(v[4]), "d"(v[5]), "d"(v[6]), "d"(v[7])
                 : "memory");
}
__device__ __forceinline__ void pr_st8(float* p, const float (&v)[8]) {
    *reinterpret_cast<float4*>(p) = make_float4(v[0], v[1], v[2], v[3]);
    *reinterpret_cast<float4*>(p + 4) = make_float4(v[4], v[5], v[6], v[7]);
}

// ---------------------------------------------------------------------------
// k_pcr_rows: CONTIGUOUS user layout, K <= 5 steps.  Every warp owns whole
// tiles of 32 RPL consecutive rows of one system (lane l rows RPL l .. RPL l +
// RPL - 1), loaded as 32-byte vectors straight into registers (one sector each:
// a warp reads 32 RPL elements contiguous per array); with PF the next tile's
// loads are issued before the current tile's steps (register double buffer).
// Measured at c3, SPLIT k = 14 (profiles/r02_ncu_split_rows*.txt,
// scripts/gpu_ab_rows.sh): RPL = 8 with prefetch 0.828 ms per solve; RPL = 16
// (3x fewer halo rows, 42 % fewer shuffles per row) 0.855 ms without prefetch
// and spills with it; RPL = 8 without prefetch 0.852 ms; a TMA-staged version
// was L1-bound on 4-way bank conflicts of the lane-blocked shared reads; CTA
// super-tiles with shared-memory boundary exchange between warps (no halo
// tiles) 0.92 ms -- the predicated boundary stores/loads cost more MIO issue
// than the halo recompute, and the warps of a CTA run in lockstep.
constexpr int PR_WARPS = 8;   // independent warps per CTA

// RPL rows per lane: a warp tile is 32 RPL rows; the halo is HL whole lanes at
// each end (RPL HL >= f(K) rows, Eq 8)
template <int K, int RPL>
struct PRGeo {
    static constexpr int ROWS = 32 * RPL;
    static constexpr int HL = ((1 << K) - 1 + RPL - 1) / RPL;
    static constexpr int H = RPL * HL;
    static constexpr int OUT = ROWS - 2 * H;  // rows a tile writes
};

template <typename T>
struct PRArgs {
    const T *a, *b, *c, *d;
    T *oA, *oC, *oD;        // mode 0: chain-interleaved [pos * C + chain]; mode 1: user layout
    int64_t n, m, n_pad;    // rows, systems, rows written per system (L 2^K)
    int64_t ntile, ntask;   // tiles per system, m * ntile
    int64_t C;              // chains of the output (m 2^K)
    int mode;
    int vec;                // a, b, c, d 32-byte aligned: vector loads
};

// 8 consecutive elements, 32-byte aligned, read once (no L1 allocation)
__device__ __forceinline__ void pr_ld8(const double* p, double* v) {
    asm("ld.global.nc.L1::no_allocate.v4.f64 {%0, %1, %2, %3}, [%4];"
        : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(p));
    asm("ld.global.nc.L1::no_allocate.v4.f64 {%0, %1, %2, %3}, [%4];"
        : "=d"(v[4]), "=d"(v[5]), "=d"(v[6]), "=d"(v[7]) : "l"(p + 4));
}
__device__ __forceinline__ void pr_ld8(const float* p, float* v) {
    asm("ld.global.nc.L1::no_allocate.v8.f32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
        : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7])
        : "l"(p));
}

template <typename T, int K, int RPL, bool PF>
__global__ void __launch_bounds__(32 * PR_WARPS, 1) k_pcr_rows(PRArgs<T> p) {
    using G = PRGeo<K, RPL>;
    constexpr int S = 1 << K;
    constexpr int EPC = 32 / (int)sizeof(T);  // elements per 32-byte vector
    const int lane = threadIdx.x & 31;
    const int64_t TW = (int64_t)gridDim.x * PR_WARPS;
    const int64_t n = p.n, N = n * p.m;

    // tile `tile` of system q covers rows [e0, e0 + 32 RPL), e0 = tile OUT - H - dq,
    // dq = (q n) mod EPC: the tiles of system q shift back by up to EPC - 1 rows
    // so that every lane's rows start on a 32-byte boundary.  Rows of the
    // neighbouring systems are replaced by identity rows below; rows outside the
    // arrays are not read.
    T va[RPL], vb[RPL], vc[RPL], vd[RPL];
    auto fetch = [&](int64_t task) {
        const int64_t q = task / p.ntile, tile = task - q * p.ntile;
        const int64_t qn = q * n;
        const int64_t f0 = qn - (qn & (EPC - 1)) + tile * G::OUT - G::H + RPL * lane;  // flat index of row 0
        if (p.vec && f0 >= 0 && f0 + RPL <= N) {
#pragma unroll
            for (int h = 0; h < RPL; h += 8) {
                pr_ld8(p.a + f0 + h, va + h); pr_ld8(p.b + f0 + h, vb + h);
                pr_ld8(p.c + f0 + h, vc + h); pr_ld8(p.d + f0 + h, vd + h);
            }
        } else {
#pragma unroll
            for (int u = 0; u < RPL; ++u) {
                const bool in = f0 + u >= 0 && f0 + u < N;
                va[u] = in ? p.a[f0 + u] : T(0); vb[u] = in ? p.b[f0 + u] : T(1);
                vc[u] = in ? p.c[f0 + u] : T(0); vd[u] = in ? p.d[f0 + u] : T(0);
            }
        }
    };
    int64_t task = (int64_t)blockIdx.x * PR_WARPS + (threadIdx.x >> 5);
    if (PF && task < p.ntask) fetch(task);
    for (; task < p.ntask; task += TW) {
        NRow<T> R[RPL];
        const int64_t q = task / p.ntile, tile = task - q * p.ntile;
        const int64_t i0 = tile * G::OUT - G::H - ((q * n) & (EPC - 1)) + RPL * lane;  // row of register 0
        if constexpr (PF) {
            // normalise this tile's rows, then issue the next tile's loads into the
            // same registers (they are free again) before the steps
#pragma unroll
            for (int u = 0; u < RPL; ++u) R[u] = pr_norm(i0 + u, n, va[u], vb[u], vc[u], vd[u]);
            if (task + TW < p.ntask) fetch(task + TW);
        } else {
            fetch(task);
#pragma unroll
            for (int u = 0; u < RPL; ++u) R[u] = pr_norm(i0 + u, n, va[u], vb[u], vc[u], vd[u]);
        }
        // PCR steps at strides 1, 2, .., 2^(K-1) (Eqs 5-6); out-of-tile neighbours of
        // the halo lanes are garbage, which only reaches rows within f(K) of the
        // tile edge -- the halo, never written
#pragma unroll
        for (int j = 0; j < K; ++j) {
            const int sg = 1 << j;
            NRow<T> N[RPL];
            if (sg < RPL) {
#pragma unroll
                for (int u = 0; u < RPL; ++u) {
                    const NRow<T> mr = u - sg >= 0 ? R[(u - sg + RPL) % RPL] : pr_shfl_up(R[(u - sg + RPL) % RPL], 1);
                    const NRow<T> pr = u + sg < RPL ? R[(u + sg) % RPL] : pr_shfl_down(R[(u + sg) % RPL], 1);
                    N[u] = pcr_combine(mr, R[u], pr);
                }
            } else {
#pragma unroll
                for (int u = 0; u < RPL; ++u)
                    N[u] = pcr_combine(pr_shfl_up(R[u], sg / RPL), R[u], pr_shfl_down(R[u], sg / RPL));
            }
#pragma unroll
            for (int u = 0; u < RPL; ++u) R[u] = N[u];
        }
        if (lane < G::HL || lane >= 32 - G::HL) continue;
        if (p.mode == 0) {
            if (K >= 3 && (i0 & 7) == 0 && i0 + RPL <= p.n_pad) {
                // 8 rows of one position, chains q 2^K + (i mod 2^K) .. + 7: 64 contiguous bytes
#pragma unroll
                for (int h = 0; h < RPL; h += 8) {
                    const int64_t i = i0 + h;
                    T* dA = p.oA + (i >> K) * p.C + q * S + (i & (S - 1));
                    const int64_t off = dA - p.oA;
                    T a8[8], c8[8], d8[8];
#pragma unroll
                    for (int u = 0; u < 8; ++u) { a8[u] = R[h + u].A; c8[u] = R[h + u].C; d8[u] = R[h + u].D; }
                    pr_st8(dA, a8);
                    pr_st8(p.oC + off, c8);
                    pr_st8(p.oD + off, d8);
                }
            } else {
#pragma unroll
                for (int u = 0; u < RPL; ++u) {
                    const int64_t i = i0 + u;
                    if (i >= 0 && i < p.n_pad) {
                        const int64_t idx = (i >> K) * p.C + q * S + (i & (S - 1));
                        p.oA[idx] = R[u].A; p.oC[idx] = R[u].C; p.oD[idx] = R[u].D;
                    }
                }
            }
        } else {
#pragma unroll
            for (int u = 0; u < RPL; ++u) {
                const int64_t i = i0 + u;
                if (i >= 0 && i < n) {
                    const int64_t gi = q * n + i;
                    p.oA[gi] = R[u].A; p.oC[gi] = R[u].C; p.oD[gi] = R[u].D;
                }
            }
        }
    }
}

// ---------------------------------------------------------------------------
// k_pcr_chains: chain-interleaved input, K <= 3 more steps.
constexpr int PC_PO = 8;    // output positions per lane per tile (>= f(3) = 7 halo positions)
constexpr int PC_NS = 4;    // ring stages: tiles t-1, t, t+1 resident, t+2 in flight

template <typename T, bool RAW>
struct PCCfg {
    static constexpr int NA = RAW ? 4 : 3;                          // arrays per stage
    static constexpr int WARPS = (RAW && sizeof(T) == 8) ? 6 : 8;   // 192 KB of stages per CTA (fp64)
    static constexpr int TILE = PC_PO * 32;                         // elements per array per tile
    static constexpr int STAGE = NA * TILE;
    static constexpr int smem_bytes() { return WARPS * PC_NS * STAGE * (int)sizeof(T) + 128; }  // + alignment slack
};

template <typename T>
struct PCArgs {
    const T* in[4];        // cp.async path: A, C, D (RAW: a, c, d, b) -- the arrays the maps describe
    T *oA, *oC, *oD;       // mode 0: chain-interleaved [pos2 * C + ch2]; mode 1: user layout
    int64_t n, m;          // original system size, systems
    int64_t L1, C1;        // input positions per chain, input chains
    int64_t C;             // output chains (C1 2^K)
    int64_t Lout;          // input positions covered: L2 2^K (L2 = output positions per chain)
    int64_t ntile_reg, nreg, nblk, ntask;
    int k1, mode, layout;  // steps applied before this pass; mode; user layout (mode 1)
};
struct PCMaps {
    CUtensorMap a, c, d, b;  // RAW: user a, c, d, b ([n][m] view); else normalised A, C, D ([L1][C1])
};

// step J + 1 (stride 2^J) on positions [2^(J+1) - 1, E - 2^(J+1) + 1), where the
// rows it reads are valid; then the steps above it (compile-time recursion keeps
// every register index static)
template <typename T, int E, int K, int J>
__device__ __forceinline__ void pc_levels(NRow<T> (&R)[E]) {
    if constexpr (J < K) {
        constexpr int sg = 1 << J, lo = (2 << J) - 1, hi = E - lo;
        NRow<T> N[E];
#pragma unroll
        for (int e = lo; e < hi; ++e) N[e] = pcr_combine(R[e - sg], R[e], R[e + sg]);
#pragma unroll
        for (int e = lo; e < hi; ++e) R[e] = N[e];
        pc_levels<T, E, K, J + 1>(R);
    }
}

// TMA: one 2D box per array per tile, lane 0 issues, an mbarrier per ring slot
// (needs a 16-byte row pitch C1 sizeof(T)); otherwise every lane copies its own
// chain's elements with cp.async (zero fill outside the batch), one commit group
// per tile -- each lane reads only what it copied, so no cross-lane handshake.
template <typename T, int K, bool RAW, bool TMA>
__global__ void __launch_bounds__(32 * PCCfg<T, RAW>::WARPS, 1) k_pcr_chains(const __grid_constant__ PCMaps tm,
                                                                             PCArgs<T> p) {
    using CF = PCCfg<T, RAW>;
    constexpr int PO = PC_PO, TILE = CF::TILE, STAGE = CF::STAGE, NW = CF::WARPS;
    constexpr int F = (1 << K) - 1;  // Eq 8
    constexpr int E = PO + 2 * F;    // positions a lane holds at level 0
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ uint64_t bar[NW][PC_NS];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    T* ring = reinterpret_cast<T*>((reinterpret_cast<uintptr_t>(smem_raw) + 127) & ~uintptr_t(127)) + warp * PC_NS * STAGE;
    const int64_t TW = (int64_t)gridDim.x * NW;
    const int k = p.k1 + K;

    if (TMA && lane == 0) {
        for (int s = 0; s < PC_NS; ++s) ptt_bar_init(&bar[warp][s]);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    uint32_t g = 0;  // loads issued by this warp so far (slot g % NS, phase g / NS)
    for (int64_t task = (int64_t)blockIdx.x * NW + warp; task < p.ntask; task += TW) {
        const int64_t blk = task % p.nblk, reg = task / p.nblk;
        const int x0 = (int)(blk * 32);
        const int64_t tb = reg * p.ntile_reg;                                         // first tile
        const int nt = (int)imin64(p.ntile_reg, (p.Lout + PO - 1) / PO - tb);      // tiles of this region
        const int64_t ch = blk * 32 + lane;
        const bool chok = ch < p.C1;
        const int64_t q = ch >> p.k1, r1 = ch & ((int64_t(1) << p.k1) - 1);
        // load l (0 .. nt + 1) = tile tb - 1 + l
        auto issue = [&](int l) {
            const uint32_t gl = g + (uint32_t)l;
            const int s = (int)(gl % PC_NS);
            T* dst = ring + s * STAGE;
            const int64_t y0 = (tb - 1 + l) * PO;
            if constexpr (TMA) {
                if (lane == 0) {
                    ptt_expect(&bar[warp][s], (unsigned)(STAGE * sizeof(T)));
                    ptt_load(dst, &tm.a, x0, (int)y0, &bar[warp][s]);
                    ptt_load(dst + TILE, &tm.c, x0, (int)y0, &bar[warp][s]);
                    ptt_load(dst + 2 * TILE, &tm.d, x0, (int)y0, &bar[warp][s]);
                    if constexpr (RAW) ptt_load(dst + 3 * TILE, &tm.b, x0, (int)y0, &bar[warp][s]);
                }
            } else {
#pragma unroll
                for (int u = 0; u < PO; ++u) {
                    const int64_t pos = y0 + u;
                    const bool ok = chok && pos >= 0 && pos < p.L1;
                    const int64_t gi = ok ? pos * p.C1 + ch : 0;
#pragma unroll
                    for (int j = 0; j < CF::NA; ++j) {
                        if constexpr (sizeof(T) == 8)
                            cp_async_8(dst + j * TILE + u * 32 + lane, p.in[j] + gi, ok ? 8 : 0);
                        else
                            cp_async_4(dst + j * TILE + u * 32 + lane, p.in[j] + gi, ok ? 4 : 0);
                    }
                }
                cp_async_commit();
            }
        };
        // TMA: wait for load l; cp.async: for every group but the `pend` newest
        auto wait = [&](int l, int pend) {
            if constexpr (TMA) {
                const uint32_t gl = g + (uint32_t)l;
                ptt_wait(&bar[warp][gl % PC_NS], (gl / PC_NS) & 1);
            } else {
                if (pend >= 2) cp_async_wait<2>();
                else if (pend == 1) cp_async_wait<1>();
                else cp_async_wait<0>();
            }
        };
        for (int l = 0; l < 3; ++l)
            if (l < nt + 2) issue(l);
            else if constexpr (!TMA) cp_async_commit();  // empty group: uniform counts
        wait(0, 2);
        wait(1, 1);
        for (int jt = 0; jt < nt; ++jt) {
            if (jt + 3 < nt + 2) issue(jt + 3);
            else if constexpr (!TMA) cp_async_commit();
            wait(jt + 2, 1);
            const T* tp = ring + ((g + jt) % PC_NS) * STAGE + lane;       // tile jt - 1
            const T* tc = ring + ((g + jt + 1) % PC_NS) * STAGE + lane;   // tile jt
            const T* tn = ring + ((g + jt + 2) % PC_NS) * STAGE + lane;   // tile jt + 1
            const int64_t t = (tb + jt) * PO;  // first output position of the tile
            NRow<T> R[E];
#pragma unroll
            for (int e = 0; e < E; ++e) {
                const T* src = e < F ? tp + (PO - F + e) * 32 : (e < F + PO ? tc + (e - F) * 32 : tn + (e - F - PO) * 32);
                if constexpr (RAW) {
                    R[e] = pr_norm(t - F + e, p.n, src[0], src[3 * TILE], src[TILE], src[2 * TILE]);
                } else {
                    R[e] = NRow<T>{src[0], src[TILE], src[2 * TILE]};
                }
            }
            __syncwarp();  // every lane has read tile jt - 1: its slot takes load jt + 4 next iteration
            // K steps at strides 1, 2, 4 of the chain positions (strides 2^k1 .. of the
            // original system)
            pc_levels<T, E, K, 0>(R);
            if (!chok) continue;
#pragma unroll
            for (int e = F; e < F + PO; ++e) {
                const int64_t pos = t + (e - F);
                if (pos >= p.Lout) break;
                const int64_t r = r1 + ((pos & ((1 << K) - 1)) << p.k1);  // residue mod 2^k
                const int64_t pos2 = pos >> K;
                if (p.mode == 0) {
                    const int64_t idx = pos2 * p.C + (q << k) + r;
                    p.oA[idx] = R[e].A; p.oC[idx] = R[e].C; p.oD[idx] = R[e].D;
                } else {
                    const int64_t i = (pos2 << k) + r;
                    if (i < p.n) {
                        const int64_t gi = elem_index(q, i, p.n, p.m, p.layout);
                        p.oA[gi] = R[e].A; p.oC[gi] = R[e].C; p.oD[gi] = R[e].D;
                    }
                }
            }
        }
        __syncwarp();
        g += (uint32_t)(nt + 2);
    }
}

}  // namespace tri
