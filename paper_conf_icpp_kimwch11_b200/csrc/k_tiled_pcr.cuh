// k_tiled_pcr.cuh -- tiled PCR with the buffered sliding window (TRI_VARIANT_SPLIT
// frontend; also tri_debug_pcr for large systems).
//
// Paper: Sec. III.A.  A CTA walks a region of one system sub-tile by
// sub-tile (two-level tiling), keeping for every PCR level j only the
// 2*sigma_j rows the next sub-tile depends on (dependency caching, Fig 8; total
// cache 2 f(k) rows, Eq 8).  Level j+1 lags level j by sigma_j = 2^j
// rows, so each level only ever needs rows that are already computed.  Regions
// of the same system run in parallel CTAs with f(k)-row halos loaded on both
// sides (Fig 11b, "overlapping tiles in the boundary of regions").
//
// B200 form: one ring buffer per level in shared memory (exactly T + 2 sigma_j
// rows, modular slots instead of the paper's buffer shifts);
// rows normalised to unit diagonal (3 values per row; X17); the last
// level writes its rows straight into the p-Thomas input layout (the interleave
// transform fused into the last store):
//     row i of system q -> chain q*2^k + (i mod 2^k), position floor(i / 2^k),
//     stored at [pos * C + chain], C = m * 2^k chains,
// padded to L = ceil(n / 2^k) positions per chain with identity rows.
#pragma once
#include "common.cuh"

namespace tri {

constexpr int TPCR_T = 256;  // sub-tile rows per level per iteration == threads

template <typename T>
struct TiledArgs {
    const T *a, *b, *c, *d;
    T *oA, *oC, *oD;   // mode 0: chain-interleaved scratch; mode 1: user layout
    int64_t n, m, n_pad, region, nreg, C;
    int layout, k, mode;
};

__host__ __device__ inline int64_t halo_f(int k) { return (int64_t(1) << k) - 1; }  // Eq 8

// Ring j holds exactly the T + 2^(j+1) rows level j can touch within one
// iteration (reads i +- 2^j of this sub-tile, the level below already wrote the
// next T rows): exact sizes instead of powers of two keep two CTAs per SM at
// k = 10 (110.5 KB fp64).  Ring slots are tracked incrementally per thread
// (32-bit, one conditional wrap per step) instead of computed from row indices.
template <int K>
struct TPCRRing {
    // closed forms (no recursion: these must fold to immediates in the unrolled level loop)
    __host__ __device__ static constexpr int size(int j) { return TPCR_T + (2 << j); }
    __host__ __device__ static constexpr int off(int j) { return j * TPCR_T + (2 << j) - 2; }  // sum of sizes below j
    __host__ __device__ static constexpr int total() { return off(K); }
};

template <typename T, int K>
__global__ void __launch_bounds__(TPCR_T, 2) k_tiled_pcr(TiledArgs<T> p) {
    using RG = TPCRRing<K>;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* rA = reinterpret_cast<T*>(smem_raw);
    T* rC = rA + RG::total();
    T* rD = rC + RG::total();

    const int tid = threadIdx.x;
    const int64_t q = blockIdx.x / p.nreg;
    const int64_t reg = blockIdx.x - q * p.nreg;
    const int64_t r0 = reg * p.region;
    const int64_t r1 = imin64(r0 + p.region, p.n_pad);
    constexpr int64_t fk = (int64_t(1) << K) - 1;  // Eq 8
    const int64_t start = r0 - fk;  // halo: level-0 rows [r0-f(k), r1+f(k)) feed outputs [r0, r1)
    const int64_t n = p.n;
    constexpr int S = 1 << K;

    for (int e = tid; e < RG::total(); e += TPCR_T) { rA[e] = T(0); rC[e] = T(0); rD[e] = T(0); }
    // slots: w0 = ring-0 slot of row s0 + tid; rs[j] = ring-j slot of the row level j
    // combines, i_j = s0 - (2^(j+1) - 1) + tid; ws[j] = ring-(j+1) slot of i_j.
    // Slot of row i in ring j = (i - base) mod size(j), base <= every row touched.
    const int64_t base = start - (int64_t(2) << K);
    int w0 = (int)((start + tid - base) % RG::size(0));
    int rs[K], ws[K];
#pragma unroll
    for (int j = 0; j < K; ++j) {
        const int64_t ij = start - ((int64_t(2) << j) - 1) + tid;
        rs[j] = (int)((ij - base) % RG::size(j));
        ws[j] = j + 1 < K ? (int)((ij - base) % RG::size(j + 1)) : 0;
    }
    __syncthreads();

    // level-0 rows of the next sub-tile are loaded into registers while the
    // current sub-tile's levels run (hides the HBM latency behind the ring work)
    T pa = T(0), pb = T(1), pc = T(0), pd = T(0);
    auto fetch = [&](int64_t s0) {
        const int64_t i = s0 + tid;
        pa = T(0); pb = T(1); pc = T(0); pd = T(0);
        if (i >= 0 && i < n) {
            const int64_t gi = elem_index(q, i, n, p.m, p.layout);
            pa = i > 0 ? ldg_stream(p.a + gi) : T(0);
            pc = i < n - 1 ? ldg_stream(p.c + gi) : T(0);
            pb = ldg_stream(p.b + gi);
            pd = ldg_stream(p.d + gi);
        }
    };
    fetch(start);
    for (int64_t s0 = start; s0 - fk < r1; s0 += TPCR_T) {
        {   // level 0: normalise this thread's prefetched row (identity outside the system)
            const NRow<T> r = normalise(pa, pb, pc, pd);
            rA[w0] = r.A; rC[w0] = r.C; rD[w0] = r.D;
        }
        fetch(s0 + TPCR_T);
        __syncthreads();
#pragma unroll
        for (int j = 0; j < K; ++j) {
            const int Z = RG::size(j), O = RG::off(j), sg = 1 << j;
            int sm = rs[j] - sg; sm += sm < 0 ? Z : 0;
            int sp = rs[j] + sg; sp -= sp >= Z ? Z : 0;
            const int so = O + rs[j];
            sm += O; sp += O;
            const NRow<T> nr = pcr_combine(NRow<T>{rA[sm], rC[sm], rD[sm]}, NRow<T>{rA[so], rC[so], rD[so]},
                                           NRow<T>{rA[sp], rC[sp], rD[sp]});
            if (j + 1 < K) {
                const int sd = RG::off(j + 1) + ws[j];
                rA[sd] = nr.A; rC[sd] = nr.C; rD[sd] = nr.D;
            } else {
                const int64_t i = s0 - ((int64_t(2) << j) - 1) + tid;
                if (i >= r0 && i < r1) {
                    if (p.mode == 0) {
                        const int64_t idx = (i >> K) * p.C + q * S + (i & (S - 1));
                        p.oA[idx] = nr.A; p.oC[idx] = nr.C; p.oD[idx] = nr.D;
                    } else if (i < n) {
                        const int64_t gi = elem_index(q, i, n, p.m, p.layout);
                        p.oA[gi] = nr.A; p.oC[gi] = nr.C; p.oD[gi] = nr.D;
                    }
                }
            }
            __syncthreads();
        }
        // every row index advances by T: advance the slots
        w0 += TPCR_T; w0 -= w0 >= RG::size(0) ? RG::size(0) : 0;
#pragma unroll
        for (int j = 0; j < K; ++j) {
            rs[j] += TPCR_T; rs[j] -= rs[j] >= RG::size(j) ? RG::size(j) : 0;
            if (j + 1 < K) { ws[j] += TPCR_T; ws[j] -= ws[j] >= RG::size(j + 1) ? RG::size(j + 1) : 0; }
        }
    }
}

// ---------------------------------------------------------------------------
// Second tiled-PCR pass (deep k, two passes): the chain-interleaved output of
// a k1-step pass is itself a batch of C1 = m 2^k1 independent systems in the
// INTERLEAVED layout (position pos of chain ch at [pos * C1 + ch]).  This pass
// applies k2 more steps (strides 2^k1 .. 2^(k1+k2-1) of the original system =
// strides 1 .. 2^(k2-1) in each chain's positions) with the same buffered
// sliding window, over TPCR_IL_CB adjacent chains per CTA so every position row
// is one 256-byte segment.  Its output is the layout a single k1 + k2 pass would
// store: chain ch2 = q 2^k + (r1 + 2^k1 (pos mod 2^k2)), position pos >> k2.
constexpr int TPCR_IL_CB = 32;                          // chains per CTA
constexpr int TPCR_IL_RPT = 2;                          // positions per thread per sub-tile
constexpr int TPCR_IL_TP = TPCR_IL_RPT * TPCR_T / TPCR_IL_CB;  // positions per sub-tile

template <typename T>
struct TiledILArgs {
    const T *iA, *iC, *iD;  // pass-1 output, [pos * C1 + ch], normalised rows
    T *oA, *oC, *oD;        // mode 0: chain-interleaved [pos2 * C + ch2]; mode 1: user layout
    int64_t n, m, L1, C1, C, region, nreg, nblk;
    int layout, k1, mode;
};

// ring j (positions): exactly TP + 2^(j+1), closed-form offsets (see TPCRRing)
template <int K2>
struct TPCRILRing {
    __host__ __device__ static constexpr int size(int j) { return TPCR_IL_TP + (2 << j); }
    __host__ __device__ static constexpr int off(int j) { return j * TPCR_IL_TP + (2 << j) - 2; }
    __host__ __device__ static constexpr int total() { return off(K2); }
};

template <typename T, int K2>
__global__ void __launch_bounds__(TPCR_T) k_tiled_pcr_il(TiledILArgs<T> p) {
    constexpr int CB = TPCR_IL_CB, TP = TPCR_IL_TP, RPT = TPCR_IL_RPT, UP = TPCR_T / CB;
    using RG = TPCRILRing<K2>;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* rA = reinterpret_cast<T*>(smem_raw);
    T* rC = rA + RG::total() * CB;
    T* rD = rC + RG::total() * CB;

    const int tid = threadIdx.x;
    const int c = tid % CB, u0 = tid / CB;  // this thread: chain c, positions u0 + UP * h
    const int64_t blk = blockIdx.x % p.nblk, reg = blockIdx.x / p.nblk;
    const int64_t ch = blk * CB + c;
    const bool chok = ch < p.C1;
    const int64_t r0 = reg * p.region;
    const int64_t r1 = imin64(r0 + p.region, p.L1);
    constexpr int64_t fk = (int64_t(1) << K2) - 1;  // Eq 8 on the chain positions
    const int64_t start = r0 - fk;
    const int k = p.k1 + K2;
    const int64_t S1 = int64_t(1) << p.k1;
    const int64_t q = ch >> p.k1, rr1 = ch & (S1 - 1);

    for (int e = tid; e < RG::total() * CB; e += TPCR_T) { rA[e] = T(0); rC[e] = T(0); rD[e] = T(0); }
    // slots (positions) of this thread's rows, advanced by TP per iteration:
    // w0[h] in ring 0 for pos = s0 + u0 + UP h; rs[j][h] in ring j and ws[j][h]
    // in ring j+1 for the row level j combines, pos_j = s0 - (2^(j+1) - 1) + u0 + UP h
    const int64_t base = start - (int64_t(2) << K2);
    int w0[RPT], rs[K2][RPT], ws[K2][RPT];
#pragma unroll
    for (int h = 0; h < RPT; ++h) {
        w0[h] = (int)((start + u0 + UP * h - base) % RG::size(0));
#pragma unroll
        for (int j = 0; j < K2; ++j) {
            const int64_t pj = start - ((int64_t(2) << j) - 1) + u0 + UP * h;
            rs[j][h] = (int)((pj - base) % RG::size(j));
            ws[j][h] = j + 1 < K2 ? (int)((pj - base) % RG::size(j + 1)) : 0;
        }
    }
    __syncthreads();

    NRow<T> nxt[RPT];  // next sub-tile's level-0 rows, loaded during this sub-tile's levels
    auto fetch = [&](int64_t s0) {
#pragma unroll
        for (int h = 0; h < RPT; ++h) {
            const int64_t pos = s0 + u0 + UP * h;
            nxt[h] = identity_row<T>();
            if (pos >= 0 && pos < p.L1 && chok) {
                const int64_t gi = pos * p.C1 + ch;
                nxt[h] = NRow<T>{ldg_stream(p.iA + gi), ldg_stream(p.iC + gi), ldg_stream(p.iD + gi)};
            }
        }
    };
    fetch(start);
    for (int64_t s0 = start; s0 - fk < r1; s0 += TP) {
#pragma unroll
        for (int h = 0; h < RPT; ++h) {
            const int sl = w0[h] * CB + c;
            rA[sl] = nxt[h].A; rC[sl] = nxt[h].C; rD[sl] = nxt[h].D;
        }
        fetch(s0 + TP);
        __syncthreads();
#pragma unroll
        for (int j = 0; j < K2; ++j) {
            const int Z = RG::size(j), O = RG::off(j), sg = 1 << j;
            NRow<T> nr[RPT];
#pragma unroll
            for (int h = 0; h < RPT; ++h) {
                int sm = rs[j][h] - sg; sm += sm < 0 ? Z : 0;
                int sp = rs[j][h] + sg; sp -= sp >= Z ? Z : 0;
                const int so = (O + rs[j][h]) * CB + c;
                sm = (O + sm) * CB + c;
                sp = (O + sp) * CB + c;
                nr[h] = pcr_combine(NRow<T>{rA[sm], rC[sm], rD[sm]}, NRow<T>{rA[so], rC[so], rD[so]},
                                    NRow<T>{rA[sp], rC[sp], rD[sp]});
            }
#pragma unroll
            for (int h = 0; h < RPT; ++h) {
                if (j + 1 < K2) {
                    const int sd = (RG::off(j + 1) + ws[j][h]) * CB + c;
                    rA[sd] = nr[h].A; rC[sd] = nr[h].C; rD[sd] = nr[h].D;
                } else {
                    const int64_t pos = s0 - ((int64_t(2) << j) - 1) + u0 + UP * h;
                    if (pos >= r0 && pos < r1 && chok) {
                        const int64_t r = rr1 + ((pos & ((int64_t(1) << K2) - 1)) << p.k1);  // residue mod 2^k
                        const int64_t pos2 = pos >> K2;
                        if (p.mode == 0) {
                            const int64_t idx = pos2 * p.C + (q << k) + r;
                            p.oA[idx] = nr[h].A; p.oC[idx] = nr[h].C; p.oD[idx] = nr[h].D;
                        } else {
                            const int64_t i = (pos2 << k) + r;
                            if (i < p.n) {
                                const int64_t gi = elem_index(q, i, p.n, p.m, p.layout);
                                p.oA[gi] = nr[h].A; p.oC[gi] = nr[h].C; p.oD[gi] = nr[h].D;
                            }
                        }
                    }
                }
            }
            __syncthreads();
        }
#pragma unroll
        for (int h = 0; h < RPT; ++h) {
            w0[h] += TP; w0[h] -= w0[h] >= RG::size(0) ? RG::size(0) : 0;
#pragma unroll
            for (int j = 0; j < K2; ++j) {
                rs[j][h] += TP; rs[j][h] -= rs[j][h] >= RG::size(j) ? RG::size(j) : 0;
                if (j + 1 < K2) { ws[j][h] += TP; ws[j][h] -= ws[j][h] >= RG::size(j + 1) ? RG::size(j + 1) : 0; }
            }
        }
    }
}

}  // namespace tri
