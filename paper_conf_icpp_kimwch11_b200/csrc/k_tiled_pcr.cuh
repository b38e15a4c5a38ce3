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
// B200 form: one ring buffer per level in shared memory (power-of-two size >=
// T + 2 sigma_j, modular indexing instead of the paper's buffer shifts);
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
    int ring_off[16];  // row offset of level j's ring inside the smem arrays
    int ring_mask[16];
    int ring_total;    // rows across all rings
};

__host__ __device__ inline int64_t halo_f(int k) { return (int64_t(1) << k) - 1; }  // Eq 8

template <typename T>
__global__ void __launch_bounds__(TPCR_T) k_tiled_pcr(TiledArgs<T> p) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* rA = reinterpret_cast<T*>(smem_raw);
    T* rC = rA + p.ring_total;
    T* rD = rC + p.ring_total;

    const int tid = threadIdx.x;
    const int64_t q = blockIdx.x / p.nreg;
    const int64_t reg = blockIdx.x - q * p.nreg;
    const int64_t r0 = reg * p.region;
    const int64_t r1 = imin64(r0 + p.region, p.n_pad);
    const int64_t fk = halo_f(p.k);
    const int64_t start = r0 - fk;  // halo: level-0 rows [r0-f(k), r1+f(k)) feed outputs [r0, r1)
    const int64_t n = p.n;
    const int S = 1 << p.k;

    // rings start as identity rows (they are only read outside the valid cone)
    for (int e = tid; e < p.ring_total; e += TPCR_T) { rA[e] = T(0); rC[e] = T(0); rD[e] = T(0); }
    __syncthreads();

    for (int64_t s0 = start; s0 - fk < r1; s0 += TPCR_T) {
        // level 0: load + normalise one row per thread
        {
            const int64_t i = s0 + tid;
            NRow<T> r = identity_row<T>();
            if (i >= 0 && i < n) {
                const int64_t gi = elem_index(q, i, n, p.m, p.layout);
                T av = i > 0 ? ldg_stream(p.a + gi) : T(0);
                T cv = i < n - 1 ? ldg_stream(p.c + gi) : T(0);
                r = normalise(av, ldg_stream(p.b + gi), cv, ldg_stream(p.d + gi));
            }
            const int s = p.ring_off[0] + (int)(i & p.ring_mask[0]);
            rA[s] = r.A; rC[s] = r.C; rD[s] = r.D;
        }
        __syncthreads();
        int64_t F = s0 + TPCR_T;  // level-j frontier (exclusive)
        for (int j = 0; j < p.k; ++j) {
            const int sg = 1 << j;
            F -= sg;
            const int64_t i = F - TPCR_T + tid;
            const int off = p.ring_off[j], msk = p.ring_mask[j];
            const int so = off + (int)(i & msk), sm = off + (int)((i - sg) & msk), sp = off + (int)((i + sg) & msk);
            NRow<T> o{rA[so], rC[so], rD[so]};
            NRow<T> mm{rA[sm], rC[sm], rD[sm]};
            NRow<T> pp{rA[sp], rC[sp], rD[sp]};
            NRow<T> nr = pcr_combine(mm, o, pp);
            if (j + 1 < p.k) {
                const int sd = p.ring_off[j + 1] + (int)(i & p.ring_mask[j + 1]);
                rA[sd] = nr.A; rC[sd] = nr.C; rD[sd] = nr.D;
            } else if (i >= r0 && i < r1) {
                if (p.mode == 0) {
                    const int64_t idx = (i >> p.k) * p.C + q * S + (i & (S - 1));
                    p.oA[idx] = nr.A; p.oC[idx] = nr.C; p.oD[idx] = nr.D;
                } else if (i < n) {
                    const int64_t gi = elem_index(q, i, n, p.m, p.layout);
                    p.oA[gi] = nr.A; p.oC[gi] = nr.C; p.oD[gi] = nr.D;
                }
            }
            __syncthreads();
        }
    }
}

}  // namespace tri
