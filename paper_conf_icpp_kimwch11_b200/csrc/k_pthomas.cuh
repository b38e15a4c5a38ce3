// k_pthomas.cuh -- thread-level parallel Thomas (p-Thomas), TRI_VARIANT_SPLIT
// backend.
//
// Paper: Sec. III.B: "each thread solves a different system ...
// memory accesses to global memory should be coalesced.  This can be achieved
// when we interleave multiple systems in global memory.  Fortunately, PCR
// naturally produces interleaved results".  Thomas Eqs 2-4.
//
// Three input modes:
//   MODE 0  normalised rows (A, C, D) produced by k_tiled_pcr, chain-interleaved:
//           position j of chain ch at [j*C + ch]  (k > 0)
//   MODE 1  raw user rows (a, b, c, d), INTERLEAVED layout: [j*m + q]  (k = 0)
//   MODE 2  raw user rows, CONTIGUOUS layout: [q*n + j]  (k = 0); a CTA of
//           TPT_CH threads stages TPT_R-row tiles of its TPT_CH systems through
//           shared memory (coalesced segment loads, transposed reads), and
//           stages x back the same way.
// The forward sweep's c', d' go to plan scratch, interleaved [j*C + ch] so
// both sweeps coalesce; the backward sweep (Eq 4) reads them in reverse.
#pragma once
#include "common.cuh"

namespace tri {

template <typename T>
struct PThomasArgs {
    const T *a, *b, *c, *d;   // MODE 1/2 inputs (raw)
    const T *iA, *iC, *iD;    // MODE 0 inputs (normalised)
    T* x;
    T *cps, *dps;             // scratch: c', d' interleaved [j*C + ch]
    int64_t n, m, C, L;       // C chains, L positions per chain
    int layout, k;
};

constexpr int PT_U = 4;  // rows prefetched ahead in modes 0/1

template <typename T, int MODE>
struct PTRow {
    using type = NRow<T>;
};
template <typename T>
struct PTRow<T, 1> {
    using type = Row4<T>;
};

template <typename T>
__device__ __forceinline__ void pt_load_into(const PThomasArgs<T>& p, int64_t ch, int64_t j, NRow<T>& r) {
    const int64_t idx = j * p.C + ch;
    r = NRow<T>{ldg_stream(p.iA + idx), ldg_stream(p.iC + idx), ldg_stream(p.iD + idx)};
}
template <typename T>
__device__ __forceinline__ void pt_load_into(const PThomasArgs<T>& p, int64_t ch, int64_t j, Row4<T>& r) {
    const int64_t idx = j * p.C + ch;
    r.a = j > 0 ? ldg_stream(p.a + idx) : T(0);          // a_1 outside A (X1)
    r.b = ldg_stream(p.b + idx);
    r.c = j < p.n - 1 ? ldg_stream(p.c + idx) : T(0);    // c_n outside A (X1)
    r.d = ldg_stream(p.d + idx);
}

template <typename T, int MODE>
__device__ __forceinline__ void pt_store_x(const PThomasArgs<T>& p, int64_t ch, int64_t j, T v) {
    if (MODE == 1) {
        __stcs(p.x + j * p.m + ch, v);
    } else {
        const int64_t q = ch >> p.k;
        const int64_t r = ch & ((int64_t(1) << p.k) - 1);
        const int64_t i = (j << p.k) + r;
        if (i < p.n) __stcs(p.x + elem_index(q, i, p.n, p.m, p.layout), v);
    }
}

// MODE 0 / MODE 1: one thread per chain, coalesced across the warp.
template <typename T, int MODE>
__global__ void __launch_bounds__(128) k_pthomas(PThomasArgs<T> p) {
    const int64_t ch = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (ch >= p.C) return;
    const int64_t L = p.L;
    T cp = T(0), dp = T(0);
    // forward sweep (Eqs 2-3) with a PT_U-row register prefetch window
    using RowT = typename PTRow<T, MODE>::type;
    RowT buf[PT_U];
#pragma unroll
    for (int u = 0; u < PT_U; ++u)
        if (u < L) pt_load_into(p, ch, u, buf[u]);
    for (int64_t j0 = 0; j0 < L; j0 += PT_U) {
        RowT nxt[PT_U];
#pragma unroll
        for (int u = 0; u < PT_U; ++u)
            if (j0 + PT_U + u < L) pt_load_into(p, ch, j0 + PT_U + u, nxt[u]);
#pragma unroll
        for (int u = 0; u < PT_U; ++u) {
            if (j0 + u < L) {
                thomas_fwd(buf[u], cp, dp);
                const int64_t idx = (j0 + u) * p.C + ch;
                p.cps[idx] = cp;
                p.dps[idx] = dp;
            }
        }
#pragma unroll
        for (int u = 0; u < PT_U; ++u) buf[u] = nxt[u];
    }
    // backward sweep (Eq 4): x_{L-1} = d'_{L-1}; x_j = d'_j - c'_j x_{j+1}
    T xv = dp;
    pt_store_x<T, MODE>(p, ch, L - 1, xv);
    int64_t j = L - 2;
    for (; j >= PT_U - 1; j -= PT_U) {
        T cs[PT_U], ds[PT_U];
#pragma unroll
        for (int u = 0; u < PT_U; ++u) {
            const int64_t idx = (j - u) * p.C + ch;
            cs[u] = p.cps[idx];
            ds[u] = p.dps[idx];
        }
#pragma unroll
        for (int u = 0; u < PT_U; ++u) {
            xv = fma(-cs[u], xv, ds[u]);
            pt_store_x<T, MODE>(p, ch, j - u, xv);
        }
    }
    for (; j >= 0; --j) {
        const int64_t idx = j * p.C + ch;
        xv = fma(-p.cps[idx], xv, p.dps[idx]);
        pt_store_x<T, MODE>(p, ch, j, xv);
    }
}

// MODE 2: contiguous raw input, k = 0, staged through shared memory.
constexpr int PT2_CH = 128;  // systems (threads) per CTA
template <typename T>
struct PT2Cfg {
    static constexpr int R = 64 / sizeof(T);  // rows per tile: one 64-byte segment per system
};

template <typename T>
__global__ void __launch_bounds__(PT2_CH) k_pthomas_contig(PThomasArgs<T> p) {
    constexpr int R = PT2Cfg<T>::R;
    constexpr int W = PT2_CH + 1;  // padded row of the transposed tile
    __shared__ T tile[4][R][W];  // [array][row][system]
    const int tid = threadIdx.x;
    const int64_t q0 = (int64_t)blockIdx.x * PT2_CH;
    const int G = (int)imin64(PT2_CH, p.m - q0);
    const int64_t n = p.n;
    const int64_t ntile = (n + R - 1) / R;
    const int64_t ch = q0 + tid;
    const bool active = tid < G;

    // cooperative loader: element e of a tile = (system e / R, row e % R)
    auto load_tile = [&](int64_t t, T (&reg)[4][R]) {
#pragma unroll
        for (int u = 0; u < R; ++u) {
            const int e = tid + u * PT2_CH;
            const int g = e / R, rr = e % R;
            const int64_t i = t * R + rr;
            T av = T(0), bv = T(1), cv = T(0), dv = T(0);
            if (g < G && i < n) {
                const int64_t gi = (q0 + g) * n + i;
                av = i > 0 ? ldg_stream(p.a + gi) : T(0);
                bv = ldg_stream(p.b + gi);
                cv = i < n - 1 ? ldg_stream(p.c + gi) : T(0);
                dv = ldg_stream(p.d + gi);
            }
            reg[0][u] = av; reg[1][u] = bv; reg[2][u] = cv; reg[3][u] = dv;
        }
    };
    auto store_tile = [&](const T (&reg)[4][R]) {
#pragma unroll
        for (int u = 0; u < R; ++u) {
            const int e = tid + u * PT2_CH;
            const int g = e / R, rr = e % R;
#pragma unroll
            for (int v = 0; v < 4; ++v) tile[v][rr][g] = reg[v][u];
        }
    };

    T cp = T(0), dp = T(0);
    T reg[4][R];
    load_tile(0, reg);
    store_tile(reg);
    __syncthreads();
    for (int64_t t = 0; t < ntile; ++t) {
        if (t + 1 < ntile) load_tile(t + 1, reg);  // in flight while we compute
        if (active) {
#pragma unroll
            for (int u = 0; u < R; ++u) {
                const int64_t j = t * R + u;
                if (j < n) {
                    Row4<T> row{tile[0][u][tid], tile[1][u][tid], tile[2][u][tid], tile[3][u][tid]};
                    thomas_fwd(row, cp, dp);
                    const int64_t idx = j * p.C + ch;
                    p.cps[idx] = cp;
                    p.dps[idx] = dp;
                }
            }
        }
        __syncthreads();
        if (t + 1 < ntile) {
            store_tile(reg);
            __syncthreads();
        }
    }
    // backward sweep, tile by tile from the end; x staged in tile[0][0]
    T xv = dp;
    for (int64_t t = ntile - 1; t >= 0; --t) {
        if (active) {
#pragma unroll
            for (int u = R - 1; u >= 0; --u) {
                const int64_t j = t * R + u;
                if (j < n) {
                    if (j < n - 1) {
                        const int64_t idx = j * p.C + ch;
                        xv = fma(-p.cps[idx], xv, p.dps[idx]);
                    }
                    tile[0][u][tid] = xv;
                }
            }
        }
        __syncthreads();
#pragma unroll
        for (int u = 0; u < R; ++u) {
            const int e = tid + u * PT2_CH;
            const int g = e / R, rr = e % R;
            const int64_t i = t * R + rr;
            if (g < G && i < n) __stcs(p.x + (q0 + g) * n + i, tile[0][rr][g]);
        }
        __syncthreads();
    }
}

}  // namespace tri
