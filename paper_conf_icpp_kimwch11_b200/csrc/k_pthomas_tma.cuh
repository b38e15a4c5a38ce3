// k_pthomas_tma.cuh -- p-Thomas for k = 0 on the CONTIGUOUS layout (the paper's
// M > P case: "straight to p-Thomas"), one warp = 32 systems, every tile
// moved by the Tensor Memory Accelerator.
//
// Paper: Sec. III.B, one thread per system; Thomas Eqs 2-4.
// B200 form:
//   forward   a, b, c, d tiles of R rows x 32 systems (128 B per system row,
//             128B-swizzled so each thread's 16-byte reads of its own row are
//             bank-conflict free) arrive by cp.async.bulk.tensor.2d into a
//             PTT_NS-stage ring, one instruction per array per tile, completion
//             on an mbarrier (expect_tx).  Each thread runs Eqs 2-3 down its
//             system and writes c', d' to plan scratch interleaved [j*m + q]
//             (a 256-byte segment per warp store).
//   backward  c', d' tiles of 32 systems x R positions come back by TMA in
//             reverse; x_j = d'_j - c'_j x_{j+1} (Eq 4) goes into a swizzled
//             x tile that a TMA tensor store writes to the user layout.
// Ragged n and m: TMA zero-fills out-of-range reads and clips out-of-range
// writes, threads of systems >= m never store scratch.
#pragma once
#include <cuda.h>
#include "common.cuh"

namespace tri {

constexpr int PTT_CH = 32;  // systems per CTA (one warp)
constexpr int PTT_NS = 3;   // forward ring stages
constexpr int PTT_NB = 3;   // backward ring stages

template <typename T>
struct PTTCfg {
    static constexpr int R = 128 / (int)sizeof(T);     // rows per tile (128 B per system)
    static constexpr int EPC = 16 / (int)sizeof(T);    // elements per 16-byte chunk
    static constexpr int TILE = PTT_CH * R;            // elements per array tile
    static constexpr int FSTAGE = 4 * TILE;            // forward stage: a, b, c, d
    static constexpr int BSTAGE = 2 * TILE;            // backward stage: c', d'
    // forward ring stages: fp64 3 (16 KB each); fp32 2 (n = 256-class systems are
    // 8 tiles long: more resident CTAs beat a deeper ring; c4 measured)
    static constexpr int NS = sizeof(T) == 8 ? 3 : 2;
    static constexpr int NB = 3;                       // backward stages (+ 2 x tiles fit the forward ring)
    static_assert(NB * BSTAGE + 2 * TILE <= NS * FSTAGE, "backward ring must fit the forward ring");
};

template <typename T>
__host__ __device__ constexpr int ptt_smem_bytes() {
    return PTTCfg<T>::NS * PTTCfg<T>::FSTAGE * (int)sizeof(T) + 1024;  // + alignment slack (128B swizzle)
}

__device__ __forceinline__ void ptt_bar_init(uint64_t* bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((unsigned)__cvta_generic_to_shared(bar)) : "memory");
}
__device__ __forceinline__ void ptt_expect(uint64_t* bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(
                     (unsigned)__cvta_generic_to_shared(bar)),
                 "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void ptt_wait(uint64_t* bar, unsigned parity) {
    const unsigned a = (unsigned)__cvta_generic_to_shared(bar);
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "W_%=:\n"
        "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 P1, [%0], %1, %2;\n"
        "@!P1 bra W_%=;\n"
        "}\n" ::"r"(a),
        "r"(parity), "r"(1000000u)
        : "memory");
}
__device__ __forceinline__ void ptt_load(void* dst, const CUtensorMap* tm, int x0, int x1, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
            (unsigned)__cvta_generic_to_shared(dst)),
        "l"(tm), "r"(x0), "r"(x1), "r"((unsigned)__cvta_generic_to_shared(bar))
        : "memory");
}
__device__ __forceinline__ void ptt_store(const CUtensorMap* tm, int x0, int x1, const void* src) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];" ::"l"(tm), "r"(x0),
                 "r"(x1), "r"((unsigned)__cvta_generic_to_shared(src))
                 : "memory");
}

// Drop a consumed scratch line from L2 without writing it back (the c', d'
// intermediates are dead once the back substitution has read them: without
// this, every dirty line still costs a DRAM write when L2 evicts it).
__device__ __forceinline__ void l2_discard(const void* p) {
    asm volatile("discard.global.L2 [%0], 128;" ::"l"(p) : "memory");
}

// Offset (elements) of row u of system s inside a 128B-swizzled [32][R] tile:
// 16-byte chunk j of 128-byte row s lives at chunk j ^ (s & 7).
template <typename T>
__device__ __forceinline__ int ptt_swz(int s, int u) {
    constexpr int EPC = PTTCfg<T>::EPC, R = PTTCfg<T>::R;
    return s * R + (((u / EPC) ^ (s & 7)) * EPC) + (u % EPC);
}

struct PTTMaps {
    CUtensorMap a, b, c, d;  // user arrays, dims {n, m}, box {R, 32}, 128B swizzle
    CUtensorMap x;           // output, same geometry
    CUtensorMap cp, dp;      // scratch [n][m], dims {m, n}, box {32, R}
};

template <typename T>
__global__ void __launch_bounds__(PTT_CH) k_pthomas_tma(const __grid_constant__ PTTMaps tm, PThomasArgs<T> p) {
    constexpr int R = PTTCfg<T>::R, EPC = PTTCfg<T>::EPC, TILE = PTTCfg<T>::TILE;
    constexpr int FSTAGE = PTTCfg<T>::FSTAGE, BSTAGE = PTTCfg<T>::BSTAGE;
    constexpr int NS_ = PTTCfg<T>::NS, NB_ = PTTCfg<T>::NB;
    extern __shared__ unsigned char smem_raw[];
    T* sm = reinterpret_cast<T*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    __shared__ uint64_t fbar[NS_], bbar[NB_];
    const int t = threadIdx.x;
    const int q0 = blockIdx.x * PTT_CH;
    const bool active = q0 + t < p.m;
    const int64_t n = p.n, M = p.m;
    const int ntile = (int)((n + R - 1) / R);
    if (t == 0) {
        for (int s = 0; s < NS_; ++s) ptt_bar_init(&fbar[s]);
        for (int s = 0; s < NB_; ++s) ptt_bar_init(&bbar[s]);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();

    auto issue_f = [&](int tt) {
        if (t == 0 && tt < ntile) {
            const int s = tt % NS_;
            T* st = sm + s * FSTAGE;
            fence_proxy_async_smem();
            ptt_expect(&fbar[s], FSTAGE * (unsigned)sizeof(T));
            ptt_load(st, &tm.a, tt * R, q0, &fbar[s]);
            ptt_load(st + TILE, &tm.b, tt * R, q0, &fbar[s]);
            ptt_load(st + 2 * TILE, &tm.c, tt * R, q0, &fbar[s]);
            ptt_load(st + 3 * TILE, &tm.d, tt * R, q0, &fbar[s]);
        }
    };
    for (int s = 0; s < NS_; ++s) issue_f(s);

    // ---- forward sweep (Eqs 2-3)
    T cp = T(0), dp = T(0);
    for (int tt = 0; tt < ntile; ++tt) {
        const int s = tt % NS_;
        ptt_wait(&fbar[s], (unsigned)((tt / NS_) & 1));
        const T* st = sm + s * FSTAGE;
        T v[4][R];
#pragma unroll
        for (int arr = 0; arr < 4; ++arr)
#pragma unroll
            for (int ck = 0; ck < R / EPC; ++ck) {
                const int4 w = *reinterpret_cast<const int4*>(st + arr * TILE + ptt_swz<T>(t, ck * EPC));
                const T* wt = reinterpret_cast<const T*>(&w);
#pragma unroll
                for (int e = 0; e < EPC; ++e) v[arr][ck * EPC + e] = wt[e];
            }
        __syncwarp();
        issue_f(tt + NS_);  // slot s consumed (values are in registers)
        const int64_t j0 = (int64_t)tt * R;
        T* cps = p.cps + j0 * M + q0 + t;
        T* dps = p.dps + j0 * M + q0 + t;
        if (j0 + R <= n && j0 > 0 && j0 + R < n) {
#pragma unroll
            for (int u = 0; u < R; ++u) {
                thomas_fwd(Row4<T>{v[0][u], v[1][u], v[2][u], v[3][u]}, cp, dp);
                if (active) { cps[u * M] = cp; dps[u * M] = dp; }
            }
        } else {
#pragma unroll
            for (int u = 0; u < R; ++u) {
                const int64_t j = j0 + u;
                if (j < n) {
                    thomas_fwd(Row4<T>{j > 0 ? v[0][u] : T(0), v[1][u], j < n - 1 ? v[2][u] : T(0), v[3][u]}, cp, dp);
                    if (active) { cps[u * M] = cp; dps[u * M] = dp; }
                }
            }
        }
    }

    // ---- back substitution (Eq 4), tiles from the end; the forward ring is
    // idle now and holds the backward ring + two x tiles
    // this warp's c', d' global stores (generic proxy) must be visible to the
    // TMA reads (async proxy) issued below by lane 0
    __threadfence_block();
    asm volatile("fence.proxy.async.global;" ::: "memory");
    __syncwarp();
    T* xt = sm + NB_ * BSTAGE;  // 2 x TILE, swizzled [32][R]
    auto issue_b = [&](int b) {
        if (t == 0 && b < ntile) {
            const int s = b % NB_;
            const int tt = ntile - 1 - b;
            T* st = sm + s * BSTAGE;
            fence_proxy_async_smem();
            ptt_expect(&bbar[s], BSTAGE * (unsigned)sizeof(T));
            ptt_load(st, &tm.cp, q0, tt * R, &bbar[s]);
            ptt_load(st + TILE, &tm.dp, q0, tt * R, &bbar[s]);
        }
    };
    for (int s = 0; s < NB_; ++s) issue_b(s);
    T xv = T(0);
    for (int b = 0; b < ntile; ++b) {
        const int s = b % NB_;
        const int tt = ntile - 1 - b;
        ptt_wait(&bbar[s], (unsigned)((b / NB_) & 1));
        const T* st = sm + s * BSTAGE;   // [R positions][32 systems] per array
        T cs[R], ds[R];
#pragma unroll
        for (int u = 0; u < R; ++u) { cs[u] = st[u * PTT_CH + t]; ds[u] = st[TILE + u * PTT_CH + t]; }
        if (p.discard && t < R && (int64_t)tt * R + t < n) {  // lane u drops row u's lines (32 systems)
            const int64_t off = ((int64_t)tt * R + t) * M + q0;
#pragma unroll
            for (int h = 0; h < PTT_CH * (int)sizeof(T) / 128; ++h) {
                l2_discard(p.cps + off + h * (128 / (int)sizeof(T)));
                l2_discard(p.dps + off + h * (128 / (int)sizeof(T)));
            }
        }
        // the x tile written two tiles ago must have been read out by its TMA store
        if (t == 0) bulk_wait_read<1>();
        __syncwarp();
        issue_b(b + NB_);
        T* xb = xt + (b & 1) * TILE;
        const int64_t j0 = (int64_t)tt * R;
#pragma unroll
        for (int u = R - 1; u >= 0; --u) {
            if (j0 + u < n) xv = fma(-cs[u], xv, ds[u]);
            xb[ptt_swz<T>(t, u)] = xv;  // rows >= n are clipped by the TMA store
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (t == 0) {
            ptt_store(&tm.x, tt * R, q0, xb);
            bulk_commit();
        }
    }
    if (t == 0) bulk_wait<0>();
}

}  // namespace tri

namespace tri {

// ---------------------------------------------------------------------------
// p-Thomas over chain-interleaved data [pos * C + ch] (MODE 0: normalised rows
// from tiled PCR; MODE 1: raw rows of the INTERLEAVED user layout, k = 0), one
// warp = 32 adjacent chains.  Tiles of 32 chains x R positions (256 B x R for
// fp64) arrive by cp.async.bulk.tensor.2d into a PTT_NS-stage ring; c', d' go to
// scratch [pos * C + ch] and come back the same way for Eq 4; x leaves by TMA
// tensor store when the user layout is a 2D [L][C] view (INTERLEAVED, or m = 1
// with n a multiple of 2^k), else by per-thread stores.
template <typename T>
struct PTICfg {
    static constexpr int R = 16;                 // positions per tile
    static constexpr int TILE = PTT_CH * R;      // elements per array tile
};

struct PTIMaps {
    CUtensorMap a, b, c, d;  // inputs (MODE 0 uses a, b, c for iA, iC, iD), dims {C, L}, box {32, R}
    CUtensorMap x;           // output view {C, L} (only when x_tma)
    CUtensorMap cp, dp;      // scratch, dims {C, L}
};

template <typename T, int MODE>
__global__ void __launch_bounds__(PTT_CH) k_pthomas_il_tma(const __grid_constant__ PTIMaps tm, PThomasArgs<T> p,
                                                         int x_tma) {
    constexpr int R = PTICfg<T>::R, TILE = PTICfg<T>::TILE;
    constexpr int NA = MODE == 1 ? 4 : 3;
    constexpr int FSTAGE = NA * TILE, BSTAGE = 2 * TILE;
    extern __shared__ unsigned char smem_raw[];
    T* sm = reinterpret_cast<T*>((reinterpret_cast<uintptr_t>(smem_raw) + 127) & ~uintptr_t(127));
    __shared__ uint64_t fbar[PTT_NS], bbar[PTT_NB];
    const int t = threadIdx.x;
    const int c0 = blockIdx.x * PTT_CH;
    const int64_t ch = c0 + t;
    const bool active = ch < p.C;
    const int64_t L = p.L, C = p.C;
    const int ntile = (int)((L + R - 1) / R);
    if (t == 0) {
        for (int s = 0; s < PTT_NS; ++s) ptt_bar_init(&fbar[s]);
        for (int s = 0; s < PTT_NB; ++s) ptt_bar_init(&bbar[s]);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    auto issue_f = [&](int tt) {
        if (t == 0 && tt < ntile) {
            const int s = tt % PTT_NS;
            T* st = sm + s * FSTAGE;
            fence_proxy_async_smem();
            ptt_expect(&fbar[s], FSTAGE * (unsigned)sizeof(T));
            ptt_load(st, &tm.a, c0, tt * R, &fbar[s]);
            ptt_load(st + TILE, &tm.b, c0, tt * R, &fbar[s]);
            ptt_load(st + 2 * TILE, &tm.c, c0, tt * R, &fbar[s]);
            if (MODE == 1) ptt_load(st + 3 * TILE, &tm.d, c0, tt * R, &fbar[s]);
        }
    };
    for (int s = 0; s < PTT_NS; ++s) issue_f(s);

    T cp = T(0), dp = T(0);
    for (int tt = 0; tt < ntile; ++tt) {
        const int s = tt % PTT_NS;
        ptt_wait(&fbar[s], (unsigned)((tt / PTT_NS) & 1));
        const T* st = sm + s * FSTAGE + t;
        T v[NA][R];
#pragma unroll
        for (int arr = 0; arr < NA; ++arr)
#pragma unroll
            for (int u = 0; u < R; ++u) v[arr][u] = st[arr * TILE + u * PTT_CH];
        __syncwarp();
        issue_f(tt + PTT_NS);
        const int64_t j0 = (int64_t)tt * R;
        T* cps = p.cps + j0 * C + ch;
        T* dps = p.dps + j0 * C + ch;
#pragma unroll
        for (int u = 0; u < R; ++u) {
            const int64_t j = j0 + u;
            if (j < L) {
                if (MODE == 1) {
                    thomas_fwd(Row4<T>{j > 0 ? v[0][u] : T(0), v[1][u], j < L - 1 ? v[2][u] : T(0), v[3][u]}, cp, dp);
                } else {
                    thomas_fwd(NRow<T>{v[0][u], v[1][u], v[2][u]}, cp, dp);
                }
                if (active) { cps[u * C] = cp; dps[u * C] = dp; }
            }
        }
    }

    __threadfence_block();
    asm volatile("fence.proxy.async.global;" ::: "memory");
    __syncwarp();
    T* xt = sm + PTT_NB * BSTAGE;  // 2 x TILE, [R][32]
    auto issue_b = [&](int b) {
        if (t == 0 && b < ntile) {
            const int s = b % PTT_NB;
            const int tt = ntile - 1 - b;
            T* st = sm + s * BSTAGE;
            fence_proxy_async_smem();
            ptt_expect(&bbar[s], BSTAGE * (unsigned)sizeof(T));
            ptt_load(st, &tm.cp, c0, tt * R, &bbar[s]);
            ptt_load(st + TILE, &tm.dp, c0, tt * R, &bbar[s]);
        }
    };
    for (int s = 0; s < PTT_NB; ++s) issue_b(s);
    T xv = T(0);
    for (int b = 0; b < ntile; ++b) {
        const int s = b % PTT_NB;
        const int tt = ntile - 1 - b;
        ptt_wait(&bbar[s], (unsigned)((b / PTT_NB) & 1));
        const T* st = sm + s * BSTAGE + t;
        T cs[R], ds[R];
#pragma unroll
        for (int u = 0; u < R; ++u) { cs[u] = st[u * PTT_CH]; ds[u] = st[TILE + u * PTT_CH]; }
        if (x_tma && t == 0) bulk_wait_read<1>();
        __syncwarp();
        issue_b(b + PTT_NB);
        T* xb = xt + (b & 1) * TILE;
        const int64_t j0 = (int64_t)tt * R;
#pragma unroll
        for (int u = R - 1; u >= 0; --u) {
            const int64_t j = j0 + u;
            if (j < L) xv = fma(-cs[u], xv, ds[u]);
            if (x_tma) {
                xb[u * PTT_CH + t] = xv;
            } else if (j < L && active) {
                pt_store_x<T, MODE>(p, ch, j, xv);
            }
        }
        if (x_tma) {
            fence_proxy_async_smem();
            __syncwarp();
            if (t == 0) {
                ptt_store(&tm.x, c0, tt * R, xb);
                bulk_commit();
            }
        }
    }
    if (x_tma && t == 0) bulk_wait<0>();
}

template <typename T, int MODE>
__host__ __device__ constexpr int pti_smem_bytes() {
    return PTT_NS * (MODE == 1 ? 4 : 3) * PTICfg<T>::TILE * (int)sizeof(T) + 128;
}

}  // namespace tri
