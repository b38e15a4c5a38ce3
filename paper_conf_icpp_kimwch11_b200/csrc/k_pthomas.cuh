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
    int discard;              // TMA kernels: L2-discard consumed c', d' lines (rows 128-B aligned)
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

// MODE 2: contiguous raw input, k = 0.  A CTA of CH threads owns CH consecutive
// systems.  An S-stage cp.async ring stages R-row tiles, smem layout
// [stage][array][system][R + pad] (80-byte system stride: conflict-free 16-byte
// reads), so each thread walks its own system's rows out of shared memory.
template <typename T>
struct PT2Cfg {
    static constexpr int R = 64 / sizeof(T);      // rows per tile: one 64-byte segment per system
    static constexpr int EPC = 16 / sizeof(T);    // elements per 16-byte chunk
    static constexpr int SROW = R + EPC;          // padded per-system stride (80 bytes)
};
constexpr int PT2_S = 6;  // pipeline stages
constexpr int PT2_UB = 16;  // backward-sweep prefetch depth (rows)

template <typename T, int CH>
__host__ __device__ constexpr int pt2_smem_bytes() {
    return PT2_S * 4 * CH * PT2Cfg<T>::SROW * (int)sizeof(T);
}

template <typename T, int CH, bool VEC16>
__global__ void __launch_bounds__(CH) k_pthomas_contig(PThomasArgs<T> p) {
    constexpr int R = PT2Cfg<T>::R, EPC = PT2Cfg<T>::EPC, SROW = PT2Cfg<T>::SROW;
    constexpr int STAGE = 4 * CH * SROW;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* sm = reinterpret_cast<T*>(smem_raw);
    const int tid = threadIdx.x;
    const int64_t q0 = (int64_t)blockIdx.x * CH;
    const int G = (int)imin64(CH, p.m - q0);
    const int64_t n = p.n;
    const int64_t ntile = (n + R - 1) / R;
    auto src = [&](int arr) { return arr == 0 ? p.a : arr == 1 ? p.b : arr == 2 ? p.c : p.d; };

    // this thread's share of a tile's 16-byte chunks: 4 arrays x CPS (system, chunk)
    // pairs, fixed for the whole sweep (only the row offset t*R changes)
    constexpr int CPS = R / EPC;
    int64_t gofs[CPS];
    int soff[CPS];
    bool gval[CPS];
#pragma unroll
    for (int jj = 0; jj < CPS; ++jj) {
        const int rem = tid + jj * CH;
        const int g = rem / CPS, ck = rem % CPS;
        gval[jj] = g < G;
        gofs[jj] = (q0 + (g < G ? g : 0)) * n + ck * EPC;
        soff[jj] = g * SROW + ck * EPC;
    }
    auto issue = [&](int64_t t) {
        T* st = sm + (int)(t % PT2_S) * STAGE;
        const int64_t r0 = t * R;
        if (VEC16) {
            const bool full_tile = r0 + R <= n;
#pragma unroll
            for (int arr = 0; arr < 4; ++arr) {
                const T* base = src(arr);
#pragma unroll
                for (int jj = 0; jj < CPS; ++jj) {
                    int bytes = 16;
                    if (!full_tile || !gval[jj]) {
                        const int64_t i = r0 + (soff[jj] % SROW);
                        bytes = (gval[jj] && i < n) ? (int)imin64(EPC, n - i) * (int)sizeof(T) : 0;
                    }
                    cp_async_16(st + arr * CH * SROW + soff[jj], bytes ? (const void*)(base + gofs[jj] + r0)
                                                                        : (const void*)base, bytes);
                }
            }
        } else {
#pragma unroll 4
            for (int e = tid; e < 4 * CH * R; e += CH) {
                const int arr = e / (CH * R);
                const int rem = e - arr * CH * R;
                const int g = rem / R, u = rem - (rem / R) * R;
                const int64_t i = t * R + u;
                int bytes = 0;
                const T* gp = src(arr);
                if (g < G && i < n) {
                    bytes = (int)sizeof(T);
                    gp = src(arr) + (q0 + g) * n + i;
                }
                if (sizeof(T) == 8) cp_async_8(st + (arr * CH + g) * SROW + u, gp, bytes);
                else cp_async_4(st + (arr * CH + g) * SROW + u, gp, bytes);
            }
        }
    };

#pragma unroll
    for (int s = 0; s < PT2_S - 1; ++s) {
        if (s < ntile) issue(s);
        cp_async_commit();
    }
    const int64_t ch = q0 + tid;
    const bool active = tid < G;
    T cp = T(0), dp = T(0);
    for (int64_t t = 0; t < ntile; ++t) {
        cp_async_wait<PT2_S - 2>();
        __syncthreads();  // tile t visible to all; stage (t-1) % S free
        if (t + PT2_S - 1 < ntile) issue(t + PT2_S - 1);
        cp_async_commit();
        if (active) {
            const T* st = sm + (int)(t % PT2_S) * STAGE + tid * SROW;
            T v[4][R];
#pragma unroll
            for (int arr = 0; arr < 4; ++arr)
#pragma unroll
                for (int c = 0; c < R / EPC; ++c) {
                    const int4 w = *reinterpret_cast<const int4*>(st + arr * CH * SROW + c * EPC);
                    const T* wt = reinterpret_cast<const T*>(&w);
#pragma unroll
                    for (int e = 0; e < EPC; ++e) v[arr][c * EPC + e] = wt[e];
                }
#pragma unroll
            for (int u = 0; u < R; ++u) {
                const int64_t j = t * R + u;
                if (j < n) {
                    Row4<T> row{j > 0 ? v[0][u] : T(0), v[1][u], j < n - 1 ? v[2][u] : T(0), v[3][u]};
                    thomas_fwd(row, cp, dp);
                    const int64_t idx = j * p.C + ch;
                    p.cps[idx] = cp;
                    p.dps[idx] = dp;
                }
            }
        }
    }
    // backward sweep (Eq 4), tiles of RB positions walked from the end; the c', d'
    // rows of this CTA's CH chains are staged by cp.async into the (now idle)
    // ring, PT2_S - 1 tiles ahead, so the scratch reads keep HBM busy.
    cp_async_wait<0>();
    __syncthreads();
    constexpr int RB = 16;                 // positions per backward tile
    constexpr int BST = 2 * RB * CH;       // elements per backward stage
    static_assert(BST <= STAGE, "backward stage must fit a forward stage");
    const int64_t nb = n - 1;              // positions n-2 .. 0 (x_{n-1} = d'_{n-1})
    const int64_t nbt = (nb + RB - 1) / RB;
    auto issue_b = [&](int64_t bt) {       // tile bt covers positions [lo, hi)
        if (bt < nbt) {
            T* st = sm + (int)(bt % PT2_S) * STAGE;
            const int64_t hi = nb - bt * RB, lo = imax64(hi - RB, 0);
            constexpr int CPR = CH * (int)sizeof(T) / 16;  // 16-byte chunks per position row
#pragma unroll
            for (int e = tid; e < 2 * RB * CPR; e += CH) {
                const int arr = e / (RB * CPR);
                const int rem = e - arr * RB * CPR;
                const int u = rem / CPR, ck = rem % CPR;
                const int64_t j = hi - 1 - u;
                const int gl = ck * (16 / (int)sizeof(T));
                const bool ok = j >= lo && q0 + gl < p.m;
                const T* base = arr == 0 ? p.cps : p.dps;
                cp_async_16(st + (arr * RB + u) * CH + gl, ok ? (const void*)(base + j * p.C + q0 + gl)
                                                              : (const void*)base, ok ? 16 : 0);
            }
        }
        cp_async_commit();
    };
    const bool vecb = ((p.C * (int64_t)sizeof(T)) % 16 == 0) && ((q0 * (int64_t)sizeof(T)) % 16 == 0) &&
                      (p.m - q0) >= CH;
    T* xq = p.x + ch * n;
    T xv = dp;
    if (active) xq[n - 1] = xv;
    if (vecb) {
#pragma unroll
        for (int s2 = 0; s2 < PT2_S - 1; ++s2) issue_b(s2);
        for (int64_t bt = 0; bt < nbt; ++bt) {
            cp_async_wait<PT2_S - 2>();
            __syncthreads();
            issue_b(bt + PT2_S - 1);
            const T* st = sm + (int)(bt % PT2_S) * STAGE;
            const int64_t hi = nb - bt * RB, lo = imax64(hi - RB, 0);
            if (active) {
#pragma unroll
                for (int u = 0; u < RB; ++u) {
                    const int64_t j = hi - 1 - u;
                    if (j >= lo) {
                        xv = fma(-st[u * CH + tid], xv, st[(RB + u) * CH + tid]);
                        xq[j] = xv;
                    }
                }
            }
        }
        cp_async_wait<0>();
    } else if (active) {
        for (int64_t j = n - 2; j >= 0; --j) {
            const int64_t idx = j * p.C + ch;
            xv = fma(-p.cps[idx], xv, p.dps[idx]);
            xq[j] = xv;
        }
    }
}


// ---------------------------------------------------------------------------
// MODE 0 / MODE 1 with few, long chains (k_pthomas_ring): a CTA of CW threads
// owns CW adjacent chains; an 8-stage cp.async ring stages RP positions x CW
// chains of every input array (RP * CW = 256, 6-8 KB per stage), so each SM
// keeps ~50 KB of loads in flight even with one 8-thread CTA, and the grid
// spreads a few thousand chains over all SMs.  The forward sweep is the
// continuant form of Eqs 2-3 (X18): the serial dependency per
// position is one FMA, the reciprocal of theta_i is off the chain.
//   theta_i = theta_{i-1} - A_i C_{i-1} theta_{i-2},  delta_i = D_i theta_{i-1} - A_i delta_{i-1}
//   c'_i = C_i theta_{i-1} / theta_i,                 d'_i = delta_i / theta_i
// theta, delta are rescaled by exact powers of two when |theta| leaves
// [2^-S, 2^S] (ratios, hence c', d', unchanged).  The back substitution (Eq 4)
// streams c', d' back through the same ring in reverse.
constexpr int PTR_NS = 8;      // ring stages
constexpr int PTR_ROWS = 256;  // RP * CW per stage

template <typename T>
struct PTRScale;
template <>
struct PTRScale<double> {
    static constexpr double lo = 0x1p-200, hi = 0x1p200, up = 0x1p200, down = 0x1p-200;
};
template <>
struct PTRScale<float> {
    static constexpr float lo = 0x1p-40f, hi = 0x1p40f, up = 0x1p40f, down = 0x1p-40f;
};

template <typename T, int CW>
__host__ __device__ constexpr int ptr_smem_bytes(bool raw) {
    return PTR_NS * (raw ? 4 : 3) * PTR_ROWS * (int)sizeof(T);
}

template <typename T, int CW, int MODE, bool VEC>
__global__ void __launch_bounds__(CW) k_pthomas_ring(PThomasArgs<T> p) {
    static_assert(MODE == 0 || MODE == 1, "ring p-Thomas takes chain-interleaved input");
    constexpr int RP = PTR_ROWS / CW;            // positions per stage
    constexpr int NA = MODE == 1 ? 4 : 3;        // input arrays
    constexpr int EPC = 16 / (int)sizeof(T);     // elements per 16-byte chunk
    constexpr int STAGE = NA * PTR_ROWS;         // elements per stage
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* sm = reinterpret_cast<T*>(smem_raw);
    const int tid = threadIdx.x;
    const int64_t ch0 = (int64_t)blockIdx.x * CW;
    const int64_t ch = ch0 + tid;
    const int64_t C = p.C, L = p.L;
    const bool active = ch < C;
    const int64_t nst = (L + RP - 1) / RP;

    // stage t holds positions [t RP, t RP + RP) of arrays src(0..NA-1), layout [arr][u][CW]
    auto issue = [&](int64_t t, int na, auto src) {
        if (t < nst) {
            T* st = sm + (int)(t % PTR_NS) * STAGE;
            const int64_t p0 = t * RP;
            if (VEC) {
                constexpr int CPR = CW / EPC;      // chunks per (array, position) row
                for (int e = tid; e < na * RP * CPR; e += CW) {
                    const int arr = e / (RP * CPR);
                    const int rem = e - arr * RP * CPR;
                    const int u = rem / CPR, h = rem - u * CPR;
                    const int64_t j = p0 + u, c0 = ch0 + h * EPC;
                    const int64_t ok = (j < L && c0 < C) ? imin64(EPC, C - c0) : 0;
                    const T* g = src(arr);
                    cp_async_16(st + (arr * RP + u) * CW + h * EPC, ok ? (const void*)(g + j * C + c0) : (const void*)g,
                                (int)ok * (int)sizeof(T));
                }
            } else {
                for (int e = tid; e < na * RP * CW; e += CW) {
                    const int arr = e / (RP * CW);
                    const int rem = e - arr * RP * CW;
                    const int u = rem / CW, h = rem - u * CW;
                    const int64_t j = p0 + u, c = ch0 + h;
                    const bool ok = j < L && c < C;
                    const T* g = src(arr);
                    if (sizeof(T) == 8) cp_async_8(st + (arr * RP + u) * CW + h, ok ? (const void*)(g + j * C + c) : (const void*)g, ok ? 8 : 0);
                    else cp_async_4(st + (arr * RP + u) * CW + h, ok ? (const void*)(g + j * C + c) : (const void*)g, ok ? 4 : 0);
                }
            }
        }
        cp_async_commit();
    };
    auto fsrc = [&](int arr) -> const T* {
        if (MODE == 1) return arr == 0 ? p.a : arr == 1 ? p.b : arr == 2 ? p.c : p.d;
        return arr == 0 ? p.iA : arr == 1 ? p.iC : p.iD;
    };
#pragma unroll 1
    for (int s = 0; s < PTR_NS - 1; ++s) issue(s, NA, fsrc);

    T th1 = T(1), th2 = T(0), de1 = T(0), Cm = T(0);  // theta_{i-1}, theta_{i-2}, delta_{i-1}, C_{i-1}
#pragma unroll 1
    for (int64_t t = 0; t < nst; ++t) {
        cp_async_wait<PTR_NS - 2>();
        __syncthreads();
        issue(t + PTR_NS - 1, NA, fsrc);
        const T* st = sm + (int)(t % PTR_NS) * STAGE + tid;
        const int64_t p0 = t * RP;
        if (active) {
#pragma unroll 4
            for (int u = 0; u < RP; ++u) {
                const int64_t j = p0 + u;
                if (j >= L) break;
                T A, Cc, D;
                if (MODE == 1) {
                    const T r = rcp(st[(1 * RP + u) * CW]);
                    A = j > 0 ? st[u * CW] * r : T(0);
                    Cc = j < L - 1 ? st[(2 * RP + u) * CW] * r : T(0);
                    D = st[(3 * RP + u) * CW] * r;
                } else {
                    A = st[u * CW]; Cc = st[(RP + u) * CW]; D = st[(2 * RP + u) * CW];
                }
                const T th = fma(-(A * Cm), th2, th1);
                const T de = fma(-A, de1, D * th1);
                const T r = rcp(th);
                const int64_t idx = j * C + ch;
                p.cps[idx] = Cc * th1 * r;
                p.dps[idx] = de * r;
                th2 = th1; th1 = th; de1 = de; Cm = Cc;
                const T ath = fabs(th1);
                if (ath < PTRScale<T>::lo || ath > PTRScale<T>::hi) {
                    const T f = ath < PTRScale<T>::lo ? PTRScale<T>::up : PTRScale<T>::down;
                    th1 *= f; th2 *= f; de1 *= f;
                }
            }
        }
    }
    // back substitution (Eq 4): stage t' holds positions [hi - RP, hi), hi = L - t' RP
    cp_async_wait<0>();
    __syncthreads();
    __threadfence_block();
    auto bsrc = [&](int arr) -> const T* { return arr == 0 ? p.cps : p.dps; };
    auto issue_b = [&](int64_t t) {
        if (t < nst) {
            T* st = sm + (int)(t % PTR_NS) * STAGE;
            const int64_t hi = L - t * RP;
            if (VEC) {
                constexpr int CPR = CW / EPC;
                for (int e = tid; e < 2 * RP * CPR; e += CW) {
                    const int arr = e / (RP * CPR);
                    const int rem = e - arr * RP * CPR;
                    const int u = rem / CPR, h = rem - u * CPR;
                    const int64_t j = hi - 1 - u, c0 = ch0 + h * EPC;
                    const int64_t ok = (j >= 0 && c0 < C) ? imin64(EPC, C - c0) : 0;
                    const T* g = bsrc(arr);
                    cp_async_16(st + (arr * RP + u) * CW + h * EPC, ok ? (const void*)(g + j * C + c0) : (const void*)g,
                                (int)ok * (int)sizeof(T));
                }
            } else {
                for (int e = tid; e < 2 * RP * CW; e += CW) {
                    const int arr = e / (RP * CW);
                    const int rem = e - arr * RP * CW;
                    const int u = rem / CW, h = rem - u * CW;
                    const int64_t j = hi - 1 - u, c = ch0 + h;
                    const bool ok = j >= 0 && c < C;
                    const T* g = bsrc(arr);
                    if (sizeof(T) == 8) cp_async_8(st + (arr * RP + u) * CW + h, ok ? (const void*)(g + j * C + c) : (const void*)g, ok ? 8 : 0);
                    else cp_async_4(st + (arr * RP + u) * CW + h, ok ? (const void*)(g + j * C + c) : (const void*)g, ok ? 4 : 0);
                }
            }
        }
        cp_async_commit();
    };
#pragma unroll 1
    for (int s = 0; s < PTR_NS - 1; ++s) issue_b(s);
    T xv = T(0);
#pragma unroll 1
    for (int64_t t = 0; t < nst; ++t) {
        cp_async_wait<PTR_NS - 2>();
        __syncthreads();
        issue_b(t + PTR_NS - 1);
        const T* st = sm + (int)(t % PTR_NS) * STAGE + tid;
        const int64_t hi = L - t * RP;
        if (active) {
#pragma unroll 4
            for (int u = 0; u < RP; ++u) {
                const int64_t j = hi - 1 - u;
                if (j < 0) break;
                xv = fma(-st[u * CW], xv, st[(RP + u) * CW]);
                pt_store_x<T, MODE>(p, ch, j, xv);
            }
        }
    }
}

}  // namespace tri
