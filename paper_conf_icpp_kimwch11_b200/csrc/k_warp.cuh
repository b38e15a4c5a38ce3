// k_warp.cuh -- WARP variant: one warp owns one system of n <= 32 R rows and
// runs the whole hybrid solve in registers (Sec. III, P:687-693,
// with the transition fixed at k = 5 = log2(warp size)).
//
// Row i lives in lane i % 32, slot t = i / 32.  PCR step j (Eqs 5-6 at stride
// s = 2^j) needs rows i - s and i + s: lane (lane -/+ s) mod 32 in
// the same slot, or the neighbouring slot when the lane index wraps.  One
// shuffle per value moves them: the sender pre-selects which of its slots the
// receiver needs.  After the five steps s = 1..16 the system has split into 32
// interleaved subsystems (Fig 4) and subsystem c = rows c + 32 t is
// exactly lane c's registers, so the interleave transform is free and the
// p-Thomas stage (Eqs 2-4, one thread per subsystem) runs on the
// registers with no shared memory, no barriers and no spill.
//
// Loads/stores: contiguous layout -> lane-consecutive rows are address-
// consecutive (one 128/256-byte segment per slot and array); interleaved
// layout -> a shared-memory transpose per slot (below).
#pragma once
#include "common.cuh"

namespace tri {

constexpr int WARP_K = 5;       // PCR steps = log2(32)
constexpr int WARP_WPB = 4;     // warps (systems) per CTA
#ifndef WARP_NO_PREFETCH
#define WARP_NO_PREFETCH 0
#endif

template <typename T>
struct WarpArgs {
    const T *a, *b, *c, *d;
    T* x;
    T *ao, *co, *do_;           // debug: reduced rows after the PCR stage
    int64_t n, m;
    int layout;
    int mode;                   // 0 solve, 1 PCR stage only
};

template <typename T>
__device__ __forceinline__ T shfl_idx(T v, int src) {
    return __shfl_sync(0xffffffffu, v, src);
}

// One PCR step at stride S over the warp's R slots, in place.  Rows outside
// [0, n) are zero rows (identity, reading X4); slot "-1" and slot "R" are zero.
template <typename T, int R, int S>
__device__ __forceinline__ void warp_pcr_step(T (&A)[R], T (&C)[R], T (&D)[R], int lane) {
    const int up_src = (lane - S) & 31, dn_src = (lane + S) & 31;
    const bool up_wrap = lane >= 32 - S;  // my slot t-1 goes to lane + S - 32, slot t
    const bool dn_wrap = lane < S;        // my slot t+1 goes to lane - S + 32, slot t
    T pA = T(0), pC = T(0), pD = T(0);    // old values of slot t-1
#pragma unroll
    for (int t = 0; t < R; ++t) {
        const T nA = t + 1 < R ? A[t + 1] : T(0);
        const T nC = t + 1 < R ? C[t + 1] : T(0);
        const T nD = t + 1 < R ? D[t + 1] : T(0);
        const T Am = shfl_idx(up_wrap ? pA : A[t], up_src);
        const T Cm = shfl_idx(up_wrap ? pC : C[t], up_src);
        const T Dm = shfl_idx(up_wrap ? pD : D[t], up_src);
        const T Ap = shfl_idx(dn_wrap ? nA : A[t], dn_src);
        const T Cp = shfl_idx(dn_wrap ? nC : C[t], dn_src);
        const T Dp = shfl_idx(dn_wrap ? nD : D[t], dn_src);
        pA = A[t]; pC = C[t]; pD = D[t];
        const NRow<T> o = pcr_combine(NRow<T>{Am, Cm, Dm}, NRow<T>{A[t], C[t], D[t]}, NRow<T>{Ap, Cp, Dp});
        A[t] = o.A; C[t] = o.C; D[t] = o.D;
    }
}

// Interleaved layout: a CTA of WARP_WPB_IL warps owns WARP_WPB_IL consecutive
// systems, so one row of the CTA's systems is a >= 32-byte contiguous segment.
// Thread th loads row 32 t + th / WPB of system q0 + th % WPB (coalesced) and a
// shared-memory transpose per slot hands each warp its system's 32 rows; x
// goes back the same way.
constexpr int WARP_WPB_IL = 8;

// measured (B200): fp32 R = 8 (c4) 1.83 -> 1.49 ms with the prefetch; fp64 R = 4
// 1.36 -> 1.60 ms (the doubled registers cost more occupancy than the overlap
// gains), larger R spill
template <typename T, int R>
__host__ __device__ constexpr bool warp_persistent() {
    return sizeof(T) == 4 && R <= 8 && !WARP_NO_PREFETCH;
}

// PCR stage + p-Thomas on one system held in registers, then x (or, in PCR
// debug mode, the reduced rows) to [base + i * stride]
template <typename T, int R>
__device__ __forceinline__ void warp_solve_and_store(const WarpArgs<T>& p, T (&A)[R], T (&C)[R], T (&D)[R], int lane,
                                                     int64_t base, int64_t stride) {
    const int64_t n = p.n;
    warp_pcr_step<T, R, 1>(A, C, D, lane);
    warp_pcr_step<T, R, 2>(A, C, D, lane);
    warp_pcr_step<T, R, 4>(A, C, D, lane);
    warp_pcr_step<T, R, 8>(A, C, D, lane);
    warp_pcr_step<T, R, 16>(A, C, D, lane);
    if (p.mode == 1) {
#pragma unroll
        for (int t = 0; t < R; ++t) {
            const int64_t i = (int64_t)t * 32 + lane;
            if (i < n) {
                const int64_t e = base + i * stride;
                p.ao[e] = A[t]; p.co[e] = C[t]; p.do_[e] = D[t];
            }
        }
        return;
    }
    T cp = T(0), dp = T(0);
#pragma unroll
    for (int t = 0; t < R; ++t) {
        thomas_fwd(NRow<T>{A[t], C[t], D[t]}, cp, dp);
        C[t] = cp; D[t] = dp;
    }
    T xv = T(0);
#pragma unroll
    for (int t = R - 1; t >= 0; --t) {
        xv = fma(-C[t], xv, D[t]);
        const int64_t i = (int64_t)t * 32 + lane;
        if (i < n) p.x[base + i * stride] = xv;
    }
}

template <typename T, int R, bool IL>
__global__ void __launch_bounds__((IL ? WARP_WPB_IL : WARP_WPB) * 32) k_warp(WarpArgs<T> p) {
    constexpr int WPB = IL ? WARP_WPB_IL : WARP_WPB;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t q = (int64_t)blockIdx.x * WPB + warp;
    const int64_t n = p.n;
    if (!IL && q >= p.m) return;
    const int64_t base = IL ? q : q * n;
    const int64_t stride = IL ? p.m : 1;

    T A[R], C[R], D[R];
    if constexpr (!IL) {
        // load + normalise (reading X17); a_0 and c_{n-1} are ignored (never
        // read into arithmetic), rows >= n are zero rows
        T ra[R], rb[R], rc[R], rd[R];
        auto load = [&](int64_t bq) {
#pragma unroll
            for (int t = 0; t < R; ++t) {
                const int64_t i = (int64_t)t * 32 + lane;
                const bool in = i < n;
                const int64_t e = bq + i;
                ra[t] = in ? ldg_stream(p.a + e) : T(0);
                rb[t] = in ? ldg_stream(p.b + e) : T(1);
                rc[t] = in ? ldg_stream(p.c + e) : T(0);
                rd[t] = in ? ldg_stream(p.d + e) : T(0);
            }
        };
        load(base);
        // persistent warps (small R): the next system's rows are in flight while
        // this one is reduced and solved; large R: one system per warp (the
        // doubled register footprint would spill)
        const int64_t qstride = warp_persistent<T, R>() ? (int64_t)gridDim.x * WPB : p.m;
        for (int64_t qq = q; qq < p.m; qq += qstride) {
#pragma unroll
            for (int t = 0; t < R; ++t) {
                const int64_t i = (int64_t)t * 32 + lane;
                const T r = rcp(rb[t]);
                A[t] = i > 0 && i < n ? ra[t] * r : T(0);
                C[t] = i < n - 1 ? rc[t] * r : T(0);
                D[t] = rd[t] * r;
            }
            if (warp_persistent<T, R>() && qq + qstride < p.m) load((qq + qstride) * n);
            warp_solve_and_store<T, R>(p, A, C, D, lane, qq * n, 1);
        }
        return;
    } else {
        __shared__ T tile[4][WPB][33];
        const int th = threadIdx.x;
        const int tq = th % WPB, tr = th / WPB;  // this thread's (system, row-in-slot) for global access
        const int64_t gq = (int64_t)blockIdx.x * WPB + tq;
        constexpr int RC = R < 8 ? R : 8;          // slots loaded per batch (bounds live registers)
#pragma unroll
        for (int t0 = 0; t0 < R; t0 += RC) {
            T raw[4][RC];
#pragma unroll
            for (int u = 0; u < RC; ++u) {
                const int64_t i = (int64_t)(t0 + u) * 32 + tr;
                const bool ok = gq < p.m && i < n;
                const int64_t e = i * p.m + gq;
                raw[0][u] = ok ? ldg_stream(p.a + e) : T(0);
                raw[1][u] = ok ? ldg_stream(p.b + e) : T(1);
                raw[2][u] = ok ? ldg_stream(p.c + e) : T(0);
                raw[3][u] = ok ? ldg_stream(p.d + e) : T(0);
            }
#pragma unroll
            for (int u = 0; u < RC; ++u) {
#pragma unroll
                for (int arr = 0; arr < 4; ++arr) tile[arr][tq][tr] = raw[arr][u];
                __syncthreads();
                const int64_t i = (int64_t)(t0 + u) * 32 + lane;
                const T av = tile[0][warp][lane], bv = tile[1][warp][lane];
                const T cv = tile[2][warp][lane], dv = tile[3][warp][lane];
                __syncthreads();
                const T r = rcp(bv);
                const bool in = i < n;
                A[t0 + u] = in && i > 0 ? av * r : T(0);
                C[t0 + u] = in && i < n - 1 ? cv * r : T(0);
                D[t0 + u] = in ? dv * r : T(0);
            }
        }
    }
    warp_pcr_step<T, R, 1>(A, C, D, lane);
    warp_pcr_step<T, R, 2>(A, C, D, lane);
    warp_pcr_step<T, R, 4>(A, C, D, lane);
    warp_pcr_step<T, R, 8>(A, C, D, lane);
    warp_pcr_step<T, R, 16>(A, C, D, lane);

    if (p.mode == 1) {
        if (q < p.m) {
#pragma unroll
            for (int t = 0; t < R; ++t) {
                const int64_t i = (int64_t)t * 32 + lane;
                if (i < n) {
                    const int64_t e = base + i * stride;
                    p.ao[e] = A[t]; p.co[e] = C[t]; p.do_[e] = D[t];
                }
            }
        }
        return;
    }
    // p-Thomas on subsystem `lane` (Eqs 2-4 on normalised rows): forward sweep
    // keeps c', d' in C, D; rows >= n are zero rows and give x = 0 (unused).
    T cp = T(0), dp = T(0);
#pragma unroll
    for (int t = 0; t < R; ++t) {
        thomas_fwd(NRow<T>{A[t], C[t], D[t]}, cp, dp);
        C[t] = cp; D[t] = dp;
    }
    T xv = T(0);
    {
        __shared__ T xt[WPB][33];
        const int th = threadIdx.x;
        const int tq = th % WPB, tr = th / WPB;
        const int64_t gq = (int64_t)blockIdx.x * WPB + tq;
#pragma unroll
        for (int t = R - 1; t >= 0; --t) {
            xv = fma(-C[t], xv, D[t]);
            xt[warp][lane] = xv;
            __syncthreads();
            const int64_t i = (int64_t)t * 32 + tr;
            const T v = xt[tq][tr];
            __syncthreads();
            if (gq < p.m && i < n) p.x[i * p.m + gq] = v;
        }
    }
}

}  // namespace tri
