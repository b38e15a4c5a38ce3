// k_stream.cuh -- TRI_VARIANT_STREAM: tiled PCR (k = 3) streamed into p-Thomas in
// one persistent kernel, Thomas intermediates kept on chip / in L2, for batches of
// long systems in the CONTIGUOUS layout (fp64, n % 8 == 0).  HBM traffic is the
// compulsory 5 arrays (read a, b, c, d once; write x once).
//
// Paper: Sec. III.C: "Tiled PCR and p-Thomas can be combined into
// one kernel ... p-Thomas can work with partial data that becomes available
// while tiled PCR kernel executes".  Tiled PCR Sec. III.A (windows
// with halos of f(k) rows, Eq 8, Fig 7); PCR step Eqs 5-6 (reading
// X3 at stride 2^j); Thomas Eqs 2-4; interleaved subsystems:
// after k = 3 steps row i belongs to chain i % 8.
//
// One CTA per SM, persistent over the systems q = blockIdx.x + j * gridDim.x;
// windows w = 0 .. NC-1 of W = 256 rows starting at row 240 w - 8 (a halo of
// 8 >= f(3) = 7 rows on each side, so the 240 middle rows are exact after three
// PCR steps).  Row 240 w + 8 t + c is position 30 w + t of chain c.  Eight
// identical warps run the steps g = j * NC + w (warp g % 8), j = 0 .. nsys:
//   * forward part (j < nsys): TMA-stage window (j, w) (2D tensor view
//     [rows/8][8], 64-byte swizzle, so the blocked register layout -- lane l
//     holds rows 8l .. 8l+7 -- reads conflict-free), normalise (X17), three PCR
//     levels in registers (shuffles only for a lane's edge rows), transpose the
//     240 reduced rows through shared memory so that lane (c, s) = (lane % 8,
//     lane / 8) holds positions 8s .. 8s+7 of chain c, and run the Thomas
//     forward sweep (Eqs 2-3) as the continuant recurrence of DESIGN.md X18 in
//     the state (theta_{t-1}, psi_t = C_{t-1} theta_{t-2}, delta_{t-1}):
//         theta_t = theta_{t-1} - A_t psi_t,  psi_{t+1} = C_t theta_{t-1},
//         delta_t = D_t theta_{t-1} - A_t delta_{t-1},
//     c'_t = psi_{t+1} / theta_t,  d'_t = delta_t / theta_t.
//     The recurrence is linear in the state: every lane builds its segment's
//     3x3 transfer matrix, a two-step shuffle scan combines the four segments
//     of a chain, and the only serial step between windows is one
//     matrix-vector product on the state handed over by the previous step's
//     warp (shared memory + mbarrier).  Each lane then replays its segment from
//     the true incoming state and stores (c', d') into the window's storage
//     slot (shared memory, or the per-CTA L2 spill region).
//   * backward part (j >= 1): Eq 4 on window (j-1, NC-1-w), segmented the same
//     way (affine maps x_start = alpha + beta x_after, a two-step shuffle scan,
//     x handed between steps), x written straight from registers.  It reads the
//     storage slot the forward part of the same step then overwrites (slot of
//     window w: w for even systems, NC-1-w for odd ones), so the slots recycle
//     with no extra synchronisation.
#pragma once
#include <cudaTypedefs.h>
#include "common.cuh"
#include "k_fused.cuh"  // fu_ld2 / fu_st2 shared-memory pair helpers

namespace tri {

constexpr int SK_K = 3;              // PCR steps
constexpr int SK_S = 1 << SK_K;      // chains per system (8)
constexpr int SK_R = 8;              // rows per lane
constexpr int SK_W = 32 * SK_R;      // window rows (256)
constexpr int SK_HALO = 8;           // >= f(3) = 7 (Eq 8), one lane of rows
constexpr int SK_V = SK_W - 2 * SK_HALO;  // valid rows per window (240)
constexpr int SK_P = SK_V / SK_S;    // positions per chain per window (30)
constexpr int SK_SEG = 8;            // positions per lane segment (4 segments: 8, 8, 8, 6)
#ifndef SK_NPCR_DEF
#define SK_NPCR_DEF 12
#endif
constexpr int SK_NPCR = SK_NPCR_DEF;  // warps
static_assert(SK_NPCR <= 15, "chain handover uses named barriers 1 .. NPCR");
constexpr int SK_THREADS = 32 * SK_NPCR;
constexpr int SK_NCMAX = 1024;       // windows per system (one mbarrier per storage slot)
constexpr int SK_TCS = 34;           // transpose buffer: chain stride (elements; bank-spread)
constexpr int SK_SCS = 33;           // storage slot: chain stride ((c', d') pairs; bank-spread)
constexpr int SK_SLOT = SK_S * SK_SCS * 2;  // elements per storage slot

struct StreamMaps {
    CUtensorMap a, b, c, d;
};

template <typename T>
struct StreamArgs {
    T* x;
    T* spill;        // per CTA: (NC - S_on) slots of SK_SLOT elements
    int64_t n, m;
    int NC;          // windows per system
    int S_on;        // resident storage slots
    T *dA, *dC, *dD; // tri_debug_pcr: emit the 3-step reduced rows instead of solving
    unsigned long long* prof;  // optional per-role cycle counters (scripts/prof_stream.py)
    int dbg;         // diagnostics: 1 = forward warps skip the PCR math
};

// shared-memory carve-up (bytes)
template <typename T>
struct SKLayout {
    static constexpr int in_bytes = 4 * SK_W * (int)sizeof(T);              // one window, 4 arrays
    static constexpr int in_stride = (in_bytes + 1023) / 1024 * 1024;        // swizzle atoms aligned
    static constexpr int off_in = 0;
    static constexpr int tr_elems = 3 * SK_S * SK_TCS;                        // [A|C|D][chain][pos]
    static constexpr int off_tr = off_in + SK_NPCR * in_stride;
    static constexpr int off_st = off_tr + SK_NPCR * tr_elems * (int)sizeof(T);  // [NPCR][theta|psi|delta][chain]
    static constexpr int off_xh = off_st + SK_NPCR * 3 * SK_S * (int)sizeof(T);  // [NPCR][chain] x handover
    static constexpr int off_bar = off_xh + SK_NPCR * SK_S * (int)sizeof(T);
    static constexpr int nbar = 3 * SK_NPCR + SK_NCMAX;                         // in_full, stfull, bfull, sfull[slot]
    static constexpr int off_store = (off_bar + nbar * 8 + 1023) / 1024 * 1024;
    static constexpr int slot_bytes = SK_SLOT * (int)sizeof(T);
};

__device__ __forceinline__ void sk_bar_init(uint64_t* bar, unsigned cnt) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(bar)), "r"(cnt)
                 : "memory");
}
__device__ __forceinline__ void sk_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"((unsigned)__cvta_generic_to_shared(bar))
                 : "memory");
}
__device__ __forceinline__ void sk_expect(uint64_t* bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(
                     (unsigned)__cvta_generic_to_shared(bar)),
                 "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void sk_wait(uint64_t* bar, unsigned parity) {
    const unsigned a = (unsigned)__cvta_generic_to_shared(bar);
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "SKW_%=:\n"
        "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 P1, [%0], %1, %2;\n"
        "@!P1 bra SKW_%=;\n"
        "}\n" ::"r"(a),
        "r"(parity), "r"(100000u)
        : "memory");
}
__device__ __forceinline__ void sk_tma2d(void* dst, const CUtensorMap* tm, int x0, int x1, uint64_t* bar,
                                         uint64_t pol) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1, {%2, %3}], [%4], %5;" ::"r"((unsigned)__cvta_generic_to_shared(dst)),
        "l"(tm), "r"(x0), "r"(x1), "r"((unsigned)__cvta_generic_to_shared(bar)), "l"(pol)
        : "memory");
}
__device__ __forceinline__ uint64_t sk_policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t sk_policy_evict_normal() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t sk_policy_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void sk_st_global_last(double* p, double a, double b, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.v2.f64 [%0], {%1, %2}, %3;" ::"l"(p), "d"(a), "d"(b), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ void sk_st_global_last(float* p, float a, float b, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.v2.f32 [%0], {%1, %2}, %3;" ::"l"(p), "f"(a), "f"(b), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ int sk_ld_volatile(const int* p) {
    int v;
    asm volatile("ld.volatile.shared.s32 %0, [%1];" : "=r"(v) : "r"((unsigned)__cvta_generic_to_shared(p)) : "memory");
    return v;
}
__device__ __forceinline__ void sk_st_release(int* p, int v) {
    asm volatile("st.release.cta.shared.s32 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(p)), "r"(v)
                 : "memory");
}
__device__ __forceinline__ int sk_ld_acquire(const int* p) {
    int v;
    asm volatile("ld.acquire.cta.shared.s32 %0, [%1];" : "=r"(v) : "r"((unsigned)__cvta_generic_to_shared(p)) : "memory");
    return v;
}
// spin (lane-uniform) until *p >= v; acquire
__device__ __forceinline__ void sk_wait_ge(const int* p, int v) {
    if (sk_ld_acquire(p) >= v) return;
    while (sk_ld_acquire(p) < v) __nanosleep(64);
}

// Before a warp refills a staging buffer it has read with generic-proxy loads by
// TMA (async proxy): every lane fences its reads against the async proxy, then
// the warp synchronises, then one lane issues the copy (the write-after-read
// hazard otherwise lets the refill land before slow shared-memory loads).
__device__ __forceinline__ void sc_release_buf() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncwarp();
}

template <typename T>
__device__ __forceinline__ T sk_exp2_scale(T v);
template <>
__device__ __forceinline__ double sk_exp2_scale<double>(double v) {
    // 2^(1023 - E) for biased exponent E, clamped to a normal number (E = 2046:
    // 2^-1022, so v s lands in [2, 4); E = 0, zero / subnormal v: 2^1023)
    const long long bits = __double_as_longlong(v);
    const int e = 2046 - (int)((bits >> 52) & 0x7ff);
    return __longlong_as_double((long long)(e < 1 ? 1 : e) << 52);
}
template <>
__device__ __forceinline__ float sk_exp2_scale<float>(float v) {
    const int bits = __float_as_int(v);
    const int e = 254 - ((bits >> 23) & 0xff);
    return __int_as_float((e < 1 ? 1 : e) << 23);
}

// storage slot -> location: the first and last S_on/2 slots are resident in
// shared memory (so that, for either parity, the windows the back substitution
// reads first -- the last ones the forward sweep wrote -- are on chip), the
// middle ones live in the per-CTA spill region.
__device__ __forceinline__ bool sk_resident(int slot, int NC, int S_on, int& idx) {
    const int lo = S_on >> 1, hi0 = NC - (S_on - lo);
    if (slot < lo) { idx = slot; return true; }
    if (slot >= hi0) { idx = lo + (slot - hi0); return true; }
    idx = slot - lo;
    return false;
}

// 3x3 transfer of the forward state (theta, psi, delta): columns = inputs
// (theta_in, psi_in, delta_in); theta and psi do not depend on delta_in.
template <typename T>
struct SKMat {
    T a, b, c, d, e, f, g;  // theta = a th + b ps; psi = c th + d ps; delta = e th + f ps + g de
};
template <typename T>
__device__ __forceinline__ SKMat<T> sk_compose(const SKMat<T>& m2, const SKMat<T>& m1) {  // m2 after m1
    SKMat<T> r;
    r.a = fma(m2.a, m1.a, m2.b * m1.c);
    r.b = fma(m2.a, m1.b, m2.b * m1.d);
    r.c = fma(m2.c, m1.a, m2.d * m1.c);
    r.d = fma(m2.c, m1.b, m2.d * m1.d);
    r.e = fma(m2.e, m1.a, fma(m2.f, m1.c, m2.g * m1.e));
    r.f = fma(m2.e, m1.b, fma(m2.f, m1.d, m2.g * m1.f));
    r.g = m2.g * m1.g;
    return r;
}
template <typename T>
__device__ __forceinline__ SKMat<T> sk_shfl_up(const SKMat<T>& m, int d) {
    SKMat<T> r;
    r.a = __shfl_up_sync(0xffffffffu, m.a, d);
    r.b = __shfl_up_sync(0xffffffffu, m.b, d);
    r.c = __shfl_up_sync(0xffffffffu, m.c, d);
    r.d = __shfl_up_sync(0xffffffffu, m.d, d);
    r.e = __shfl_up_sync(0xffffffffu, m.e, d);
    r.f = __shfl_up_sync(0xffffffffu, m.f, d);
    r.g = __shfl_up_sync(0xffffffffu, m.g, d);
    return r;
}

template <typename T>
__device__ __forceinline__ bool sk_test(uint64_t* bar, unsigned parity) {
    unsigned r;
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "mbarrier.test_wait.parity.acquire.cta.shared::cta.b64 P1, [%1], %2;\n"
        "selp.u32 %0, 1, 0, P1;\n"
        "}\n"
        : "=r"(r)
        : "r"((unsigned)__cvta_generic_to_shared(bar)), "r"(parity)
        : "memory");
    return r != 0;
}
__device__ __forceinline__ void sk_ldg2(const double* p, double& a, double& b) {
    asm volatile("ld.global.v2.f64 {%0, %1}, [%2];" : "=d"(a), "=d"(b) : "l"(p));
}

template <typename T, bool PROF>
__global__ void __launch_bounds__(SK_THREADS, 1) k_stream(const __grid_constant__ StreamMaps tm, StreamArgs<T> p) {
    using L = SKLayout<T>;
    extern __shared__ __align__(16) unsigned char sk_smem_raw[];
    // dynamic smem is only guaranteed 16-byte aligned: align the carve-up to 1 KB
    unsigned char* sbase = sk_smem_raw + ((1024 - ((unsigned)__cvta_generic_to_shared(sk_smem_raw) & 1023)) & 1023);
    uint64_t* in_full = reinterpret_cast<uint64_t*>(sbase + L::off_bar);  // [NPCR] TMA -> warp
    uint64_t* bfull = in_full + 2 * SK_NPCR;                               // (layout only)
    // sfull[slot]: one phase per system written into the slot.  A reader waits
    // for phase j-1 only after the write of system j-2 completed: that write was
    // in step (j-2) NC + w', >= 2 NC > NPCR + 1 steps back, and its warp has
    // since finished a later step whose state the chain has consumed (NC >= 8).
    uint64_t* sfull = bfull + SK_NPCR;                                     // [NC]
    T* stt = reinterpret_cast<T*>(sbase + L::off_st);
    T* xh = reinterpret_cast<T*>(sbase + L::off_xh);
    T* store = reinterpret_cast<T*>(sbase + L::off_store);
    const int NC = p.NC;

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int i = 0; i < SK_NPCR; ++i) {
            sk_bar_init(&in_full[i], 1);
        }
        for (int i = 0; i < NC; ++i) sk_bar_init(&sfull[i], 32);  // every lane releases its own slot stores
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    __syncthreads();

    const int64_t n = p.n;
    const int nsys = (int)((p.m - blockIdx.x + gridDim.x - 1) / gridDim.x);
    const int nfwd = nsys * NC;             // forward steps
    const int total = p.dA ? nfwd : (nsys + 1) * NC;  // + the back substitution of the last system
    const int nspill = NC - p.S_on;
    T* spill_cta = p.spill + (int64_t)blockIdx.x * (int64_t)(nspill > 0 ? nspill : 0) * SK_SLOT;
    constexpr bool prof = PROF;
    const int c = lane & (SK_S - 1), sg = lane >> 3;  // (chain, segment) of the Thomas phases
    const int nvs = sg == 3 ? SK_P - 3 * SK_SEG : SK_SEG;  // valid positions of this lane's segment

    const int pw = warp;
    T* ib = reinterpret_cast<T*>(sbase + L::off_in + pw * L::in_stride);
    T* tr = reinterpret_cast<T*>(sbase + L::off_tr) + pw * L::tr_elems;
    constexpr int EPC = 16 / (int)sizeof(T);   // elements per 16-byte chunk
    constexpr int CPL = SK_R / EPC;            // chunks per lane-row
    const int swz = sizeof(T) == 8 ? ((lane >> 1) & 3) : ((lane >> 2) & 1);
    const uint64_t pol_in = sk_policy_evict_first();
    const uint64_t pol_sp = sk_policy_evict_last();
    int j = 0, w = pw;
    while (w >= NC) { w -= NC; ++j; }
    auto issue = [&](int jj, int ww) {
        const int64_t q = blockIdx.x + (int64_t)jj * gridDim.x;
        const int64_t row0 = q * n + (int64_t)ww * SK_V - SK_HALO;  // multiple of 8 (n % 8 == 0)
        const int y = (int)(row0 >> 3);                              // may be -1: TMA zero-fills
        // (the generic-proxy reads of the buffer completed: their values were
        // consumed before this point, as in a consumer-release / producer-acquire pipeline)
        sk_expect(&in_full[pw], (unsigned)(4 * SK_W * sizeof(T)));
        sk_tma2d(ib + 0 * SK_W, &tm.a, 0, y, &in_full[pw], pol_in);
        sk_tma2d(ib + 1 * SK_W, &tm.b, 0, y, &in_full[pw], pol_in);
        sk_tma2d(ib + 2 * SK_W, &tm.c, 0, y, &in_full[pw], pol_in);
        sk_tma2d(ib + 3 * SK_W, &tm.d, 0, y, &in_full[pw], pol_in);
    };
    if (lane == 0 && pw < nfwd) issue(j, w);
    unsigned ph = 0;
    unsigned long long t_in = 0, t_st = 0, t_bx = 0, t_sf = 0, t0 = prof ? clock64() : 0;
    unsigned long long ph_t[7] = {0, 0, 0, 0, 0, 0, 0}, tq = 0;
#define SK_PH(k) do { if (prof) { const unsigned long long tn_ = clock64(); ph_t[k] += tn_ - tq; tq = tn_; } } while (0)
    // slot of step gg (read by its backward part, then written by its forward part)
    auto slot_of = [&](int jj, int ww) { return (jj & 1) ? NC - 1 - ww : ww; };
    auto seg_ptr = [&](int sl, bool& res) -> T* {
        int idx;
        res = sk_resident(sl, NC, p.S_on, idx);
        return (res ? store : spill_cta) + (size_t)idx * SK_SLOT + (c * SK_SCS + sg * SK_SEG) * 2;
    };
    // spilled slot of the warp's next step, prefetched into its (then idle)
    // transpose buffer by cp.async; `pref` says whether that happened
    bool pref = false;
    auto prefetch = [&](int jj, int ww) {  // step (jj, ww): backward reads slot_of(jj, ww) of system jj - 1
        pref = false;
        if (jj < 1 || jj > nsys) return;
        const int sl = slot_of(jj, ww);
        int idx;
        if (sk_resident(sl, NC, p.S_on, idx)) return;
        if (!sk_test<T>(&sfull[sl], (unsigned)((jj - 1) & 1))) return;  // not written yet: load at use
        const T* src = spill_cta + (size_t)idx * SK_SLOT;
        constexpr int E16 = 16 / (int)sizeof(T);
        for (int ci = lane; ci < SK_SLOT / E16; ci += 32) cp_async_16(tr + ci * E16, src + ci * E16, 16);
        cp_async_commit();
        pref = true;
    };
    if (pw < total) prefetch(j, w);
    const int pi = (pw + SK_NPCR - 1) % SK_NPCR;  // warp of step g - 1
    int it = 0;                                   // this warp's step count
    for (int g = pw; g < total; g += SK_NPCR, ++it) {
        if (prof) tq = clock64();
        const int cj = j, cw = w;
        w += SK_NPCR;
        while (w >= NC) { w -= NC; ++j; }
        const bool fwd = cj < nsys, bwd = cj >= 1 && !p.dA;
        const int wb = NC - 1 - cw;     // backward window (system cj - 1)
        const int slot = slot_of(cj, cw);
        bool res;
        T* sp = seg_ptr(slot, res);
        // The forward and the backward work of a step are computed unconditionally
        // (on identity data when a part is inactive: the first and the last NC
        // steps) so that the compiler can interleave their dependency chains;
        // only waits and stores are conditional.

        // ---- forward: stage, normalise (X17), K PCR levels (Eqs 5-6; X3/X4)
        NRow<T> v[SK_R];
        if (fwd) {
            const unsigned long long ta = prof ? clock64() : 0;
            sk_wait(&in_full[pw], ph);
            if (prof) t_in += clock64() - ta;
            ph ^= 1u;
            const int64_t ws = (int64_t)cw * SK_V - SK_HALO;
            const bool interior = cw > 0 && ws + SK_W <= n;
            const int64_t i0 = ws + lane * SK_R;
            const T* st = ib + lane * SK_R;
#pragma unroll
            for (int cc = 0; cc < CPL; ++cc) {  // EPC rows at a time: load and normalise
                T raw[4][EPC];
#pragma unroll
                for (int arr = 0; arr < 4; ++arr) {
                    const int4 v4 = *reinterpret_cast<const int4*>(st + arr * SK_W + (cc ^ swz) * EPC);
                    const T* vt = reinterpret_cast<const T*>(&v4);
#pragma unroll
                    for (int e = 0; e < EPC; ++e) raw[arr][e] = vt[e];
                }
#pragma unroll
                for (int e = 0; e < EPC; ++e) {
                    const int u = cc * EPC + e;
                    if (interior) {
                        v[u] = normalise(raw[0][e], raw[1][e], raw[2][e], raw[3][e]);
                    } else {  // rows outside [0, n): identity (X4); a_0, c_{n-1} outside A (X1)
                        const int64_t i = i0 + u;
                        const T av = i == 0 ? T(0) : raw[0][e];
                        const T cv = i == n - 1 ? T(0) : raw[2][e];
                        v[u] = (i >= 0 && i < n) ? normalise(av, raw[1][e], cv, raw[3][e]) : identity_row<T>();
                    }
                }
            }
            sc_release_buf();  // this warp's reads of the buffer before the TMA refill
            if (lane == 0 && g + SK_NPCR < nfwd) issue(j, w);
        } else {
#pragma unroll
            for (int u = 0; u < SK_R; ++u) v[u] = identity_row<T>();
        }
        SK_PH(1);
        if (p.dbg != 1) {
#pragma unroll
            for (int lv = 0; lv < SK_K; ++lv) {
                const int sgm = 1 << lv;
                NRow<T> nv[SK_R];
#pragma unroll
                for (int u = 0; u < SK_R; ++u) {
                    NRow<T> mm, pp;
                    if (u - sgm >= 0) {
                        mm = v[u - sgm];
                    } else {
                        const NRow<T>& s = v[u - sgm + SK_R];
                        mm.A = __shfl_up_sync(0xffffffffu, s.A, 1);
                        mm.C = __shfl_up_sync(0xffffffffu, s.C, 1);
                        mm.D = __shfl_up_sync(0xffffffffu, s.D, 1);
                    }
                    if (u + sgm < SK_R) {
                        pp = v[u + sgm];
                    } else {
                        const NRow<T>& s = v[u + sgm - SK_R];
                        pp.A = __shfl_down_sync(0xffffffffu, s.A, 1);
                        pp.C = __shfl_down_sync(0xffffffffu, s.C, 1);
                        pp.D = __shfl_down_sync(0xffffffffu, s.D, 1);
                    }
                    nv[u] = pcr_combine(mm, v[u], pp);
                }
#pragma unroll
                for (int u = 0; u < SK_R; ++u) v[u] = nv[u];
            }
        }
        SK_PH(2);
        if (p.dA) {  // tri_debug_pcr: the reduced rows, normalised (X17)
            const int64_t q = blockIdx.x + (int64_t)cj * gridDim.x;
            if (lane >= 1 && lane <= SK_P) {
#pragma unroll
                for (int u = 0; u < SK_R; ++u) {
                    const int64_t row = (int64_t)cw * SK_V + (lane - 1) * SK_R + u;
                    if (row < n) {
                        p.dA[q * n + row] = v[u].A;
                        p.dC[q * n + row] = v[u].C;
                        p.dD[q * n + row] = v[u].D;
                    }
                }
            }
            continue;
        }

        // ---- backward: the (c', d') pairs of window (cj - 1, wb), segment sg
        T cpb[SK_SEG], dpb[SK_SEG];
        if (bwd) {
            if (!res && pref) {  // prefetched into the transpose buffer by the previous step
                cp_async_wait<0>();
                __syncwarp();
                const T* pb = tr + (c * SK_SCS + sg * SK_SEG) * 2;
#pragma unroll
                for (int t = 0; t < SK_SEG; ++t) fu_ld2(pb + 2 * t, cpb[t], dpb[t]);
                __syncwarp();
            } else {
                const unsigned long long tb = prof ? clock64() : 0;
                sk_wait(&sfull[slot], (unsigned)((cj - 1) & 1));  // system cj - 1 stored in the slot
                if (prof) t_sf += clock64() - tb;
                if (res) {
#pragma unroll
                    for (int t = 0; t < SK_SEG; ++t) fu_ld2(sp + 2 * t, cpb[t], dpb[t]);
                } else {
#pragma unroll
                    for (int t = 0; t < SK_SEG; ++t) sk_ldg2(sp + 2 * t, cpb[t], dpb[t]);
                }
            }
#pragma unroll
            for (int t = 0; t < SK_SEG; ++t)
                if (t >= nvs) { cpb[t] = T(-1); dpb[t] = T(0); }  // padding: x_t = x_{t+1}
        } else {
#pragma unroll
            for (int t = 0; t < SK_SEG; ++t) { cpb[t] = T(-1); dpb[t] = T(0); }
        }
        SK_PH(3);

        // ---- forward: transpose so that lane (c, sg) holds positions 8 sg .. 8 sg + 7 of chain c
        if (lane >= 1 && lane <= SK_P) {
#pragma unroll
            for (int u = 0; u < SK_R; ++u) {
                tr[u * SK_TCS + lane - 1] = v[u].A;
                tr[SK_S * SK_TCS + u * SK_TCS + lane - 1] = v[u].C;
                tr[2 * SK_S * SK_TCS + u * SK_TCS + lane - 1] = v[u].D;
            }
        }
        __syncwarp();
        T A[SK_SEG], C[SK_SEG], D[SK_SEG];
        {
            const T* tA = tr + c * SK_TCS + sg * SK_SEG;
#pragma unroll
            for (int t = 0; t < SK_SEG; t += 2) {
                fu_ld2(tA + t, A[t], A[t + 1]);
                fu_ld2(tA + SK_S * SK_TCS + t, C[t], C[t + 1]);
                fu_ld2(tA + 2 * SK_S * SK_TCS + t, D[t], D[t + 1]);
            }
        }
        __syncwarp();  // the transpose buffer is free: prefetch the next step's spilled slot
        prefetch(j, w);
        SK_PH(4);

        // ---- both sweeps' segment maps (independent chains, one loop)
        SKMat<T> M;
        T al = T(0), be = T(1);  // backward: x_start = al + be * x_after
        {
            T t1 = T(1), p1 = T(0), d1 = T(0);  // forward response to theta_in
            T t2 = T(0), p2 = T(1), d2 = T(0);  // ... to psi_in
            T d3 = T(1);                        // ... to delta_in
#pragma unroll
            for (int t = 0; t < SK_SEG; ++t) {
                if (t < nvs) {
                    const T nt1 = fma(-A[t], p1, t1), np1 = C[t] * t1, nd1 = fma(-A[t], d1, D[t] * t1);
                    const T nt2 = fma(-A[t], p2, t2), np2 = C[t] * t2, nd2 = fma(-A[t], d2, D[t] * t2);
                    d3 = -A[t] * d3;
                    t1 = nt1; p1 = np1; d1 = nd1;
                    t2 = nt2; p2 = np2; d2 = nd2;
                }
                const int tb = SK_SEG - 1 - t;  // backward runs the positions in reverse
                al = fma(-cpb[tb], al, dpb[tb]);
                be = -cpb[tb] * be;
            }
            M = SKMat<T>{t1, t2, p1, p2, d1, d2, d3};
        }
        {  // scans over the four segments of a chain: forward inclusive (lanes c + 8 sg
           // ascending), backward suffix (descending)
            SKMat<T> o = sk_shfl_up(M, 8);
            T oa = __shfl_down_sync(0xffffffffu, al, 8), ob = __shfl_down_sync(0xffffffffu, be, 8);
            if (sg >= 1) M = sk_compose(M, o);
            if (sg <= 2) { al = fma(be, oa, al); be = be * ob; }
            o = sk_shfl_up(M, 16);
            oa = __shfl_down_sync(0xffffffffu, al, 16);
            ob = __shfl_down_sync(0xffffffffu, be, 16);
            if (sg >= 2) M = sk_compose(M, o);
            if (sg <= 1) { al = fma(be, oa, al); be = be * ob; }
        }
        SK_PH(5);

        // ---- the two serial steps: x (backward) and the state (forward) of step g - 1,
        // handed over through the hardware named barrier 1 + pi (warp pi -> warp pw,
        // 64 threads): a waiting warp is descheduled, nothing polls.  Warp pw arrives
        // on barrier 1 + pw again only after the successor's sync for this step
        // (its next arrival depends, through the chain, on the successor's step g + 1).
        if (g > 0) {
            const unsigned long long tb = prof ? clock64() : 0;
            asm volatile("bar.sync %0, 64;" ::"r"(1 + pi) : "memory");
            if (prof) t_st += clock64() - tb;
        }
        const T xw = (bwd && wb < NC - 1) ? xh[pi * SK_S + c] : T(0);  // x at position 0 of window wb + 1
        T th = T(1), ps = T(0), de = T(0);  // theta_{-1} = 1, psi_0 = C_{-1} theta_{-2} = 0 (a_0 = 0)
        if (fwd && cw > 0) {
            const T* si = stt + pi * 3 * SK_S + c;
            th = si[0];
            ps = si[SK_S];
            de = si[2 * SK_S];
        }
        const T xs = fma(be, xw, al);  // x at the first position of segment sg
        const T ot = fma(M.a, th, M.b * ps);
        const T op = fma(M.c, th, M.d * ps);
        const T od = fma(M.e, th, fma(M.f, ps, M.g * de));
        if (sg == 0) xh[pw * SK_S + c] = xs;
        if (sg == 3) {  // window end: exact power-of-two rescale, hand over
            const T sc = sk_exp2_scale(ot);
            T* so = stt + pw * 3 * SK_S + c;
            so[0] = ot * sc;
            so[SK_S] = op * sc;
            so[2 * SK_S] = od * sc;
        }
        if (g + 1 < total) {
            __threadfence_block();
            asm volatile("bar.arrive %0, 64;" ::"r"(1 + pw) : "memory");
        }
        T x = __shfl_down_sync(0xffffffffu, xs, 8);  // x after segment sg
        if (sg == 3) x = xw;
        {  // incoming state of this lane's segment = outgoing state of segment sg - 1
            const T it_ = __shfl_up_sync(0xffffffffu, ot, 8);
            const T ip = __shfl_up_sync(0xffffffffu, op, 8);
            const T id = __shfl_up_sync(0xffffffffu, od, 8);
            if (sg > 0) { th = it_; ps = ip; de = id; }
        }
        SK_PH(6);

        // ---- both replays: x (Eq 4) of window (cj - 1, wb); c', d' (Eqs 2-3) of (cj, cw)
        const int64_t qb = blockIdx.x + (int64_t)(cj - 1) * gridDim.x;
        const int64_t xr = (int64_t)wb * SK_V + (sg * SK_SEG) * SK_S + c;  // row of position 8 sg
        T* xo = p.x + qb * n + xr;
        const int64_t rmax = bwd ? n - xr : 0;
#pragma unroll
        for (int t = 0; t < SK_SEG; ++t) {
            const int tb = SK_SEG - 1 - t;
            x = fma(-cpb[tb], x, dpb[tb]);
            if (tb < nvs && tb * SK_S < rmax) __stcs(xo + tb * SK_S, x);
            if (t < nvs) {
                const T nt = fma(-A[t], ps, th);
                const T np = C[t] * th;
                const T nd = fma(-A[t], de, D[t] * th);
                const T inv = rcp(nt);
                const T cpv = np * inv, dpv = nd * inv;
                if (fwd) {
                    if (res) fu_st2(sp + 2 * t, cpv, dpv);
                    else sk_st_global_last(sp + 2 * t, cpv, dpv, pol_sp);
                }
                th = nt; ps = np; de = nd;
            }
        }
        __syncwarp();
        if (fwd) sk_arrive(&sfull[slot]);
        SK_PH(0);
    }
    cp_async_wait<0>();
    if (prof && lane == 0) {
        atomicAdd(&p.prof[0], clock64() - t0);
        atomicAdd(&p.prof[1], t_in);
        atomicAdd(&p.prof[2], t_st);
        atomicAdd(&p.prof[3], t_bx);
        atomicAdd(&p.prof[4], t_sf);
        for (int k = 0; k < 7; ++k) atomicAdd(&p.prof[5 + k], ph_t[k]);
    }
}

}  // namespace tri
