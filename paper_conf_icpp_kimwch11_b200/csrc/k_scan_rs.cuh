// k_scan_rs.cuh -- the SCAN kernel (k_scan.cuh; X21) for the CONTIGUOUS
// layout with ROLE-SPLIT warps: RS_NF forward warps run the forward chain
// (window loads, segment maps, scan, state handover, replay -> c', d' into a
// storage slot) and RS_NB backward warps run the back-substitution chain (slot
// -> affine maps, scan, x handover, replay -> x), each chain through its own
// named barriers.  A backward warp holds no rows and a forward warp no (c', d'),
// so each role needs fewer registers (124 vs 156 at fp64) and a shorter step.
// MEASURED SLOWER than the paired k_scan (c5 shape: 2.06-2.08 ms for 10+4,
// 11+4, 9+5 warps vs 1.86 ms), so it is off by default (TRI_SCAN_RS=1 selects
// it for A/B measurements; tested by the SCAN parity tests under that switch).
//
// Slots: forward step f (window f of the CTA's sequence, system f / NC, window
// f % NC) stores into a slot; backward step b (system b / NC, window NC - 1 -
// b % NC) reads the window stored by forward step f'(b) = (b / NC) NC + NC - 1 -
// b % NC <= b + NC - 1.  Forward step f >= NS = NC + delta reuses the slot read
// by backward step f - NS (published in fre[] after that step's handover); the
// first NS forward steps take fresh slots.  tab[] maps a stored window to its
// slot, with a per-system tag (k_scan.cuh).  Both tables are written after the
// writer's chain handover, so the chains order every overwrite after the read.
#pragma once
#include "k_scan.cuh"

namespace tri {

#ifndef RS_NF_DEF
#define RS_NF_DEF 10
#endif
#ifndef RS_NB_DEF
#define RS_NB_DEF 4
#endif
constexpr int RS_NF = RS_NF_DEF;   // forward warps
constexpr int RS_NB = RS_NB_DEF;   // backward warps
static_assert(RS_NF + RS_NB <= 15, "two chains of named barriers 1 .. NF + NB");
constexpr int RS_THREADS = 32 * (RS_NF + RS_NB);

template <typename T>
struct RSLayout {
    static constexpr int in_stride = (4 * SC_W * (int)sizeof(T) + 1023) / 1024 * 1024;
    static constexpr int off_st = RS_NF * in_stride;                        // [NF][4] forward state
    static constexpr int off_xh = off_st + RS_NF * 4 * (int)sizeof(T);      // [NB] x handover
    static constexpr int off_bar = (off_xh + RS_NB * (int)sizeof(T) + 7) / 8 * 8;  // [NF] in_full
    static constexpr int off_tab = off_bar + RS_NF * 8;                     // [K][NC] tag | slot
    static constexpr int slot_bytes = sc_slot_elems<T>() * (int)sizeof(T);
    // fre[Q], Q = NS + NC = 2 NC + delta: tag(b) << 16 | slot freed by backward step b
    static __host__ __device__ constexpr int off_fre(int NC, int D) { return off_tab + 4 * (3 * NC + D); }
    static __host__ __device__ constexpr int off_store(int NC, int D) {
        return (off_fre(NC, D) + 4 * (2 * NC + D) + 1023) / 1024 * 1024;
    }
    static __host__ __device__ constexpr int smem_bytes(int NC, int D, int S_on) {
        return off_store(NC, D) + S_on * slot_bytes + 1024;
    }
};

__device__ __forceinline__ unsigned rs_wait_tag(const unsigned* e, unsigned tg) {
    const int* ei = reinterpret_cast<const int*>(e);
    unsigned v = (unsigned)sk_ld_acquire(ei);
    while ((v >> 16) != tg) {
        __nanosleep(32);
        v = (unsigned)sk_ld_acquire(ei);
    }
    return v;
}

template <typename T>
__global__ void __launch_bounds__(RS_THREADS, 1) k_scan_rs(const __grid_constant__ StreamMaps tm, ScanArgs<T> p) {
    using L = RSLayout<T>;
    extern __shared__ __align__(16) unsigned char rs_smem_raw[];
    unsigned char* sbase = rs_smem_raw + ((1024 - ((unsigned)__cvta_generic_to_shared(rs_smem_raw) & 1023)) & 1023);
    const int NC = p.NC, D = p.delta;
    uint64_t* in_full = reinterpret_cast<uint64_t*>(sbase + L::off_bar);
    unsigned* tab = reinterpret_cast<unsigned*>(sbase + L::off_tab);
    unsigned* fre = reinterpret_cast<unsigned*>(sbase + L::off_fre(NC, D));
    T* stt = reinterpret_cast<T*>(sbase + L::off_st);
    T* xh = reinterpret_cast<T*>(sbase + L::off_xh);
    const unsigned store_s = (unsigned)__cvta_generic_to_shared(sbase + L::off_store(NC, D));
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int i = 0; i < RS_NF; ++i) sk_bar_init(&in_full[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    for (int i = threadIdx.x; i < 3 * NC + D; i += blockDim.x) tab[i] = 0u;
    for (int i = threadIdx.x; i < 2 * NC + D; i += blockDim.x) fre[i] = 0u;
    __syncthreads();

    const int64_t n = p.n;
    const int nsys = (int)((p.m - blockIdx.x + gridDim.x - 1) / gridDim.x);
    const int nsteps = nsys * NC;            // forward steps = backward steps
    const int NS = NC + D, Q = 2 * NC + D;
    const int K = 3 + (D - 1) / NC;
    const int nspill = NS - p.S_on;
    T* spill_cta = p.spill + (int64_t)blockIdx.x * (int64_t)(nspill > 0 ? nspill : 0) * sc_slot_elems<T>();
    const uint64_t pol_sp = sk_policy_evict_last();

    if (warp < RS_NF) {
        // ======================= forward chain =======================
        const int pw = warp, pi = (pw + RS_NF - 1) % RS_NF;
        T* ib = reinterpret_cast<T*>(sbase + pw * L::in_stride);
        const uint64_t pol_in = sk_policy_evict_first();
        auto issue = [&](int f) {
            const int q = (int)(blockIdx.x + (int64_t)(f / NC) * gridDim.x);
            const int y = (f % NC) * (SC_W / 8);
            sk_expect(&in_full[pw], (unsigned)(4 * SC_W * sizeof(T)));
            sc_tma3d(ib + 0 * SC_W, &tm.a, y, q, &in_full[pw], pol_in);
            sc_tma3d(ib + 1 * SC_W, &tm.b, y, q, &in_full[pw], pol_in);
            sc_tma3d(ib + 2 * SC_W, &tm.c, y, q, &in_full[pw], pol_in);
            sc_tma3d(ib + 3 * SC_W, &tm.d, y, q, &in_full[pw], pol_in);
        };
        if (lane == 0 && pw < nsteps) issue(pw);
        unsigned ph = 0;
        for (int f = pw; f < nsteps; f += RS_NF) {
            const int j = f / NC, w = f - j * NC;
            int slot = f;  // fresh slot
            if (f >= NS) {
                const int b = f - NS;
                slot = (int)(rs_wait_tag(&fre[b % Q], (unsigned)(b % 65535 + 1)) & 0xffffu);
            }
            const int64_t i0 = (int64_t)w * SC_W + lane * SC_R;
            const bool edge = w == 0 || (int64_t)(w + 1) * SC_W > n;
            sk_wait(&in_full[pw], ph);
            ph ^= 1u;
            SKMat<T> M;
            {
                T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
                sc_ld_rows(ib, lane, ra, rb, rc, rd);
                if (edge) sc_fix_rows<T>(i0, n, ra, rb, rc, rd);
                M = sc_fwd_map(ra, rb, rc, rd);
            }
            sc_fwd_scan(M, lane);
            if (f > 0) asm volatile("bar.sync %0, 64;" ::"r"(1 + pi) : "memory");
            T th = T(1), ps = T(0), de = T(0);
            if (w > 0) { th = stt[pi * 4 + 0]; ps = stt[pi * 4 + 1]; de = stt[pi * 4 + 2]; }
            const T ot = fma(M.a, th, M.b * ps);
            const T op = fma(M.c, th, M.d * ps);
            const T od = fma(M.e, th, fma(M.f, ps, M.g * de));
            if (lane == 31) {
                const T sc = sk_exp2_scale(ot);
                stt[pw * 4 + 0] = ot * sc; stt[pw * 4 + 1] = op * sc; stt[pw * 4 + 2] = od * sc;
            }
            if (f + 1 < nsteps) asm volatile("bar.arrive %0, 64;" ::"r"(1 + pw) : "memory");
            {
                const T it_ = __shfl_up_sync(0xffffffffu, ot, 1);
                const T ip = __shfl_up_sync(0xffffffffu, op, 1);
                const T id = __shfl_up_sync(0xffffffffu, od, 1);
                if (lane > 0) { th = it_; ps = ip; de = id; }
            }
            T ra[SC_R], rb[SC_R], rc[SC_R], rd[SC_R];
            sc_ld_rows(ib, lane, ra, rb, rc, rd);
            if (edge) sc_fix_rows<T>(i0, n, ra, rb, rc, rd);
            sc_release_buf();  // this warp's reads of the buffer before the TMA refill
            if (lane == 0 && f + RS_NF < nsteps) issue(f + RS_NF);
            T cpf[SC_R], dpf[SC_R];
            sc_fwd_replay(ra, rb, rc, rd, th, ps, de, cpf, dpf);
            const bool res = slot < p.S_on;
            if (res) sc_store_slot_s(store_s + (unsigned)(slot * L::slot_bytes), lane, cpf, dpf);
            else sc_store_slot_g(spill_cta + (size_t)(slot - p.S_on) * sc_slot_elems<T>(), lane, cpf, dpf, pol_sp);
            __syncwarp();
            if (lane == 0)
                sk_st_release(reinterpret_cast<int*>(&tab[(j % K) * NC + w]),
                              (int)(((unsigned)(j % 65535 + 1) << 16) | (unsigned)slot));
        }
    } else {
        // ======================= backward chain =======================
        const int bw = warp - RS_NF, bpi = (bw + RS_NB - 1) % RS_NB;
        for (int b = bw; b < nsteps; b += RS_NB) {
            const int bj = b / NC, wb = NC - 1 - (b - bj * NC);
            const unsigned v = rs_wait_tag(&tab[(bj % K) * NC + wb], (unsigned)(bj % 65535 + 1));
            const int slot = (int)(v & 0xffffu);
            T cpb[SC_R], dpb[SC_R];
            if (slot < p.S_on) sc_load_slot_s(store_s + (unsigned)(slot * L::slot_bytes), lane, cpb, dpb);
            else sc_load_slot_g(spill_cta + (size_t)(slot - p.S_on) * sc_slot_elems<T>(), lane, cpb, dpb);
            T al, be;
            sc_bwd_map(cpb, dpb, al, be);
            sc_bwd_scan(al, be, lane);
            if (b > 0) asm volatile("bar.sync %0, 64;" ::"r"(1 + RS_NF + bpi) : "memory");
            const T xw = wb < NC - 1 ? xh[bpi] : T(0);  // x at the first row of window wb + 1
            const T xs = fma(be, xw, al);
            if (lane == 0) xh[bw] = xs;
            if (b + 1 < nsteps) asm volatile("bar.arrive %0, 64;" ::"r"(1 + RS_NF + bw) : "memory");
            // the slot's values are in registers (consumed by the map): free it
            __syncwarp();
            if (lane == 0)
                sk_st_release(reinterpret_cast<int*>(&fre[b % Q]),
                              (int)(((unsigned)(b % 65535 + 1) << 16) | (unsigned)slot));
            T x = __shfl_down_sync(0xffffffffu, xs, 1);
            if (lane == 31) x = xw;
            T xv[SC_R];
#pragma unroll
            for (int t = SC_R - 1; t >= 0; --t) {
                x = fma(-cpb[t], x, dpb[t]);
                xv[t] = x;
            }
            const int64_t qb = blockIdx.x + (int64_t)bj * gridDim.x;
            const int64_t xr = (int64_t)wb * SC_W + lane * SC_R;
            sc_store_x(p.x + qb * n + xr, n - xr, xv);
        }
    }
}

}  // namespace tri
