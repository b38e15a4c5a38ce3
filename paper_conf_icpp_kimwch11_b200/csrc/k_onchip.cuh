// k_onchip.cuh -- TRI_VARIANT_ONCHIP: one CTA owns G whole systems in shared
// memory, runs k PCR steps there, then p-Thomas with one thread per subsystem.
//
// Paper: "When the whole input can fit into shared memory, our method no longer
// manages the buffered sliding window and it reduces to [16][17]" (P:687,
// Fig 11a); several systems per block is Fig 11c.  PCR Eqs 5-6,
// interleaved subsystems after k steps (Fig 6), p-Thomas Eqs 2-4
// (P:91-127).
//
// B200 layout: rows are normalised to unit diagonal on load (X17), so
// smem holds 3 arrays (A, C, D) of G systems x P rows, P = n padded so that the
// 2^k-chain walk of p-Thomas is bank-conflict free.  HBM traffic is the
// compulsory 5 arrays (read a, b, c, d once; write x once).
#pragma once
#include "common.cuh"

namespace tri {

template <typename T>
struct OnchipArgs {
    const T *a, *b, *c, *d;
    T* x;                 // solve output (mode 0)
    T *ao, *co, *do_;     // debug-PCR outputs (mode 1)
    int64_t n, m;
    int layout, k, G, P, mode;
};

template <typename T, int RPT>
__global__ void __launch_bounds__(512) k_onchip(OnchipArgs<T> p) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    T* sA = reinterpret_cast<T*>(smem_raw);
    T* sC = sA + (int64_t)p.G * p.P;
    T* sD = sC + (int64_t)p.G * p.P;

    const int n = (int)p.n;
    const int64_t q0 = (int64_t)blockIdx.x * p.G;
    const int G = (int)imin64(p.G, p.m - q0);
    const int rows = G * n;
    const int tid = threadIdx.x;
    const int nt = blockDim.x;

    // ---- load + normalise (coalesced: contiguous block, or G-wide row segments)
    for (int e = tid; e < rows; e += nt) {
        int g, i;
        int64_t gi;
        if (p.layout == 0) {
            g = e / n; i = e - g * n;
            gi = q0 * p.n + e;
        } else {
            i = e / G; g = e - i * G;
            gi = (int64_t)i * p.m + q0 + g;
        }
        T av = i > 0 ? ldg_stream(p.a + gi) : T(0);       // a_1 outside A (X1)
        T cv = i < n - 1 ? ldg_stream(p.c + gi) : T(0);   // c_n outside A (X1)
        NRow<T> r = normalise(av, ldg_stream(p.b + gi), cv, ldg_stream(p.d + gi));
        int s = g * p.P + i;
        sA[s] = r.A; sC[s] = r.C; sD[s] = r.D;
    }
    __syncthreads();

    // ---- k PCR steps in place (register-staged: read all, sync, write all)
    for (int j = 0; j < p.k; ++j) {
        const int sg = 1 << j;
        NRow<T> nr[RPT];
#pragma unroll
        for (int u = 0; u < RPT; ++u) {
            int e = tid + u * nt;
            if (e < rows) {
                int g = e / n, i = e - (e / n) * n;
                int s = g * p.P + i;
                NRow<T> o{sA[s], sC[s], sD[s]};
                NRow<T> mm = i - sg >= 0 ? NRow<T>{sA[s - sg], sC[s - sg], sD[s - sg]} : identity_row<T>();
                NRow<T> pp = i + sg < n ? NRow<T>{sA[s + sg], sC[s + sg], sD[s + sg]} : identity_row<T>();
                nr[u] = pcr_combine(mm, o, pp);
            }
        }
        __syncthreads();
#pragma unroll
        for (int u = 0; u < RPT; ++u) {
            int e = tid + u * nt;
            if (e < rows) {
                int g = e / n, i = e - (e / n) * n;
                int s = g * p.P + i;
                sA[s] = nr[u].A; sC[s] = nr[u].C; sD[s] = nr[u].D;
            }
        }
        __syncthreads();
    }

    if (p.mode == 1) {  // debug: emit the reduced (normalised) system
        for (int e = tid; e < rows; e += nt) {
            int g, i;
            int64_t gi;
            if (p.layout == 0) { g = e / n; i = e - g * n; gi = q0 * p.n + e; }
            else { i = e / G; g = e - i * G; gi = (int64_t)i * p.m + q0 + g; }
            int s = g * p.P + i;
            p.ao[gi] = sA[s]; p.co[gi] = sC[s]; p.do_[gi] = sD[s];
        }
        return;
    }

    // ---- p-Thomas: one thread per subsystem (g, r), rows r, r+2^k, ...
    const int S = 1 << p.k;
    const int chains = G * S;
    for (int ch = tid; ch < chains; ch += nt) {
        const int g = ch >> p.k, r = ch & (S - 1);
        if (r >= n) continue;
        const int base = g * p.P;
        T cp = T(0), dp = T(0);
        int i = r;
        for (; i < n; i += S) {
            NRow<T> row{sA[base + i], sC[base + i], sD[base + i]};
            thomas_fwd(row, cp, dp);
            sC[base + i] = cp;
            sD[base + i] = dp;
        }
        i -= S;                      // last row of the chain: x = d'
        T xv = sD[base + i];
        for (i -= S; i >= 0; i -= S) {  // Eq 4: x_i = d'_i - c'_i x_{i+1}
            xv = fma(-sC[base + i], xv, sD[base + i]);
            sD[base + i] = xv;
        }
    }
    __syncthreads();

    // ---- store x (same coalesced mapping as the load)
    for (int e = tid; e < rows; e += nt) {
        int g, i;
        int64_t gi;
        if (p.layout == 0) { g = e / n; i = e - g * n; gi = q0 * p.n + e; }
        else { i = e / G; g = e - i * G; gi = (int64_t)i * p.m + q0 + g; }
        __stcs(p.x + gi, sD[g * p.P + i]);
    }
}

}  // namespace tri
