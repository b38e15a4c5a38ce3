// l_split.cu -- TRI_VARIANT_SPLIT: the paper's two-stage method as separate
// kernels (Sec. III): tiled-PCR passes (Sec. III.A, sliding window,
// Figs 8-10, region split with f(k) halos, Fig 11b / Eq 8) writing the reduced
// system chain-interleaved (the interleave transform fused into the last store,
// P:647), then p-Thomas with one thread per subsystem (Sec. III.B).
//
// Any 0 <= k <= floor(log2 n).  Pass 1 works on the user layout,
// every further pass on the chain-interleaved batch the previous pass wrote
// (strides 2^K.. of the original system are strides 1.. of each chain),
// ping-ponging between two scratch buffers; the last pass writes the p-Thomas
// input.  Two kernel families (PassKind):
//   register tiles (k_pcr_reg.cuh, TMA-fed, the default): pass 1 up to 5 steps
//     on CONTIGUOUS rows (3 on the user's INTERLEAVED rows), later passes up to 3
//     steps each, the remaining steps balanced over the fewest passes;
//   the paper's shared-memory sliding window (k_tiled_pcr.cuh): pass 1 up to 10
//     steps, later passes up to 5 -- with TRI_OPT_TMA off, the BATCHED layout,
//     and shapes the TMA maps cannot describe.
#include <algorithm>

#include "plan.cuh"
#include "common.cuh"
#include "k_tiled_pcr.cuh"
#include "k_pcr_reg.cuh"
#include "k_pthomas.cuh"
#include "k_pthomas_tma.cuh"

using namespace tri;

namespace trih {
namespace {

constexpr int SPLIT_K1MAX = 10;   // deepest k one sliding-window pass on the user layout holds in smem (T = 256)
constexpr int SPLIT_KNMAX = 5;    // steps of a later (interleaved-batch) pass
constexpr int TILED_WAVES1 = 1;   // regions per SM slot, pass 1
constexpr int TILED_WAVES2 = 3;   // regions per SM slot, later passes (measured best at c3: 1 vs 3)

template <typename T, int K>
int tiled_occ_k() {
    const int smem = 3 * TPCRRing<K>::total() * (int)sizeof(T);
    if (set_smem((const void*)k_tiled_pcr<T, K>, smem) != cudaSuccess) { cudaGetLastError(); return 1; }
    int occ = 1;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_tiled_pcr<T, K>, TPCR_T, smem) != cudaSuccess) {
        cudaGetLastError();
        occ = 1;
    }
    return std::max(1, occ);
}
template <typename T>
int tiled_occ(int k1) {
    switch (k1) {
        case 1: return tiled_occ_k<T, 1>();
        case 2: return tiled_occ_k<T, 2>();
        case 3: return tiled_occ_k<T, 3>();
        case 4: return tiled_occ_k<T, 4>();
        case 5: return tiled_occ_k<T, 5>();
        case 6: return tiled_occ_k<T, 6>();
        case 7: return tiled_occ_k<T, 7>();
        case 8: return tiled_occ_k<T, 8>();
        case 9: return tiled_occ_k<T, 9>();
        default: return tiled_occ_k<T, 10>();
    }
}
template <typename T, int K2>
int tiled_il_occ_k() {
    const int smem = 3 * TPCRILRing<K2>::total() * TPCR_IL_CB * (int)sizeof(T);
    if (set_smem((const void*)k_tiled_pcr_il<T, K2>, smem) != cudaSuccess) { cudaGetLastError(); return 1; }
    int occ = 1;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_tiled_pcr_il<T, K2>, TPCR_T, smem) != cudaSuccess) {
        cudaGetLastError();
        occ = 1;
    }
    return std::max(1, occ);
}
template <typename T>
int tiled_il_occ(int k2) {
    switch (k2) {
        case 1: return tiled_il_occ_k<T, 1>();
        case 2: return tiled_il_occ_k<T, 2>();
        case 3: return tiled_il_occ_k<T, 3>();
        case 4: return tiled_il_occ_k<T, 4>();
        default: return tiled_il_occ_k<T, 5>();
    }
}

// cumulative PCR steps after pass i
int ksum(const tri_plan_s* p, int i) {
    int s = 0;
    for (int j = 0; j <= i; ++j) s += p->kp[j];
    return s;
}

// elements of the largest intermediate (not last) pass output, per array
int64_t inter_elems(const tri_plan_s* p) {
    int64_t e = 0;
    for (int i = 0; i + 1 < p->npass; ++i) e = std::max<int64_t>(e, p->Cp[i] * p->Lp[i]);
    return e;
}

// ---- launches -----------------------------------------------------------------
template <typename T, int K>
cudaError_t launch_tiled_k(const TiledArgs<T>& A, int64_t grid, cudaStream_t st) {
    const int smem = 3 * TPCRRing<K>::total() * (int)sizeof(T);
    cudaError_t e = set_smem((const void*)k_tiled_pcr<T, K>, smem);
    if (e != cudaSuccess) return e;
    k_tiled_pcr<T, K><<<(unsigned)grid, TPCR_T, smem, st>>>(A);
    return cudaGetLastError();
}

// pass 0: user layout -> chain-interleaved (mode 0) or the user layout (mode 1)
template <typename T>
cudaError_t launch_pass0(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* oA,
                         void* oC, void* oD, int mode, cudaStream_t st) {
    TiledArgs<T> A;
    A.a = (const T*)a; A.b = (const T*)b; A.c = (const T*)c; A.d = (const T*)d;
    A.oA = (T*)oA; A.oC = (T*)oC; A.oD = (T*)oD;
    const int k1 = p->kp[0];
    A.n = p->n; A.m = p->m; A.n_pad = p->Lp[0] << k1; A.region = p->region[0]; A.nreg = p->nreg[0];
    A.C = p->Cp[0];
    A.layout = p->layout; A.k = k1; A.mode = mode;
    const int64_t grid = p->m * p->nreg[0];
    switch (k1) {
        case 1: return launch_tiled_k<T, 1>(A, grid, st);
        case 2: return launch_tiled_k<T, 2>(A, grid, st);
        case 3: return launch_tiled_k<T, 3>(A, grid, st);
        case 4: return launch_tiled_k<T, 4>(A, grid, st);
        case 5: return launch_tiled_k<T, 5>(A, grid, st);
        case 6: return launch_tiled_k<T, 6>(A, grid, st);
        case 7: return launch_tiled_k<T, 7>(A, grid, st);
        case 8: return launch_tiled_k<T, 8>(A, grid, st);
        case 9: return launch_tiled_k<T, 9>(A, grid, st);
        case 10: return launch_tiled_k<T, 10>(A, grid, st);
        default: return cudaErrorInvalidValue;
    }
}

template <typename T, int K2>
cudaError_t launch_tiled_il_k(const TiledILArgs<T>& A, int64_t grid, cudaStream_t st) {
    const int smem = 3 * TPCRILRing<K2>::total() * TPCR_IL_CB * (int)sizeof(T);
    cudaError_t e = set_smem((const void*)k_tiled_pcr_il<T, K2>, smem);
    if (e != cudaSuccess) return e;
    k_tiled_pcr_il<T, K2><<<(unsigned)grid, TPCR_T, smem, st>>>(A);
    return cudaGetLastError();
}

// pass i >= 1: chain-interleaved batch of pass i-1 -> pass i's chains
template <typename T>
cudaError_t launch_pass(const tri_plan_s* p, int i, const void* iA, const void* iC, const void* iD, void* oA,
                        void* oC, void* oD, int mode, cudaStream_t st) {
    TiledILArgs<T> A;
    A.iA = (const T*)iA; A.iC = (const T*)iC; A.iD = (const T*)iD;
    A.oA = (T*)oA; A.oC = (T*)oC; A.oD = (T*)oD;
    A.n = p->n; A.m = p->m; A.L1 = p->Lp[i - 1]; A.C1 = p->Cp[i - 1]; A.C = p->Cp[i];
    A.region = p->region[i]; A.nreg = p->nreg[i]; A.nblk = p->nblk[i];
    A.layout = p->layout; A.k1 = ksum(p, i - 1); A.mode = mode;
    const int64_t grid = p->nblk[i] * p->nreg[i];
    switch (p->kp[i]) {
        case 1: return launch_tiled_il_k<T, 1>(A, grid, st);
        case 2: return launch_tiled_il_k<T, 2>(A, grid, st);
        case 3: return launch_tiled_il_k<T, 3>(A, grid, st);
        case 4: return launch_tiled_il_k<T, 4>(A, grid, st);
        case 5: return launch_tiled_il_k<T, 5>(A, grid, st);
        default: return cudaErrorInvalidValue;
    }
}

// ---- register-tile passes (k_pcr_reg.cuh) --------------------------------------
#ifndef PR_RPL
#define PR_RPL 8   // rows per lane of k_pcr_rows (A/B builds: -DPR_RPL=16)
#endif
#ifndef PR_PF
#define PR_PF 1    // k_pcr_rows register prefetch of the next tile
#endif

template <typename T, int K>
cudaError_t launch_rows_k(const PRArgs<T>& A, int sms, cudaStream_t st) {
    auto kern = k_pcr_rows<T, K, PR_RPL, PR_PF != 0>;
    int occ = 1;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, 32 * PR_WARPS, 0) != cudaSuccess) {
        cudaGetLastError();
        occ = 1;
    }
    const int64_t grid = std::max<int64_t>(1, std::min<int64_t>(cdiv(A.ntask, PR_WARPS), (int64_t)std::max(1, occ) * sms));
    kern<<<(unsigned)grid, 32 * PR_WARPS, 0, st>>>(A);
    return cudaGetLastError();
}

// pass 0 on CONTIGUOUS rows
template <typename T>
cudaError_t launch_rows(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* oA, void* oC,
                        void* oD, int mode, cudaStream_t st) {
    const int K = p->kp[0];
    PRArgs<T> A;
    A.a = (const T*)a; A.b = (const T*)b; A.c = (const T*)c; A.d = (const T*)d;
    A.oA = (T*)oA; A.oC = (T*)oC; A.oD = (T*)oD;
    A.n = p->n; A.m = p->m; A.n_pad = p->Lp[0] << K;
    A.ntile = p->region[0]; A.ntask = p->m * p->region[0];
    A.C = p->Cp[0]; A.mode = mode;
    A.vec = (((uintptr_t)a | (uintptr_t)b | (uintptr_t)c | (uintptr_t)d) & 31) == 0;
    switch (K) {
        case 1: return launch_rows_k<T, 1>(A, p->sms, st);
        case 2: return launch_rows_k<T, 2>(A, p->sms, st);
        case 3: return launch_rows_k<T, 3>(A, p->sms, st);
        case 4: return launch_rows_k<T, 4>(A, p->sms, st);
        case 5: return launch_rows_k<T, 5>(A, p->sms, st);
        default: return cudaErrorInvalidValue;
    }
}

template <typename T, bool RAW>
int chains_ctas(const tri_plan_s* p) {
    const int occ = std::max(1, (227 * 1024) / PCCfg<T, RAW>::smem_bytes());
    return occ * p->sms;
}

template <typename T, int K, bool RAW>
cudaError_t launch_chains_k(const PCMaps& tm, const PCArgs<T>& A, bool tma, int grid, cudaStream_t st) {
    constexpr int smem = PCCfg<T, RAW>::smem_bytes();
    auto kern = tma ? k_pcr_chains<T, K, RAW, true> : k_pcr_chains<T, K, RAW, false>;
    cudaError_t e = set_smem((const void*)kern, smem);
    if (e != cudaSuccess) return e;
    kern<<<grid, 32 * PCCfg<T, RAW>::WARPS, smem, st>>>(tm, A);
    return cudaGetLastError();
}

// pass i on a chain-interleaved batch (the previous pass's output, or -- RAW, pass
// 0 -- the user's INTERLEAVED arrays a, b, c, d)
template <typename T, bool RAW>
cudaError_t launch_chains(tri_plan_s* p, int i, const void* in0, const void* in1, const void* in2, const void* in3,
                          void* oA, void* oC, void* oD, int mode, cudaStream_t st) {
    const int K = p->kp[i];
    const int64_t C1 = i == 0 ? p->m : p->Cp[i - 1], L1 = i == 0 ? p->n : p->Lp[i - 1];
    PCMaps tm;
    const void* key[4] = {in0, in1, in2, in3};
    const int nk = RAW ? 4 : 3;
    const int tag = 0x7200 + 16 * i + (int)sizeof(T);
    // TMA needs a 16-byte row pitch and 16-byte aligned bases; cp.async otherwise
    bool tma = (C1 * (int64_t)sizeof(T)) % 16 == 0 && C1 < INT32_MAX && L1 + 4 * PC_PO + 64 < INT32_MAX;
    for (int j = 0; j < nk; ++j) tma = tma && ((uintptr_t)key[j] % 16) == 0;
    if (tma && !tm_lookup(p, tag, key, nk, &tm.a, nk)) {
        const uint64_t dims[2] = {(uint64_t)C1, (uint64_t)L1}, str[1] = {(uint64_t)C1 * sizeof(T)};
        const uint32_t box[2] = {32u, (uint32_t)PC_PO};
        CUtensorMap* dst[4] = {&tm.a, &tm.c, &tm.d, &tm.b};
        for (int j = 0; j < nk && tma; ++j)
            tma = tma_encode(dst[j], sizeof(T), 2, key[j], dims, str, box, CU_TENSOR_MAP_SWIZZLE_NONE);
        if (tma) tm_store(p, tag, key, nk, &tm.a, nk);
    }
    PCArgs<T> A;
    for (int j = 0; j < 4; ++j) A.in[j] = (const T*)key[j];
    A.oA = (T*)oA; A.oC = (T*)oC; A.oD = (T*)oD;
    A.n = p->n; A.m = p->m; A.L1 = L1; A.C1 = C1; A.C = p->Cp[i];
    A.Lout = p->Lp[i] << K;
    A.ntile_reg = p->region[i]; A.nreg = p->nreg[i]; A.nblk = p->nblk[i]; A.ntask = p->nreg[i] * p->nblk[i];
    A.k1 = i == 0 ? 0 : ksum(p, i - 1); A.mode = mode; A.layout = p->layout;
    const int grid = (int)std::max<int64_t>(
        1, std::min<int64_t>(cdiv(A.ntask, PCCfg<T, RAW>::WARPS), chains_ctas<T, RAW>(p)));
    switch (K) {
        case 1: return launch_chains_k<T, 1, RAW>(tm, A, tma, grid, st);
        case 2: return launch_chains_k<T, 2, RAW>(tm, A, tma, grid, st);
        case 3: return launch_chains_k<T, 3, RAW>(tm, A, tma, grid, st);
        default: return cudaErrorInvalidValue;
    }
}

// all PCR passes; the last one writes (fA, fC, fD) in `mode` (0: chain-
// interleaved p-Thomas input, 1: the user layout for tri_debug_pcr)
template <typename T>
cudaError_t run_passes(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* fA,
                       void* fC, void* fD, int mode, cudaStream_t st) {
    const size_t ce = (size_t)p->C * (size_t)p->L;
    const size_t ie = (size_t)inter_elems(p);
    T* X = (T*)p->scratch + 5 * ce;  // intermediates: two 3-array buffers
    T* bufs[2] = {X, X + 3 * ie};
    const void* in[3] = {nullptr, nullptr, nullptr};
    for (int i = 0; i < p->npass; ++i) {
        const bool last = i + 1 == p->npass;
        T* o = bufs[i & 1];
        void* oA = last ? fA : (void*)o;
        void* oC = last ? fC : (void*)(o + ie);
        void* oD = last ? fD : (void*)(o + 2 * ie);
        const int md = last ? mode : 0;
        cudaError_t e;
        switch (p->pk[i]) {
            case PK_ROWS: e = launch_rows<T>(p, a, b, c, d, oA, oC, oD, md, st); break;
            case PK_RAW: e = launch_chains<T, true>(p, i, a, c, d, b, oA, oC, oD, md, st); break;
            case PK_CHAINS: e = launch_chains<T, false>(p, i, in[0], in[1], in[2], nullptr, oA, oC, oD, md, st); break;
            case PK_RING: e = launch_pass0<T>(p, a, b, c, d, oA, oC, oD, md, st); break;
            default: e = launch_pass<T>(p, i, in[0], in[1], in[2], oA, oC, oD, md, st); break;
        }
        if (e != cudaSuccess) return e;
        in[0] = oA; in[1] = oC; in[2] = oD;
    }
    return cudaSuccess;
}

// k = 0, CONTIGUOUS: the TMA kernel when both row strides (n and m elements)
// are 16-byte multiples; returns cudaErrorNotSupported to request the fallback.
template <typename T>
cudaError_t launch_contig_tma(tri_plan_s* p, const PThomasArgs<T>& A, cudaStream_t st) {
    constexpr int R = PTTCfg<T>::R;
    if ((p->n * (int64_t)sizeof(T)) % 16 || (p->m * (int64_t)sizeof(T)) % 16) return cudaErrorNotSupported;
    if (p->n > INT32_MAX || p->m > INT32_MAX) return cudaErrorNotSupported;
    PTTMaps tm;
    const void* key[7] = {A.a, A.b, A.c, A.d, A.x, A.cps, A.dps};
    if (!tm_lookup(p, 0x5000 + (int)sizeof(T), key, 7, &tm.a, 7)) {
        const uint64_t n = (uint64_t)p->n, m = (uint64_t)p->m;
        const uint64_t dx[2] = {n, m}, sx[1] = {n * sizeof(T)}, dc[2] = {m, n}, sc[1] = {m * sizeof(T)};
        const uint32_t bx[2] = {(uint32_t)R, (uint32_t)PTT_CH}, bc[2] = {(uint32_t)PTT_CH, (uint32_t)R};
        const void* rows[5] = {A.a, A.b, A.c, A.d, A.x};
        CUtensorMap* dst[5] = {&tm.a, &tm.b, &tm.c, &tm.d, &tm.x};
        bool ok = true;
        for (int i = 0; i < 5 && ok; ++i) ok = tma_encode(dst[i], sizeof(T), 2, rows[i], dx, sx, bx, CU_TENSOR_MAP_SWIZZLE_128B);
        ok = ok && tma_encode(&tm.cp, sizeof(T), 2, A.cps, dc, sc, bc, CU_TENSOR_MAP_SWIZZLE_NONE) &&
             tma_encode(&tm.dp, sizeof(T), 2, A.dps, dc, sc, bc, CU_TENSOR_MAP_SWIZZLE_NONE);
        if (!ok) return cudaErrorNotSupported;
        tm_store(p, 0x5000 + (int)sizeof(T), key, 7, &tm.a, 7);
    }
    constexpr int smem = ptt_smem_bytes<T>();
    cudaError_t e = set_smem((const void*)k_pthomas_tma<T>, smem);
    if (e != cudaSuccess) return e;
    k_pthomas_tma<T><<<(unsigned)cdiv(p->m, PTT_CH), PTT_CH, smem, st>>>(tm, A);
    return cudaGetLastError();
}

template <typename T, int CH>
cudaError_t launch_contig(const tri_plan_s* p, const PThomasArgs<T>& A, bool vec, cudaStream_t st) {
    constexpr int smem = pt2_smem_bytes<T, CH>();
    auto kern = vec ? k_pthomas_contig<T, CH, true> : k_pthomas_contig<T, CH, false>;
    cudaError_t e = set_smem((const void*)kern, smem);
    if (e != cudaSuccess) return e;
    kern<<<(unsigned)cdiv(p->m, CH), CH, smem, st>>>(A);
    return cudaGetLastError();
}

// p-Thomas over chain-interleaved input (MODE 0 scratch, MODE 1 user
// INTERLEAVED).  Few chains (< 8 warps' worth per SM): the ring-staged kernel
// with CW chains per CTA, CW the largest of 32/16/8 that still gives every SM
// a CTA; many chains: one thread per chain with a register prefetch window.
template <typename T, int CW, int MODE>
cudaError_t launch_ring(const tri_plan_s* p, const PThomasArgs<T>& A, bool vec, cudaStream_t st) {
    const int smem = ptr_smem_bytes<T, CW>(MODE == 1);
    auto kern = vec ? k_pthomas_ring<T, CW, MODE, true> : k_pthomas_ring<T, CW, MODE, false>;
    cudaError_t e = set_smem((const void*)kern, smem);
    if (e != cudaSuccess) return e;
    kern<<<(unsigned)cdiv(p->C, CW), CW, smem, st>>>(A);
    return cudaGetLastError();
}

// chain-interleaved p-Thomas through TMA (C >= 32 x SMs); cudaErrorNotSupported
// asks for the fallback kernels
template <typename T, int MODE>
cudaError_t launch_pthomas_il_tma(tri_plan_s* p, const PThomasArgs<T>& A, cudaStream_t st) {
    constexpr int R = PTICfg<T>::R;
    const int64_t C = p->C, L = p->L;
    if ((C * (int64_t)sizeof(T)) % 16 || C > INT32_MAX || L > INT32_MAX) return cudaErrorNotSupported;
    PTIMaps tm;
    const void* in[4] = {MODE == 1 ? (const void*)A.a : (const void*)A.iA, MODE == 1 ? (const void*)A.b : (const void*)A.iC,
                         MODE == 1 ? (const void*)A.c : (const void*)A.iD, MODE == 1 ? (const void*)A.d : (const void*)A.iD};
    // x as a [L][C] view: INTERLEAVED user layout (MODE 1), or one system whose
    // rows pos * 2^k + r are exactly [pos * C + r] (m = 1, n = L * 2^k)
    const bool x_view = MODE == 1 || (p->m == 1 && p->n == L * C);
    const void* key[7] = {in[0], in[1], in[2], in[3], A.cps, A.dps, x_view ? (const void*)A.x : nullptr};
    const int tag = 0x6000 + 16 * MODE + (int)sizeof(T);
    int x_tma = 0;
    if (tm_lookup(p, tag, key, 7, &tm.a, 7)) {
        x_tma = x_view ? 1 : 0;
    } else {
        const uint64_t dims[2] = {(uint64_t)C, (uint64_t)L}, str[1] = {(uint64_t)C * sizeof(T)};
        const uint32_t box[2] = {(uint32_t)PTT_CH, (uint32_t)R};
        bool ok = true;
        for (int i = 0; i < 4 && ok; ++i) ok = tma_encode(&tm.a + i, sizeof(T), 2, in[i], dims, str, box, CU_TENSOR_MAP_SWIZZLE_NONE);
        ok = ok && tma_encode(&tm.cp, sizeof(T), 2, A.cps, dims, str, box, CU_TENSOR_MAP_SWIZZLE_NONE) &&
             tma_encode(&tm.dp, sizeof(T), 2, A.dps, dims, str, box, CU_TENSOR_MAP_SWIZZLE_NONE);
        if (!ok) return cudaErrorNotSupported;
        if (x_view) x_tma = tma_encode(&tm.x, sizeof(T), 2, A.x, dims, str, box, CU_TENSOR_MAP_SWIZZLE_NONE) ? 1 : 0;
        if (x_tma == (x_view ? 1 : 0)) tm_store(p, tag, key, 7, &tm.a, 7);
    }
    constexpr int smem = pti_smem_bytes<T, MODE>();
    cudaError_t e = set_smem((const void*)k_pthomas_il_tma<T, MODE>, smem);
    if (e != cudaSuccess) return e;
    k_pthomas_il_tma<T, MODE><<<(unsigned)cdiv(C, PTT_CH), PTT_CH, smem, st>>>(tm, A, x_tma);
    return cudaGetLastError();
}

template <typename T, int MODE>
cudaError_t launch_pthomas_il(tri_plan_s* p, const PThomasArgs<T>& A, cudaStream_t st) {
    const int64_t C = p->C, sms = p->sms;
    if (C >= 32 * sms && p->opt_tma) {
        const cudaError_t et = launch_pthomas_il_tma<T, MODE>(p, A, st);
        if (et != cudaErrorNotSupported) return et;
    }
    if (C >= 32 * 8 * sms) {
        k_pthomas<T, MODE><<<(unsigned)cdiv(C, 128), 128, 0, st>>>(A);
        return cudaGetLastError();
    }
    const T* in0 = MODE == 1 ? A.a : A.iA;
    const bool vec = ((C * (int64_t)sizeof(T)) % 16) == 0 && ((uintptr_t)in0 % 16) == 0;
    if (C >= 32 * sms) return launch_ring<T, 32, MODE>(p, A, vec, st);
    if (C >= 16 * sms) return launch_ring<T, 16, MODE>(p, A, vec, st);
    return launch_ring<T, 8, MODE>(p, A, vec, st);
}

template <typename T>
cudaError_t split_t(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                    cudaStream_t st) {
    const size_t ce = (size_t)p->C * (size_t)p->L;
    T* base = (T*)p->scratch;
    PThomasArgs<T> A;
    A.a = (const T*)a; A.b = (const T*)b; A.c = (const T*)c; A.d = (const T*)d;
    A.x = (T*)x;
    A.n = p->n; A.m = p->m; A.C = p->C; A.L = p->L; A.layout = p->layout; A.k = p->k;
    // 32 chains x s bytes per scratch row segment start on 128-byte lines when
    // the row pitch C s is a multiple of 128 (and the scratch base is 256-aligned)
    A.discard = ((p->C * (int64_t)sizeof(T)) % 128 == 0) ? 1 : 0;
    if (p->k > 0) {
        T *rA = base, *rC = base + ce, *rD = base + 2 * ce;
        cudaError_t e = run_passes<T>(p, a, b, c, d, rA, rC, rD, 0, st);
        if (e != cudaSuccess) return e;
        A.iA = rA; A.iC = rC; A.iD = rD;
        A.cps = base + 3 * ce; A.dps = base + 4 * ce;
        return launch_pthomas_il<T, 0>(p, A, st);
    }
    A.iA = A.iC = A.iD = nullptr;
    A.cps = base; A.dps = base + ce;
    if (p->layout == TRI_LAYOUT_INTERLEAVED) return launch_pthomas_il<T, 1>(p, A, st);
    if (p->opt_tma) {
        const cudaError_t et = launch_contig_tma<T>(p, A, st);
        if (et != cudaErrorNotSupported) return et;
    }
    const bool vec = ((p->n * (int64_t)sizeof(T)) % 16) == 0 && ((uintptr_t)a % 16) == 0;
    // 16 systems per CTA when the batch is thin (finer balance over the SMs)
    const bool thin = cdiv(p->m, 32) < 6 * (int64_t)p->sms;
    return thin ? launch_contig<T, 16>(p, A, vec, st) : launch_contig<T, 32>(p, A, vec, st);
}

}  // namespace

// register-tile passes: can the TMA maps describe pass 1's input / a batch of C1 chains?
bool rows_ok(const tri_plan_s* p) {
    return p->opt_tma && p->layout == TRI_LAYOUT_CONTIGUOUS;
}
bool chains_ok(const tri_plan_s* p) {
    return p->opt_tma && p->layout != TRI_LAYOUT_BATCHED;
}

void split_geometry(tri_plan_s* p) {
    const int64_t n = p->n, m = p->m;
    const int S = 1 << p->k;
    p->L = cdiv(n, S);
    p->n_pad = p->L * S;
    p->C = m * S;
    p->npass = 0;
    for (int i = 0; i < 8; ++i) {
        p->kp[i] = p->pk[i] = 0;
        p->Lp[i] = p->Cp[i] = p->region[i] = p->nreg[i] = p->nblk[i] = 0;
    }
    if (p->k == 0) return;
    const bool f64 = p->dtype == TRI_F64;
    int rem = p->k;
    if (rows_ok(p) || (p->layout == TRI_LAYOUT_INTERLEAVED && chains_ok(p))) {
        // register tiles: pass 1 up to 5 (rows) / 3 (interleaved) steps, then the
        // remaining steps over the fewest passes of <= 3, balanced
        const bool rows = rows_ok(p);
        const int k1 = std::min(rem, rows ? 5 : 3);
        p->kp[0] = k1;
        p->pk[0] = rows ? PK_ROWS : PK_RAW;
        p->npass = 1;
        rem -= k1;
        const int np = (int)cdiv(rem, 3);
        for (int j = 0; j < np; ++j) {
            p->kp[p->npass] = rem / np + (j < rem % np ? 1 : 0);
            p->pk[p->npass] = PK_CHAINS;
            ++p->npass;
        }
    } else {
        // sliding window: pass 1 up to 10 steps; two passes split as (k - 5, 5)
        // beyond that; deeper k adds passes of 5 steps
        int k1 = std::min(rem, SPLIT_K1MAX);
        if (rem > SPLIT_K1MAX && rem <= SPLIT_K1MAX + SPLIT_KNMAX && rem - k1 > SPLIT_KNMAX) k1 = rem - SPLIT_KNMAX;
        p->kp[0] = k1;
        p->pk[0] = PK_RING;
        p->npass = 1;
        rem -= k1;
        while (rem > 0) {
            const int kk = std::min(rem, SPLIT_KNMAX);
            p->pk[p->npass] = PK_IL;
            p->kp[p->npass++] = kk;
            rem -= kk;
        }
    }
    int K = 0;
    for (int i = 0; i < p->npass; ++i) {
        K += p->kp[i];
        p->Lp[i] = cdiv(n, int64_t(1) << K);
        p->Cp[i] = m << K;
        const int64_t C1 = i == 0 ? m : p->Cp[i - 1], L1 = i == 0 ? n : p->Lp[i - 1];
        if (p->pk[i] == PK_ROWS) {
            // tiles of OUT rows cover the L 2^K rows pass 1 writes per system (from
            // up to 3 (fp64) / 7 (fp32) rows before row 0: 32-byte aligned lane rows)
            const int h = ((1 << p->kp[0]) - 1 + PR_RPL - 1) / PR_RPL * PR_RPL;
            p->region[0] = cdiv((p->Lp[0] << p->kp[0]) + 32 / (int64_t)esize(p->dtype) - 1, 32 * PR_RPL - 2 * h);
            p->nreg[0] = 1;
            p->nblk[0] = m;
        } else if (p->pk[i] == PK_CHAINS || p->pk[i] == PK_RAW) {
            // tasks = (32-chain block, region of tiles): about two per resident warp,
            // regions of >= 4 tiles (two halo tiles per region: at most a third of the
            // loads, and only on passes too small to fill the GPU otherwise)
            const int64_t ntile = cdiv(p->Lp[i] << p->kp[i], PC_PO);
            const bool raw = p->pk[i] == PK_RAW;
            const int64_t warps = (int64_t)(raw ? (f64 ? chains_ctas<double, true>(p) * PCCfg<double, true>::WARPS
                                                       : chains_ctas<float, true>(p) * PCCfg<float, true>::WARPS)
                                                : (f64 ? chains_ctas<double, false>(p) * PCCfg<double, false>::WARPS
                                                       : chains_ctas<float, false>(p) * PCCfg<float, false>::WARPS));
            p->nblk[i] = cdiv(C1, 32);
            int64_t nreg = std::max<int64_t>(1, cdiv(2 * warps, p->nblk[i]));
            nreg = std::max<int64_t>(1, std::min<int64_t>(nreg, ntile / 4));
            p->region[i] = cdiv(ntile, nreg);
            p->nreg[i] = cdiv(ntile, p->region[i]);
        } else if (i == 0) {
            const int occ = f64 ? tiled_occ<double>(p->kp[0]) : tiled_occ<float>(p->kp[0]);
            const int64_t target = (int64_t)occ * p->sms * TILED_WAVES1;
            const int64_t n_pad1 = p->Lp[0] << p->kp[0];
            int64_t nreg = std::max<int64_t>(1, cdiv(target, m));
            // regions no shorter than 4 f(k1) + T so halos stay a small fraction
            const int64_t minreg = 4 * halo_f(p->kp[0]) + TPCR_T;
            nreg = std::max<int64_t>(1, std::min<int64_t>(nreg, n_pad1 / minreg));
            p->region[0] = cdiv(n_pad1, nreg);
            p->nreg[0] = cdiv(n_pad1, p->region[0]);
            p->nblk[0] = m;
        } else {  // over the Cp[i-1] chains, TPCR_IL_CB per CTA
            const int k2 = p->kp[i];
            p->nblk[i] = cdiv(C1, TPCR_IL_CB);
            const int occ2 = f64 ? tiled_il_occ<double>(k2) : tiled_il_occ<float>(k2);
            int64_t nreg2 = std::max<int64_t>(1, cdiv((int64_t)occ2 * p->sms * TILED_WAVES2, p->nblk[i]));
            const int64_t minreg2 = 4 * halo_f(k2) + TPCR_IL_TP;
            nreg2 = std::max<int64_t>(1, std::min<int64_t>(nreg2, L1 / minreg2));
            p->region[i] = cdiv(L1, nreg2);
            p->nreg[i] = cdiv(L1, p->region[i]);
        }
    }
}

size_t split_scratch(const tri_plan_s* p) {
    const size_t s = esize(p->dtype);
    const size_t chain_elems = (size_t)p->C * (size_t)p->L;
    // k > 0: normalised reduced rows (3 arrays) + c', d' (2 arrays) + two 3-array
    // intermediate buffers when there are several passes; k = 0: c', d'
    if (p->k == 0) return 2 * chain_elems * s;
    return (5 * chain_elems + (p->npass > 1 ? 6 * (size_t)inter_elems(p) : 0)) * s;
}

cudaError_t launch_split(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                         cudaStream_t st) {
    return p->dtype == TRI_F64 ? split_t<double>(p, a, b, c, d, x, st) : split_t<float>(p, a, b, c, d, x, st);
}

cudaError_t launch_split_pcr(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* ao,
                             void* co, void* do_, cudaStream_t st) {
    if (p->k == 0) return cudaErrorInvalidValue;
    return p->dtype == TRI_F64 ? run_passes<double>(p, a, b, c, d, ao, co, do_, 1, st)
                               : run_passes<float>(p, a, b, c, d, ao, co, do_, 1, st);
}

}  // namespace trih
