// l_scan.cu -- launchers of TRI_VARIANT_SCAN (k_scan.cuh) and TRI_VARIANT_SCAN_MC
// (k_scan_mc.cuh): p-Thomas at k = 0 (the paper's rule for M > P) with
// each system's sweeps spread over a warp's lanes (X21).
#include <algorithm>

#include "plan.cuh"
#include "k_scan.cuh"
#include "k_scan_mc.cuh"
#include "k_scan_cl.cuh"
#include "k_scan_grid.cuh"
#include "k_scan_w512.cuh"

#ifndef SMC_DISCARD
#define SMC_DISCARD 1            // SCAN_MC pass 2: discard the read (c', d') lines (A/B macro)
#endif
#ifndef SMC_KEEP_MB
#define SMC_KEEP_MB 64           // SCAN_MC: L2 megabytes kept between passes (A/B macro)
#endif

using namespace tri;

namespace trih {
namespace {

// CONTIGUOUS: tensor view [m][n/r][r] (r = 8, or 128 bytes of elements with w128),
// box [1][256/r][r] = one 256-row window of one system per array; every
// coordinate fits int32 for any n, m of the API
template <typename T>
bool map_sys_rows(CUtensorMap* tm, const void* base, int64_t n, int64_t m, bool w128) {
    const int rw = w128 ? 128 / (int)sizeof(T) : 8;  // elements per tensor row
    // one system: its stride is never stepped, but must still be a 16-byte multiple
    const uint64_t sys = m == 1 ? ((uint64_t)n * sizeof(T) + 15) / 16 * 16 : (uint64_t)n * sizeof(T);
    const uint64_t dims[3] = {(uint64_t)rw, (uint64_t)(n / rw), (uint64_t)m};
    const uint64_t str[2] = {(uint64_t)rw * sizeof(T), sys};
    const uint32_t box[3] = {(uint32_t)rw, (uint32_t)(SC_W / rw), 1u};
    const CUtensorMapSwizzle swz =
        w128 ? CU_TENSOR_MAP_SWIZZLE_128B : sizeof(T) == 8 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B;
    return tma_encode(tm, sizeof(T), 3, base, dims, str, box, swz);
}

// SCAN, unit element stride (CONTIGUOUS, STRIDED x-lines): tensor view
// [nb][ms][n/r][r] with the plan's system / batch strides, box [1][1][256/r][r]
template <typename T>
bool map_sys_rows4(CUtensorMap* tm, const void* base, const tri_plan_s* p, bool w128) {
    const int rw = w128 ? 128 / (int)sizeof(T) : 8;
    const uint64_t dims[4] = {(uint64_t)rw, (uint64_t)(p->n / rw), (uint64_t)p->ms, (uint64_t)p->nb};
    const uint64_t str[3] = {(uint64_t)rw * sizeof(T), (uint64_t)p->ss * sizeof(T), (uint64_t)p->bs * sizeof(T)};
    const uint32_t box[4] = {(uint32_t)rw, (uint32_t)(SC_W / rw), 1u, 1u};
    const CUtensorMapSwizzle swz =
        w128 ? CU_TENSOR_MAP_SWIZZLE_128B : sizeof(T) == 8 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B;
    return tma_encode(tm, sizeof(T), 4, base, dims, str, box, swz);
}

// ... one batch: 3D view [ms][n/r][r] with the plan's system stride
template <typename T>
bool map_sys_rows3(CUtensorMap* tm, const void* base, const tri_plan_s* p, bool w128) {
    const int rw = w128 ? 128 / (int)sizeof(T) : 8;
    const uint64_t sys = p->ms == 1 ? ((uint64_t)p->ss * sizeof(T) + 15) / 16 * 16 : (uint64_t)p->ss * sizeof(T);
    const uint64_t dims[3] = {(uint64_t)rw, (uint64_t)(p->n / rw), (uint64_t)p->ms};
    const uint64_t str[2] = {(uint64_t)rw * sizeof(T), sys};
    const uint32_t box[3] = {(uint32_t)rw, (uint32_t)(SC_W / rw), 1u};
    const CUtensorMapSwizzle swz =
        w128 ? CU_TENSOR_MAP_SWIZZLE_128B : sizeof(T) == 8 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B;
    return tma_encode(tm, sizeof(T), 3, base, dims, str, box, swz);
}

// SCAN, unit system stride (INTERLEAVED / BATCHED / STRIDED y- and z-lines):
// tensor [nb][n][ms] (row stride es, batch stride bs elements), box [1][256 / S rows][S systems]
template <typename T>
bool map_il(CUtensorMap* tm, const void* base, int64_t n, int64_t ms, int64_t nb, int S, int64_t es, int64_t bs) {
    const uint64_t dims[3] = {(uint64_t)ms, (uint64_t)n, (uint64_t)nb};
    const uint64_t str[2] = {(uint64_t)es * sizeof(T), (uint64_t)bs * sizeof(T)};
    const uint32_t box[3] = {(uint32_t)S, (uint32_t)(SC_W / S), 1u};
    return tma_encode(tm, sizeof(T), 3, base, dims, str, box, CU_TENSOR_MAP_SWIZZLE_NONE);
}

template <typename T>
bool scan_maps(tri_plan_s* p, int tag, const void* a, const void* b, const void* c, const void* d, bool w128,
               StreamMaps& tm) {
    const void* key[4] = {a, b, c, d};
    if (tm_lookup(p, tag, key, 4, &tm.a, 4)) return true;
    const void* src[4] = {a, b, c, d};
    CUtensorMap* dst[4] = {&tm.a, &tm.b, &tm.c, &tm.d};
    for (int i = 0; i < 4; ++i) {
        const bool ok = p->variant == TRI_VARIANT_SCAN_MC ? map_sys_rows<T>(dst[i], src[i], p->n, p->m, w128)
                        : p->sk_S == 1 ? (p->nb == 1 ? map_sys_rows3<T>(dst[i], src[i], p, w128)
                                                     : map_sys_rows4<T>(dst[i], src[i], p, w128))
                                       : map_il<T>(dst[i], src[i], p->n, p->ms, p->nb, p->sk_S, p->es, p->bs);
        if (!ok) return false;
    }
    tm_store(p, tag, key, 4, &tm.a, 4);
    return true;
}

// fp32 one-window systems, two per TMA box (k_scan1_r16): tensor [m][n/32][32],
// box [2][n/32][32], 128B swizzle
bool map_pairs(CUtensorMap* tm, const void* base, int64_t n, int64_t m) {
    const uint64_t dims[3] = {32, (uint64_t)(n / 32), (uint64_t)m};
    const uint64_t str[2] = {128, (uint64_t)n * 4};
    const uint32_t box[3] = {32, (uint32_t)(n / 32), 2u};
    return tma_encode(tm, 4, 3, base, dims, str, box, CU_TENSOR_MAP_SWIZZLE_128B);
}

template <typename T, int S>
void* scan_kernel(bool prof) {
    return prof ? (void*)k_scan<T, S, true> : (void*)k_scan<T, S, false>;
}

// TRI_OPT_SCAN_CLUSTER: INTERLEAVED batches of few 8-system groups (no more groups
// than SMs: the chained kernel leaves SMs idle and walks every window in sequence)
// through one cluster of CL CTAs per group (k_scan_cl.cuh), CL the smallest of
// 2 / 4 / 8 whose CTAs are all resident at once; cudaErrorNotSupported leaves the
// shape to the chained kernel.  Measured slower at c2 (27.5 vs 21.0 us in ncu):
// every warp walks its windows three times (maps, replay, back substitution) with
// one load in flight, at 16 warps per SM (registers).
template <typename T>
int scan_cl_choose(const tri_plan_s* p, int& wpw) {
    const int64_t ngrp = cdiv(p->m, SCL_S), nwin = cdiv(p->n, SCL_WR);
    if (ngrp > p->sms || nwin < 2 * SCL_NW) return 0;
    const int smem = SCL_NW * SCLayout<T>::in_stride + 1024;
    int occ = 0;
    if (set_smem((const void*)k_scan_cl<T, 2>, smem) != cudaSuccess ||
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_scan_cl<T, 2>, 32 * SCL_NW, smem) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    for (int cl = 2; cl <= 8; cl *= 2) {
        wpw = (int)cdiv(nwin, (int64_t)cl * SCL_NW);
        if (wpw <= SCL_WMAX && ngrp * cl <= (int64_t)occ * p->sms) return cl;
    }
    return 0;
}

template <typename T, int CL>
cudaError_t scan_cl_launch(const tri_plan_s* p, const StreamMaps& tm, const SCLArgs<T>& A, cudaStream_t st) {
    const int smem = SCL_NW * SCLayout<T>::in_stride + 1024;
    cudaError_t e = set_smem((const void*)k_scan_cl<T, CL>, smem);
    if (e != cudaSuccess) return e;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(cdiv(p->m, SCL_S) * CL));
    cfg.blockDim = dim3(32 * SCL_NW);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = CL;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_scan_cl<T, CL>, tm, A);
}

template <typename T>
cudaError_t scan_cl_t(tri_plan_s* p, const StreamMaps& tm, void* x, cudaStream_t st) {
    int wpw = 0;
    const int cl = scan_cl_choose<T>(p, wpw);
    if (cl == 0) return cudaErrorNotSupported;
    SCLArgs<T> A;
    A.x = (T*)x;
    A.n = p->n; A.m = p->m; A.wpw = wpw;
    return cl == 2 ? scan_cl_launch<T, 2>(p, tm, A, st)
                   : cl == 4 ? scan_cl_launch<T, 4>(p, tm, A, st) : scan_cl_launch<T, 8>(p, tm, A, st);
}

// k_scan_grid (the planner's sg_Q > 0): tensor [nb][n][ms] (row stride es, batch
// stride bs), box [1][4 rows][32 systems]; blocks x Q CTAs in clusters of Q (the
// Q row pieces of a 32-system block exchange their aggregates through DSMEM)
template <typename T>
cudaError_t scan_grid_t(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                        cudaStream_t st) {
    StreamMaps tm;
    const void* key[4] = {a, b, c, d};
    if (!tm_lookup(p, 0x2800 + (int)sizeof(T), key, 4, &tm.a, 4)) {
        const void* src[4] = {a, b, c, d};
        CUtensorMap* dst[4] = {&tm.a, &tm.b, &tm.c, &tm.d};
        for (int i = 0; i < 4; ++i) {
            const uint64_t dims[3] = {(uint64_t)p->ms, (uint64_t)p->n, (uint64_t)p->nb};
            const uint64_t str[2] = {(uint64_t)p->es * sizeof(T), (uint64_t)p->bs * sizeof(T)};
            const uint32_t box[3] = {32u, (uint32_t)SG_SR, 1u};
            if (!tma_encode(dst[i], sizeof(T), 3, src[i], dims, str, box, CU_TENSOR_MAP_SWIZZLE_NONE))
                return cudaErrorNotSupported;
        }
        tm_store(p, 0x2800 + (int)sizeof(T), key, 4, &tm.a, 4);
    }
    const int ctas = p->sg_Q * p->sg_bpb * (int)p->nb;
    SGArgs<T> A;
    A.x = (T*)x;
    A.n = p->n; A.ms = p->ms; A.xel = p->es; A.xbat = p->bs;
    A.bpb = p->sg_bpb; A.Q = p->sg_Q;
    A.prof = (unsigned long long*)g_fused_prof;  // tri_debug_set_profile: [CTAs][16][16] phase timestamps
    A.dbg = g_fused_dbg_mode;
    const int nst = p->sg_R / SG_SR;
    void* kern = nst == 1 ? (void*)k_scan_grid<T, 1> : nst == 2 ? (void*)k_scan_grid<T, 2>
                 : nst == 3 ? (void*)k_scan_grid<T, 3> : (void*)k_scan_grid<T, 4>;
    const int smem = SGLayout<T>::smem_bytes;
    cudaError_t e = set_smem(kern, smem);
    if (e != cudaSuccess) return e;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)ctas);
    cfg.blockDim = dim3(SG_THREADS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = (unsigned)p->sg_Q;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    void* args[] = {(void*)&tm, (void*)&A};
    return cudaLaunchKernelExC(&cfg, kern, args);
}

template <typename T>
bool scan_grid_fits_t(const tri_plan_s* p, int Q, int R, int64_t nblk) {
    const int nst = R / SG_SR;
    const void* kern = nst == 1 ? (const void*)k_scan_grid<T, 1> : nst == 2 ? (const void*)k_scan_grid<T, 2>
                       : nst == 3 ? (const void*)k_scan_grid<T, 3> : (const void*)k_scan_grid<T, 4>;
    const int smem = SGLayout<T>::smem_bytes;
    if (set_smem(kern, smem) != cudaSuccess) { cudaGetLastError(); return false; }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(nblk * Q));
    cfg.blockDim = dim3(SG_THREADS);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = (unsigned)Q;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int ncl = 0;
    if (cudaOccupancyMaxActiveClusters(&ncl, kern, &cfg) != cudaSuccess) { cudaGetLastError(); return false; }
    return (int64_t)ncl >= nblk;
}

// k_scan_w512 (the planner's s5): tensor view [m][n/16][16] (128-byte rows), box
// [1][32][16] = one 512-row window of one array, 128B swizzle
cudaError_t scan_w512_t(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                        cudaStream_t st) {
    StreamMaps tm;
    const void* key[4] = {a, b, c, d};
    if (!tm_lookup(p, 0x3008, key, 4, &tm.a, 4)) {
        const void* src[4] = {a, b, c, d};
        CUtensorMap* dst[4] = {&tm.a, &tm.b, &tm.c, &tm.d};
        const uint64_t sys = p->m == 1 ? ((uint64_t)p->n * 8 + 15) / 16 * 16 : (uint64_t)p->n * 8;
        for (int i = 0; i < 4; ++i) {
            const uint64_t dims[3] = {16, (uint64_t)(p->n / 16), (uint64_t)p->m};
            const uint64_t str[2] = {128, sys};
            const uint32_t box[3] = {16, (uint32_t)(S5_W / 16), 1u};
            if (!tma_encode(dst[i], 8, 3, src[i], dims, str, box, CU_TENSOR_MAP_SWIZZLE_128B))
                return cudaErrorNotSupported;
        }
        tm_store(p, 0x3008, key, 4, &tm.a, 4);
    }
    ScanArgs<double> A{};
    A.x = (double*)x;
    A.spill = (double*)p->scratch;
    A.n = p->n; A.m = p->m; A.ms = p->ms; A.NC = p->sk_nc; A.S_on = p->sk_son; A.delta = p->sk_delta;
    A.xsys = p->ss; A.xbat = p->bs; A.xel = p->es; A.nb = 1;
    A.x32 = ((uintptr_t)x % 32 == 0 && (p->ss * 8) % 32 == 0) ? 1 : 0;
    const int smem = S5Layout::smem_bytes(p->sk_nc, p->sk_delta, p->sk_son);
    cudaError_t e = set_smem((const void*)k_scan_w512<double>, smem);
    if (e != cudaSuccess) return e;
    k_scan_w512<double><<<p->sk_grid, S5_THREADS, smem, st>>>(tm, A);
    return cudaGetLastError();
}

template <typename T>
cudaError_t scan_t(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                   cudaStream_t st) {
    if (p->sg_Q > 0) return scan_grid_t<T>(p, a, b, c, d, x, st);
    if (p->s5) return scan_w512_t(p, a, b, c, d, x, st);
    const int S = p->sk_S;
    const bool contig = p->layout == TRI_LAYOUT_CONTIGUOUS;  // the one-window kernels assume system stride n
    if constexpr (sizeof(T) == 4) {
        // fp32 one-window systems, n % 32 == 0 (c4): two systems per warp, 16 rows per lane
        if (contig && S == 1 && p->sk_nc == 1 && p->n % 32 == 0) {
            StreamMaps tm;
            const void* key[4] = {a, b, c, d};
            if (!tm_lookup(p, 0x1800, key, 4, &tm.a, 4)) {
                if (!map_pairs(&tm.a, a, p->n, p->m) || !map_pairs(&tm.b, b, p->n, p->m) ||
                    !map_pairs(&tm.c, c, p->n, p->m) || !map_pairs(&tm.d, d, p->n, p->m))
                    return cudaErrorNotSupported;
                tm_store(p, 0x1800, key, 4, &tm.a, 4);
            }
            ScanArgs<float> A{};
            A.x = (float*)x;
            A.n = p->n; A.m = p->m; A.ms = p->ms; A.NC = 1;
            cudaError_t e = set_smem((const void*)k_scan1_r16<float>, S16::smem_bytes);
            if (e != cudaSuccess) return e;
            const unsigned grid = (unsigned)std::min<int64_t>((p->m + 1) / 2, p->sms);
            k_scan1_r16<float><<<grid, S16_NW * 32, S16::smem_bytes, st>>>(tm, A);
            return cudaGetLastError();
        }
    }
    // one-window systems shorter than 3/4 of a window (many idle rows: compute-heavy)
    // run the chain-free kernel with more warps (fp32 n = 128: 1.19 ms vs 1.50 ms
    // per 2^28 rows); at n = 256 the 12-warp kernel is faster (c4: 0.99 vs 1.02 ms)
    const bool one = contig && S == 1 && p->sk_nc == 1 && p->n <= 3 * SC_W / 4;
    // 128-byte TMA rows (n % 32 fp32 / n % 16 fp64; the k_scan chain and one-window
    // paths): one TMA request per 128 bytes (fp32 c4: 0.99 -> 0.84 ms)
    const bool w128 = S == 1 && p->n % (128 / (int)sizeof(T)) == 0 && !one;
    StreamMaps tm;
    if (one) {  // k_scan1: 3D view [m][n/8][8]
        const void* key[4] = {a, b, c, d};
        if (!tm_lookup(p, 0x1400 + (int)sizeof(T), key, 4, &tm.a, 4)) {
            if (!map_sys_rows<T>(&tm.a, a, p->n, p->m, false) || !map_sys_rows<T>(&tm.b, b, p->n, p->m, false) ||
                !map_sys_rows<T>(&tm.c, c, p->n, p->m, false) || !map_sys_rows<T>(&tm.d, d, p->n, p->m, false))
                return cudaErrorNotSupported;
            tm_store(p, 0x1400 + (int)sizeof(T), key, 4, &tm.a, 4);
        }
    } else if (!scan_maps<T>(p, 0x1000 + (int)sizeof(T) + 16 * (w128 ? 1 : 0), a, b, c, d, w128, tm)) {
        return cudaErrorNotSupported;
    }
    if (S == 8 && p->nb == 1 && p->opt_cluster) {
        const cudaError_t ec = scan_cl_t<T>(p, tm, x, st);
        if (ec != cudaErrorNotSupported) return ec;
    }
    ScanArgs<T> A;
    A.x = (T*)x;
    A.spill = (T*)p->scratch;
    A.n = p->n; A.m = p->m; A.ms = p->ms; A.NC = p->sk_nc; A.S_on = p->sk_son; A.delta = p->sk_delta;
    A.xsys = p->ss; A.xbat = p->bs; A.xel = p->es; A.nb = (int)p->nb;
    A.x32 = ((uintptr_t)x % 32 == 0 && (p->ss * (int64_t)sizeof(T)) % 32 == 0 &&
             (p->nb == 1 || (p->bs * (int64_t)sizeof(T)) % 32 == 0)) ? 1 : 0;
    A.w128 = w128 ? 1 : 0;
    A.ga = (const T*)a; A.gb = (const T*)b; A.gc = (const T*)c; A.gd = (const T*)d;
    {
        const int64_t rw = S > 1 ? 1 : w128 ? 128 / (int64_t)sizeof(T) : 8;
        A.n_al = p->n / rw * rw;  // ragged n: the rows past the tensor map's last row group (sc_patch_tail)
    }
    A.prof = (unsigned long long*)g_fused_prof;
    A.dbg = g_fused_dbg_mode;
    if (one) {
        cudaError_t e = set_smem((const void*)k_scan1<T>, SC1<T>::smem_bytes);
        if (e != cudaSuccess) return e;
        k_scan1<T><<<p->sk_grid, SC1<T>::NW * 32, SC1<T>::smem_bytes, st>>>(tm, A);
        return cudaGetLastError();
    }
    // one-window systems (S = 1): the slot area holds the warps' second staging buffers
    const int son_or_buf = (S == 1 && p->sk_nc == 1)
                               ? (SC_NW * SCLayout<T>::in_stride + SCLayout<T>::slot_bytes - 1) / SCLayout<T>::slot_bytes
                               : p->sk_son;
    const int smem = SCLayout<T>::smem_bytes(p->sk_nc, p->sk_delta, son_or_buf);
    const bool pr = A.prof != nullptr;
    void* kern = S == 1 ? scan_kernel<T, 1>(pr) : S == 2 ? scan_kernel<T, 2>(pr) : S == 4 ? scan_kernel<T, 4>(pr)
                 : S == 8 ? scan_kernel<T, 8>(pr) : S == 16 ? scan_kernel<T, 16>(pr) : scan_kernel<T, 32>(pr);
    cudaError_t e = set_smem(kern, smem);
    if (e != cudaSuccess) return e;
    void* args[] = {(void*)&tm, (void*)&A};
    return cudaLaunchKernel(kern, dim3(p->sk_grid), dim3(SC_THREADS), args, smem, st);
}

template <typename T>
cudaError_t scan_mc_setup(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                          StreamMaps& tm, ScanMCArgs<T>& A, int& smem, bool cache) {
    const int64_t n = p->n;
    const bool w = n % (128 / (int)sizeof(T)) == 0;
    if (a) {
        bool ok;
        if (cache) {
            ok = scan_maps<T>(p, 0x2000 + (int)sizeof(T), a, b, c, d, w, tm);
        } else {
            ok = map_sys_rows<T>(&tm.a, a, n, p->m, w) && map_sys_rows<T>(&tm.b, b, n, p->m, w) &&
                 map_sys_rows<T>(&tm.c, c, n, p->m, w) && map_sys_rows<T>(&tm.d, d, n, p->m, w);
        }
        if (!ok) return cudaErrorNotSupported;
    }
    A = ScanMCArgs<T>{};
    A.w128 = w ? 1 : 0;
    A.ga = (const T*)a; A.gb = (const T*)b; A.gc = (const T*)c; A.gd = (const T*)d;
    A.n_al = n / (w ? 128 / (int64_t)sizeof(T) : 8) * (w ? 128 / (int64_t)sizeof(T) : 8);
    A.x = (T*)x;
    A.x32 = ((uintptr_t)x % 32 == 0 && (n * (int64_t)sizeof(T)) % 32 == 0) ? 1 : 0;
    A.cd = (T*)p->scratch;
    const int64_t mp = p->m * (int64_t)p->mc_P;
    A.cmap = reinterpret_cast<double*>(A.cd + p->m * (int64_t)p->sk_nc * sc_slot_elems<T>());  // 2 KB multiples
    A.cbm = A.cmap + 8 * mp;
    A.n = p->n; A.m = p->m; A.NC = p->sk_nc; A.NCW = p->mc_NCW; A.P = p->mc_P;
    // L2 reuse between the passes (~SMC_KEEP_MB of each pass's last data per pass;
    // only when the system does not fit L2 anyway)
    {
        const int64_t kb = (int64_t)SMC_KEEP_MB << 20;
        const int64_t in_w = 4 * SC_W * (int64_t)sizeof(T), cd_w = (int64_t)sc_slot_elems<T>() * sizeof(T);
        const int64_t chunks = p->m * (int64_t)p->mc_P;
        const bool big = chunks * p->mc_NCW * in_w > 2 * kb;
        A.keep0 = big ? (int)std::min<int64_t>(p->mc_NCW, kb / (chunks * in_w)) : 0;
        A.keep1 = big ? (int)std::min<int64_t>(p->mc_NCW, kb / (chunks * cd_w)) : 0;
        A.discard = SMC_DISCARD;
    }
    smem = SMCLayout<T>::smem_bytes(p->mc_NCW);
    for (auto k : {k_scan_mc<T, 0>, k_scan_mc<T, 1>, k_scan_mc<T, 2>}) {
        cudaError_t e = set_smem((const void*)k, smem);
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}
// the 16 values after the fp64 chunk maps: the slice's incoming state (3) and x after it (1)
template <typename T>
T* scan_mc_slice_vals(const tri_plan_s* p) {
    double* maps = reinterpret_cast<double*>((T*)p->scratch + p->m * (int64_t)p->sk_nc * sc_slot_elems<T>());
    return reinterpret_cast<T*>(maps + 16 * p->m * (int64_t)p->mc_P);
}

template <typename T>
cudaError_t scan_mc_t(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                      cudaStream_t st) {
    StreamMaps tm;
    ScanMCArgs<T> A;
    int smem = 0;
    cudaError_t e = scan_mc_setup<T>(p, a, b, c, d, x, tm, A, smem, true);
    if (e != cudaSuccess) return e;
    if (p->mc_lb) {
        ScanMCLB<T> lb;
        lb.rec = reinterpret_cast<double*>(scan_mc_slice_vals<T>(p) + 16);  // 16 T values: 8-byte aligned
        const int64_t nrec = p->m * (int64_t)p->mc_Ps;
        lb.Pb = (p->mc_Ps + 31) / 32;
        const int64_t nblk = p->m * (int64_t)lb.Pb;
        lb.brec = lb.rec + nrec * SMC_REC;
        lb.flag = (unsigned*)(lb.brec + nblk * 8);
        lb.NCWs = p->mc_NCWs;
        lb.Ps = p->mc_Ps;
        lb.prof = (unsigned long long*)g_fused_prof;
        const int smem_lb = LBLayout<T>::smem_bytes;
        e = set_smem((const void*)k_scan_mc_lb<T>, smem_lb);
        if (e != cudaSuccess) return e;
        e = cudaMemsetAsync(lb.flag, 0, (size_t)(nrec + 1 + nblk) * sizeof(unsigned), st);
        if (e != cudaSuccess) return e;
        const int grid = (int)std::min<int64_t>(p->sms, nrec);
        k_scan_mc_lb<T><<<grid, LB_THREADS, smem_lb, st>>>(tm, A, lb);
        A.xafter = lb.rec;
        A.NCWs = p->mc_NCWs;
        A.Ps = p->mc_Ps;
        k_scan_mc<T, 2><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
        return cudaGetLastError();
    }
    k_scan_mc<T, 0><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
    k_scan_mc<T, 1><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
    k_scan_mc<T, 2><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
    return cudaGetLastError();
}

// sliced solve of one system over devices (NEXT-4): phase 0 = pass 0 + the
// slice's forward map; 1 = incoming state from every slice's map, pass 1, the
// slice's backward map; 2 = x after the slice from every backward map, pass 2
template <typename T>
cudaError_t scan_mc_slice_t(tri_plan_s* p, int phase, int slice, int nslices, const void* a, const void* b,
                            const void* c, const void* d, const void* maps, void* out, cudaStream_t st) {
    StreamMaps tm;
    ScanMCArgs<T> A;
    int smem = 0;
    cudaError_t e = scan_mc_setup<T>(p, phase < 2 ? a : nullptr, b, c, d, phase == 2 ? out : nullptr, tm, A, smem,
                                     false);
    if (e != cudaSuccess) return e;
    A.keep_a0 = slice > 0;
    A.keep_cn = slice < nslices - 1;
    T* vals = scan_mc_slice_vals<T>(p);
    if (phase == 0) {
        k_scan_mc<T, 0><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
        k_scan_mc_slice_map<T, 0><<<1, 32, 0, st>>>(A, (T*)out);
    } else if (phase == 1) {
        k_scan_mc_slice_link<T, 0><<<1, 32, 0, st>>>((const T*)maps, nslices, slice, vals);
        A.s0 = vals;
        k_scan_mc<T, 1><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
        k_scan_mc_slice_map<T, 1><<<1, 32, 0, st>>>(A, (T*)out);
    } else {
        k_scan_mc_slice_link<T, 1><<<1, 32, 0, st>>>((const T*)maps, nslices, slice, vals + 4);
        A.xe = vals + 4;
        k_scan_mc<T, 2><<<p->sk_grid, SC_THREADS, smem, st>>>(tm, A);
    }
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_scan(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                        cudaStream_t st) {
    return p->dtype == TRI_F64 ? scan_t<double>(p, a, b, c, d, x, st) : scan_t<float>(p, a, b, c, d, x, st);
}
cudaError_t launch_scan_mc(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                           cudaStream_t st) {
    return p->dtype == TRI_F64 ? scan_mc_t<double>(p, a, b, c, d, x, st) : scan_mc_t<float>(p, a, b, c, d, x, st);
}
cudaError_t launch_scan_mc_slice(tri_plan_s* p, int phase, int slice, int nslices, const void* a, const void* b,
                                 const void* c, const void* d, const void* maps, void* out, cudaStream_t st) {
    return p->dtype == TRI_F64 ? scan_mc_slice_t<double>(p, phase, slice, nslices, a, b, c, d, maps, out, st)
                               : scan_mc_slice_t<float>(p, phase, slice, nslices, a, b, c, d, maps, out, st);
}
int scan_smem_fixed(tri_dtype t, int NC, int delta) {
    return t == TRI_F64 ? SCLayout<double>::smem_bytes(NC, delta, 0) : SCLayout<float>::smem_bytes(NC, delta, 0);
}
int scan_slot_bytes(tri_dtype t) { return t == TRI_F64 ? SCLayout<double>::slot_bytes : SCLayout<float>::slot_bytes; }
int scan_in_stride(tri_dtype t) { return t == TRI_F64 ? SCLayout<double>::in_stride : SCLayout<float>::in_stride; }
int scan_mc_wmax() { return SMC_WMAX; }
bool scan_grid_fits(const tri_plan_s* p, int Q, int R, int64_t nblk) {
    return p->dtype == TRI_F64 ? scan_grid_fits_t<double>(p, Q, R, nblk) : scan_grid_fits_t<float>(p, Q, R, nblk);
}
int scan_mc_lb_maxw() { return LB_MAXW; }

}  // namespace trih
