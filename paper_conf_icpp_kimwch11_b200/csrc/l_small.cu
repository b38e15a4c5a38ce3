// l_small.cu -- launchers of the whole-system variants: TRI_VARIANT_WARP
// (k_warp.cuh: one warp per system, 5 shuffle PCR steps + in-register p-Thomas)
// and TRI_VARIANT_ONCHIP (k_onchip.cuh: whole systems in one CTA's shared
// memory, Fig 11a/c).
#include <algorithm>

#include "plan.cuh"
#include "k_onchip.cuh"
#include "k_warp.cuh"

using namespace tri;

namespace trih {
namespace {

constexpr int ONCHIP_THREADS = 512;

template <typename T, int RPT>
cudaError_t onchip_rpt(const tri_plan_s* p, OnchipArgs<T> a, cudaStream_t st) {
    const int smem = 3 * p->G * p->P * (int)sizeof(T);
    cudaError_t e = set_smem((const void*)k_onchip<T, RPT>, smem);
    if (e != cudaSuccess) return e;
    const int64_t grid = cdiv(p->m, p->G);
    k_onchip<T, RPT><<<(unsigned)grid, ONCHIP_THREADS, smem, st>>>(a);
    return cudaGetLastError();
}

template <typename T>
cudaError_t onchip_t(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                     void* ao, void* co, void* do_, int mode, cudaStream_t st) {
    OnchipArgs<T> A;
    A.a = (const T*)a; A.b = (const T*)b; A.c = (const T*)c; A.d = (const T*)d;
    A.x = (T*)x; A.ao = (T*)ao; A.co = (T*)co; A.do_ = (T*)do_;
    A.n = p->n; A.m = p->m; A.layout = p->layout; A.k = p->k; A.G = p->G; A.P = p->P; A.mode = mode;
    switch (p->rpt) {
        case 1: return onchip_rpt<T, 1>(p, A, st);
        case 2: return onchip_rpt<T, 2>(p, A, st);
        case 4: return onchip_rpt<T, 4>(p, A, st);
        case 8: return onchip_rpt<T, 8>(p, A, st);
        case 16: return onchip_rpt<T, 16>(p, A, st);
        default: return cudaErrorInvalidValue;
    }
}

template <typename T>
cudaError_t warp_t(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                   void* ao, void* co, void* do_, int mode, cudaStream_t st) {
    WarpArgs<T> A;
    A.a = (const T*)a; A.b = (const T*)b; A.c = (const T*)c; A.d = (const T*)d;
    A.x = (T*)x; A.ao = (T*)ao; A.co = (T*)co; A.do_ = (T*)do_;
    A.n = p->n; A.m = p->m; A.layout = p->layout; A.mode = mode;
    const bool il = p->layout == TRI_LAYOUT_INTERLEAVED && p->m > 1;
    const int wpb = il ? WARP_WPB_IL : WARP_WPB;
    const int64_t need = cdiv(p->m, wpb);
    // contiguous: persistent warps (one resident wave), each walking systems
    // q, q + grid*WPB, ... with the next system's loads in flight
    auto contig_grid = [&](auto kern) {
        int occ = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, wpb * 32, 0) != cudaSuccess || occ < 1) {
            cudaGetLastError();
            occ = 1;
        }
        return (unsigned)std::min<int64_t>(need, (int64_t)occ * p->sms);
    };
#define TRI_WARP_CASE(R)                                                                  \
    case R:                                                                               \
        if (il) k_warp<T, R, true><<<(unsigned)need, wpb * 32, 0, st>>>(A);               \
        else k_warp<T, R, false><<<warp_persistent<T, R>() ? contig_grid(k_warp<T, R, false>) : (unsigned)need, \
                                   wpb * 32, 0, st>>>(A);                                 \
        break;
    switch (p->rpt) {
        TRI_WARP_CASE(1) TRI_WARP_CASE(2) TRI_WARP_CASE(4) TRI_WARP_CASE(8) TRI_WARP_CASE(16) TRI_WARP_CASE(32)
        default: return cudaErrorInvalidValue;
    }
#undef TRI_WARP_CASE
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_warp(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                        void* ao, void* co, void* do_, int mode, cudaStream_t st) {
    return p->dtype == TRI_F64 ? warp_t<double>(p, a, b, c, d, x, ao, co, do_, mode, st)
                               : warp_t<float>(p, a, b, c, d, x, ao, co, do_, mode, st);
}
cudaError_t launch_onchip(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                          void* ao, void* co, void* do_, int mode, cudaStream_t st) {
    return p->dtype == TRI_F64 ? onchip_t<double>(p, a, b, c, d, x, ao, co, do_, mode, st)
                               : onchip_t<float>(p, a, b, c, d, x, ao, co, do_, mode, st);
}

}  // namespace trih
