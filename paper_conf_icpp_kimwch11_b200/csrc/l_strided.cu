// l_strided.cu -- TRI_LAYOUT_STRIDED fallback (ADI line solves
// on pitched / sub-grid views of a 3D array): when the caller's strides are not
// what a TMA tensor map can describe (16-byte multiples), the solve gathers a, b,
// c, d into a packed CONTIGUOUS ([q][i]) or INTERLEAVED ([i][q]) copy, runs the
// inner plan on it and scatters x back.  Element (q = b ms + s, i) of the caller's
// arrays is at i es + s ss + b bs.  The packed order follows the unit stride of
// the source so the gathers coalesce on the side that has it.
#include "plan.cuh"

namespace trih {
namespace {

template <typename T>
__global__ void k_pack4(const T* __restrict__ a, const T* __restrict__ b, const T* __restrict__ c,
                        const T* __restrict__ d, T* __restrict__ pa, T* __restrict__ pb, T* __restrict__ pc,
                        T* __restrict__ pd, int64_t n, int64_t ms, int64_t m, int64_t es, int64_t ss, int64_t bs,
                        int il) {
    const int64_t N = n * m;
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < N; k += (int64_t)gridDim.x * blockDim.x) {
        int64_t q, i;
        if (il) { i = k / m; q = k - i * m; } else { q = k / n; i = k - q * n; }
        const int64_t bt = q / ms, s = q - bt * ms;
        const int64_t o = i * es + s * ss + bt * bs;
        pa[k] = __ldcs(a + o); pb[k] = __ldcs(b + o); pc[k] = __ldcs(c + o); pd[k] = __ldcs(d + o);
    }
}

template <typename T>
__global__ void k_unpack(const T* __restrict__ px, T* __restrict__ x, int64_t n, int64_t ms, int64_t m, int64_t es,
                         int64_t ss, int64_t bs, int il) {
    const int64_t N = n * m;
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < N; k += (int64_t)gridDim.x * blockDim.x) {
        int64_t q, i;
        if (il) { i = k / m; q = k - i * m; } else { q = k / n; i = k - q * n; }
        const int64_t bt = q / ms, s = q - bt * ms;
        __stcs(x + i * es + s * ss + bt * bs, __ldcs(px + k));
    }
}

unsigned grid_for(int64_t N, int sms) {
    const int64_t g = cdiv(N, 256);
    return (unsigned)(g < 8 * (int64_t)sms ? g : 8 * (int64_t)sms);
}

}  // namespace

cudaError_t launch_pack(const tri_plan_s* p, const void* const src[4], void* const dst[4], cudaStream_t st) {
    const int il = p->inner->layout == TRI_LAYOUT_INTERLEAVED ? 1 : 0;
    const unsigned g = grid_for(p->n * p->m, p->sms);
    if (p->dtype == TRI_F64)
        k_pack4<double><<<g, 256, 0, st>>>((const double*)src[0], (const double*)src[1], (const double*)src[2],
                                           (const double*)src[3], (double*)dst[0], (double*)dst[1], (double*)dst[2],
                                           (double*)dst[3], p->n, p->ms, p->m, p->es, p->ss, p->bs, il);
    else
        k_pack4<float><<<g, 256, 0, st>>>((const float*)src[0], (const float*)src[1], (const float*)src[2],
                                          (const float*)src[3], (float*)dst[0], (float*)dst[1], (float*)dst[2],
                                          (float*)dst[3], p->n, p->ms, p->m, p->es, p->ss, p->bs, il);
    return cudaGetLastError();
}

cudaError_t launch_unpack(const tri_plan_s* p, const void* src, void* dst, cudaStream_t st) {
    const int il = p->inner->layout == TRI_LAYOUT_INTERLEAVED ? 1 : 0;
    const unsigned g = grid_for(p->n * p->m, p->sms);
    if (p->dtype == TRI_F64)
        k_unpack<double><<<g, 256, 0, st>>>((const double*)src, (double*)dst, p->n, p->ms, p->m, p->es, p->ss, p->bs, il);
    else
        k_unpack<float><<<g, 256, 0, st>>>((const float*)src, (float*)dst, p->n, p->ms, p->m, p->es, p->ss, p->bs, il);
    return cudaGetLastError();
}

}  // namespace trih
