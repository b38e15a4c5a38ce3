// l_fused.cu -- launcher of TRI_VARIANT_FUSED (k_fused.cuh): streaming tiled PCR
// (k = 4) feeding p-Thomas in one persistent kernel (Sec. III.C).
#include "plan.cuh"
#include "k_fused.cuh"

using namespace tri;

namespace trih {
namespace {
template <typename T>
cudaError_t fused_t(const tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                    cudaStream_t st, void* dA, void* dC, void* dD) {
    FusedArgs<T> A;
    A.dA = (T*)dA; A.dC = (T*)dC; A.dD = (T*)dD;
    A.prof = (unsigned long long*)g_fused_prof;
    A.dbg_mode = g_fused_dbg_mode;
    A.a = (const T*)a; A.b = (const T*)b; A.c = (const T*)c; A.d = (const T*)d; A.x = (T*)x;
    A.spill = (T*)p->scratch;
    A.n = p->n; A.m = p->m; A.L = p->L; A.NC = p->fu_nc; A.S_on = p->fu_son;
    const bool vec = p->fu_vec && ((uintptr_t)a | (uintptr_t)b | (uintptr_t)c | (uintptr_t)d) % 16 == 0;
    const int smem = fused_fixed_smem<T>() + (vec ? fused_stage_smem<T>() : 0) + p->fu_son * FU_S * 2 * (int)sizeof(T);
    auto kern = vec ? k_fused<T, true> : k_fused<T, false>;
    cudaError_t e = set_smem((const void*)kern, smem);
    if (e != cudaSuccess) return e;
    kern<<<p->fu_grid, FU_THREADS, smem, st>>>(A);
    return cudaGetLastError();
}
}  // namespace

cudaError_t launch_fused(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                         cudaStream_t st, void* dA, void* dC, void* dD) {
    return p->dtype == TRI_F64 ? fused_t<double>(p, a, b, c, d, x, st, dA, dC, dD)
                               : fused_t<float>(p, a, b, c, d, x, st, dA, dC, dD);
}
int fused_smem_fixed(tri_dtype t, bool vec) {
    return t == TRI_F64 ? fused_fixed_smem<double>() + (vec ? fused_stage_smem<double>() : 0)
                        : fused_fixed_smem<float>() + (vec ? fused_stage_smem<float>() : 0);
}

}  // namespace trih
