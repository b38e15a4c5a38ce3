// l_stream.cu -- launcher of TRI_VARIANT_STREAM (k_stream.cuh): tiled PCR (k = 3)
// streamed into a segmented p-Thomas in one persistent kernel (Sec. III.C,
// P:687-693).
#include "plan.cuh"
#include "k_stream.cuh"

using namespace tri;

namespace trih {

// tensor maps [n m / 8][8] (64-byte rows, 64B swizzle, box 8 x 32)
cudaError_t launch_stream(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                          cudaStream_t st, void* ao, void* co, void* do_) {
    StreamMaps tm;
    const void* key[4] = {a, b, c, d};
    if (!tm_lookup(p, 0x3000, key, 4, &tm.a, 4)) {
        const uint64_t rows8 = (uint64_t)(p->n / 8) * (uint64_t)p->m;
        const uint64_t dims[2] = {8, rows8}, str[1] = {8 * sizeof(double)};
        const uint32_t box[2] = {8, 32};
        CUtensorMap* dst[4] = {&tm.a, &tm.b, &tm.c, &tm.d};
        for (int i = 0; i < 4; ++i)
            if (!tma_encode(dst[i], 8, 2, key[i], dims, str, box, CU_TENSOR_MAP_SWIZZLE_64B)) return cudaErrorNotSupported;
        tm_store(p, 0x3000, key, 4, &tm.a, 4);
    }
    StreamArgs<double> A;
    A.x = (double*)x;
    A.spill = (double*)p->scratch;
    A.n = p->n; A.m = p->m; A.NC = p->sk_nc; A.S_on = p->sk_son;
    A.dA = (double*)ao; A.dC = (double*)co; A.dD = (double*)do_;
    A.prof = (unsigned long long*)g_fused_prof;
    A.dbg = g_fused_dbg_mode;
    const int smem = SKLayout<double>::off_store + p->sk_son * SKLayout<double>::slot_bytes + 1024;
    auto kern = A.prof ? k_stream<double, true> : k_stream<double, false>;
    cudaError_t e = set_smem((const void*)kern, smem);
    if (e != cudaSuccess) return e;
    kern<<<p->sk_grid, SK_THREADS, smem, st>>>(tm, A);
    return cudaGetLastError();
}

}  // namespace trih
