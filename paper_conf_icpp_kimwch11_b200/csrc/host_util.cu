// host_util.cu -- host-side helpers shared by the launchers (plan.cuh): the TMA
// descriptor encoder, the per-plan tensor-map cache and the per-kernel
// shared-memory attribute cache.  No kernels here.
#include <cstring>
#include <mutex>

#include "plan.cuh"

namespace trih {

void* g_fused_prof = nullptr;
int g_fused_dbg_mode = 0;

namespace {
PFN_cuTensorMapEncodeTiled_v12000 tma_encoder() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (PFN_cuTensorMapEncodeTiled_v12000)f;
        else
            cudaGetLastError();
    });
    return fn;
}
}  // namespace

bool tma_encode(CUtensorMap* tm, size_t es, int rank, const void* base, const uint64_t* dims,
                const uint64_t* strides, const uint32_t* box, CUtensorMapSwizzle swz) {
    auto enc = tma_encoder();
    if (!enc || rank < 1 || rank > 5) return false;
    cuuint64_t d[5], s[4];
    cuuint32_t b[5], e[5];
    for (int i = 0; i < rank; ++i) {
        d[i] = dims[i];
        b[i] = box[i];
        e[i] = 1;
        if (i + 1 < rank) s[i] = strides[i];
    }
    return enc(tm, es == 8 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, (cuuint32_t)rank,
               const_cast<void*>(base), d, s, b, e, CU_TENSOR_MAP_INTERLEAVE_NONE, swz,
               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool tm_lookup(tri_plan_s* p, int tag, const void* const* key, int nkey, CUtensorMap* maps, int nmaps) {
    if (nkey > TM_MAX || nmaps > TM_MAX) return false;
    for (const TmEntry& c : p->tmc.e) {
        if (!c.valid || c.tag != tag) continue;
        bool same = true;
        for (int i = 0; i < TM_MAX && same; ++i) same = c.key[i] == (i < nkey ? key[i] : nullptr);
        if (!same) continue;
        std::memcpy(maps, c.maps, sizeof(CUtensorMap) * nmaps);
        return true;
    }
    return false;
}

void tm_store(tri_plan_s* p, int tag, const void* const* key, int nkey, const CUtensorMap* maps, int nmaps) {
    if (nkey > TM_MAX || nmaps > TM_MAX) return;
    // the entry of the same launcher (tag) is replaced; otherwise the round-robin victim
    int v = -1;
    for (int i = 0; i < TM_ENT && v < 0; ++i)
        if (p->tmc.e[i].valid && p->tmc.e[i].tag == tag) v = i;
    if (v < 0) { v = p->tmc.next; p->tmc.next = (v + 1) % TM_ENT; }
    TmEntry& c = p->tmc.e[v];
    for (int i = 0; i < TM_MAX; ++i) c.key[i] = i < nkey ? key[i] : nullptr;
    std::memcpy(c.maps, maps, sizeof(CUtensorMap) * nmaps);
    c.tag = tag;
    c.valid = true;
}

cudaError_t set_smem(const void* func, int bytes) {
    // (kernel, device) -> largest size already set; a linear table is plenty
    // (a few dozen kernel instantiations x devices)
    struct Ent { const void* f; int dev; int bytes; };
    static Ent tab[512];
    static int nt = 0;
    static std::mutex mu;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return cudaGetLastError();
    std::lock_guard<std::mutex> lk(mu);
    for (int i = 0; i < nt; ++i)
        if (tab[i].f == func && tab[i].dev == dev) {
            if (tab[i].bytes >= bytes) return cudaSuccess;
            const cudaError_t e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
            if (e == cudaSuccess) tab[i].bytes = bytes;
            return e;
        }
    const cudaError_t e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess && nt < 512) tab[nt++] = Ent{func, dev, bytes};
    return e;
}

}  // namespace trih
