// plan.cuh -- internal (non-exported) host-side declarations shared by the
// translation units of libtri.so: the plan object, small host helpers, the TMA
// descriptor encoder, the per-kernel shared-memory attribute cache, and the
// launchers each kernel family's .cu file defines.  Not part of the C ABI
// (include/tri.h is); built with -fvisibility=hidden so none of this is exported.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <cstddef>
#include <cstdint>

#include "tri.h"

namespace trih {

constexpr int HOST_CHUNKS = 16;  // tri_solve_host pipeline depth (chunks of systems)
constexpr int TM_MAX = 8;        // tensor maps per cache entry
constexpr int TM_ENT = 6;        // cache entries per plan (one per launch of a multi-kernel solve)

// Tensor maps of the last pointer sets the launchers saw (tri_solve then does no
// cuTensorMapEncode work when the caller reuses its buffers, as bench.py and a
// time-stepping ADI code do).  `tag` names the launcher (and its geometry);
// any plan change (k, variant, option) clears the cache.
struct TmEntry {
    bool valid = false;
    int tag = 0;
    const void* key[TM_MAX] = {};
    alignas(64) CUtensorMap maps[TM_MAX];
};
struct TmCache {
    TmEntry e[TM_ENT];
    int next = 0;  // round-robin victim
    void clear() {
        for (auto& x : e) x.valid = false;
    }
};

}  // namespace trih

struct tri_plan_s {
    int64_t n = 0, m = 0;
    tri_dtype dtype = TRI_F64;
    tri_layout layout = TRI_LAYOUT_CONTIGUOUS;
    int device = 0, sms = 0;
    int k = 0;
    tri_variant variant = TRI_VARIANT_SCAN;
    bool forced = false;          // variant or k set by the caller (tri_solve_host sub-plans inherit it)
    int opt_tma = 1;              // TRI_OPT_TMA: 0 = p-Thomas through the non-TMA kernels
    int opt_lookback = -1;        // TRI_OPT_SCAN_MC_LOOKBACK: windows per look-back chunk (0 = three passes, -1 = auto)
    int opt_cluster = 0;          // TRI_OPT_SCAN_CLUSTER: interleaved SCAN through thread-block clusters
    int opt_grid = -1;            // TRI_OPT_SCAN_GRID: interleaved SCAN split over the grid (k_scan_grid; -1 auto)
    int opt_w512 = -1;            // TRI_OPT_SCAN_W512: fp64 contiguous SCAN with 512-row windows (k_scan_w512; -1 auto)
    int G = 0, P = 0, rpt = 0;    // ONCHIP geometry
    int64_t n_pad = 0, L = 0, C = 0;  // SPLIT: chain length, chains
    int npass = 0;                // SPLIT: tiled-PCR passes (0 at k = 0)
    int kp[8] = {};               // SPLIT: PCR steps of each pass
    int pk[8] = {};               // SPLIT: kernel of each pass (trih::PassKind)
    int64_t Lp[8] = {}, Cp[8] = {};   // SPLIT: positions per chain, chains AFTER pass i
    // SPLIT: region length (rows / positions; tiles for the register kernels), regions per
    // system or chain block, chain blocks of pass i
    int64_t region[8] = {}, nreg[8] = {}, nblk[8] = {};
    int fu_grid = 0, fu_son = 0;  // FUSED: persistent CTAs, on-chip positions per chain
    bool fu_vec = false;          // FUSED: staged 8-row-aligned path
    int64_t fu_nc = 0;            // FUSED: windows per system
    int sk_grid = 0, sk_nc = 0, sk_son = 0;  // STREAM / SCAN: persistent CTAs, windows per system, resident slots
    int sk_delta = 8;             // SCAN: back-substitution lag (steps)
    int sk_S = 1;                 // SCAN: systems per window (1 contiguous; 8 interleaved)
    int s5 = 0;                   // SCAN through k_scan_w512 (sk_nc / sk_son then count 512-row windows / 8 KB slots)
    int sg_Q = 0, sg_R = 0, sg_bpb = 0;  // SCAN, k_scan_grid: CTAs per 32-system block, rows per warp, blocks per batch
    int64_t ms = 0;               // systems per batch (BATCHED / STRIDED; m otherwise)
    // element (system q = b ms + s, row i) at offset i es + s ss + b bs (elements) of
    // every array, for every layout: CONTIGUOUS (1, n, n m), INTERLEAVED (m, 1, n m),
    // BATCHED (ms, 1, n ms), STRIDED (caller's)
    int64_t es = 1, ss = 0, bs = 0, nb = 1;
    tri_plan_s* inner = nullptr;  // STRIDED, strides no TMA map can describe: packed CONTIGUOUS / INTERLEAVED plan
    void* packbuf = nullptr;      // ... and its 5 packed arrays
    size_t packbuf_bytes = 0;
    int mc_P = 0, mc_NCW = 0;     // SCAN_MC: chunks per system, windows per chunk
    int mc_lb = 0, mc_NCWs = 0, mc_Ps = 0;  // SCAN_MC look-back path: on, windows per small chunk, small chunks
    size_t smem_optin = 0;
    void* scratch = nullptr;
    size_t scratch_bytes = 0;
    void* stage = nullptr;        // tri_solve_host staging (5 arrays), lazily allocated
    size_t stage_bytes = 0;
    // tri_solve_host pipeline (CONTIGUOUS, m >= 2 HOST_CHUNKS): chunks of systems
    // flow H2D -> solve -> D2H on three streams; sub-plans for the chunk sizes
    tri_plan_s* sub[2] = {nullptr, nullptr};
    int64_t sub_m[2] = {0, 0};
    cudaStream_t hs[3] = {nullptr, nullptr, nullptr};
    cudaEvent_t ev[3 * trih::HOST_CHUNKS + 1] = {};
    const void* seen[8] = {};     // pointers whose device residency was last verified
    trih::TmCache tmc;
};

namespace trih {

// SPLIT pass kernels: the shared-memory sliding window of the paper (first pass
// on the user layout, later passes on chain-interleaved batches), or the
// register-resident tiles (k_pcr_reg.cuh: rows of the CONTIGUOUS layout, chains
// of a chain-interleaved batch, the user's INTERLEAVED rows)
enum PassKind { PK_RING = 0, PK_IL = 1, PK_ROWS = 2, PK_CHAINS = 3, PK_RAW = 4 };

inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }
inline size_t esize(tri_dtype t) { return t == TRI_F64 ? 8 : 4; }
inline int floor_log2(int64_t v) {
    int r = -1;
    while (v > 0) { v >>= 1; ++r; }
    return r;
}
inline int ceil_log2(int64_t v) {
    int r = 0;
    while ((int64_t(1) << r) < v) ++r;
    return r;
}

// ---- TMA descriptors (cuTensorMapEncodeTiled through the runtime's driver entry
// point: no link-time dependency on libcuda) ---------------------------------
// rank-R tiled map of elements of `es` bytes: dims[0] innermost; strides[i] =
// byte stride of dim i+1.  false if the encoder is unavailable or rejects it.
bool tma_encode(CUtensorMap* tm, size_t es, int rank, const void* base, const uint64_t* dims,
                const uint64_t* strides, const uint32_t* box, CUtensorMapSwizzle swz);

// Tensor maps for the plan's current launcher and pointer set: true (and
// `maps` filled from the cache) when `key[0..nkey)` and `tag` match the cached
// set; otherwise the caller encodes into `maps` and calls tm_store.
bool tm_lookup(tri_plan_s* p, int tag, const void* const* key, int nkey, CUtensorMap* maps, int nmaps);
void tm_store(tri_plan_s* p, int tag, const void* const* key, int nkey, const CUtensorMap* maps, int nmaps);

// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) once per (kernel, device,
// size): later launches with the same or a smaller size skip the call.
cudaError_t set_smem(const void* func, int bytes);

// ---- per-family launchers (one .cu file each) --------------------------------
// SCAN / SCAN_MC (l_scan.cu)
cudaError_t launch_scan(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                        cudaStream_t st);
cudaError_t launch_scan_mc(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                           cudaStream_t st);
cudaError_t launch_scan_mc_slice(tri_plan_s* p, int phase, int slice, int nslices, const void* a, const void* b,
                                 const void* c, const void* d, const void* maps, void* out, cudaStream_t st);
int scan_smem_fixed(tri_dtype t, int NC, int delta);  // SCLayout<T>::smem_bytes(NC, delta, 0)
int scan_slot_bytes(tri_dtype t);
int scan_in_stride(tri_dtype t);
int scan_mc_wmax();
// k_scan_grid: nblk clusters of Q CTAs (R rows per warp) all resident at once
bool scan_grid_fits(const tri_plan_s* p, int Q, int R, int64_t nblk);
int scan_mc_lb_maxw();
// STREAM (l_stream.cu)
cudaError_t launch_stream(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                          cudaStream_t st, void* ao, void* co, void* do_);
// FUSED (l_fused.cu)
cudaError_t launch_fused(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                         cudaStream_t st, void* dA, void* dC, void* dD);
int fused_smem_fixed(tri_dtype t, bool vec);
// WARP / ONCHIP (l_small.cu)
cudaError_t launch_warp(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                        void* ao, void* co, void* do_, int mode, cudaStream_t st);
cudaError_t launch_onchip(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                          void* ao, void* co, void* do_, int mode, cudaStream_t st);
// SPLIT: tiled-PCR passes + p-Thomas (l_split.cu)
cudaError_t launch_split(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* x,
                         cudaStream_t st);
cudaError_t launch_split_pcr(tri_plan_s* p, const void* a, const void* b, const void* c, const void* d, void* ao,
                             void* co, void* do_, cudaStream_t st);  // tri_debug_pcr: the PCR passes only
void split_geometry(tri_plan_s* p);
// STRIDED fallback (l_strided.cu): gather a, b, c, d into the inner plan's layout,
// scatter its x back (one thread per element)
cudaError_t launch_pack(const tri_plan_s* p, const void* const src[4], void* const dst[4], cudaStream_t st);
cudaError_t launch_unpack(const tri_plan_s* p, const void* src, void* dst, cudaStream_t st);
size_t split_scratch(const tri_plan_s* p);

extern void* g_fused_prof;    // tri_debug_set_profile: device counters (diagnostics)
extern int g_fused_dbg_mode;  // TRI_FUSED_DBG_MODE read by tri_debug_set_profile (diagnostics)

}  // namespace trih
