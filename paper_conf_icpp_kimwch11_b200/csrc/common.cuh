// common.cuh -- device helpers shared by the sm_100a kernels of the solver.
// Part of the CUDA path only; nothing here is shared with oracle/.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace tri {

__host__ __device__ __forceinline__ int64_t imin64(int64_t a, int64_t b) { return a < b ? a : b; }
__host__ __device__ __forceinline__ int64_t imax64(int64_t a, int64_t b) { return a > b ? a : b; }

// Reciprocal used for every division of the method (Eqs 2-6).  fp64: MUFU seed
// (rcp.approx, relative error e0 < 2^-22) refined by one cubic Newton step on the
// FMA pipe, r (1 + e + e^2) with e = 1 - x r: error O(e0^3) below fp64 rounding,
// ~1 ulp, three dependent FMAs; fp32: the MUFU result itself (<= 1 ulp, far
// inside the 1e-4 fp32 tolerance).  Pure mantissa arithmetic, so scaling the
// argument by 2^p scales the result by 2^-p exactly (metamorphic tests rely on
// it).  Inputs are pivots of diagonally dominant systems: never 0/denormal.
__device__ __forceinline__ double rcp(double x) {
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
    const double e = fma(-x, r, 1.0);
    return fma(r, fma(e, e, e), r);
}
__device__ __forceinline__ float rcp(float x) {
    float r;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
    return r;
}

template <typename T>
__device__ __forceinline__ T ldg_stream(const T* p) {
    return __ldcs(p);  // evict-first streaming load: inputs are read once
}

// A row of the system normalised to unit diagonal: A x_{i-s} + x_i + C x_{i+s} = D.
// (a/b, c/b, d/b) -- scaling a row by 1/b_i is a row operation; X17.
template <typename T>
struct NRow {
    T A, C, D;
};

template <typename T>
__device__ __forceinline__ NRow<T> identity_row() {
    return NRow<T>{T(0), T(0), T(0)};
}

// Normalise a raw row (a, b, c, d) -> (a/b, c/b, d/b) with one reciprocal.
template <typename T>
__device__ __forceinline__ NRow<T> normalise(T a, T b, T c, T d) {
    T r = rcp(b);
    return NRow<T>{a * r, c * r, d * r};
}

// One PCR step (Eqs 5-6, at stride s; reading X3) on normalised rows:
// row i combines with rows i-s (m) and i+s (p):
//   k1 = a_i/b_{i-s}, k2 = c_i/b_{i+s}  -> with b == 1 these are A_i, C_i and
//   a'_i = -A_i A_m,  c'_i = -C_i C_p,  b'_i = 1 - A_i C_m - C_i A_p,
//   d'_i = D_i - A_i D_m - C_i D_p,     then renormalise by 1/b'_i.
// Out-of-range neighbours are identity rows (reading X4): all-zero NRow.
template <typename T>
__device__ __forceinline__ NRow<T> pcr_combine(const NRow<T>& m, const NRow<T>& o, const NRow<T>& p) {
    T bp = fma(-o.A, m.C, fma(-o.C, p.A, T(1)));
    T dp = fma(-o.A, m.D, fma(-o.C, p.D, o.D));
    T r = rcp(bp);
    NRow<T> out;
    out.A = (-o.A * m.A) * r;
    out.C = (-o.C * p.C) * r;
    out.D = dp * r;
    return out;
}

// Raw row (a, b, c, d) of Eq 1.
template <typename T>
struct Row4 {
    T a, b, c, d;
};

// Thomas forward step (Eqs 2-3) on a raw row:
//   den = b - a c'_{prev};  c' = c/den;  d' = (d - a d'_{prev})/den.
template <typename T>
__device__ __forceinline__ void thomas_fwd(const Row4<T>& r, T& cp, T& dp) {
    T den = fma(-r.a, cp, r.b);
    T inv = rcp(den);
    cp = r.c * inv;
    dp = fma(-r.a, dp, r.d) * inv;
}

// Thomas forward step (Eqs 2-3) on a normalised row, given the previous c', d':
//   den = 1 - A c'_{prev};  c' = C/den;  d' = (D - A d'_{prev})/den.
template <typename T>
__device__ __forceinline__ void thomas_fwd(const NRow<T>& r, T& cp, T& dp) {
    T den = fma(-r.A, cp, T(1));
    T inv = rcp(den);
    cp = r.C * inv;
    dp = fma(-r.A, dp, r.D) * inv;
}

__host__ __device__ __forceinline__ int64_t elem_index(int64_t q, int64_t i, int64_t n, int64_t m, int layout) {
    return layout == 0 ? q * n + i : i * m + q;
}

}  // namespace tri

namespace tri {

// ---- cp.async (LDGSTS) helpers: global -> shared without a register round trip
__device__ __forceinline__ void cp_async_16(void* smem, const void* gmem, int src_bytes) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(s), "l"(gmem), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cp_async_8(void* smem, const void* gmem, int src_bytes) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(s), "l"(gmem), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cp_async_4(void* smem, const void* gmem, int src_bytes) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(s), "l"(gmem), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

}  // namespace tri

namespace tri {

// ---- TMA bulk copy shared -> global (cp.async.bulk, bulk_group completion)
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void bulk_store_s2g(void* gdst, const void* ssrc, unsigned bytes) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(ssrc);
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst), "r"(s), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait() {
    asm volatile("cp.async.bulk.wait_group %0;" ::"n"(N) : "memory");
}

}  // namespace tri
