// Microbenchmark: one warp doing the fused kernel's back-substitution batch loop
// (16 positions x 8 chains per batch from shared memory, FMA chain, x stores),
// alone on the SM or next to 2 fp64-busy warps on its SMSP.
#include <cstdio>
#include <cuda_runtime.h>
constexpr int U = 16, S = 8;

template <int STORE, int NOISE>
__global__ void bench(double* x, long long* cyc, int batches) {
    __shared__ __align__(16) double st[256 * S * 2];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int e = threadIdx.x; e < 256 * S * 2; e += blockDim.x) st[e] = (e & 1) ? 1e-3 * (e & 15) : 0.3;
    __syncthreads();
    if (warp != 0) {  // fp64-busy neighbours on the same SMSP (warps 4, 8)
        if (NOISE && (warp % 4) == 0) {
            double a = lane, b = 1.0000001;
            for (int i = 0; i < batches * 64; ++i) {
#pragma unroll
                for (int j = 0; j < 8; ++j) a = fma(a, b, 1e-9);
            }
            x[1000000 + threadIdx.x] = a;
        }
        return;
    }
    const int r = lane & 7;
    double xv = 0;
    double* xp = x + r + (long long)blockIdx.x * 65536;
    long long t0 = clock64();
    const double* base = st + r * 2;
    double cs[U], ds[U];
#pragma unroll
    for (int u = 0; u < U; ++u) { const double2 v = *reinterpret_cast<const double2*>(base + u * S * 2); cs[u] = v.x; ds[u] = v.y; }
    for (int bi = 0; bi < batches; ++bi) {
        double c0[U], d0[U];
#pragma unroll
        for (int u = 0; u < U; ++u) { c0[u] = cs[u]; d0[u] = ds[u]; }
        const double* p = base + ((bi + 1) % 16) * U * S * 2;
#pragma unroll
        for (int u = 0; u < U; ++u) { const double2 v = *reinterpret_cast<const double2*>(p + u * S * 2); cs[u] = v.x; ds[u] = v.y; }
        double xs[U];
#pragma unroll
        for (int u = 0; u < U; ++u) { xv = fma(-c0[u], xv, d0[u]); xs[u] = xv; }
        if (STORE && lane < 8) {
#pragma unroll
            for (int u = 0; u < U; ++u) xp[(bi % 256) * U * S + u * S] = xs[u];
        }
    }
    long long t1 = clock64();
    if (lane == 0) cyc[blockIdx.x] = t1 - t0;
    if (!STORE) x[lane] = xv;
}

int main() {
    double* x;
    long long* cyc;
    long long h;
    cudaMalloc(&x, 148 * 65536 * 8 + 8 * 1000000 * 2);
    cudaMalloc(&cyc, 148 * 8);
    const int B = 1000;
    auto run = [&](auto k, const char* name) {
        k<<<148, 384>>>(x, cyc, B);
        k<<<148, 384>>>(x, cyc, B);
        cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
        printf("%-40s %.1f cycles/batch (%.1f per position)\n", name, (double)h / B, (double)h / B / U);
    };
    run(bench<0, 0>, "no stores, alone");
    run(bench<1, 0>, "stores, alone");
    run(bench<0, 1>, "no stores, 2 fp64 warps on SMSP");
    run(bench<1, 1>, "stores, 2 fp64 warps on SMSP");
    printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
