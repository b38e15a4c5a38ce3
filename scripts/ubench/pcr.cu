// Microbenchmark: the fused kernel's register PCR (k = 3 levels on 8 rows per
// lane) in isolation, no memory traffic.  Cycles per window per warp vs warps/SM.
#include <cstdio>
#include <cuda_runtime.h>
#include "common.cuh"
using namespace tri;

template <int K>
__device__ __forceinline__ void pcr_levels(NRow<double> (&v)[8]) {
#pragma unroll
    for (int j = 0; j < K; ++j) {
        const int sg = 1 << j;
        NRow<double> nv[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            NRow<double> mm, pp;
            if (u - sg >= 0) mm = v[u - sg];
            else {
                const NRow<double>& s = v[u - sg + 8];
                mm.A = __shfl_up_sync(0xffffffffu, s.A, 1);
                mm.C = __shfl_up_sync(0xffffffffu, s.C, 1);
                mm.D = __shfl_up_sync(0xffffffffu, s.D, 1);
            }
            if (u + sg < 8) pp = v[u + sg];
            else {
                const NRow<double>& s = v[u + sg - 8];
                pp.A = __shfl_down_sync(0xffffffffu, s.A, 1);
                pp.C = __shfl_down_sync(0xffffffffu, s.C, 1);
                pp.D = __shfl_down_sync(0xffffffffu, s.D, 1);
            }
            nv[u] = pcr_combine(mm, v[u], pp);
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) v[u] = nv[u];
    }
}

template <int K>
__global__ void bench(double* out, long long* cyc, int iters) {
    NRow<double> v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = NRow<double>{0.1 + 1e-3 * u, 0.2 - 1e-3 * threadIdx.x, 1.0 + u};
    __syncthreads();
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
        // fresh "window": normalise-like perturbation keeps values bounded
#pragma unroll
        for (int u = 0; u < 8; ++u) { v[u].A *= 0.5; v[u].C *= 0.5; }
        pcr_levels<K>(v);
    }
    __syncthreads();
    long long t1 = clock64();
    double s = 0;
#pragma unroll
    for (int u = 0; u < 8; ++u) s += v[u].A + v[u].C + v[u].D;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

int main() {
    double* out;
    long long *cyc, h[8];
    cudaMalloc(&out, 1 << 22);
    cudaMalloc(&cyc, 64);
    const int it = 2000;
    for (int warps : {1, 2, 4, 5, 8}) {
        bench<3><<<1, 32 * warps>>>(out, cyc, it);
        cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
        printf("K=3: %d warps/SM: %.0f cycles per window per warp, %.1f cycles per window per SM\n", warps,
               (double)h[0] / it, (double)h[0] / it / warps);
    }
    for (int warps : {1, 4, 8}) {
        bench<4><<<1, 32 * warps>>>(out, cyc, it);
        cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
        printf("K=4: %d warps/SM: %.0f cycles per window per warp, %.1f per SM\n", warps, (double)h[0] / it,
               (double)h[0] / it / warps);
    }
    printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    return 0;
}
