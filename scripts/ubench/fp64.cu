// Microbenchmarks: fp64 DFMA / MUFU.RCP64H latency and per-SMSP throughput,
// SHFL and LDS throughput, on the B200 (sm_100a).  nvcc -arch=sm_100a -O3.
#include <cstdio>
#include <cuda_runtime.h>

__global__ void dfma_lat(double* out, long long* cyc, int iters) {
    double x = threadIdx.x * 1e-3 + 1.0, y = 0.999999, z = 1e-9;
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int u = 0; u < 16; ++u) x = fma(x, y, z);
    }
    long long t1 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) *cyc = t1 - t0;
}
template <int ILP>
__global__ void dfma_tput(double* out, long long* cyc, int iters) {
    double x[ILP];
#pragma unroll
    for (int j = 0; j < ILP; ++j) x[j] = threadIdx.x * 1e-3 + j;
    const double y = 0.999999, z = 1e-9;
    __syncthreads();
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < ILP; ++j) x[j] = fma(x[j], y, z);
    }
    __syncthreads();
    long long t1 = clock64();
    double s = 0;
#pragma unroll
    for (int j = 0; j < ILP; ++j) s += x[j];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
__global__ void rcp_lat(double* out, long long* cyc, int iters) {
    double x = threadIdx.x * 1e-3 + 1.5;
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int u = 0; u < 16; ++u) {
            double r;
            asm volatile("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
            x = r + 1.0;
        }
    }
    long long t1 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) *cyc = t1 - t0;
}
template <int ILP>
__global__ void rcp_tput(double* out, long long* cyc, int iters) {
    double x[ILP];
#pragma unroll
    for (int j = 0; j < ILP; ++j) x[j] = threadIdx.x * 1e-3 + j + 1.5;
    __syncthreads();
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < ILP; ++j) {
            double r;
            asm volatile("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x[j]));
            x[j] = r;
        }
    }
    __syncthreads();
    long long t1 = clock64();
    double s = 0;
#pragma unroll
    for (int j = 0; j < ILP; ++j) s += x[j];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
template <int ILP>
__global__ void shfl_tput(double* out, long long* cyc, int iters) {
    double x[ILP];
#pragma unroll
    for (int j = 0; j < ILP; ++j) x[j] = threadIdx.x * 1e-3 + j;
    __syncthreads();
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < ILP; ++j) x[j] = __shfl_down_sync(0xffffffffu, x[j], 1);
    }
    __syncthreads();
    long long t1 = clock64();
    double s = 0;
#pragma unroll
    for (int j = 0; j < ILP; ++j) s += x[j];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

int main() {
    double* out;
    long long *cyc, h[4096];
    cudaMalloc(&out, 1 << 24);
    cudaMalloc(&cyc, 4096 * 8);
    const int it = 4096;
    dfma_lat<<<1, 32>>>(out, cyc, it);
    cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("DFMA dependent latency: %.2f cycles\n", (double)h[0] / (it * 16));
    rcp_lat<<<1, 32>>>(out, cyc, it);
    cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("MUFU.RCP64H + DADD dependent latency: %.2f cycles\n", (double)h[0] / (it * 16));
    for (int warps : {1, 2, 4, 8, 16}) {
        dfma_tput<8><<<1, 32 * warps>>>(out, cyc, it);
        cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
        printf("DFMA throughput, %2d warps x ILP8 on one SM: %.3f warp-instr/cycle/SM (%.1f lanes/clk)\n", warps,
               (double)warps * it * 8 / h[0], 32.0 * warps * it * 8 / h[0]);
    }
    for (int warps : {1, 4, 8}) {
        rcp_tput<8><<<1, 32 * warps>>>(out, cyc, it);
        cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
        printf("RCP64H throughput, %2d warps x ILP8: %.3f warp-instr/cycle/SM\n", warps, (double)warps * it * 8 / h[0]);
    }
    for (int warps : {1, 4, 8}) {
        shfl_tput<8><<<1, 32 * warps>>>(out, cyc, it);
        cudaMemcpy(h, cyc, 8, cudaMemcpyDeviceToHost);
        printf("SHFL(f64 = 2 SHFL) throughput, %2d warps x ILP8: %.3f f64-shuffles(warp)/cycle/SM\n", warps,
               (double)warps * it * 8 / h[0]);
    }
    cudaError_t e = cudaDeviceSynchronize();
    printf("status %s\n", cudaGetErrorString(e));
    return 0;
}
