// Microbenchmark: the continuant chain (X18) of the STREAM kernel's TC warp,
// one warp alone on an SM: (0) chain on register data, (1) + 3 STS per
// position, (2) + LDS of the inputs from a chain-major slot, (3) two
// positions per step (2x2 transfer), on register data.
#include <cstdio>
#include <cuda_runtime.h>
constexpr int P = 30, S = 8, V = 240;

template <int MODE>
__global__ void bench(double* out, long long* cyc, int windows) {
    __shared__ __align__(16) double hand[3 * V];
    __shared__ __align__(16) double scr[3 * V];
    const int lane = threadIdx.x & 31;
    for (int e = threadIdx.x; e < 3 * V; e += blockDim.x) hand[e] = 0.01 * (e % 7) + (e >= 2 * V ? 1.0 : 0.0);
    __syncthreads();
    const int c = lane & 7;
    double th1 = 1, th2 = 1, de1 = 0, Cp = 0;
    double Ar[P], Cr[P], Dr[P];
#pragma unroll
    for (int t = 0; t < P; ++t) { Ar[t] = 0.01 * (t % 5) + lane * 1e-4; Cr[t] = 0.02 * (t % 3); Dr[t] = 1.0 + t * 1e-3; }
    long long t0 = clock64();
    for (int w = 0; w < windows; ++w) {
        if (MODE == 2) {
            const double* hs = hand + c * P;
#pragma unroll
            for (int t = 0; t < P; t += 2) {
                double2 a = *reinterpret_cast<const double2*>(hs + t);
                double2 cc = *reinterpret_cast<const double2*>(hs + V + t);
                double2 d = *reinterpret_cast<const double2*>(hs + 2 * V + t);
                Ar[t] = a.x; Ar[t + 1] = a.y; Cr[t] = cc.x; Cr[t + 1] = cc.y; Dr[t] = d.x; Dr[t + 1] = d.y;
            }
        }
        if (MODE == 3) {
#pragma unroll
            for (int t = 0; t < P; t += 2) {
                // (th_{t+1}, th_t) from (th_{t-1}, th_{t-2}): th_t = th1 + x_t th2, th_{t+1} = th_t + x_{t+1} th1
                const double x0 = -Ar[t] * Cp, x1 = -Ar[t + 1] * Cr[t];
                const double a11 = 1.0 + x1, b1 = x1 * 0.0 + x0;  // placeholder algebra kept cheap
                const double th = fma(x0, th2, th1);
                const double thn = fma(a11, th1, b1 * th2);
                th2 = th; th1 = thn;
                Cp = Cr[t + 1];
            }
        } else {
#pragma unroll
            for (int t = 0; t < P; ++t) {
                const double th = fma(-Ar[t] * Cp, th2, th1);
                const double de = fma(-Ar[t], de1, Dr[t] * th1);
                const double gg = Cr[t] * th1;
                if (MODE >= 1 && lane < S) {
                    scr[t * S + c] = gg;
                    scr[V + t * S + c] = th;
                    scr[2 * V + t * S + c] = de;
                }
                th2 = th1; th1 = th; de1 = de; Cp = Cr[t];
            }
        }
        const long long bits = __double_as_longlong(th1);
        const double sc = __longlong_as_double((long long)(1023 - ((int)((bits >> 52) & 0x7ff) - 1023)) << 52);
        th1 *= sc; th2 *= sc; de1 *= sc;
        __syncwarp();
    }
    long long t1 = clock64();
    if (lane == 0) { cyc[blockIdx.x] = t1 - t0; out[blockIdx.x] = th1 + de1 + scr[lane] + scr[5]; }
}

int main() {
    double* out; long long* cyc; long long h;
    cudaMalloc(&out, 4096); cudaMalloc(&cyc, 4096);
    const int W = 2000;
    bench<0><<<148, 32>>>(out, cyc, W); bench<0><<<148, 32>>>(out, cyc, W);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("chain only (registers):      %.0f cycles/window\n", (double)h / W);
    bench<1><<<148, 32>>>(out, cyc, W); bench<1><<<148, 32>>>(out, cyc, W);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("+ 3 STS per position:        %.0f cycles/window\n", (double)h / W);
    bench<2><<<148, 32>>>(out, cyc, W); bench<2><<<148, 32>>>(out, cyc, W);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("+ LDS of the window:         %.0f cycles/window\n", (double)h / W);
    bench<3><<<148, 32>>>(out, cyc, W); bench<3><<<148, 32>>>(out, cyc, W);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("two positions per step:      %.0f cycles/window\n", (double)h / W);
    printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
