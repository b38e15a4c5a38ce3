// Microbenchmark: the fused kernel's PCR-warp loop pieces, 8 warps per SM, to
// find where the per-window time goes: (0) PCR only, (1) + smem read/normalise,
// (2) + cp.async staging from HBM, (3) + handoff stores.
#include <cstdio>
#include <cuda_runtime.h>
#include "common.cuh"
using namespace tri;
constexpr int R = 8, W = 256, EPC = 2, CPL = 4;

__device__ __forceinline__ void pcr3(NRow<double> (&v)[8]) {
#pragma unroll
    for (int j = 0; j < 3; ++j) {
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

template <int MODE>
__global__ void __launch_bounds__(256, 1) bench(const double* a, const double* b, const double* c, const double* d,
                                                double* out, long long* cyc, int windows) {
    extern __shared__ __align__(16) double sm[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    double* st = sm + warp * 4 * W;
    double* hand = sm + 8 * 4 * W + warp * 3 * W;
    const int swz = (lane >> 1) & 3;
    const long long base0 = ((long long)blockIdx.x * 8 + warp) * (long long)windows * W;
    auto issue = [&](int w) {
        if (MODE >= 2 && w < windows) {
            const long long base = base0 + (long long)w * W;
#pragma unroll
            for (int arr = 0; arr < 4; ++arr) {
                const double* src = arr == 0 ? a : arr == 1 ? b : arr == 2 ? c : d;
#pragma unroll
                for (int j = 0; j < W / EPC / 32; ++j) {
                    const int ci = lane + 32 * j, o = ci / CPL, cc = ci % CPL;
                    const int os = (o >> 1) & 3;
                    cp_async_16(st + arr * W + o * R + (cc ^ os) * EPC, src + base + ci * EPC, 16);
                }
            }
        }
        cp_async_commit();
    };
    // initialise the stage once for modes 0/1
    for (int e = lane; e < 4 * W; e += 32) st[e] = (e % W) * 1e-3 + (e / W == 1 ? 3.0 : 0.1);
    __syncwarp();
    NRow<double> v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = NRow<double>{0.1, 0.2, 1.0 + u};
    issue(0);
    long long t0 = clock64();
    for (int w = 0; w < windows; ++w) {
        if (MODE >= 1) {
            cp_async_wait<0>();
            __syncwarp();
            const double* s2 = st + lane * R;
#pragma unroll
            for (int cc = 0; cc < CPL; ++cc) {
                double raw[4][EPC];
#pragma unroll
                for (int arr = 0; arr < 4; ++arr) {
                    const int4 q = *reinterpret_cast<const int4*>(s2 + arr * W + (cc ^ swz) * EPC);
                    const double* qt = reinterpret_cast<const double*>(&q);
                    raw[arr][0] = qt[0];
                    raw[arr][1] = qt[1];
                }
#pragma unroll
                for (int e = 0; e < EPC; ++e) v[cc * EPC + e] = normalise(raw[0][e], raw[1][e], raw[2][e], raw[3][e]);
            }
            __syncwarp();
            issue(w + 1);
        } else {
#pragma unroll
            for (int u = 0; u < 8; ++u) { v[u].A *= 0.5; v[u].C *= 0.5; }
        }
        pcr3(v);
        if (MODE >= 3) {
            const int t = lane - 1;
            if (t >= 0 && t < 30) {
                double* hs = hand + t;
#pragma unroll
                for (int u = 0; u < 8; ++u) {
                    hs[u * 30] = v[u].A;
                    hs[(8 + u) * 30] = v[u].C;
                    hs[(16 + u) * 30] = v[u].D;
                }
            }
            __syncwarp();
        }
    }
    long long t1 = clock64();
    double s = 0;
#pragma unroll
    for (int u = 0; u < 8; ++u) s += v[u].A + v[u].C + v[u].D;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (lane == 0) cyc[blockIdx.x * 8 + warp] = t1 - t0;
}

int main() {
    const int windows = 64, ctas = 148;
    const size_t N = (size_t)ctas * 8 * windows * W;
    double *a, *b, *c, *d, *out;
    long long* cyc;
    cudaMalloc(&a, N * 8); cudaMalloc(&b, N * 8); cudaMalloc(&c, N * 8); cudaMalloc(&d, N * 8);
    cudaMemset(a, 0, N * 8); cudaMemset(c, 0, N * 8); cudaMemset(d, 0, N * 8);
    {
        double* hb = (double*)malloc(N * 8);
        for (size_t i = 0; i < N; ++i) hb[i] = 2.0;
        cudaMemcpy(b, hb, N * 8, cudaMemcpyHostToDevice);
        free(hb);
    }
    cudaMalloc(&out, ctas * 256 * 8);
    cudaMalloc(&cyc, ctas * 8 * 8);
    const int smem = (8 * 4 * W + 8 * 3 * W) * 8;
    long long h[148 * 8];
    auto run = [&](auto kern, const char* name) {
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        kern<<<ctas, 256, smem>>>(a, b, c, d, out, cyc, windows);
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0); cudaEventCreate(&e1);
        cudaEventRecord(e0);
        kern<<<ctas, 256, smem>>>(a, b, c, d, out, cyc, windows);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < ctas * 8; ++i) avg += h[i];
        avg /= ctas * 8;
        printf("%-34s %7.0f cycles/window/warp  %.3f ms  %.0f GB/s input\n", name, avg / windows, ms,
               4.0 * N * 8 / ms / 1e6);
    };
    run(bench<0>, "PCR only");
    run(bench<1>, "+ smem read & normalise");
    run(bench<2>, "+ cp.async staging from HBM");
    run(bench<3>, "+ handoff stores");
    printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
