// Microbenchmark: register PCR throughput per SM for the streaming kernel design.
// Each warp repeatedly: reads a 256-row window (8 rows/lane, blocked, swizzled) from
// shared memory, normalises, K PCR levels with shuffles, writes the reduced rows
// chain-major to a per-warp smem buffer.  Reports rows/clk/SM (valid rows).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I../../paper_conf_icpp_kimwch11_b200/csrc pcr3.cu
#include <cstdio>
#include <cuda_runtime.h>
#include "common.cuh"
using namespace tri;

__device__ __forceinline__ double rcp3(double x) {  // MUFU + one cubic Newton step
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
    double e = fma(-x, r, 1.0);
    double t = fma(e, e, e);
    return fma(r, t, r);
}

template <int RC>
__device__ __forceinline__ double rc(double x) { return RC == 0 ? rcp(x) : rcp3(x); }

template <int RC>
__device__ __forceinline__ NRow<double> comb(const NRow<double>& m, const NRow<double>& o, const NRow<double>& p) {
    double bp = fma(-o.A, m.C, fma(-o.C, p.A, 1.0));
    double dp = fma(-o.A, m.D, fma(-o.C, p.D, o.D));
    double r = rc<RC>(bp);
    NRow<double> out;
    out.A = (-o.A * m.A) * r;
    out.C = (-o.C * p.C) * r;
    out.D = dp * r;
    return out;
}

template <int K, int RC>
__device__ __forceinline__ void pcr(NRow<double> (&v)[8]) {
#pragma unroll
    for (int j = 0; j < K; ++j) {
        const int sg = 1 << j;
        NRow<double> nv[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            NRow<double> mm, pp;
            if (u - sg >= 0) mm = v[u - sg];
            else {
                const NRow<double>& s = v[(u - sg + 64) % 8];
                const int dl = (sg + 7) / 8 > 0 ? ((u - sg) >= -8 ? 1 : 2) : 1;
                mm.A = __shfl_up_sync(0xffffffffu, s.A, dl);
                mm.C = __shfl_up_sync(0xffffffffu, s.C, dl);
                mm.D = __shfl_up_sync(0xffffffffu, s.D, dl);
            }
            if (u + sg < 8) pp = v[u + sg];
            else {
                const NRow<double>& s = v[(u + sg) % 8];
                const int dl = (u + sg) < 16 ? 1 : 2;
                pp.A = __shfl_down_sync(0xffffffffu, s.A, dl);
                pp.C = __shfl_down_sync(0xffffffffu, s.C, dl);
                pp.D = __shfl_down_sync(0xffffffffu, s.D, dl);
            }
            nv[u] = comb<RC>(mm, v[u], pp);
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) v[u] = nv[u];
    }
}

template <int K, int NW, int RC, int OUT>
__global__ void __launch_bounds__(NW * 32, 1) bench(double* out, long long* cyc, int windows) {
    extern __shared__ __align__(16) double sm[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    double* st = sm;
    double* hand = sm + 4 * 256 + warp * 3 * 256;
    if (warp == 0) for (int e = lane; e < 4 * 256; e += 32) st[e] = (e % 256) * 1e-3 + (e / 256 == 1 ? 3.0 : 0.1);
    __syncthreads();
    const int swz = (lane >> 1) & 3;
    NRow<double> acc{0, 0, 0};
    long long t0 = clock64();
    for (int w = 0; w < windows; ++w) {
        NRow<double> v[8];
        const double* s2 = st + lane * 8;
#pragma unroll
        for (int cc = 0; cc < 4; ++cc) {
            double raw[4][2];
#pragma unroll
            for (int arr = 0; arr < 4; ++arr) {
                const double2 q = *reinterpret_cast<const double2*>(s2 + arr * 256 + ((cc ^ swz) & 3) * 2);
                raw[arr][0] = q.x;
                raw[arr][1] = q.y;
            }
#pragma unroll
            for (int e = 0; e < 2; ++e) {
                const double r = rc<RC>(raw[1][e] + w);
                v[cc * 2 + e] = NRow<double>{raw[0][e] * r, raw[2][e] * r, raw[3][e] * r};
            }
        }
        pcr<K, RC>(v);
        if (OUT) {
            // chain-major handoff: row i = 8 lane + u -> chain i % S, position i / S
            constexpr int S = 1 << K;
            constexpr int P = 256 / S;
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                const int i = lane * 8 + u;
                const int ch = i % S, t = i / S;
                hand[ch * P + t] = v[u].A;
                hand[256 + ch * P + t] = v[u].C;
                hand[512 + ch * P + t] = v[u].D;
            }
            __syncwarp();
            acc.A += hand[lane];
        } else {
#pragma unroll
            for (int u = 0; u < 8; ++u) { acc.A += v[u].A; acc.C += v[u].C; acc.D += v[u].D; }
        }
    }
    long long t1 = clock64();
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc.A + acc.C + acc.D;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int K, int NW, int RC, int OUT>
void run(double* out, long long* cyc) {
    const int windows = 256, ctas = 148;
    const int smem = (4 * 256 + NW * 3 * 256) * 8;
    auto kern = bench<K, NW, RC, OUT>;
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    kern<<<ctas, NW * 32, smem>>>(out, cyc, windows);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<<<ctas, NW * 32, smem>>>(out, cyc, windows);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    long long h[148];
    cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < ctas; ++i) avg += h[i];
    avg /= ctas;
    const double halo = 2.0 * (1 << K);
    const double rows = (double)NW * windows * (256 - halo);
    printf("K=%d NW=%2d rcp=%s out=%d: %7.0f cyc/window/warp, %.3f valid rows/clk/SM (%.3f ms)  %s\n", K, NW,
           RC ? "cubic" : "2newton", OUT, avg / windows, rows / avg, ms, cudaGetErrorString(cudaGetLastError()));
}

int main() {
    double* out;
    long long* cyc;
    cudaMalloc(&out, 148 * 1024 * 8);
    cudaMalloc(&cyc, 148 * 8);
    run<3, 8, 0, 0>(out, cyc);
    run<3, 8, 1, 0>(out, cyc);
    run<3, 12, 1, 0>(out, cyc);
    run<3, 16, 1, 0>(out, cyc);
    run<3, 8, 1, 1>(out, cyc);
    run<3, 12, 1, 1>(out, cyc);
    run<3, 16, 1, 1>(out, cyc);
    run<4, 8, 1, 0>(out, cyc);
    run<4, 12, 1, 0>(out, cyc);
    run<4, 16, 1, 1>(out, cyc);
    run<4, 12, 1, 1>(out, cyc);
    return 0;
}
