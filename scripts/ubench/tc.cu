// Microbenchmark: the fused kernel's chain-warp (TC) window loop in isolation:
// 30 positions x 8 chains from a chain-major handoff slot, continuant recurrence,
// (theta, delta) pairs to a scratch buffer.  Optionally with the mbarrier
// handshakes of the real kernel (a partner warp that immediately acknowledges).
#include <cstdio>
#include <cuda_runtime.h>
#include "common.cuh"
__device__ __forceinline__ void fu_ld2_ub(const double* s, double& a, double& b) { const double2 v = *reinterpret_cast<const double2*>(s); a = v.x; b = v.y; }
using namespace tri;
constexpr int S = 8, PPC = 30, TCH = 10;

__device__ __forceinline__ void mbar_init(uint64_t* bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"((unsigned)__cvta_generic_to_shared(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, unsigned parity) {
    const unsigned a = (unsigned)__cvta_generic_to_shared(bar);
    asm volatile("{\n.reg .pred P1;\nWAIT_%=:\nmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 P1, [%0], %1;\n@!P1 bra WAIT_%=;\n}\n" ::"r"(a), "r"(parity) : "memory");
}

template <int SYNC>
__global__ void bench(double* out, long long* cyc, int windows) {
    __shared__ __align__(16) double hand[4][3 * S * PPC];
    __shared__ __align__(16) double scr[2][(PPC + 1) * S * 2];
    __shared__ uint64_t full[4], empty[4];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int e = threadIdx.x; e < 4 * 3 * S * PPC; e += blockDim.x) (&hand[0][0])[e] = 0.01 * (e % 7) + ((e / (S * PPC)) % 3 == 2 ? 1.0 : 0.0);
    if (threadIdx.x == 0) for (int s = 0; s < 4; ++s) { mbar_init(&full[s], 32); mbar_init(&empty[s], 32); }
    __syncthreads();
    if (warp == 1) {  // partner: produces "full" and consumes "empty" immediately
        if (SYNC) for (int g = 0; g < windows; ++g) {
            const int slot = g & 3;
            mbar_wait(&empty[slot], ((g >> 2) & 1) ^ 1);
            mbar_arrive(&full[slot]);
        }
        return;
    }
    if (warp != 0) return;
    const int r = lane & 7;
    const bool w8 = lane < 8;
    double th1 = 1, th2 = 1, del1 = 0, Cprev = 0;
    long long t0 = clock64();
    for (int g = 0; g < windows; ++g) {
        const int slot = g & 3;
        if (SYNC) mbar_wait(&full[slot], (g >> 2) & 1);
        const double* hs = hand[slot] + r * PPC;
        double* ss = scr[g & 1] + r * 2;
        if (w8) { ss[0] = th1; ss[1] = del1; }
        // rolled chunk loop: the next chunk's loads are loop-carried, so ptxas
        // cannot sink them next to their uses (it cannot move them past the back-edge)
        double An[TCH], Cn[TCH], Dn[TCH];
#pragma unroll
        for (int t = 0; t < TCH; t += 2) {
            fu_ld2_ub(hs + t, An[t], An[t + 1]);
            fu_ld2_ub(hs + S * PPC + t, Cn[t], Cn[t + 1]);
            fu_ld2_ub(hs + 2 * S * PPC + t, Dn[t], Dn[t + 1]);
        }
#pragma unroll 1
        for (int ch = 0; ch < PPC / TCH; ++ch) {
            double Ac[TCH], Cc[TCH], Dc[TCH];
#pragma unroll
            for (int t = 0; t < TCH; ++t) { Ac[t] = An[t]; Cc[t] = Cn[t]; Dc[t] = Dn[t]; }
            const int nx = (ch + 1 < PPC / TCH) ? (ch + 1) * TCH : 0;
#pragma unroll
            for (int t = 0; t < TCH; t += 2) {
                fu_ld2_ub(hs + nx + t, An[t], An[t + 1]);
                fu_ld2_ub(hs + S * PPC + nx + t, Cn[t], Cn[t + 1]);
                fu_ld2_ub(hs + 2 * S * PPC + nx + t, Dn[t], Dn[t + 1]);
            }
            double thv[TCH], dev[TCH];
#pragma unroll
            for (int e = 0; e < TCH; ++e) {
                const double th = fma(-Ac[e] * Cprev, th2, th1);
                const double de = fma(-Ac[e], del1, Dc[e] * th1);
                thv[e] = th; dev[e] = de;
                th2 = th1; th1 = th; del1 = de; Cprev = Cc[e];
            }
            if (w8) {
#pragma unroll
                for (int e = 0; e < TCH; ++e) { double2* d2 = reinterpret_cast<double2*>(ss + (ch * TCH + e + 1) * S * 2); *d2 = make_double2(thv[e], dev[e]); }
            }
        }
        const long long bits = __double_as_longlong(th1);
        const double sc = __longlong_as_double((long long)(1023 - ((int)((bits >> 52) & 0x7ff) - 1023)) << 52);
        th1 *= sc; th2 *= sc; del1 *= sc;
        __syncwarp();
        if (SYNC) mbar_arrive(&empty[slot]);
    }
    long long t1 = clock64();
    if (lane == 0) { cyc[blockIdx.x] = t1 - t0; out[blockIdx.x] = th1 + del1 + scr[0][lane] + scr[1][5]; }
}

int main() {
    double* out; long long* cyc; long long h;
    cudaMalloc(&out, 4096); cudaMalloc(&cyc, 4096);
    const int W = 2000;
    bench<0><<<148, 64>>>(out, cyc, W); bench<0><<<148, 64>>>(out, cyc, W);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("TC loop, no sync:       %.0f cycles/window\n", (double)h / W);
    bench<1><<<148, 64>>>(out, cyc, W); bench<1><<<148, 64>>>(out, cyc, W);
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("TC loop, mbarrier sync: %.0f cycles/window\n", (double)h / W);
    printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
