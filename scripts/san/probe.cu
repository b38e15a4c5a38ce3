// Probe of compute-sanitizer racecheck's model of the synchronisation idioms
// the solver's kernels use: two warps hand a shared-memory
// buffer from a producer to a consumer through
//   mode 0: __syncthreads()                        (modelled: expect 0 hazards)
//   mode 1: st.release / ld.acquire flag (cta)     (PTX memory model)
//   mode 2: atom.release.exch / atom.acquire.or flag
//   mode 3: mbarrier.arrive.release / mbarrier.try_wait.parity.acquire
//   mode 4: bar.arrive (producer) / bar.sync (consumer) on a named barrier
// Every mode is correct under the PTX memory model; the run shows which ones
// racecheck reports as hazards.  usage: probe <mode>
#include <cstdio>
#include <cstdlib>
#include <cstdint>

__global__ void k(int mode, float* out) {
    __shared__ float buf[64];
    __shared__ int flag;
    __shared__ __align__(8) uint64_t bar;
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        flag = 0;
        asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(&bar)), "r"(32));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const unsigned fa = (unsigned)__cvta_generic_to_shared(&flag);
    const unsigned ba = (unsigned)__cvta_generic_to_shared(&bar);
    if (w == 0) {  // producer
        buf[l] = 1.0f + l;
        buf[32 + l] = 2.0f + l;
        if (mode == 0) { __syncthreads(); }
        if (mode == 1) { __syncwarp(); if (l == 0) asm volatile("st.release.cta.shared::cta.u32 [%0], %1;" ::"r"(fa), "r"(1) : "memory"); }
        if (mode == 2) { __syncwarp(); if (l == 0) { int o; asm volatile("atom.release.cta.shared::cta.exch.b32 %0, [%1], %2;" : "=r"(o) : "r"(fa), "r"(1) : "memory"); } }
        if (mode == 3) asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(ba) : "memory");
        if (mode == 4) asm volatile("bar.arrive 1, 64;" ::: "memory");
    } else {  // consumer
        if (mode == 0) __syncthreads();
        if (mode == 1) { unsigned v = 0; do { asm volatile("ld.acquire.cta.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(fa) : "memory"); } while (v == 0); }
        if (mode == 2) { int v = 0; do { asm volatile("atom.acquire.cta.shared::cta.or.b32 %0, [%1], 0;" : "=r"(v) : "r"(fa) : "memory"); } while (v == 0); }
        if (mode == 3) {
            asm volatile("{\n.reg .pred P;\nW_%=:\nmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 P, [%0], %1;\n@!P bra W_%=;\n}\n" ::"r"(ba), "r"(0) : "memory");
        }
        if (mode == 4) asm volatile("bar.sync 1, 64;" ::: "memory");
        out[l] = buf[(l + 1) & 31] + buf[32 + ((l + 5) & 31)];
    }
}

int main(int argc, char** argv) {
    const int mode = argc > 1 ? atoi(argv[1]) : 0;
    float* out;
    cudaMalloc(&out, 64 * sizeof(float));
    k<<<1, 64>>>(mode, out);
    float h[32];
    cudaMemcpy(h, out, sizeof h, cudaMemcpyDeviceToHost);
    const cudaError_t e = cudaGetLastError();
    printf("mode %d: out[0] = %g (expect %g) %s\n", mode, h[0], 2.0 + 2.0 + 5, cudaGetErrorString(e));
    return 0;
}
