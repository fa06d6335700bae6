// Micro-benchmark (JP tail diagnosis): does a grid of CTAs polling ONE barrier word
// slow down another warp's random atomics / loads?  CTA 0 warp 0 does K returning
// atomicSub (or loads) per lane into a 180 MB array, then releases a flag; every
// other CTA's thread 0 polls the flag: 0 = nobody polls, 1 = ld.acquire.gpu spin,
// 2 = ld.relaxed.gpu spin, 3 = ld.acquire.gpu + __nanosleep(256).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/bpi tools/bench_poll_interference.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint64_t gt() { uint64_t t; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)); return t; }
__device__ __forceinline__ uint32_t hsh(uint32_t x) { x ^= x >> 16; x *= 0x85EBCA6Bu; x ^= x >> 13; x *= 0xC2B2AE35u; x ^= x >> 16; return x; }
__device__ __forceinline__ uint32_t ld_acq(const uint32_t *p) { uint32_t v; asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v; }
__device__ __forceinline__ uint32_t ld_rlx(const uint32_t *p) { uint32_t v; asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v; }
template <int MODE, bool ATOM>
__global__ void k(uint32_t *a, uint64_t nwords, uint32_t *flag, uint32_t gen, uint64_t *out) {
    constexpr int K = 8;
    if (blockIdx.x == 0) {
        if (threadIdx.x >= 32) return;
        const int lane = threadIdx.x;
        // wait until the pollers are running
        uint64_t tw = gt(); while (gt() - tw < 20000) {}
        uint32_t idx[K], v[K];
#pragma unroll
        for (int u = 0; u < K; u++) idx[u] = (uint32_t)(((uint64_t)hsh(gen * 977u ^ (u * 32 + lane)) * 4) % nwords);
        const uint64_t t0 = gt();
#pragma unroll
        for (int u = 0; u < K; u++) v[u] = ATOM ? atomicSub(a + idx[u], 1u) : __ldcg(a + idx[u]);
        uint32_t x = 0;
#pragma unroll
        for (int u = 0; u < K; u++) x ^= v[u];
        if (__ballot_sync(0xffffffffu, x == 0x12345u) == 0xffffffffu) a[0] = 0;
        const uint64_t t1 = gt();
        if (lane == 0) { out[0] = t1 - t0; asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(flag), "r"(gen) : "memory"); }
        return;
    }
    if (threadIdx.x != 0) return;
    if (MODE == 0) return;
    if (MODE == 1) while (ld_acq(flag) != gen) {}
    if (MODE == 2) while (ld_rlx(flag) != gen) {}
    if (MODE == 3) while (ld_acq(flag) != gen) __nanosleep(256);
}
template <int MODE, bool ATOM>
void run(uint32_t *a, uint64_t bytes, uint32_t *flag, uint64_t *out, int ctas) {
    static uint32_t gen = 1;
    double s = 0; uint64_t h;
    for (int rep = 0; rep < 6; rep++) {
        k<MODE, ATOM><<<ctas, 512>>>(a, bytes / 4, flag, ++gen, out);
        cudaDeviceSynchronize();
        cudaMemcpy(&h, out, 8, cudaMemcpyDeviceToHost);
        if (rep) s += h;
    }
    printf("%s poll mode %d ctas %d: %.2f us (%s)\n", ATOM ? "atomicSub" : "load     ", MODE, ctas, s / 5 / 1e3,
           cudaGetErrorString(cudaGetLastError()));
}
int main() {
    uint32_t *a, *flag; uint64_t *out;
    const uint64_t bytes = 180ull << 20;
    cudaMalloc(&a, bytes); cudaMalloc(&flag, 4096); cudaMalloc(&out, 4096); cudaMemset(a, 0x7f, bytes); cudaMemset(flag, 0, 4096);
    for (int ctas : {296}) {
        run<0, true>(a, bytes, flag, out, ctas); run<1, true>(a, bytes, flag, out, ctas);
        run<2, true>(a, bytes, flag, out, ctas); run<3, true>(a, bytes, flag, out, ctas);
        run<0, false>(a, bytes, flag, out, ctas); run<1, false>(a, bytes, flag, out, ctas);
        run<2, false>(a, bytes, flag, out, ctas); run<3, false>(a, bytes, flag, out, ctas);
    }
    return 0;
}
