// Micro-benchmark (JP tail diagnosis): how long does ONE warp (per SM, W warps in all)
// take for K random 4-B accesses per lane into an array of S bytes -- returning
// atomicSub vs plain loads vs atomicSub on pre-touched (L2-resident) lines.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/bga tools/bench_gather_atomics.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include <initializer_list>
__device__ __forceinline__ uint64_t gt() { uint64_t t; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)); return t; }
__device__ __forceinline__ uint32_t hsh(uint32_t x) { x ^= x >> 16; x *= 0x85EBCA6Bu; x ^= x >> 13; x *= 0xC2B2AE35u; x ^= x >> 16; return x; }
template <int K, int MODE>
__global__ void k(uint32_t *a, uint64_t nwords, uint32_t seed, uint64_t *out) {
    const int lane = threadIdx.x & 31;
    const uint32_t w = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    uint32_t idx[K], v[K];
#pragma unroll
    for (int u = 0; u < K; u++) idx[u] = (uint32_t)(((uint64_t)hsh(seed ^ (w * 1024 + u * 32 + lane)) * 4) % nwords);
    __syncwarp();
    const uint64_t t0 = gt();
#pragma unroll
    for (int u = 0; u < K; u++) {
        if (MODE == 0) v[u] = atomicSub(a + idx[u], 1u);
        else if (MODE == 1) v[u] = __ldcg(a + idx[u]);
        else { atomicSub(a + idx[u], 1u); v[u] = 0; }
    }
    uint32_t x = 0;
#pragma unroll
    for (int u = 0; u < K; u++) x ^= v[u];
    if (__ballot_sync(0xffffffffu, x == 0x12345u) == 0xffffffffu) a[0] = 0;
    const uint64_t t1 = gt();
    if (lane == 0) out[w] = t1 - t0;
}
template <int K, int MODE>
void run(const char *name, uint32_t *a, uint64_t bytes, int ctas, int warps, uint64_t *out) {
    static uint64_t h[1 << 16];
    double best = 1e30, worst = 0;
    for (int rep = 0; rep < 5; rep++) {
        k<K, MODE><<<ctas, warps * 32>>>(a, bytes / 4, 12345u + rep * 7919u, out);
        cudaDeviceSynchronize();
        cudaMemcpy(h, out, sizeof(uint64_t) * ctas * warps, cudaMemcpyDeviceToHost);
        double s = 0, mx = 0;
        for (int i = 0; i < ctas * warps; i++) { s += h[i]; if (h[i] > mx) mx = h[i]; }
        if (rep > 0) { best = s / (ctas * warps) < best ? s / (ctas * warps) : best; worst = mx > worst ? mx : worst; }
    }
    printf("%-10s K/lane %2d array %7.1f MB ctas %4d warps/cta %2d: mean %7.2f us  max %7.2f us (%s)\n", name, K,
           bytes / 1e6, ctas, warps, best / 1e3, worst / 1e3, cudaGetErrorString(cudaGetLastError()));
}
int main() {
    uint32_t *a; uint64_t *out;
    const uint64_t big = 2ull << 30;
    cudaMalloc(&a, big); cudaMalloc(&out, 1 << 20); cudaMemset(a, 0x7f, big);
    const uint64_t sizes[3] = {16ull << 20, 180ull << 20, big};
    for (uint64_t bytes : sizes) {
        for (int ctas : {16, 148, 296}) {
            run<8, 0>("atomicSub", a, bytes, ctas, 1, out);
            run<8, 1>("load", a, bytes, ctas, 1, out);
            run<8, 2>("red", a, bytes, ctas, 1, out);
            run<1, 0>("atomicSub", a, bytes, ctas, 1, out);
            run<1, 1>("load", a, bytes, ctas, 1, out);
        }
        run<8, 0>("atomicSub", a, bytes, 296, 16, out);
        run<8, 1>("load", a, bytes, 296, 16, out);
    }
    return 0;
}
