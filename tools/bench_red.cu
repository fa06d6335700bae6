// Micro-benchmark: scattered ATOM (returning) vs RED throughput and scattered loads,
// 2368 warps x 32 lanes x U ops at once over a 16.8M-entry array.
#include <cstdio>
#include <cstdint>
#include <algorithm>
#include <vector>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t h32(uint32_t h) { h ^= h >> 16; h *= 0x85EBCA6Bu; h ^= h >> 13; h *= 0xC2B2AE35u; h ^= h >> 16; return h; }
template <int MODE, int U>
__global__ void k(uint32_t *cnt, uint32_t n, uint32_t seed, long long *out) {
    const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    uint32_t w[U];
    for (int u = 0; u < U; u++) w[u] = (h32(seed ^ (warp * 32 * U + u * 32 + lane)) % n) * 8;  // 32-B records
    __syncthreads();
    long long t0 = clock64();
    uint32_t acc = 0;
#pragma unroll
    for (int u = 0; u < U; u++) {
        if (MODE == 0) acc |= atomicSub(cnt + w[u], 1u);
        if (MODE == 1) atomicSub(cnt + w[u], 1u);
        if (MODE == 2) acc |= __ldcg(cnt + w[u]);
        if (MODE == 3) { acc |= atomicSub(cnt + w[u], 1u); atomicOr(cnt + w[u] + 4, 1u << lane); }
    }
    if (MODE == 1 || MODE == 3) __threadfence();
    acc = __reduce_or_sync(0xffffffffu, acc);
    long long t1 = clock64();
    if (lane == 0) out[warp] = (t1 - t0) + (acc == 0x12345 ? 1 : 0);
}
int main() {
    uint32_t *cnt; long long *out;
    uint32_t n = 1u << 24;
    cudaMalloc(&cnt, 32ull * n); cudaMalloc(&out, 1 << 20);
    cudaMemset(cnt, 0x7f, 32ull * n);
    std::vector<long long> h(65536);
    const char *names[] = {"ATOM (returning)", "RED + fence", "LDG.cg", "ATOM + RED(same sector) + fence"};
    for (int mode = 0; mode < 4; mode++) {
        int blocks = 148, threads = 512;
        for (int rep = 0; rep < 3; rep++) {
            if (mode == 0) k<0, 4><<<blocks, threads>>>(cnt, n, rep * 7919, out);
            if (mode == 1) k<1, 4><<<blocks, threads>>>(cnt, n, rep * 7919, out);
            if (mode == 2) k<2, 4><<<blocks, threads>>>(cnt, n, rep * 7919, out);
            if (mode == 3) k<3, 4><<<blocks, threads>>>(cnt, n, rep * 7919, out);
        }
        int nw = blocks * threads / 32;
        cudaMemcpy(h.data(), out, sizeof(long long) * nw, cudaMemcpyDeviceToHost);
        std::sort(h.begin(), h.begin() + nw);
        printf("%-34s 4/lane x %d warps: median %6lld p90 %6lld max %6lld cycles -> %.1f ops/cycle %s\n", names[mode], nw,
               h[nw / 2], h[nw * 9 / 10], h[nw - 1], (double)nw * 32 * 4 * (mode == 3 ? 2 : 1) / h[nw - 1],
               cudaGetErrorString(cudaGetLastError()));
    }
}
