// Micro-benchmark: latency of a JP-like push (8 random targets per lane: 2 row-pointer
// loads + 1 returning atomic each) for 2368 warps at once, vs array footprint.
#include <cstdio>
#include <cstdint>
#include <algorithm>
#include <vector>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t h32(uint32_t h) { h ^= h >> 16; h *= 0x85EBCA6Bu; h ^= h >> 13; h *= 0xC2B2AE35u; h ^= h >> 16; return h; }
template <int MODE>
__global__ void k(const int64_t *rp, uint32_t *cnt, uint32_t n, uint32_t seed, long long *out) {
    const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    uint32_t w[8];
    for (int u = 0; u < 8; u++) w[u] = h32(seed ^ (warp * 256 + u * 32 + lane)) % n;
    __syncthreads();
    long long t0 = clock64();
    int64_t acc = 0;
    uint32_t old[8];
#pragma unroll
    for (int u = 0; u < 8; u++) {
        if (MODE & 1) acc += rp[w[u]] + rp[w[u] + 1];
        if (MODE & 2) old[u] = atomicSub(cnt + w[u], 1u); else old[u] = 0;
    }
    uint32_t o = 0;
    for (int u = 0; u < 8; u++) o |= old[u];
    o = __reduce_or_sync(0xffffffffu, o) + (uint32_t)__reduce_add_sync(0xffffffffu, (uint32_t)acc);
    long long t1 = clock64();
    if (lane == 0) out[warp] = (t1 - t0) + (o == 0x12345 ? 1 : 0);
}
int main() {
    int64_t *rp; uint32_t *cnt; long long *out;
    size_t maxn = 1ull << 27;
    cudaMalloc(&rp, 8 * (maxn + 1)); cudaMalloc(&cnt, 4 * maxn); cudaMalloc(&out, 1 << 20);
    cudaMemset(rp, 0, 8 * (maxn + 1)); cudaMemset(cnt, 0x7f, 4 * maxn);
    std::vector<long long> h(65536);
    for (int mode = 1; mode <= 3; mode++)
    for (uint32_t n : {1u << 16, 1u << 20, 1u << 22, 1u << 24, 1u << 27}) {
        int blocks = 148, threads = 512;
        for (int rep = 0; rep < 3; rep++) {
            if (mode == 1) k<1><<<blocks, threads>>>(rp, cnt, n, rep * 7919, out);
            if (mode == 2) k<2><<<blocks, threads>>>(rp, cnt, n, rep * 7919, out);
            if (mode == 3) k<3><<<blocks, threads>>>(rp, cnt, n, rep * 7919, out);
        }
        int nw = blocks * threads / 32;
        cudaMemcpy(h.data(), out, sizeof(long long) * nw, cudaMemcpyDeviceToHost);
        std::sort(h.begin(), h.begin() + nw);
        printf("mode %d (1=rp 2=atom 3=both) n 2^%2d: median %6lld p90 %6lld max %6lld cycles %s\n", mode, 31 - __builtin_clz(n),
               h[nw / 2], h[nw * 9 / 10], h[nw - 1], cudaGetErrorString(cudaGetLastError()));
    }
}
