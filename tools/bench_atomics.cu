// Micro-benchmark: latency of returning atomics when W warps hit K distinct addresses at once.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__global__ void k(uint32_t *cnt, int K, int stride, int per_lane, long long *out) {
    const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    __syncthreads();
    long long t0 = clock64();
    uint32_t acc = 0;
    if (lane < per_lane) acc = atomicSub(cnt + (size_t)((warp * per_lane + lane) % K) * stride, 1u);
    acc = __reduce_add_sync(0xffffffffu, acc);
    long long t1 = clock64();
    if (lane == 0) out[warp] = (t1 - t0) + (acc == 0x7fffffff ? 1 : 0);
}
int main() {
    uint32_t *cnt; long long *out;
    cudaMalloc(&cnt, 64 << 20); cudaMalloc(&out, 1 << 20);
    cudaMemset(cnt, 0x7f, 64 << 20);
    static long long h[65536];
    for (int per_lane : {1, 8, 32})
    for (int K : {1, 4, 16, 64, 256, 4096, 1 << 20}) {
        for (int stride : {1, 32}) {
            int blocks = 148 * 2, threads = 512;
            k<<<blocks, threads>>>(cnt, K, stride, per_lane, out);
            k<<<blocks, threads>>>(cnt, K, stride, per_lane, out);
            cudaMemcpy(h, out, sizeof(long long) * blocks * threads / 32, cudaMemcpyDeviceToHost);
            int nw = blocks * threads / 32; double s = 0; long long mx = 0;
            for (int i = 0; i < nw; i++) { s += h[i]; if (h[i] > mx) mx = h[i]; }
            printf("lanes/warp %2d K %8d stride %2d: mean %8.0f max %8lld cycles (%s)\n", per_lane, K, stride, s / nw, mx, cudaGetErrorString(cudaGetLastError()));
        }
    }
}
