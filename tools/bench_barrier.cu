// Micro-benchmark: software grid barrier cost on the GPU (diagnostic for JP levels).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
template <int MODE>
__global__ void k(uint32_t *bar, uint32_t *gen_p, int iters, uint32_t *sink) {
    uint32_t gen = 0;
    for (int i = 0; i < iters; i++) {
        __syncthreads();
        if (threadIdx.x == 0) {
            if (MODE == 0) __threadfence();
            if (MODE == 2) asm volatile("fence.acq_rel.gpu;" ::: "memory");
            uint32_t old;
            if (MODE == 2) asm volatile("atom.add.release.gpu.u32 %0, [%1], 1;" : "=r"(old) : "l"(bar) : "memory");
            else old = atomicAdd(bar, 1u);
            if (old == gridDim.x - 1) {
                atomicExch(bar, 0u);
                if (MODE != 2) __threadfence();
                if (MODE == 2) asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(gen_p) : "memory");
                else atomicAdd(gen_p, 1u);
            } else {
                if (MODE == 2) { while (ld_relaxed_u32(gen_p) == gen) {} asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
                else while (ld_acquire_u32(gen_p) == gen) {}
            }
        }
        gen++;
        __syncthreads();
    }
    if (threadIdx.x == 0 && gen == 12345) *sink = gen;
}
int main() {
    uint32_t *buf;
    cudaMalloc(&buf, 4096);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (int mode = 0; mode < 3; mode++)
    for (int threads : {128, 512}) {
        cudaMemset(buf, 0, 4096);
        int iters = 5000;
        cudaEvent_t a, b;
        cudaEventCreate(&a); cudaEventCreate(&b);
        void (*kp)(uint32_t*, uint32_t*, int, uint32_t*) = mode == 0 ? k<0> : mode == 1 ? k<1> : k<2>;
        kp<<<sms, threads>>>(buf, buf + 64, 10, buf + 128);
        cudaMemset(buf, 0, 4096);
        cudaEventRecord(a);
        kp<<<sms, threads>>>(buf, buf + 64, iters, buf + 128);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        printf("mode %d threads %d: %.3f us per barrier (%s)\n", mode, threads, ms * 1000 / iters, cudaGetErrorString(cudaGetLastError()));
    }
}
