// common.cuh -- device-side building blocks shared by the sm_100a kernels.
//
// Hash contract (DESIGN.md §3 H; the paper is silent on its RNG):
//   K(seed,tag,round) = mix64(mix64(seed ^ 0x9E3779B97F4A7C15) ^ (tag<<32 | round))
//   pv(v)       = fmix32(v ^ Klo) ^ Khi                 vertex priority
//   pe(lo,hi)   = fmix32(lo*0x9E3779B1 ^ hi ^ Klo) ^ Khi edge priority
//   label(v)    = (pv_RAND(v) * p) >> 32                 RAND part (Alg 2 l.3)
// Vertices are ordered by the 64-bit key (pv(v) << 32 | v); edges at a fixed
// endpoint u by (pe(u,w) << 32 | w), which agrees with the global (pe, lo, hi)
// order (DESIGN §3 H).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace sym {

constexpr uint32_t TAG_VERTEX = 1, TAG_EDGE = 2, TAG_RAND = 3;
constexpr unsigned FULL = 0xffffffffu;

// MIS vertex status (1 byte per vertex)
constexpr uint8_t ST_UNDEC = 0, ST_IN = 1, ST_OUT = 2, ST_INACTIVE = 3;

__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z ^= z >> 30;
    z *= 0xBF58476D1CE4E5B9ULL;
    z ^= z >> 27;
    z *= 0x94D049BB133111EBULL;
    z ^= z >> 31;
    return z;
}

__host__ __device__ __forceinline__ uint32_t fmix32(uint32_t h) {
    h ^= h >> 16;
    h *= 0x85EBCA6Bu;
    h ^= h >> 13;
    h *= 0xC2B2AE35u;
    h ^= h >> 16;
    return h;
}

struct Key {
    uint32_t lo, hi;
};

inline Key stream_key(uint64_t seed, uint32_t tag, uint32_t round) {
    uint64_t k = mix64(mix64(seed ^ 0x9E3779B97F4A7C15ULL) ^ (((uint64_t)tag << 32) | round));
    return Key{(uint32_t)k, (uint32_t)(k >> 32)};
}

__device__ __forceinline__ uint32_t pv(Key k, uint32_t v) { return fmix32(v ^ k.lo) ^ k.hi; }

// 64-bit vertex order key: larger wins; unique because ids are unique
__device__ __forceinline__ uint64_t vkey(Key k, uint32_t v) { return ((uint64_t)pv(k, v) << 32) | v; }

__device__ __forceinline__ uint32_t pe(Key k, uint32_t a, uint32_t b) {
    uint32_t lo = min(a, b), hi = max(a, b);
    return fmix32((lo * 0x9E3779B1u) ^ hi ^ k.lo) ^ k.hi;
}

// edge key seen from endpoint u towards w: (pe << 32) | w
__device__ __forceinline__ uint64_t ekey(Key k, uint32_t u, uint32_t w) { return ((uint64_t)pe(k, u, w) << 32) | w; }

__device__ __forceinline__ uint32_t rand_label(Key k, uint32_t v, uint32_t p) {
    return (uint32_t)(((uint64_t)pv(k, v) * (uint64_t)p) >> 32);
}

// ---------------------------------------------------------------- warp helpers
__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

// warp-aggregated append: every lane with `pred` gets a unique slot in list
// (returns the slot; -1 for lanes without pred).  Must be called by all lanes of
// the warp in converged control flow.
__device__ __forceinline__ int64_t warp_append(bool pred, uint32_t *counter) {
    unsigned m = __ballot_sync(FULL, pred);
    if (!m) return -1;
    int leader = __ffs(m) - 1;
    uint32_t base = 0;
    if (lane_id() == leader) base = atomicAdd(counter, (uint32_t)__popc(m));
    base = __shfl_sync(FULL, base, leader);
    if (!pred) return -1;
    return (int64_t)base + __popc(m & ((1u << lane_id()) - 1));
}

// Two-class list append, aggregated per CTA: class-0 vertices from the front of vlist,
// class-1 from the back (slot n-1-k), ONE atomic per CTA and class instead of one per
// warp (per-warp appends to one counter serialise at the L2: 0.7 ms for 16 M vertices).
// Every thread of the CTA must call it in block-uniform control flow; the list order
// is immaterial to its users.
__device__ __forceinline__ void cta_append2(bool c0, bool c1, int32_t v, int64_t n, int32_t *vlist,
                                            uint32_t *cnt0, uint32_t *cnt1) {
    __shared__ uint32_t w0[32], w1[32], b0, b1;
    const unsigned m0 = __ballot_sync(FULL, c0), m1 = __ballot_sync(FULL, c1);
    const int wid = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
    if (lane_id() == 0) {
        w0[wid] = __popc(m0);
        w1[wid] = __popc(m1);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t t0 = 0, t1 = 0;
        for (int q = 0; q < nw; q++) {
            const uint32_t a0 = w0[q], a1 = w1[q];
            w0[q] = t0;
            w1[q] = t1;
            t0 += a0;
            t1 += a1;
        }
        b0 = t0 ? atomicAdd(cnt0, t0) : 0u;
        b1 = t1 ? atomicAdd(cnt1, t1) : 0u;
    }
    __syncthreads();
    const unsigned lt = (1u << lane_id()) - 1u;
    if (c0) vlist[b0 + w0[wid] + __popc(m0 & lt)] = v;
    if (c1) vlist[n - 1 - (int64_t)(b1 + w1[wid] + __popc(m1 & lt))] = v;
    __syncthreads();  // the scratch is reused by the next call
}

// Same, into two separate lists (list0 / cnt0, list1 / cnt1), u32 entries.
__device__ __forceinline__ void cta_append2x(bool c0, bool c1, uint32_t v, uint32_t *list0, uint32_t *cnt0,
                                             uint32_t *list1, uint32_t *cnt1) {
    __shared__ uint32_t x0[32], x1[32], xb0, xb1;
    const unsigned m0 = __ballot_sync(FULL, c0), m1 = __ballot_sync(FULL, c1);
    const int wid = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
    if (lane_id() == 0) {
        x0[wid] = __popc(m0);
        x1[wid] = __popc(m1);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t t0 = 0, t1 = 0;
        for (int q = 0; q < nw; q++) {
            const uint32_t a0 = x0[q], a1 = x1[q];
            x0[q] = t0;
            x1[q] = t1;
            t0 += a0;
            t1 += a1;
        }
        xb0 = t0 ? atomicAdd(cnt0, t0) : 0u;
        xb1 = t1 ? atomicAdd(cnt1, t1) : 0u;
    }
    __syncthreads();
    const unsigned lt = (1u << lane_id()) - 1u;
    if (c0) list0[xb0 + x0[wid] + __popc(m0 & lt)] = v;
    if (c1) list1[xb1 + x1[wid] + __popc(m1 & lt)] = v;
    __syncthreads();
}

__device__ __forceinline__ uint64_t ld_volatile_u64(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ uint32_t ld_volatile_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.volatile.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// Predicated PTX loads/atomics (no branch per element): with `p ? load : default` the
// compiler branched around each access and, short of registers, consumed its result
// inside the branch, so K independent accesses ran one after another (~1 us each).
__device__ __forceinline__ uint32_t ld_cg_pred(const uint32_t *addr, bool p) {  // 0xffffffff if !p
    uint32_t v = 0xffffffffu;
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q ld.global.cg.u32 %0, [%1];\n\t}"
                 : "+r"(v)
                 : "l"(addr), "r"((uint32_t)p)
                 : "memory");
    return v;
}

__device__ __forceinline__ uint4 ld_cg_v4_pred(const uint4 *addr, bool p) {  // {1,0,0,0} if !p
    uint4 v = make_uint4(1u, 0u, 0u, 0u);
    asm volatile(
        "{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %5, 0;\n\t@q ld.global.cg.v4.u32 {%0, %1, %2, %3}, [%4];\n\t}"
        : "+r"(v.x), "+r"(v.y), "+r"(v.z), "+r"(v.w)
        : "l"(addr), "r"((uint32_t)p)
        : "memory");
    return v;
}

__device__ __forceinline__ uint32_t atom_add_pred(uint32_t *addr, uint32_t val, bool p) {  // 0 if !p
    uint32_t old = 0u;
    asm volatile(
        "{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q atom.global.add.u32 %0, [%1], %3;\n\t}"
        : "+r"(old)
        : "l"(addr), "r"((uint32_t)p), "r"(val)
        : "memory");
    return old;
}

// returning 64-bit atomic decrement under a predicate (0 when !p), no branch
__device__ __forceinline__ uint64_t atom_dec64_pred(unsigned long long *addr, bool p) {
    unsigned long long old = 0ull;
    asm volatile(
        "{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q atom.global.add.u64 %0, [%1], %3;\n\t}"
        : "+l"(old)
        : "l"(addr), "r"((uint32_t)p), "l"(0xffffffffffffffffull)
        : "memory");
    return old;
}

// streaming (evict-first) 4-B load under a predicate (0 when !p), no branch
__device__ __forceinline__ uint32_t ld_cs_pred(const uint32_t *addr, bool p) {
    uint32_t v = 0u;
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q ld.global.cs.u32 %0, [%1];\n\t}"
                 : "+r"(v)
                 : "l"(addr), "r"((uint32_t)p)
                 : "memory");
    return v;
}

// read-only 8-B load under a predicate ({0,0} when !p), no branch
__device__ __forceinline__ uint2 ld_nc_v2_pred(const uint2 *addr, bool p) {
    uint2 v = make_uint2(0u, 0u);
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %3, 0;\n\t@q ld.global.nc.v2.u32 {%0, %1}, [%2];\n\t}"
                 : "+r"(v.x), "+r"(v.y)
                 : "l"(addr), "r"((uint32_t)p));
    return v;
}

// 1-B load under a predicate (dflt when !p), no branch
__device__ __forceinline__ uint8_t ld_u8_pred(const uint8_t *addr, bool p, uint8_t dflt) {
    uint32_t v = dflt;
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q ld.global.u8 %0, [%1];\n\t}"
                 : "+r"(v)
                 : "l"(addr), "r"((uint32_t)p)
                 : "memory");
    return (uint8_t)v;
}

// read-only 4-B load under a predicate (0 when !p), no branch
__device__ __forceinline__ uint32_t ld_nc_pred(const uint32_t *addr, bool p) {
    uint32_t v = 0u;
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q ld.global.nc.u32 %0, [%1];\n\t}"
                 : "+r"(v)
                 : "l"(addr), "r"((uint32_t)p));
    return v;
}

}  // namespace sym
