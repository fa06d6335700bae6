// jp.cu -- Jones-Plassmann colouring and the COLOR flows.
//
// JP ([18]) with fixed priorities colours v once every higher-(pv,id)
// neighbour of its phase set S is coloured, with the smallest colour >= 1 not held by
// any coloured neighbour: exactly first-fit greedy in priority order (DESIGN §3 C1).
//
// Push form over a compact oriented DAG, built once per call:
//   ids     the S vertices with phase arcs get compact ids h (rows of degree > 2
//           first, so the hot records of a power-law core are contiguous); a vertex
//           without any phase arc takes colour 1 at once.
//   segment seg[boff .. boff+R) = h's forbidden-colour bitmap, R = ceil(cap/32)
//           words for cap = (#higher + #fixed-coloured neighbours) + 1 >= mex, then
//           seg[boff+R .. boff+R+ldeg) = compact ids of h's LOWER S-neighbours: the
//           only arcs a push needs (half of the phase arcs, no hash at level time).
//   record  rec[h] (8 B) = cnt | min(R,255) << 24 | boff << 32, cnt = higher
//           S-neighbours not yet coloured.  A push to w is ONE returning 64-bit
//           atomic (the decrement returns w's segment address; w's lower degree is
//           loaded beside it, so a vertex that becomes ready needs no further load)
//           plus one RED of the colour bit; records + bitmaps are ~90 MB at R-MAT
//           s24 (vs 0.5 GB of 32-B records per vertex id before).
//   level   every ready vertex is split into tasks of <= JP_CHUNK lower arcs; a
//           task computes colour(h) = mex of h's bitmap (complete: every higher
//           neighbour pushed in an earlier level) and pushes it to its lower
//           neighbours; the decrement reaching 0 stages w for the next level.
// Levels = the JP dependency depth (~5e3 on R-MAT scale 24), all in ONE persistent
// cooperative kernel (k_jp_levels) with a software grid barrier between levels.
#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include "internal.h"

namespace sym {

constexpr int JP_THREADS = 256;
constexpr int JP_HUGE_THREADS = 512;
constexpr int JP_SMALL = 32;     // build: rows <= JP_SMALL arcs are handled by one lane
constexpr int JP_BUDGET = 4096;  // build: rows > JP_BUDGET arcs are split into pieces
constexpr int JP_PIECE = 8192;   // arcs per CTA piece of a huge row in the build passes
constexpr int JP_TILE = 2048;    // build: compact ids per scan tile (JP_THREADS x 8)
constexpr int JP_TPT = JP_TILE / JP_THREADS;
#ifndef SYM_JP_CHUNK
#define SYM_JP_CHUNK 64
#endif
constexpr int JP_CHUNK = SYM_JP_CHUNK;  // lower arcs per warp task (2 per lane)
constexpr int JP_LANE = 8;              // lower lists of <= JP_LANE arcs are a lane task
constexpr unsigned long long JP_CNT_MASK = (1ull << 24) - 1;
constexpr uint32_t JP_RSAT = 255;       // R field saturated: the word count is in rfull[h]

// a task: one chunk of a ready vertex's lower list
struct __align__(16) JpTask {
    int64_t b, e;     // h's lower list: seg[b .. e)
    int32_t h;
    uint32_t j;       // chunk index
    uint64_t bm;      // h's bitmap: boff << 32 | R
};
static_assert(sizeof(JpTask) == 32, "JpTask layout");

struct JpArgs {
    const int64_t *rp;   // phase CSR (original ids)
    const int32_t *ci;
    const uint8_t *inS;  // nullable: S = all vertices
    uint32_t *color;     // output (original ids); fixed colours of non-S neighbours
    const int32_t *in_list;  // S as a list (nullable = implicit 0..implicit_n-1)
    const uint32_t *in_cnt;
    int64_t implicit_n;
    int32_t *cid;        // [n] original -> compact id
    int32_t *ov;         // [n] compact id -> original
    uint32_t *ldeg;      // [n] lower degree
    uint32_t *rfull;     // [n] bitmap words R
    unsigned long long *rec;  // [n+1] cnt | Rsat << 24 | boff << 32
    uint32_t *seg;       // per compact vertex: bitmap (R words), lower list (ldeg ids)
    uint32_t *ccol;      // [n] colours by compact id (build: fill cursor of huge rows)
    uint32_t *tcnt;      // scan scratch: per tile class counts (2 per tile)
    unsigned long long *tsum;  // scan scratch: per tile (lower arcs, bitmap words)
    uint32_t *nc;        // [0] = compact count n', [1] = rows of degree > 2
    JpTask *tout;        // the task queue (monotone; level r owns [lo_r, hi_r))
    uint32_t *out_cnt;   // level-0 task counter (the low half of the levels kernel's W)
    int64_t *huge;       // (piece << 32 | h) items of the huge rows
    uint32_t *huge_cnt;
    uint32_t *err;       // 2 = a count exceeds the record field
    uint32_t *hist;
    uint32_t *trace;     // nullable: per-level spans (SYM_JP_TRACE diagnostics)
    unsigned long long *prof;  // algorithmic bytes of the levels pass (nullable)
    Key k;
};

__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ bool in_set(const uint8_t *inS, uint32_t w) { return inS == nullptr || inS[w] != 0; }

__device__ __forceinline__ uint32_t n_tasks(int64_t ldeg) {
    return ldeg <= 0 ? 1u : (uint32_t)((ldeg + JP_CHUNK - 1) / JP_CHUNK);
}

__device__ __forceinline__ void write_task(JpTask *q, int64_t b, int64_t e, int32_t h, uint32_t j, uint64_t bm) {
    longlong2 *p = reinterpret_cast<longlong2 *>(q);
    p[0] = make_longlong2(b, e);
    p[1] = make_longlong2((long long)(((uint64_t)j << 32) | (uint32_t)h), (long long)bm);
}

// warp-aggregated reservation of k_lane consecutive slots per lane; returns this
// lane's first slot.  All lanes must call it.
__device__ __forceinline__ int64_t warp_reserve(uint32_t k_lane, uint32_t *counter) {
    uint32_t incl = k_lane;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        uint32_t y = __shfl_up_sync(FULL, incl, d);
        if (lane_id() >= d) incl += y;
    }
    uint32_t total = __shfl_sync(FULL, incl, 31);
    uint32_t base = 0;
    if (total) {
        if (lane_id() == 0) base = atomicAdd(counter, total);
        base = __shfl_sync(FULL, base, 0);
    }
    return (int64_t)base + incl - k_lane;
}

// bitmap word count of a record (saturated field -> rfull)
__device__ __forceinline__ uint32_t rec_words(const JpArgs &A, unsigned long long r, uint32_t h) {
    const uint32_t R = (uint32_t)(r >> 24) & 0xffu;
    return R == JP_RSAT ? __ldg(A.rfull + h) : R;
}

// CTA-wide exclusive scan of one value per thread (blockDim.x == JP_THREADS);
// returns the exclusive prefix, *total = the CTA sum.  sm scratch: >= 8 entries.
template <class T>
__device__ __forceinline__ T block_excl_scan(T x, T *sm, T *total) {
    T incl = x;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const T y = __shfl_up_sync(FULL, incl, d);
        if (lane_id() >= d) incl += y;
    }
    const int wid = threadIdx.x >> 5;
    if (lane_id() == 31) sm[wid] = incl;
    __syncthreads();
    T before = 0, all = 0;
#pragma unroll
    for (int q = 0; q < JP_THREADS / 32; q++) {
        const T s = sm[q];
        if (q < wid) before += s;
        all += s;
    }
    __syncthreads();
    *total = all;
    return before + incl - x;
}

// ---------------------------------------------------------------- build: compact ids
// class of position i of S: 0 = degree > 2, 1 = 1..2 arcs, 2 = no phase arc
__device__ __forceinline__ int jp_class(const JpArgs &A, int64_t i, uint32_t cnt, int32_t &v) {
    v = -1;
    if (i >= cnt) return 2;
    v = A.in_list ? A.in_list[i] : (int32_t)i;
    const int64_t d = A.rp[v + 1] - A.rp[v];
    return d > 2 ? 0 : (d > 0 ? 1 : 2);
}

__device__ __forceinline__ uint32_t s_count(const JpArgs &A) {
    return A.in_list ? *A.in_cnt : (uint32_t)A.implicit_n;
}

// per tile of JP_TILE positions of S: the number of class-0 and class-1 vertices
__global__ void __launch_bounds__(JP_THREADS) k_jpc_tiles(JpArgs A) {
    const uint32_t cnt = s_count(A);
    const int64_t base = (int64_t)blockIdx.x * JP_TILE;
    if (base >= cnt) return;
    int c0 = 0, c1 = 0;
    for (int u = 0; u < JP_TPT; u++) {
        int32_t v;
        const int c = jp_class(A, base + u * JP_THREADS + threadIdx.x, cnt, v);
        c0 += c == 0;
        c1 += c == 1;
    }
    __shared__ int s0, s1;
    if (threadIdx.x == 0) s0 = s1 = 0;
    __syncthreads();
    c0 = __reduce_add_sync(FULL, c0);
    c1 = __reduce_add_sync(FULL, c1);
    if (lane_id() == 0) {
        if (c0) atomicAdd(&s0, c0);
        if (c1) atomicAdd(&s1, c1);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        A.tcnt[2 * blockIdx.x] = (uint32_t)s0;
        A.tcnt[2 * blockIdx.x + 1] = (uint32_t)s1;
    }
}

// one CTA: exclusive prefix of the tile counts per class (class 1 after all class 0)
__global__ void __launch_bounds__(1024) k_jpc_tiles_scan(JpArgs A, int64_t ntiles) {
    const uint32_t cnt = s_count(A);
    const int64_t need = ((int64_t)cnt + JP_TILE - 1) / JP_TILE;
    const int64_t used = need < ntiles ? need : ntiles;
    const int64_t per = (used + blockDim.x - 1) / blockDim.x;
    const int64_t t0 = (int64_t)threadIdx.x * per, t1 = used < t0 + per ? used : t0 + per;
    uint32_t s0 = 0, s1 = 0;
    for (int64_t t = t0; t < t1; t++) {
        s0 += A.tcnt[2 * t];
        s1 += A.tcnt[2 * t + 1];
    }
    __shared__ uint32_t w0[32], w1[32];
    uint32_t i0 = s0, i1 = s1;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y0 = __shfl_up_sync(FULL, i0, d), y1 = __shfl_up_sync(FULL, i1, d);
        if (lane_id() >= d) {
            i0 += y0;
            i1 += y1;
        }
    }
    const int wid = threadIdx.x >> 5;
    if (lane_id() == 31) {
        w0[wid] = i0;
        w1[wid] = i1;
    }
    __syncthreads();
    uint32_t b0 = 0, b1 = 0, T0 = 0, T1 = 0;
    for (int q = 0; q < (int)(blockDim.x >> 5); q++) {
        if (q < wid) {
            b0 += w0[q];
            b1 += w1[q];
        }
        T0 += w0[q];
        T1 += w1[q];
    }
    uint32_t o0 = b0 + i0 - s0, o1 = T0 + b1 + i1 - s1;
    for (int64_t t = t0; t < t1; t++) {
        const uint32_t a0 = A.tcnt[2 * t], a1 = A.tcnt[2 * t + 1];
        A.tcnt[2 * t] = o0;
        A.tcnt[2 * t + 1] = o1;
        o0 += a0;
        o1 += a1;
    }
    if (threadIdx.x == 0) {
        A.nc[0] = T0 + T1;
        A.nc[1] = T0;
    }
}

// compact ids in (class, position) order; vertices without phase arcs: colour 1
__global__ void __launch_bounds__(JP_THREADS) k_jpc_assign(JpArgs A) {
    const uint32_t cnt = s_count(A);
    const int64_t base = (int64_t)blockIdx.x * JP_TILE;
    if (base >= cnt) return;
    __shared__ uint32_t sm0[8], sm1[8];
    uint32_t o0 = A.tcnt[2 * blockIdx.x], o1 = A.tcnt[2 * blockIdx.x + 1];
    for (int u = 0; u < JP_TPT; u++) {
        int32_t v;
        const int c = jp_class(A, base + u * JP_THREADS + threadIdx.x, cnt, v);
        uint32_t t0, t1;
        const uint32_t r0 = block_excl_scan<uint32_t>(c == 0, sm0, &t0);
        const uint32_t r1 = block_excl_scan<uint32_t>(c == 1, sm1, &t1);
        if (c < 2) {
            const uint32_t h = c == 0 ? o0 + r0 : o1 + r1;
            A.cid[v] = (int32_t)h;
            A.ov[h] = v;
        } else if (v >= 0) {
            A.color[v] = 1u;
        }
        o0 += t0;
        o1 += t1;
    }
}

// ---------------------------------------------------------------- build: DAG
// count pass: rec[h] = #higher S-neighbours, ldeg[h] = #lower S-neighbours; rows
// longer than JP_BUDGET arcs are deferred as JP_PIECE-arc pieces
__global__ void __launch_bounds__(JP_THREADS) k_jpc_count(JpArgs A) {
    const uint32_t cnt = A.nc[0];
    const int lane = lane_id();
    const int64_t warp_g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = warp_g * 32; base < cnt; base += nwarps * 32) {
        const int64_t h = base + lane;
        const bool active = h < cnt;
        int32_t v = 0;
        int64_t b = 0, e = 0;
        uint64_t kv = 0;
        if (active) {
            v = A.ov[h];
            b = A.rp[v];
            e = A.rp[v + 1];
            kv = vkey(A.k, (uint32_t)v);
        }
        uint32_t hi = 0, lo = 0;
        if (active && e - b <= JP_SMALL) {
            for (int64_t x = b; x < e; x++) {
                const uint32_t w = (uint32_t)__ldg(A.ci + x);
                if (in_set(A.inS, w)) {
                    const bool up = vkey(A.k, w) > kv;
                    hi += up;
                    lo += !up;
                }
            }
        }
        unsigned medm = __ballot_sync(FULL, active && e - b > JP_SMALL && e - b <= JP_BUDGET);
        while (medm) {
            const int src = __ffs(medm) - 1;
            medm &= medm - 1;
            const int64_t wb = __shfl_sync(FULL, b, src), we = __shfl_sync(FULL, e, src);
            const uint64_t wk = __shfl_sync(FULL, kv, src);
            uint32_t lh = 0, ll = 0;
            for (int64_t x = wb + lane; x < we; x += 32) {
                const uint32_t w = (uint32_t)__ldg(A.ci + x);
                if (in_set(A.inS, w)) {
                    const bool up = vkey(A.k, w) > wk;
                    lh += up;
                    ll += !up;
                }
            }
            lh = __reduce_add_sync(FULL, lh);
            ll = __reduce_add_sync(FULL, ll);
            if (lane == src) {
                hi = lh;
                lo = ll;
            }
        }
        const bool huge = active && e - b > JP_BUDGET;
        if (active) {
            A.rec[h] = hi;
            A.ldeg[h] = lo;
        }
        const uint32_t np = huge ? (uint32_t)((e - b + JP_PIECE - 1) / JP_PIECE) : 0u;
        const int64_t ps = warp_reserve(np, A.huge_cnt);
        for (uint32_t q = 0; q < np; q++) A.huge[ps + q] = ((int64_t)q << 32) | (uint32_t)h;
    }
}

// counts of the huge rows, one CTA per JP_PIECE-arc piece
__global__ void __launch_bounds__(JP_HUGE_THREADS) k_jpc_count_huge(JpArgs A) {
    const uint32_t cnt = *A.huge_cnt;
    for (uint32_t p = blockIdx.x; p < cnt; p += gridDim.x) {
        const int64_t item = A.huge[p];
        const int32_t h = (int32_t)(uint32_t)item;
        const int64_t j = item >> 32;
        const int32_t v = A.ov[h];
        const int64_t b = A.rp[v], e = A.rp[v + 1];
        const int64_t pb = b + j * JP_PIECE, pe_ = min(e, pb + JP_PIECE);
        const uint64_t kv = vkey(A.k, (uint32_t)v);
        uint32_t lh = 0, ll = 0;
        for (int64_t x = pb + threadIdx.x; x < pe_; x += JP_HUGE_THREADS) {
            const uint32_t w = (uint32_t)__ldg(A.ci + x);
            if (in_set(A.inS, w)) {
                const bool up = vkey(A.k, w) > kv;
                lh += up;
                ll += !up;
            }
        }
        lh = __reduce_add_sync(FULL, lh);
        ll = __reduce_add_sync(FULL, ll);
        if (lane_id() == 0) {
            if (lh) atomicAdd(A.rec + h, (unsigned long long)lh);
            if (ll) atomicAdd(A.ldeg + h, ll);
        }
    }
}

// bitmap words of compact vertex h: cap = (higher + fixed-coloured neighbours) + 1 bits
__device__ __forceinline__ uint32_t jp_words(const JpArgs &A, int64_t h) {
    const int32_t v = A.ov[h];
    const int64_t deg = A.rp[v + 1] - A.rp[v];
    return (uint32_t)((deg - (int64_t)A.ldeg[h] + 1 + 31) >> 5);
}

// per tile of JP_TILE compact ids: (lower arcs, bitmap words)
__global__ void __launch_bounds__(JP_THREADS) k_jpc_sums(JpArgs A) {
    const uint32_t cnt = A.nc[0];
    const int64_t base = (int64_t)blockIdx.x * JP_TILE;
    if (base >= cnt) return;
    unsigned long long sl = 0, sw = 0;
    for (int u = 0; u < JP_TPT; u++) {
        const int64_t h = base + u * JP_THREADS + threadIdx.x;
        if (h < cnt) {
            sl += A.ldeg[h];
            sw += jp_words(A, h) + A.ldeg[h];
        }
    }
    for (int d = 16; d; d >>= 1) {
        sl += __shfl_xor_sync(FULL, sl, d);
        sw += __shfl_xor_sync(FULL, sw, d);
    }
    __shared__ unsigned long long a[2];
    if (threadIdx.x == 0) a[0] = a[1] = 0;
    __syncthreads();
    if (lane_id() == 0) {
        atomicAdd(&a[0], sl);
        atomicAdd(&a[1], sw);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        A.tsum[2 * blockIdx.x] = a[0];
        A.tsum[2 * blockIdx.x + 1] = a[1];
    }
}

// one CTA: exclusive prefix of the tile sums (segment offsets must fit 32 bits)
__global__ void __launch_bounds__(1024) k_jpc_sums_scan(JpArgs A, int64_t ntiles) {
    const uint32_t cnt = A.nc[0];
    const int64_t need = ((int64_t)cnt + JP_TILE - 1) / JP_TILE;
    const int64_t used = need < ntiles ? need : ntiles;
    const int64_t per = (used + blockDim.x - 1) / blockDim.x;
    const int64_t t0 = (int64_t)threadIdx.x * per, t1 = used < t0 + per ? used : t0 + per;
    unsigned long long s0 = 0, s1 = 0;
    for (int64_t t = t0; t < t1; t++) {
        s0 += A.tsum[2 * t];
        s1 += A.tsum[2 * t + 1];
    }
    __shared__ unsigned long long w0[32], w1[32];
    unsigned long long i0 = s0, i1 = s1;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const unsigned long long y0 = __shfl_up_sync(FULL, i0, d), y1 = __shfl_up_sync(FULL, i1, d);
        if (lane_id() >= d) {
            i0 += y0;
            i1 += y1;
        }
    }
    const int wid = threadIdx.x >> 5;
    if (lane_id() == 31) {
        w0[wid] = i0;
        w1[wid] = i1;
    }
    __syncthreads();
    unsigned long long b0 = 0, b1 = 0, T0 = 0, T1 = 0;
    for (int q = 0; q < (int)(blockDim.x >> 5); q++) {
        if (q < wid) {
            b0 += w0[q];
            b1 += w1[q];
        }
        T0 += w0[q];
        T1 += w1[q];
    }
    unsigned long long o0 = b0 + i0 - s0, o1 = b1 + i1 - s1;
    for (int64_t t = t0; t < t1; t++) {
        const unsigned long long a0 = A.tsum[2 * t], a1 = A.tsum[2 * t + 1];
        A.tsum[2 * t] = o0;
        A.tsum[2 * t + 1] = o1;
        o0 += a0;
        o1 += a1;
    }
    if (threadIdx.x == 0 && T1 >= (1ull << 32)) atomicOr(A.err, 2u);
}

// per compact id: the record (count, segment address), a zeroed bitmap, level-0 tasks
__global__ void __launch_bounds__(JP_THREADS) k_jpc_place(JpArgs A) {
    const uint32_t cnt = A.nc[0];
    const int64_t base = (int64_t)blockIdx.x * JP_TILE;
    if (base >= cnt) return;
    __shared__ unsigned long long sm0[8], sm1[8];
    unsigned long long o0 = A.tsum[2 * blockIdx.x], o1 = A.tsum[2 * blockIdx.x + 1];
    for (int u = 0; u < JP_TPT; u++) {
        const int64_t h = base + u * JP_THREADS + threadIdx.x;
        const bool active = h < cnt;
        unsigned long long ld = 0, R = 0, hi = 0;
        if (active) {
            ld = A.ldeg[h];
            R = jp_words(A, h);
            hi = A.rec[h];
        }
        unsigned long long t0, t1;
        const unsigned long long p0 = block_excl_scan<unsigned long long>(ld, sm0, &t0);
        const unsigned long long p1 = block_excl_scan<unsigned long long>(R + ld, sm1, &t1);
        (void)p0;
        uint32_t nt = 0;
        int64_t b = 0;
        unsigned long long boff = 0;
        if (active) {
            boff = o1 + p1;
            b = (int64_t)(boff + R);
            if (hi > JP_CNT_MASK) atomicOr(A.err, 2u);
            A.rec[h] = hi | ((R < JP_RSAT ? R : (unsigned long long)JP_RSAT) << 24) | (boff << 32);
            A.rfull[h] = (uint32_t)R;
            A.ccol[h] = 0;  // fill cursor
            for (unsigned long long q = 0; q < R; q++) A.seg[boff + q] = 0u;
            nt = hi == 0 ? n_tasks((int64_t)ld) : 0u;
        }
        // algorithmic bytes of the levels pass: the lower list (4 B/arc) + per vertex its
        // tasks (32 B written + read), lp pair (16 B), record read (8 B), colour (4 B)
        prof_add(A.prof, active ? 4ull * ld + 92ull : 0ull);
        const int64_t slot = warp_reserve(nt, A.out_cnt);
        for (uint32_t q = 0; q < nt; q++)
            write_task(A.tout + slot + q, b, b + (int64_t)ld, (int32_t)h, q, (boff << 32) | R);
        o0 += t0;
        o1 += t1;
    }
}

// fill pass: lower lists (compact ids, CSR order) and the fixed colours of neighbours
// outside S (COLOR-Rand recolouring) as forbidden bits
__device__ __forceinline__ void jp_fixed(const JpArgs &A, unsigned long long r, int64_t h, uint32_t w) {
    const uint32_t c = A.color[w];
    if (c == 0) return;
    const uint32_t q = (c - 1) >> 5;
    if (q < rec_words(A, r, (uint32_t)h)) atomicOr(A.seg + (r >> 32) + q, 1u << ((c - 1) & 31));
}

__global__ void __launch_bounds__(JP_THREADS) k_jpc_fill(JpArgs A) {
    const uint32_t cnt = A.nc[0];
    const int lane = lane_id();
    const int64_t warp_g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = warp_g * 32; base < cnt; base += nwarps * 32) {
        const int64_t h = base + lane;
        const bool active = h < cnt;
        int32_t v = 0;
        int64_t b = 0, e = 0, o = 0;
        uint64_t kv = 0;
        unsigned long long r = 0;
        if (active) {
            v = A.ov[h];
            b = A.rp[v];
            e = A.rp[v + 1];
            kv = vkey(A.k, (uint32_t)v);
            r = A.rec[h];
            o = (int64_t)(r >> 32) + rec_words(A, r, (uint32_t)h);
        }
        if (active && e - b <= JP_SMALL) {
            for (int64_t x = b; x < e; x++) {
                const uint32_t w = (uint32_t)__ldg(A.ci + x);
                if (!in_set(A.inS, w)) jp_fixed(A, r, h, w);
                else if (vkey(A.k, w) < kv) A.seg[o++] = (uint32_t)A.cid[w];
            }
        }
        unsigned medm = __ballot_sync(FULL, active && e - b > JP_SMALL && e - b <= JP_BUDGET);
        while (medm) {
            const int src = __ffs(medm) - 1;
            medm &= medm - 1;
            const int64_t wb = __shfl_sync(FULL, b, src), we = __shfl_sync(FULL, e, src);
            const uint64_t wk = __shfl_sync(FULL, kv, src);
            const int64_t wh = base + src;
            const unsigned long long wr = __shfl_sync(FULL, r, src);
            int64_t wo = __shfl_sync(FULL, o, src);
            for (int64_t x0 = wb; x0 < we; x0 += 32) {
                const int64_t x = x0 + lane;
                bool low = false;
                uint32_t w = 0;
                if (x < we) {
                    w = (uint32_t)__ldg(A.ci + x);
                    if (!in_set(A.inS, w)) jp_fixed(A, wr, wh, w);
                    else low = vkey(A.k, w) < wk;
                }
                const unsigned m = __ballot_sync(FULL, low);
                if (low) A.seg[wo + __popc(m & ((1u << lane) - 1u))] = (uint32_t)A.cid[w];
                wo += __popc(m);
            }
        }
    }
}

// huge rows: one CTA per piece, positions reserved per warp on the row's cursor
__global__ void __launch_bounds__(JP_HUGE_THREADS) k_jpc_fill_huge(JpArgs A) {
    const uint32_t cnt = *A.huge_cnt;
    const int lane = lane_id();
    for (uint32_t p = blockIdx.x; p < cnt; p += gridDim.x) {
        const int64_t item = A.huge[p];
        const int32_t h = (int32_t)(uint32_t)item;
        const int64_t j = item >> 32;
        const int32_t v = A.ov[h];
        const int64_t b = A.rp[v], e = A.rp[v + 1];
        const int64_t pb = b + j * JP_PIECE, pe_ = min(e, pb + JP_PIECE);
        const uint64_t kv = vkey(A.k, (uint32_t)v);
        const unsigned long long r = A.rec[h];
        const int64_t o = (int64_t)(r >> 32) + rec_words(A, r, (uint32_t)h);
        for (int64_t x0 = pb + (threadIdx.x & ~31); x0 < pe_; x0 += JP_HUGE_THREADS) {
            const int64_t x = x0 + lane;
            bool low = false;
            uint32_t w = 0;
            if (x < pe_) {
                w = (uint32_t)__ldg(A.ci + x);
                if (!in_set(A.inS, w)) jp_fixed(A, r, h, w);
                else low = vkey(A.k, w) < kv;
            }
            const unsigned m = __ballot_sync(FULL, low);
            uint32_t pos = 0;
            if (m && lane == 0) pos = atomicAdd(A.ccol + h, (uint32_t)__popc(m));
            pos = __shfl_sync(FULL, pos, 0);
            if (low) A.seg[o + pos + __popc(m & ((1u << lane) - 1u))] = (uint32_t)A.cid[w];
        }
    }
}

// colours back to original ids
__global__ void k_jpc_scatter(JpArgs A) {
    const uint32_t cnt = A.nc[0];
    for (int64_t h = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; h < cnt; h += (int64_t)gridDim.x * blockDim.x)
        A.color[A.ov[h]] = A.ccol[h];
}

// ---------------------------------------------------------------- one level
// Tasks live in ONE monotone queue (every vertex is enqueued exactly once): level r
// owns slots [lo_r, hi_r).  A 64-bit word W = (arrivals << 32 | tasks reserved) is
// both the grid barrier and the task allocator: at the end of a level each CTA adds
// (1 << 32 | its staged tasks) once -- reservation and arrival in one atomic -- then
// writes its tasks; the last arriver publishes (r+1 << 32 | hi_{r+1}) in the word G
// that the other CTAs poll.  Tasks may land after the barrier, so the queue is
// pre-filled with -1 and a reader waits until its task's three 8-byte words are
// written.  Ready vertices are staged in shared memory (one reservation per CTA and
// level, a hub's tasks written by the whole CTA); a full stage reserves per warp.
constexpr int JP_STAGE = 1024;

struct JpStage {
    uint32_t n;                  // entries appended this level (may exceed JP_STAGE)
    uint32_t base;               // global slot of the CTA's first task
    uint32_t total;              // tasks of the staged entries
    uint32_t wsum[32];           // scan scratch (one per warp)
    int32_t v[JP_STAGE];         // compact ids
    uint32_t deg[JP_STAGE];      // lower degrees
    int64_t b[JP_STAGE];         // lower-list starts
    uint64_t bm[JP_STAGE];       // bitmaps: boff << 32 | R
    uint32_t off[JP_STAGE + 1];  // exclusive prefix of the task counts
};

struct JlCtl {
    unsigned long long *W;  // (arrivals << 32) | tasks reserved (low half = the build's counter)
    unsigned long long *G;  // (level + 1) << 32 | end of that level's tasks, by the last arriver
    uint32_t *err;          // 1 = timeout / max levels, 2 = record field overflow
    uint32_t *levels;       // out: number of levels run
    uint32_t max_levels;
};

__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_release_u64(unsigned long long *p, unsigned long long v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// a task of the current level; waits (bounded by the writer CTA's progress: all CTAs
// are co-resident) until its writer's stores are visible
__device__ __forceinline__ void read_task(const JpTask *q, int64_t &b, int64_t &e, int32_t &h, uint32_t &j,
                                          uint64_t &bm) {
    const volatile long long *p = reinterpret_cast<const volatile long long *>(q);
    long long x0, x1, x2, x3;
    do {
        x0 = p[0];
        x1 = p[1];
        x2 = p[2];
        x3 = p[3];
    } while (x0 == -1 || x1 == -1 || x2 == -1 || x3 == -1);
    b = x0;
    e = x1;
    h = (int32_t)(uint32_t)(unsigned long long)x2;
    j = (uint32_t)((unsigned long long)x2 >> 32);
    bm = (uint64_t)x3;
}

// w became ready: its record r (returned by the decrement) gives the segment address
__device__ __forceinline__ void stage_ready(const JpArgs &A, const JlCtl &C, JpStage &st, int32_t w,
                                            unsigned long long r, uint32_t deg) {
    const uint32_t R = rec_words(A, r, (uint32_t)w);
    const int64_t b = (int64_t)(r >> 32) + R;
    const uint64_t bm = (r >> 32 << 32) | R;
    asm volatile("prefetch.global.L2 [%0];" ::"l"(A.seg + b));  // the list is read next level
    const uint32_t slot = atomicAdd(&st.n, 1u);
    if (slot < JP_STAGE) {
        st.v[slot] = w;
        st.deg[slot] = deg;
        st.b[slot] = b;
        st.bm[slot] = bm;
    } else {  // stage full: reserve directly (no arrival)
        const uint32_t nt = n_tasks(deg);
        const uint32_t base = (uint32_t)atomicAdd(C.W, (unsigned long long)nt);
        for (uint32_t q = 0; q < nt; q++) write_task(A.tout + base + q, b, b + deg, w, q, bm);
    }
}

// CTA-wide end of a level: one atomic = arrival + reservation of the staged entries'
// tasks, then the tasks, then wait for the level's last arrival; returns hi_{r+1}
__device__ __forceinline__ uint32_t stage_flush_barrier(const JpArgs &A, const JlCtl &C, JpStage &st, uint32_t r,
                                                        uint32_t arrivals_expected, uint32_t *trace, uint64_t ts) {
    __syncthreads();
    const uint64_t tw = trace ? globaltimer_ns() : 0;
    const uint32_t n = min(st.n, (uint32_t)JP_STAGE);
    const uint32_t per = (JP_STAGE + blockDim.x - 1) / blockDim.x;
    const uint32_t i0 = threadIdx.x * per;
    uint32_t loc = 0;
    for (uint32_t i = i0; i < min(n, i0 + per); i++) loc += n_tasks(st.deg[i]);
    uint32_t incl = loc;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, incl, d);
        if (lane_id() >= d) incl += y;
    }
    const int wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
    if (lane_id() == 31) st.wsum[wid] = incl;
    __syncthreads();
    if (wid == 0) {
        const uint32_t x = lane_id() < nw ? st.wsum[lane_id()] : 0u;
        uint32_t xi = x;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(FULL, xi, d);
            if (lane_id() >= d) xi += y;
        }
        if (lane_id() < nw) st.wsum[lane_id()] = xi - x;
        if (lane_id() == 31) {
            __threadfence();  // this CTA's pushes (counts, bits, colours) before its arrival
            const unsigned long long old = atomicAdd(C.W, (1ull << 32) | xi);
            st.total = xi;
            st.base = (uint32_t)old;
            if ((uint32_t)(old >> 32) + 1u == arrivals_expected)  // last arriver: publish the level's end
                st_release_u64(C.G, ((unsigned long long)(r + 1) << 32) | (uint32_t)(old + xi));
            if (trace && r < 1024) {  // stats: slowest CTA's work span and flush+arrival span
                const uint64_t ta = globaltimer_ns();
                atomicMax(trace + r, (uint32_t)((tw - ts) >> 5));
                atomicMax(trace + 1024 + r, (uint32_t)((ta - tw) >> 5));
            }
        }
    }
    __syncthreads();
    uint32_t o = st.wsum[wid] + incl - loc;
    for (uint32_t i = i0; i < min(n, i0 + per); i++) {
        st.off[i] = o;
        o += n_tasks(st.deg[i]);
    }
    __syncthreads();
    const uint32_t total = st.total, base = st.base;
    for (uint32_t q = threadIdx.x; q < total; q += blockDim.x) {
        uint32_t lo = 0, hi = n - 1;  // last entry with off <= q
        while (lo < hi) {
            const uint32_t mid = (lo + hi + 1) >> 1;
            if (st.off[mid] <= q) lo = mid;
            else hi = mid - 1;
        }
        write_task(A.tout + base + q, st.b[lo], st.b[lo] + st.deg[lo], st.v[lo], q - st.off[lo], st.bm[lo]);
    }
    if (threadIdx.x == 0) {
        st.n = 0;
        unsigned long long g;
        while (((g = ld_acquire_u64(C.G)) >> 32) < r + 1) {
        }
        st.base = (uint32_t)g;
    }
    __syncthreads();
    return st.base;
}

// decrement the counts of the lower neighbours w[0..U) (flags act[]); each returns
// the neighbour's whole record (count before the push + segment address); the lower
// degrees are loaded beside the atomics (needed only by the vertices that become ready)
template <int U>
__device__ __forceinline__ void jp_decrement(const JpArgs &A, const uint32_t (&w)[U], const bool (&act)[U],
                                             unsigned long long (&old)[U], uint32_t (&ld)[U]) {
#pragma unroll
    for (int u = 0; u < U; u++) old[u] = act[u] ? atomicAdd(A.rec + w[u], ~0ull) : 0ull;
#pragma unroll
    for (int u = 0; u < U; u++) ld[u] = act[u] ? __ldg(A.ldeg + w[u]) : 0u;
}

// forbidden bit of colour c for the lower neighbours (fire-and-forget; skipped when c
// lies beyond w's mex range), then the vertices that became ready go to the stage
template <int U>
__device__ __forceinline__ void jp_mark(const JpArgs &A, const JlCtl &C, JpStage &st, const uint32_t (&w)[U],
                                        const bool (&act)[U], const unsigned long long (&old)[U],
                                        const uint32_t (&ld)[U], uint32_t c) {
    const uint32_t q = (c - 1) >> 5, bit = 1u << ((c - 1) & 31);
#pragma unroll
    for (int u = 0; u < U; u++)
        if (act[u] && q < rec_words(A, old[u], w[u])) atomicOr(A.seg + (old[u] >> 32) + q, bit);
#pragma unroll
    for (int u = 0; u < U; u++)
        if (act[u] && (old[u] & JP_CNT_MASK) == 1ull) stage_ready(A, C, st, (int32_t)w[u], old[u], ld[u]);
}

// mex of h's bitmap (bm = boff << 32 | R), warp-cooperative (a zero lies within the
// first cap bits)
__device__ __forceinline__ uint32_t warp_mex(const JpArgs &A, uint64_t bmw) {
    const uint32_t R = (uint32_t)bmw;
    const uint32_t *bm = A.seg + (bmw >> 32);
    for (uint32_t k0 = 0; k0 < R; k0 += 32) {
        const uint32_t z = k0 + lane_id() < R ? ~__ldcg(bm + k0 + lane_id()) : 0u;
        const unsigned bal = __ballot_sync(FULL, z != 0);
        if (bal) {
            const int src = __ffs(bal) - 1;
            const uint32_t zz = __shfl_sync(FULL, z, src);
            return (k0 + src) * 32 + __ffs(zz);
        }
    }
    return R * 32 + 1;  // unreachable: at most cap-1 of the first cap bits are set
}

// mex by one lane (usually the first word decides)
__device__ __forceinline__ uint32_t lane_mex(const JpArgs &A, uint64_t bmw) {
    const uint32_t R = (uint32_t)bmw;
    const uint32_t *bm = A.seg + (bmw >> 32);
    for (uint32_t k = 0; k < R; k++) {
        const uint32_t z = ~__ldcg(bm + k);
        if (z) return k * 32 + __ffs(z);
    }
    return R * 32 + 1;
}

// One level of push JP over the tasks [lo, hi) of the queue: every task colours its
// vertex (the first chunk writes the colour) and pushes it to the lower neighbours of
// its chunk; vertices whose count reaches 0 are staged for the next level.
__device__ __forceinline__ void jp_level(const JpArgs &A, const JlCtl &C, JpStage &st, uint32_t lo, uint32_t hi,
                                         int64_t warp_g, int64_t nwarps) {
    const int lane = lane_id();
    const uint32_t cnt = hi - lo;
    // task index t = it*32*nwarps + lane*nwarps + warp: consecutive tasks (the chunks
    // of one hub) land on different warps
    for (int64_t base = warp_g; base - warp_g < cnt; base += nwarps * 32) {
        const int64_t t = base + (int64_t)lane * nwarps;
        int32_t h = -1;
        uint32_t j = 0;
        int64_t b = 0, e = 0;
        uint64_t bmw = 0;
        if (t < cnt) read_task(A.tout + lo + t, b, e, h, j, bmw);
        // ---- short lists: one lane does the whole task
        const bool small = h >= 0 && e - b <= JP_LANE;
        if (__any_sync(FULL, small)) {
            uint32_t w[JP_LANE];
            bool act[JP_LANE];
#pragma unroll
            for (int u = 0; u < JP_LANE; u++) {
                act[u] = small && b + u < e;
                w[u] = act[u] ? __ldcs(A.seg + b + u) : 0u;
            }
            unsigned long long old[JP_LANE];
            uint32_t ld[JP_LANE];
            jp_decrement<JP_LANE>(A, w, act, old, ld);
            uint32_t c = 1;
            if (small) {
                c = lane_mex(A, bmw);
                A.ccol[h] = c;
            }
            jp_mark<JP_LANE>(A, C, st, w, act, old, ld, c);
        }
        // ---- longer lists: the warp takes these tasks one by one (<= JP_CHUNK arcs)
        unsigned bigm = __ballot_sync(FULL, h >= 0 && !small);
        while (bigm) {
            const int src = __ffs(bigm) - 1;
            bigm &= bigm - 1;
            const int32_t th = __shfl_sync(FULL, h, src);
            const uint32_t tj = __shfl_sync(FULL, j, src);
            const int64_t tb = __shfl_sync(FULL, b, src), te = __shfl_sync(FULL, e, src);
            const uint64_t tbm = __shfl_sync(FULL, bmw, src);
            const int64_t cb = tb + (int64_t)tj * JP_CHUNK;
            constexpr int U = JP_CHUNK / 32;
            uint32_t w[U];
            bool act[U];
#pragma unroll
            for (int u = 0; u < U; u++) {
                const int64_t x = cb + u * 32 + lane;
                act[u] = x < te;
                w[u] = act[u] ? __ldcs(A.seg + x) : 0u;
            }
            unsigned long long old[U];
            uint32_t ld[U];
            jp_decrement<U>(A, w, act, old, ld);  // the decrements do not wait for the mex
            const uint32_t c = warp_mex(A, tbm);
            if (tj == 0 && lane == 0) A.ccol[th] = c;
            jp_mark<U>(A, C, st, w, act, old, ld, c);
        }
    }
}

// ---------------------------------------------------------------- persistent levels
// All levels in ONE cooperative launch (grid = one or more CTAs per SM, all
// co-resident): level r = jp_level over [lo_r, hi_r), then stage_flush_barrier.  The
// barrier orders the pushes of level r before the mex reads of level r+1, so no
// per-push fence is needed.
constexpr int JL_THREADS = 512;
#ifndef SYM_JL_MINB
#define SYM_JL_MINB 1
#endif
constexpr uint64_t JL_TIMEOUT_NS = 20ull * 1000 * 1000 * 1000;

__global__ void __launch_bounds__(JL_THREADS, SYM_JL_MINB) k_jp_levels(JpArgs A, JlCtl C) {
    __shared__ JpStage st;
    if (threadIdx.x == 0) st.n = 0;
    __syncthreads();
    // warp-in-CTA major: consecutive tasks (the chunks of one row) go to different SMs
    const int64_t warp_g = (int64_t)(threadIdx.x >> 5) * gridDim.x + blockIdx.x;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t t0 = globaltimer_ns();
    uint32_t lo = 0, hi = (uint32_t)__ldcg(C.W);  // level 0 = the build pass's tasks
    uint32_t r = 0;
    uint32_t *trace = A.trace;
    for (;; r++) {
        if (hi == lo || __ldcg(C.err) != 0) break;
        const uint64_t ts = trace ? globaltimer_ns() : 0;
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            if (A.hist && r < 1024) {  // stats: tasks and start time (32 ns units) of the first levels
                A.hist[r] = hi - lo;
                A.hist[1024 + r] = (uint32_t)((globaltimer_ns() - t0) >> 5);
            }
            if (r + 1 >= C.max_levels || globaltimer_ns() - t0 > JL_TIMEOUT_NS) atomicOr(C.err, 1u);
        }
        jp_level(A, C, st, lo, hi, warp_g, nwarps);
        const uint32_t next = stage_flush_barrier(A, C, st, r, (r + 1) * gridDim.x, trace, ts);
        lo = hi;
        hi = next;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) *C.levels = r;
}

// ---------------------------------------------------------------- fix-up kernels
// COLOR-Degk (Alg 9): L colours are shifted past max(C_H)
__global__ void k_color_max_h(const uint32_t *color, const uint32_t *hbits, int64_t n, uint32_t *mx) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    uint32_t m = 0;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
        if ((hbits[v >> 5] >> (v & 31)) & 1u) m = max(m, color[v]);
    for (int d = 16; d; d >>= 1) m = max(m, __shfl_xor_sync(FULL, m, d));
    if (lane_id() == 0 && m) atomicMax(mx, m);
}

__global__ void k_color_shift_l(uint32_t *color, const uint32_t *hbits, int64_t n, const uint32_t *mx) {
    const uint32_t M = *mx;
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
        if (!((hbits[v >> 5] >> (v & 31)) & 1u)) color[v] += M;
}

// COLOR-Rand (Alg 8): V' = endpoints of monochromatic cross arcs
__global__ void k_color_conflicts(const int64_t *__restrict__ rp_x, const int32_t *__restrict__ ci_x, int64_t n,
                                  const uint32_t *color, uint8_t *mark, int32_t *list, uint32_t *cnt) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n; base += stride) {
        int64_t v = base + threadIdx.x;
        bool conf = false;
        if (v < n) {
            uint32_t cv = color[v];
            for (int64_t x = rp_x[v]; x < rp_x[v + 1] && !conf; x++) conf = color[ci_x[x]] == cv;
            mark[v] = conf ? 1 : 0;
        }
        int64_t s = warp_append(conf, cnt);
        if (s >= 0) list[s] = (int32_t)v;
    }
}

__global__ void k_color_reset(const int32_t *list, const uint32_t *cnt, uint32_t *color) {
    const uint32_t c = *cnt;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < c; i += gridDim.x * blockDim.x) color[list[i]] = 0;
}

__global__ void k_color_max(const uint32_t *color, int64_t n, uint32_t *mx) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    uint32_t m = 0;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) m = max(m, color[v]);
    for (int d = 16; d; d >>= 1) m = max(m, __shfl_xor_sync(FULL, m, d));
    if (lane_id() == 0 && m) atomicMax(mx, m);
}

// ---------------------------------------------------------------- host side
void carve_color_ws(Arena &a, int64_t n, int64_t nnz, ColorWs &w) {
    const int64_t ntiles = (n + JP_TILE - 1) / JP_TILE + 1;
    w.cid = a.take<int32_t>((size_t)n + 1);
    w.ov = a.take<int32_t>((size_t)n + 1);
    w.ldeg = a.take<uint32_t>((size_t)n + 1);
    w.rfull = a.take<uint32_t>((size_t)n + 1);
    w.ccol = a.take<uint32_t>((size_t)n + 1);
    w.rec = a.take<unsigned long long>((size_t)n + 2);
    // segments: bitmaps, sum of ceil(cap/32) <= (nnz + n)/32 + n words, and lower
    // lists, one id per S-S edge (<= nnz/2)
    w.seg_words = (nnz + n) / 32 + n + nnz / 2 + 2;
    w.seg = a.take<uint32_t>((size_t)w.seg_words);
    w.tcnt = a.take<uint32_t>(2 * (size_t)ntiles);
    w.tsum = a.take<unsigned long long>(2 * (size_t)ntiles);
    w.ntiles = ntiles;
    w.queue_cap = n + nnz / (2 * JP_CHUNK) + 2;  // every vertex is enqueued once
    w.task = a.take<int64_t>((size_t)w.queue_cap * (sizeof(JpTask) / sizeof(int64_t)));
    w.vlist = a.take<int32_t>((size_t)n + 1);
    w.mark = a.take<uint8_t>((size_t)n + 1);
    w.queue = a.take<int64_t>((size_t)(nnz / JP_BUDGET + 2));  // huge-row pieces (<= nnz/JP_BUDGET)
    w.sync = a.take<uint32_t>(64);  // levels kernel: barrier words, apart from the task counters
}

// JP over (rp, ci) for the vertex set S (list/implicit) with membership inS.
// Build: compact ids, the oriented lower-neighbour DAG, records + bitmaps, and the
// level-0 tasks at the head of the queue (counter = the low half of W).
static int jp_build(const FlowArgs &f, ColorWs &w, JpArgs &A, uint32_t *color, const int64_t *rp,
                    const int32_t *ci, const uint8_t *inS, const int32_t *list0, const uint32_t *cnt0,
                    int64_t implicit_n, JpTask *q, uint32_t *qcnt, uint32_t *err) {
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
    const int64_t n = f.g.n;
    SYM_CUDA(cudaMemsetAsync(ctl->huge, 0, sizeof(ctl->huge), s));
    A.rp = rp;
    A.ci = ci;
    A.inS = inS;
    A.color = color;
    A.in_list = list0;
    A.in_cnt = cnt0;
    A.implicit_n = implicit_n;
    A.cid = w.cid;
    A.ov = w.ov;
    A.ldeg = w.ldeg;
    A.rfull = w.rfull;
    A.rec = w.rec;
    A.seg = w.seg;
    A.ccol = w.ccol;
    A.tcnt = w.tcnt;
    A.tsum = w.tsum;
    A.nc = w.sync + 40;
    A.tout = q;
    A.out_cnt = qcnt;
    A.huge = w.queue;
    A.huge_cnt = &ctl->huge[1];
    A.err = err;
    A.hist = nullptr;
    A.trace = nullptr;
    A.prof = prof_counter(s);
    A.k = stream_key(f.p.seed, TAG_VERTEX, 0);
    const int64_t smax = list0 ? n : implicit_n;  // positions of S (upper bound for a list)
    const unsigned tiles_s = (unsigned)((smax + JP_TILE - 1) / JP_TILE);
    const unsigned tiles_c = (unsigned)((n + JP_TILE - 1) / JP_TILE);  // compact ids <= n
    prof_begin("jp_build", s);
    if (tiles_s) {
        k_jpc_tiles<<<tiles_s, JP_THREADS, 0, s>>>(A);
        SYM_LAUNCH_CHECK();
    }
    k_jpc_tiles_scan<<<1, 1024, 0, s>>>(A, tiles_s);
    SYM_LAUNCH_CHECK();
    if (tiles_s) {
        k_jpc_assign<<<tiles_s, JP_THREADS, 0, s>>>(A);
        SYM_LAUNCH_CHECK();
    }
    k_jpc_count<<<num_sms() * (2048 / JP_THREADS), JP_THREADS, 0, s>>>(A);
    SYM_LAUNCH_CHECK();
    k_jpc_count_huge<<<num_sms() * 4, JP_HUGE_THREADS, 0, s>>>(A);
    SYM_LAUNCH_CHECK();
    if (tiles_c) {
        k_jpc_sums<<<tiles_c, JP_THREADS, 0, s>>>(A);
        SYM_LAUNCH_CHECK();
    }
    k_jpc_sums_scan<<<1, 1024, 0, s>>>(A, tiles_c);
    SYM_LAUNCH_CHECK();
    if (tiles_c) {
        k_jpc_place<<<tiles_c, JP_THREADS, 0, s>>>(A);
        SYM_LAUNCH_CHECK();
    }
    k_jpc_fill<<<num_sms() * (2048 / JP_THREADS), JP_THREADS, 0, s>>>(A);
    SYM_LAUNCH_CHECK();
    k_jpc_fill_huge<<<num_sms() * 4, JP_HUGE_THREADS, 0, s>>>(A);
    SYM_LAUNCH_CHECK();
    prof_end(s, -1);
    return SYM_OK;
}

// every level in one persistent cooperative launch
static int jp_run(const FlowArgs &f, ColorWs &w, uint32_t *color, const int64_t *rp, const int32_t *ci,
                  const uint8_t *inS, const int32_t *list0, const uint32_t *cnt0, int64_t implicit_n, int phase) {
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
    if (f.g.n == 0) return SYM_OK;
    static int grid = 0;
    if (grid == 0) {
        int dev = 0, coop = 0, per_sm = 0;
        SYM_CUDA(cudaGetDevice(&dev));
        SYM_CUDA(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, dev));
        if (!coop) {
            set_error("JP needs cooperative launch (persistent levels kernel), unsupported on this device");
            return SYM_ECUDA;
        }
        SYM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_jp_levels, JL_THREADS, 0));
        if (per_sm < 1) {
            set_error("k_jp_levels does not fit on an SM");
            return SYM_ECUDA;
        }
        grid = num_sms() * per_sm;
    }
    JpTask *q = reinterpret_cast<JpTask *>(w.task);
    const int64_t qcap = w.queue_cap;
    if (qcap >= (int64_t)0xffffffff) {
        set_error("JP task queue exceeds 2^32 entries");
        return SYM_EINVAL;
    }
    // W (u64) = sync[0..1], G (u64) = sync[2..3], err = sync[32], levels = sync[33],
    // build counts = sync[40..41]
    SYM_CUDA(cudaMemsetAsync(w.sync, 0, 64 * sizeof(uint32_t), s));
    SYM_CUDA(cudaMemsetAsync(q, 0xff, sizeof(JpTask) * (size_t)qcap, s));
    JlCtl C;
    C.W = reinterpret_cast<unsigned long long *>(w.sync);
    C.G = reinterpret_cast<unsigned long long *>(w.sync + 2);
    C.err = &w.sync[32];
    C.levels = &w.sync[33];
    C.max_levels = f.p.max_rounds ? f.p.max_rounds : 0xffffffffu;
    // arrivals (levels x grid) must not overflow the high half of W
    C.max_levels = std::min<uint64_t>(C.max_levels, 0xffffffffull / (uint64_t)grid - 1);
    JpArgs A;
    SYM_TRY(jp_build(f, w, A, color, rp, ci, inS, list0, cnt0, implicit_n, q, w.sync /* low half of W */, C.err));
    // stats: per-level task counts and start times; phase 0 also traces the level
    // spans into hist[2048..4095] (SYM_JP_TRACE=1 in the environment)
    static const bool jp_trace = getenv("SYM_JP_TRACE") != nullptr;
    A.hist = f.stats ? ctl->hist + phase * 2048 : nullptr;
    A.trace = jp_trace && phase == 0 && A.hist ? ctl->hist + 2048 : nullptr;
    if (A.trace) SYM_CUDA(cudaMemsetAsync(A.trace, 0, 2048 * sizeof(uint32_t), s));
    unsigned long long *ctr = A.prof;
    A.prof = nullptr;
    void *args[] = {&A, &C};
    prof_begin("jp_levels", s);
    SYM_CUDA(cudaLaunchCooperativeKernel((const void *)k_jp_levels, dim3(grid), dim3(JL_THREADS), args, 0, s));
    prof_end_dev(s, ctr);
    k_jpc_scatter<<<num_sms() * 8, 256, 0, s>>>(A);
    SYM_LAUNCH_CHECK();
    uint32_t err = 0, levels = 0;
    SYM_TRY(read_u32(C.err, &err, s));
    if (err) {
        SYM_TRY(read_u32(C.levels, &levels, s));
        if (err & 2u) {
            set_error("JP: a vertex count or bitmap offset exceeds the record fields (degree >= 2^24)");
            return SYM_EINVAL;
        }
        const bool rounds = f.p.max_rounds && levels + 1 >= f.p.max_rounds;
        set_error(rounds ? "JP did not converge within max_rounds" : "JP levels kernel timed out");
        return rounds ? SYM_EROUNDS : SYM_ECUDA;
    }
    if (f.stats) {
        SYM_TRY(read_u32(C.levels, &levels, s));
        f.stats->rounds[phase] = levels;
    }
    return SYM_OK;
}

int run_color(const FlowArgs &f, ColorWs &w, uint32_t *color) {
    const Graph &g = f.g;
    cudaStream_t s = f.stream;
    Ctl *ctl = f.ctl;
    const int kind = f.p.kind;
    SYM_CUDA(cudaMemsetAsync(color, 0, sizeof(uint32_t) * (size_t)g.n, s));
    if (kind == SYM_DECOMP_NONE) {
        SYM_TRY(jp_run(f, w, color, g.rp, g.ci, nullptr, nullptr, nullptr, g.n, 0));
    } else if (kind == SYM_DECOMP_DEGK) {
        // C_H on G_H and C_L on G_L: both are components of the intra CSR
        SYM_TRY(launch_classify_degk(g, f.p.param, f.hbits, nullptr, ctl, s));
        SYM_TRY(jp_run(f, w, color, f.split.rp_in, f.split.ci_in, nullptr, nullptr, nullptr, g.n, 0));
        SYM_CUDA(cudaMemsetAsync(&ctl->max_color, 0, sizeof(uint32_t), s));
        k_color_max_h<<<num_sms() * 8, 256, 0, s>>>(color, f.hbits, g.n, &ctl->max_color);
        SYM_LAUNCH_CHECK();
        k_color_shift_l<<<num_sms() * 8, 256, 0, s>>>(color, f.hbits, g.n, &ctl->max_color);
        SYM_LAUNCH_CHECK();
    } else {
        // C_IS on the induced subgraphs with one palette
        SYM_TRY(jp_run(f, w, color, f.split.rp_in, f.split.ci_in, nullptr, nullptr, nullptr, g.n, 0));
        // V' = endpoints of monochromatic cross edges; uncolour them
        SYM_CUDA(cudaMemsetAsync(&ctl->conflicts, 0, sizeof(uint32_t), s));
        k_color_conflicts<<<num_sms() * 8, 256, 0, s>>>(f.split.rp_x, f.split.ci_x, g.n, color, w.mark, w.vlist,
                                                          &ctl->conflicts);
        SYM_LAUNCH_CHECK();
        k_color_reset<<<num_sms() * 4, 256, 0, s>>>(w.vlist, &ctl->conflicts, color);
        SYM_LAUNCH_CHECK();
        // recolour V' by JP against all of G
        SYM_TRY(jp_run(f, w, color, g.rp, g.ci, w.mark, w.vlist, &ctl->conflicts, 0, 1));
    }
    if (f.stats) {
        SYM_CUDA(cudaMemsetAsync(&ctl->flag, 0, sizeof(uint32_t), s));
        k_color_max<<<num_sms() * 8, 256, 0, s>>>(color, g.n, &ctl->flag);
        SYM_LAUNCH_CHECK();
        uint32_t mx = 0, conf = 0;
        SYM_TRY(read_u32(&ctl->flag, &mx, s));
        SYM_TRY(read_u32(&ctl->conflicts, &conf, s));
        f.stats->max_color = mx;
        f.stats->result_size = mx;
        f.stats->conflicts = conf;
    }
    return SYM_OK;
}

}  // namespace sym
