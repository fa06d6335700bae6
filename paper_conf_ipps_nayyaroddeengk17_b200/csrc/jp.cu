// jp.cu -- Jones-Plassmann colouring and the COLOR flows.
//
// JP ([18]) with fixed priorities colours v once every higher-(pv,id)
// neighbour of its phase set S is coloured, with the smallest colour >= 1 not held by
// any coloured neighbour: exactly first-fit greedy in priority order (DESIGN §3 C1).
//
// Push form with forbidden-colour sets (the FORBIDDEN array of P:214/P:234):
//   record  every S vertex owns one 32-byte record {cnt, deg, row start, bits of the
//           colours 1..JP_WIN}: a push to w touches ONE sector and needs no row-pointer
//           load.  Colours > JP_WIN (the dense core only: ~1 % of pushes at R-MAT s24)
//           go to an overflow bitmap addressed by the row (bit offset row_ptr[w] + w,
//           deg+1 bits, since mex <= deg+1).
//   init    cnt[v] = #higher S-neighbours; fixed colours of neighbours outside S
//           (COLOR-Rand recolouring) are pre-set; cnt == 0 -> ready (a ready vertex
//           without phase arcs takes colour 1 at once).
//   level   every ready vertex v is split into tasks of <= JP_CHUNK arcs that carry
//           v's row bounds.  A task computes colour(v) = mex of v's forbidden set
//           (complete: every higher neighbour pushed in an earlier level) and, for
//           each lower S-neighbour w of its chunk, decrements cnt[w] and sets bit
//           colour(v) of w; the decrement reaching 0 appends w's tasks for the next
//           level.  Rows <= JP_LANE arcs are one lane's task, longer chunks a warp's.
// Levels = the JP dependency depth (~5e3 on R-MAT scale 24); each level is a burst of
// ~5e4 scattered pushes, so the cost per level is the latency of that burst plus one
// grid barrier: all levels run inside ONE persistent cooperative kernel (k_jp_levels)
// with a software grid barrier between levels.
#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include "internal.h"

namespace sym {

constexpr int JP_SMALL = 32;     // init: rows <= JP_SMALL arcs are counted by one lane
constexpr int JP_BUDGET = 4096;  // init: rows > JP_BUDGET arcs are split into pieces
constexpr int JP_THREADS = 256;
constexpr int JP_HUGE_THREADS = 512;
#ifndef SYM_JP_CHUNK
#define SYM_JP_CHUNK 64
#endif
constexpr int JP_CHUNK = SYM_JP_CHUNK;  // arcs per warp task (2 per lane: few pushes in flight per warp)
constexpr int JP_LANE = 8;              // rows with <= JP_LANE arcs are a lane task
constexpr int JP_PIECE = 8192;          // arcs per CTA piece of a huge row in the init pass
constexpr uint32_t JP_WIN = 128;        // colours held in the record
#ifndef JP_LDCI
#define JP_LDCI __ldcs  // column loads: streaming, so the hot records stay in L2
#endif

// per-vertex record (one 32-byte sector)
struct __align__(32) JpRec {
    uint32_t cnt;       // higher S-neighbours not yet coloured
    uint32_t deg;       // phase degree
    int64_t b;          // row_ptr[v] of the phase CSR
    uint32_t win[4];    // forbidden colours 1..JP_WIN
};
static_assert(sizeof(JpRec) == 32, "JpRec layout");

// a task: one chunk of a ready vertex's row, with the row bounds
struct __align__(16) JpTask {
    int64_t b, e;     // row_ptr[v], row_ptr[v+1]
    int32_t v;
    uint32_t j;       // chunk index
    int64_t pad;
};
static_assert(sizeof(JpTask) == 32, "JpTask layout");

struct JpArgs {
    const int64_t *rp;
    const int32_t *ci;
    const uint8_t *inS;  // nullable: S = all vertices
    uint32_t *color;
    JpRec *rec;
    uint32_t *bits;      // overflow bitmaps (colours > JP_WIN)
    const int32_t *in_list;    // init: vertex list (nullable = implicit)
    const uint32_t *in_cnt;
    int64_t implicit_n;
    JpTask *tout;         // the task queue (monotone; level r owns [lo_r, hi_r))
    uint32_t *out_cnt;    // init: task counter (the low half of the levels kernel's W)
    int64_t *huge;        // init: (piece << 32 | v) items of the huge rows
    uint32_t *huge_cnt;
    uint32_t *hist;
    Key k;
};

__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ bool in_set(const uint8_t *inS, uint32_t w) { return inS == nullptr || inS[w] != 0; }

__device__ __forceinline__ uint32_t n_tasks(int64_t deg) {
    return deg <= 0 ? 1u : (uint32_t)((deg + JP_CHUNK - 1) / JP_CHUNK);
}

__device__ __forceinline__ void put_tasks(JpTask *out, int64_t slot, int32_t v, int64_t b, int64_t e, uint32_t nt) {
    for (uint32_t q = 0; q < nt; q++) {
        JpTask t;
        t.b = b;
        t.e = e;
        t.v = v;
        t.j = q;
        t.pad = 0;
        out[slot + q] = t;
    }
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

// overflow bit of colour c (> JP_WIN) in the bitmap of a vertex with row start b, degree d
__device__ __forceinline__ void set_overflow(uint32_t *bits, int64_t b, int32_t v, uint32_t d, uint32_t c) {
    if (c <= d + 1) {
        const int64_t pos = b + v + c - 1;
        atomicOr(bits + (pos >> 5), 1u << (pos & 31));
    }
}

// colour c is forbidden for v (window bits accumulated by the caller; overflow direct)
__device__ __forceinline__ void note_colour(uint32_t (&win)[4], uint32_t *bits, int64_t b, int32_t v, uint32_t d,
                                            uint32_t c) {
    if (c == 0) return;
    if (c <= JP_WIN) win[(c - 1) >> 5] |= 1u << ((c - 1) & 31);
    else set_overflow(bits, b, v, d, c);
}

__device__ __forceinline__ void store_rec(JpRec *r, uint32_t cnt, uint32_t deg, int64_t b, const uint32_t (&win)[4]) {
    uint4 *p = reinterpret_cast<uint4 *>(r);
    p[0] = make_uint4(cnt, deg, (uint32_t)(uint64_t)b, (uint32_t)((uint64_t)b >> 32));
    p[1] = make_uint4(win[0], win[1], win[2], win[3]);
}

// mex of v's forbidden set (colours 1..deg+1), warp-cooperative: window first, then
// the overflow bitmap from colour JP_WIN+1
__device__ __forceinline__ uint32_t warp_mex(const JpRec *r, const uint32_t *bits, int64_t B, uint32_t deg) {
    const int lane = lane_id();
    const uint32_t nbits = deg + 1;
    {
        const uint4 wv = __ldcg(reinterpret_cast<const uint4 *>(r) + 1);
        const uint32_t wd[4] = {wv.x, wv.y, wv.z, wv.w};
#pragma unroll
        for (int q = 0; q < 4; q++) {
            const uint32_t lo = 32u * q;
            if (lo >= nbits) break;
            const uint32_t width = min(32u, nbits - lo);
            const uint32_t z = ~wd[q] & (width >= 32 ? 0xffffffffu : ((1u << width) - 1u));
            if (z) return lo + __ffs(z);
        }
    }
    // overflow: bit positions B + JP_WIN .. B + nbits - 1 (colour = position - B + 1)
    const int64_t end = B + nbits;
    const int64_t w0 = (B + JP_WIN) >> 5, w1 = (end - 1) >> 5;
    for (int64_t k0 = w0; k0 <= w1; k0 += 32) {
        const int64_t wi = k0 + lane;
        uint32_t zeros = 0;
        if (wi <= w1) {
            const uint32_t word = __ldcg(bits + wi);
            const int64_t lo = max(B + (int64_t)JP_WIN, wi * 32) - wi * 32, hi = min(end, wi * 32 + 32) - wi * 32;
            const uint32_t width = (uint32_t)(hi - lo);
            const uint32_t mask = (width >= 32 ? 0xffffffffu : ((1u << width) - 1u)) << lo;
            zeros = ~word & mask;
        }
        const unsigned bal = __ballot_sync(FULL, zeros != 0);
        if (bal) {
            const int src = __ffs(bal) - 1;
            const uint32_t z = __shfl_sync(FULL, zeros, src);
            const int64_t pos = (k0 + src) * 32 + __ffs(z) - 1;
            return (uint32_t)(pos - B + 1);
        }
    }
    return nbits;  // unreachable: at most deg bits can be set
}

// mex of a short row (deg <= JP_LANE < 32): window word 0 only
__device__ __forceinline__ uint32_t lane_mex(const JpRec *r, uint32_t deg) {
    const uint32_t w0 = __ldcg(&r->win[0]);
    return (uint32_t)__ffs(~w0 & ((1u << (deg + 1)) - 1u));
}

// ---------------------------------------------------------------- init
// record of every S vertex: cnt = #higher S-neighbours, fixed colours of non-S
// neighbours; ready vertices enqueue their level-0 tasks; huge rows are deferred
__global__ void __launch_bounds__(JP_THREADS) k_jp_init(JpArgs A) {
    const uint32_t cnt = A.in_list ? *A.in_cnt : (uint32_t)A.implicit_n;
    const int lane = lane_id();
    const int64_t warp_g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = warp_g * 32; base < cnt; base += nwarps * 32) {
        const int64_t i = base + lane;
        int32_t v = -1;
        if (i < cnt) v = A.in_list ? A.in_list[i] : (int32_t)i;
        const bool active = v >= 0;
        int64_t b = 0, e = 0;
        uint64_t kv = 0;
        if (active) {
            b = A.rp[v];
            e = A.rp[v + 1];
            kv = vkey(A.k, (uint32_t)v);
        }
        const uint32_t deg = (uint32_t)(e - b);
        uint32_t c = 0;
        uint32_t win[4] = {0u, 0u, 0u, 0u};
        if (active && e - b <= JP_SMALL) {
            for (int64_t x = b; x < e; x++) {
                const uint32_t w = (uint32_t)__ldg(A.ci + x);
                if (in_set(A.inS, w)) c += vkey(A.k, w) > kv ? 1u : 0u;
                else note_colour(win, A.bits, b, v, deg, A.color[w]);
            }
        }
        unsigned medm = __ballot_sync(FULL, active && e - b > JP_SMALL && e - b <= JP_BUDGET);
        while (medm) {
            const int src = __ffs(medm) - 1;
            medm &= medm - 1;
            const int64_t wb = __shfl_sync(FULL, b, src), we = __shfl_sync(FULL, e, src);
            const uint64_t wk = __shfl_sync(FULL, kv, src);
            const int32_t wv = __shfl_sync(FULL, v, src);
            uint32_t lc = 0;
            uint32_t lw[4] = {0u, 0u, 0u, 0u};
            for (int64_t x = wb + lane; x < we; x += 32) {
                const uint32_t w = (uint32_t)__ldg(A.ci + x);
                if (in_set(A.inS, w)) lc += vkey(A.k, w) > wk ? 1u : 0u;
                else note_colour(lw, A.bits, wb, wv, (uint32_t)(we - wb), A.color[w]);
            }
            lc = __reduce_add_sync(FULL, lc);
#pragma unroll
            for (int q = 0; q < 4; q++) lw[q] = __reduce_or_sync(FULL, lw[q]);
            if (lane == src) {
                c = lc;
#pragma unroll
                for (int q = 0; q < 4; q++) win[q] = lw[q];
            }
        }
        const bool huge = active && e - b > JP_BUDGET;
        if (active) store_rec(A.rec + v, huge ? 0u : c, deg, b, win);
        bool ready = active && !huge && c == 0;
        if (ready && e == b) {  // no phase neighbour: colour 1 now, no task
            A.color[v] = 1u;
            ready = false;
        }
        const uint32_t nt = ready ? n_tasks(e - b) : 0u;
        const int64_t slot = warp_reserve(nt, A.out_cnt);
        put_tasks(A.tout, slot, v, b, e, nt);
        // huge rows: one (v, piece) entry per JP_PIECE arcs, counted by k_jp_init_huge
        const uint32_t np = huge ? (uint32_t)((e - b + JP_PIECE - 1) / JP_PIECE) : 0u;
        const int64_t ps = warp_reserve(np, A.huge_cnt);
        for (uint32_t q = 0; q < np; q++) A.huge[ps + q] = ((int64_t)q << 32) | (uint32_t)v;
    }
}

// counts of the huge rows, one CTA per JP_PIECE-arc piece (a 4e5-arc hub is spread
// over ~50 CTAs instead of serialising one CTA)
__global__ void __launch_bounds__(JP_HUGE_THREADS) k_jp_init_huge(JpArgs A) {
    const uint32_t cnt = *A.huge_cnt;
    for (uint32_t h = blockIdx.x; h < cnt; h += gridDim.x) {
        const int64_t item = A.huge[h];
        const int32_t v = (int32_t)(uint32_t)item;
        const int64_t j = item >> 32;
        const int64_t b = A.rp[v], e = A.rp[v + 1];
        const uint32_t deg = (uint32_t)(e - b);
        const int64_t pb = b + j * JP_PIECE, pe_ = min(e, pb + JP_PIECE);
        const uint64_t kv = vkey(A.k, (uint32_t)v);
        uint32_t lc = 0;
        uint32_t lw[4] = {0u, 0u, 0u, 0u};
        for (int64_t x = pb + threadIdx.x; x < pe_; x += JP_HUGE_THREADS) {
            const uint32_t w = (uint32_t)__ldg(A.ci + x);
            if (in_set(A.inS, w)) lc += vkey(A.k, w) > kv ? 1u : 0u;
            else note_colour(lw, A.bits, b, v, deg, A.color[w]);
        }
        lc = __reduce_add_sync(FULL, lc);
#pragma unroll
        for (int q = 0; q < 4; q++) lw[q] = __reduce_or_sync(FULL, lw[q]);
        if (lane_id() == 0) {
            if (lc) atomicAdd(&A.rec[v].cnt, lc);
#pragma unroll
            for (int q = 0; q < 4; q++)
                if (lw[q]) atomicOr(&A.rec[v].win[q], lw[q]);
        }
    }
}

// huge rows whose count is 0 are ready for level 0
__global__ void k_jp_huge_ready(JpArgs A) {
    const uint32_t cnt = *A.huge_cnt;
    for (uint32_t h = blockIdx.x * blockDim.x + threadIdx.x; h < cnt; h += gridDim.x * blockDim.x) {
        const int64_t item = A.huge[h];
        if ((item >> 32) != 0) continue;
        const int32_t v = (int32_t)(uint32_t)item;
        if (A.rec[v].cnt != 0) continue;
        const int64_t b = A.rp[v], e = A.rp[v + 1];
        const uint32_t nt = n_tasks(e - b);
        const int64_t slot = atomicAdd(A.out_cnt, nt);
        put_tasks(A.tout, slot, v, b, e, nt);
    }
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
    int32_t v[JP_STAGE];
    uint32_t deg[JP_STAGE];
    int64_t b[JP_STAGE];
    uint32_t off[JP_STAGE + 1];  // exclusive prefix of the task counts
};

struct JlCtl {
    unsigned long long *W;  // (arrivals << 32) | tasks reserved (low half = init's counter)
    unsigned long long *G;  // (level + 1) << 32 | end of that level's tasks, by the last arriver
    uint32_t *err;          // 1 = timeout / max levels
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

__device__ __forceinline__ void write_task(JpTask *q, int64_t b, int64_t e, int32_t v, uint32_t j) {
    longlong2 *p = reinterpret_cast<longlong2 *>(q);
    p[0] = make_longlong2(b, e);
    p[1] = make_longlong2((long long)(((uint64_t)j << 32) | (uint32_t)v), 0);
}

// a task of the current level; waits (bounded by the writer CTA's progress: all CTAs
// are co-resident) until its writer's stores are visible
__device__ __forceinline__ void read_task(const JpTask *q, int64_t &b, int64_t &e, int32_t &v, uint32_t &j) {
    const volatile long long *p = reinterpret_cast<const volatile long long *>(q);
    long long x0, x1, x2;
    do {
        x0 = p[0];
        x1 = p[1];
        x2 = p[2];
    } while (x0 == -1 || x1 == -1 || x2 == -1);
    b = x0;
    e = x1;
    v = (int32_t)(uint32_t)(unsigned long long)x2;
    j = (uint32_t)((unsigned long long)x2 >> 32);
}

__device__ __forceinline__ void stage_ready(const JpArgs &A, const JlCtl &C, JpStage &st, int32_t w, int64_t b,
                                            uint32_t deg) {
    asm volatile("prefetch.global.L2 [%0];" ::"l"(A.ci + b));  // the row is read next level
    const uint32_t slot = atomicAdd(&st.n, 1u);
    if (slot < JP_STAGE) {
        st.v[slot] = w;
        st.deg[slot] = deg;
        st.b[slot] = b;
    } else {  // stage full: reserve directly (no arrival)
        const uint32_t nt = n_tasks(deg);
        const uint32_t base = (uint32_t)atomicAdd(C.W, (unsigned long long)nt);
        for (uint32_t q = 0; q < nt; q++) write_task(A.tout + base + q, b, b + deg, w, q);
    }
}

// CTA-wide end of a level: one atomic = arrival + reservation of the staged entries'
// tasks, then the tasks, then wait for the level's last arrival; returns hi_{r+1}
__device__ __forceinline__ uint32_t stage_flush_barrier(const JpArgs &A, const JlCtl &C, JpStage &st, uint32_t r,
                                                        uint32_t arrivals_expected) {
    __syncthreads();
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
        write_task(A.tout + base + q, st.b[lo], st.b[lo] + st.deg[lo], st.v[lo], q - st.off[lo]);
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

// Decrement the counts of the lower S-neighbours w[0..U) (flags low[]); returns the
// previous counts (1 = the push that makes w ready)
template <int U>
__device__ __forceinline__ void jp_decrement(const JpArgs &A, const uint32_t (&w)[U], const bool (&low)[U],
                                             uint32_t (&old)[U]) {
#pragma unroll
    for (int u = 0; u < U; u++) old[u] = low[u] ? atomicSub(&A.rec[w[u]].cnt, 1u) : 0u;
}

// forbidden bit of colour c for the lower S-neighbours (fire-and-forget), then the
// records of the vertices that became ready go to the stage
template <int U>
__device__ __forceinline__ void jp_mark(const JpArgs &A, const JlCtl &C, JpStage &st, const uint32_t (&w)[U],
                                        const bool (&low)[U], const uint32_t (&old)[U], uint32_t c) {
    if (c <= JP_WIN) {
        const uint32_t q = (c - 1) >> 5, bit = 1u << ((c - 1) & 31);
#pragma unroll
        for (int u = 0; u < U; u++)
            if (low[u]) atomicOr(&A.rec[w[u]].win[q], bit);
    } else {  // dense core: the overflow bitmap needs the row of w
#pragma unroll
        for (int u = 0; u < U; u++) {
            if (low[u]) {
                const uint4 h = __ldcg(reinterpret_cast<const uint4 *>(A.rec + w[u]));
                set_overflow(A.bits, (int64_t)(((uint64_t)h.w << 32) | h.z), (int32_t)w[u], h.y, c);
            }
        }
    }
#pragma unroll
    for (int u = 0; u < U; u++) {
        if (low[u] && old[u] == 1u) {
            const uint4 h = __ldcg(reinterpret_cast<const uint4 *>(A.rec + w[u]));
            stage_ready(A, C, st, (int32_t)w[u], (int64_t)(((uint64_t)h.w << 32) | h.z), h.y);
        }
    }
}

// One level of push JP over the tasks [lo, hi) of the queue: every task colours its
// vertex (the first chunk writes the colour) and pushes it to the lower S-neighbours
// of its chunk; vertices whose count reaches 0 are staged for the next level.
__device__ __forceinline__ void jp_level(const JpArgs &A, const JlCtl &C, JpStage &st, uint32_t lo, uint32_t hi,
                                         int64_t warp_g, int64_t nwarps) {
    const int lane = lane_id();
    const uint32_t cnt = hi - lo;
    // task index t = it*32*nwarps + lane*nwarps + warp: consecutive tasks (the chunks
    // of one hub) land on different warps
    for (int64_t base = warp_g; base - warp_g < cnt; base += nwarps * 32) {
        const int64_t t = base + (int64_t)lane * nwarps;
        int32_t v = -1;
        uint32_t j = 0;
        int64_t b = 0, e = 0;
        if (t < cnt) read_task(A.tout + lo + t, b, e, v, j);
        const uint64_t kv = v >= 0 ? vkey(A.k, (uint32_t)v) : 0;
        // ---- short rows: one lane does the whole task
        const bool small = v >= 0 && e - b <= JP_LANE;
        if (__any_sync(FULL, small)) {
            uint32_t w[JP_LANE];
            bool low[JP_LANE];
#pragma unroll
            for (int u = 0; u < JP_LANE; u++) {
                low[u] = small && b + u < e;
                w[u] = low[u] ? (uint32_t)JP_LDCI(A.ci + b + u) : 0u;
            }
#pragma unroll
            for (int u = 0; u < JP_LANE; u++) low[u] = low[u] && in_set(A.inS, w[u]) && vkey(A.k, w[u]) < kv;
            uint32_t old[JP_LANE];
            jp_decrement<JP_LANE>(A, w, low, old);
            uint32_t c = 1;
            if (small) {
                c = lane_mex(A.rec + v, (uint32_t)(e - b));
                A.color[v] = c;
            }
            jp_mark<JP_LANE>(A, C, st, w, low, old, c);
        }
        // ---- longer rows: the warp takes these tasks one by one (<= JP_CHUNK arcs)
        unsigned bigm = __ballot_sync(FULL, v >= 0 && !small);
        while (bigm) {
            const int src = __ffs(bigm) - 1;
            bigm &= bigm - 1;
            const int32_t tv = __shfl_sync(FULL, v, src);
            const uint32_t tj = __shfl_sync(FULL, j, src);
            const int64_t tb = __shfl_sync(FULL, b, src), te = __shfl_sync(FULL, e, src);
            const uint64_t tk = __shfl_sync(FULL, kv, src);
            const int64_t cb = tb + (int64_t)tj * JP_CHUNK;
            constexpr int U = JP_CHUNK / 32;
            uint32_t w[U];
            bool low[U];
#pragma unroll
            for (int u = 0; u < U; u++) {
                const int64_t x = cb + u * 32 + lane;
                low[u] = x < te;
                w[u] = low[u] ? (uint32_t)JP_LDCI(A.ci + x) : 0u;
            }
#pragma unroll
            for (int u = 0; u < U; u++) low[u] = low[u] && in_set(A.inS, w[u]) && vkey(A.k, w[u]) < tk;
            uint32_t old[U];
            jp_decrement<U>(A, w, low, old);  // the decrements do not wait for the mex
            const uint32_t c = warp_mex(A.rec + tv, A.bits, tb + tv, (uint32_t)(te - tb));
            if (tj == 0 && lane == 0) A.color[tv] = c;
            jp_mark<U>(A, C, st, w, low, old, c);
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
    uint32_t lo = 0, hi = (uint32_t)__ldcg(C.W);  // level 0 = the init pass's tasks
    uint32_t r = 0;
    for (;; r++) {
        if (hi == lo || __ldcg(C.err) != 0) break;
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            if (A.hist && r < 1024) {  // stats: tasks and start time (32 ns units) of the first levels
                A.hist[r] = hi - lo;
                A.hist[1024 + r] = (uint32_t)((globaltimer_ns() - t0) >> 5);
            }
            if (r + 1 >= C.max_levels || globaltimer_ns() - t0 > JL_TIMEOUT_NS) atomicExch(C.err, 1u);
        }
        jp_level(A, C, st, lo, hi, warp_g, nwarps);
        const uint32_t next = stage_flush_barrier(A, C, st, r, (r + 1) * gridDim.x);
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
    w.rec = a.take<uint8_t>(((size_t)n + 1) * sizeof(JpRec));
    w.bits = a.take<uint32_t>((size_t)((nnz + n) / 32 + 2));
    w.bits_words = (nnz + n) / 32 + 2;
    w.queue_cap = n + nnz / JP_CHUNK + 2;  // tasks in one level <= all tasks
    w.task = a.take<int64_t>(2 * (size_t)w.queue_cap * (sizeof(JpTask) / sizeof(int64_t)));
    w.vlist = a.take<int32_t>((size_t)n + 1);
    w.mark = a.take<uint8_t>((size_t)n + 1);
    w.queue = a.take<int64_t>((size_t)(nnz / JP_BUDGET + 2));  // huge-row pieces (<= nnz/JP_BUDGET)
    w.sync = a.take<uint32_t>(64);  // levels kernel: barrier words, apart from the task counters
}

// JP over (rp, ci) for the vertex set S (list/implicit) with membership inS; the
// overflow bitmap layout follows this CSR (offset rp[v] + v, deg+1 bits).
// Init pass: records and the level-0 tasks at the head of the queue (counter *qcnt).
static int jp_init(const FlowArgs &f, ColorWs &w, JpArgs &A, uint32_t *color, const int64_t *rp, const int32_t *ci,
                   const uint8_t *inS, const int32_t *list0, const uint32_t *cnt0, int64_t implicit_n, JpTask *q,
                   uint32_t *qcnt) {
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
    SYM_CUDA(cudaMemsetAsync(ctl->huge, 0, sizeof(ctl->huge), s));
    SYM_CUDA(cudaMemsetAsync(w.bits, 0, sizeof(uint32_t) * (size_t)w.bits_words, s));
    A.rp = rp;
    A.ci = ci;
    A.inS = inS;
    A.color = color;
    A.rec = reinterpret_cast<JpRec *>(w.rec);
    A.bits = w.bits;
    A.k = stream_key(f.p.seed, TAG_VERTEX, 0);
    A.huge = w.queue;
    A.hist = nullptr;
    A.in_list = list0;
    A.in_cnt = cnt0;
    A.implicit_n = implicit_n;
    A.tout = q;
    A.out_cnt = qcnt;
    A.huge_cnt = &ctl->huge[1];
    prof_begin("jp_init", s);
    k_jp_init<<<num_sms() * (2048 / JP_THREADS), JP_THREADS, 0, s>>>(A);
    SYM_LAUNCH_CHECK();
    k_jp_init_huge<<<num_sms() * 4, JP_HUGE_THREADS, 0, s>>>(A);
    SYM_LAUNCH_CHECK();
    k_jp_huge_ready<<<num_sms(), 256, 0, s>>>(A);
    prof_end(s, -1);
    SYM_LAUNCH_CHECK();
    return SYM_OK;
}

// algorithmic bytes of the level pass: every arc of the phase CSR read
// once (4 B) + per vertex its task (32 B written + read) and colour write (4 B); the
// pushes are L2 atomics on the 32-B records (not HBM bytes)
static double jp_alg_bytes(const FlowArgs &f, const int64_t *rp) {
    const int64_t phase_nnz = rp == f.g.rp ? f.g.nnz : (rp == f.split.rp_in ? f.split.nnz_in : -1);
    return phase_nnz >= 0 ? 4.0 * (double)phase_nnz + 68.0 * (double)f.g.n : -1.0;
}

// every level in one persistent cooperative launch
static int jp_run(const FlowArgs &f, ColorWs &w, uint32_t *color, const int64_t *rp, const int32_t *ci,
                  const uint8_t *inS, const int32_t *list0, const uint32_t *cnt0, int64_t implicit_n, int phase) {
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
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
    const int64_t qcap = 2 * w.queue_cap;  // >= n + nnz/JP_CHUNK: every vertex is enqueued once
    if (qcap >= (int64_t)0xffffffff) {
        set_error("JP task queue exceeds 2^32 entries");
        return SYM_EINVAL;
    }
    // W (u64) = sync[0..1], G (u64) = sync[2..3], err = sync[32], levels = sync[33]
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
    SYM_TRY(jp_init(f, w, A, color, rp, ci, inS, list0, cnt0, implicit_n, q, w.sync /* low half of W */));
    A.hist = f.stats ? ctl->hist + phase * 2048 : nullptr;
    void *args[] = {&A, &C};
    prof_begin("jp_levels", s);
    SYM_CUDA(cudaLaunchCooperativeKernel((const void *)k_jp_levels, dim3(grid), dim3(JL_THREADS), args, 0, s));
    prof_end(s, jp_alg_bytes(f, rp));
    uint32_t err = 0, levels = 0;
    SYM_TRY(read_u32(C.err, &err, s));
    if (err) {
        SYM_TRY(read_u32(C.levels, &levels, s));
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
