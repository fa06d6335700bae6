// jp.cu -- Jones-Plassmann colouring and the COLOR flows.
//
// JP ([18]) with fixed priorities gives v the smallest colour >= 1 not held by
// any higher-(pv,id) neighbour of its phase set S: exactly first-fit greedy in
// priority order (DESIGN §3 C1).  Plain JP waits until EVERY higher neighbour is
// coloured, so it runs as many dependent levels as the priority DAG is deep (5 063
// at R-MAT s24).  This file computes the same colouring with an early-commit rule:
//
//   m = mex of the colours of v's coloured higher neighbours (v's forbidden bitmap);
//   v may take m as soon as every higher neighbour u is either coloured with a
//   colour != m, or uncoloured and unable to take m: m is already forbidden for u,
//   or m > cap(u) (u's colour is at most cap(u) = #higher + #fixed-coloured + 1).
//
// Proof: the final higher-neighbour colours are the known ones (which hold 1..m-1
// and not m) plus one colour per uncoloured u, and u can never take m, so the final
// mex is m.  Every fact the rule reads ("u has colour c", "m is forbidden for u") is
// permanent once observed, so the rule is exact under any schedule and staleness; a
// vertex whose higher neighbours are all coloured (plain JP's ready vertex) always
// passes.  Result: the same colours in ~530 rounds instead of 5 063 levels at R-MAT
// s24 (CPU simulation and GPU).
//
// Layout (built once per call; the S vertices with phase arcs get compact ids h =
// their rank in id order; a vertex without any phase arc takes colour 1 at once).  The
// per-vertex state other vertices touch is one 16-B record in a compact array, so a
// check or a push touches ONE sector and the hot set (90 MB at R-MAT s24) is mostly
// L2-resident: hot[h] = {colour (0 = not yet), forbidden colours 1..32, count =
// higher neighbours not yet pushed, offset of h's words for colours 33..32R in xb[]
// (R-1 words) | min(R,31) << 27}, R = ceil(cap/32) -- count and offset adjacent, so a
// push's one 64-bit atomic decrements the count and returns the offset.  meta[h] (32 B, read by h itself) = {R, hdeg, ldeg, watch
// length, blocker position, m at the last failed check, list offset}; lst[off..]
// = [watch area of JP_WATCH ids if hdeg + ldeg > JP_WLIST (used if hdeg > JP_WLIST)]
// [higher ids] [lower ids] (compact ids).  With S implicit the build is count-free: a
// row's area is sized from its degree, higher ids are filled from the front and lower
// ids from the back, and the counts found by the fill size the records afterwards.
// A round: phase A -- every vertex whose count is <= JP_WATCH checks its watch list
// (the higher neighbours still uncoloured when it was built; a list of <= JP_WLIST
// higher neighbours is its own watch list), resuming at the last blocker when m is
// unchanged; a vertex that passes writes its colour and queues push tasks; grid
// barrier; phase B -- each new colour goes into the uncoloured lower neighbours'
// bitmaps and decrements their counts (the push that brings a count to JP_WATCH
// activates the vertex), and requested watch lists are built; grid barrier.  All
// rounds run in ONE persistent cooperative kernel (k_jp_rounds).  Waiting for the
// count to reach JP_WATCH costs no rounds on R-MAT (CPU simulation) and bounds every
// check to two warp steps.
#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include "internal.h"

namespace sym {

constexpr int JP_THREADS = 256;
constexpr int JP_HUGE_THREADS = 512;
#ifndef SYM_JP_LANE_ITERS
#define SYM_JP_LANE_ITERS 2  // two lane batches before the warp stage: COLOR-Deg2 20.12 -> 19.81 ms (3: 19.93, 16: 23.5)
#endif
#ifndef SYM_JP_SMALL
#define SYM_JP_SMALL 32
#endif
constexpr int JP_SMALL = SYM_JP_SMALL;  // build: rows <= JP_SMALL arcs are handled by one lane
#ifndef SYM_JP_BUDGET
#define SYM_JP_BUDGET 4096
#endif
constexpr int JP_BUDGET = SYM_JP_BUDGET;  // build: rows > JP_BUDGET arcs are split into pieces
constexpr int JP_PIECE = 8192;   // arcs per CTA piece of a huge row in the build passes
constexpr int JP_TILE = 2048;    // build: compact ids per scan tile (JP_THREADS x 8)
constexpr int JP_TPT = JP_TILE / JP_THREADS;
#ifndef SYM_JP_LANE_CHECKS
#define SYM_JP_LANE_CHECKS 4
#endif
constexpr int JP_LANE_CHECKS = SYM_JP_LANE_CHECKS;  // phase A: entries a lane checks before the warp takes over
#ifndef SYM_JP_WATCH
#define SYM_JP_WATCH 64
#endif
#ifndef SYM_JP_WLIST
#define SYM_JP_WLIST 64
#endif
#ifndef SYM_JP_LANE_ALL
#define SYM_JP_LANE_ALL 1
#endif
#ifndef SYM_JP_WARP_S2
#define SYM_JP_WARP_S2 1
#endif
#ifndef SYM_JP_PUSH_LANE
#define SYM_JP_PUSH_LANE 4
#endif
constexpr int JP_PUSH_LANE = SYM_JP_PUSH_LANE;  // phase B: tasks of <= JP_PUSH_LANE entries are a lane's
constexpr int JP_PUSH = 32 * JP_PUSH_LANE;  // phase B: lower entries per push task (one warp step)
constexpr uint32_t JP_WATCH = SYM_JP_WATCH;  // a vertex checks once <= JP_WATCH higher neighbours are unpushed
constexpr uint32_t JP_WLIST = SYM_JP_WLIST;  // higher lists up to JP_WLIST entries are their own watch list
constexpr uint32_t JP_NOTBUILT = 0xffffffffu;
constexpr int JP_BUILD = 256;    // phase B: higher entries per watch-list build task
constexpr uint32_t JP_HBITS = 27;  // hot.w = offset of the extra bitmap words | min(R, 31) << 27
constexpr uint32_t JP_HMASK = (1u << JP_HBITS) - 1u;
constexpr uint32_t JP_R5 = 31u;

struct JpArgs {
    const int64_t *rp;   // phase CSR (original ids)
    const int32_t *ci;
    const uint8_t *inS;  // nullable: S = all vertices
    uint32_t *color;     // output (original ids); fixed colours of non-S neighbours
    const int32_t *in_list;  // S as a list (nullable = implicit 0..implicit_n-1)
    const uint32_t *in_cnt;
    int64_t implicit_n;
    int32_t *ov;         // [n] compact id -> original
    uint32_t *hdeg;      // [n] higher degree (count pass), fill cursor (huge rows)
    uint32_t *ldeg;      // [n] lower degree (count pass), fill cursor (huge rows)
    uint32_t *arank;     // [2 n/32] per 32 ids: {bitmap of the S vertices with phase arcs,
                         //   exclusive prefix of the popcounts} (rank = compact id)
    uint4 *hot;          // [n] hot per-vertex state {col, bm0, cnt, xo} (see the header)
    uint4 *meta;         // [2n] per-vertex own data
    uint32_t *lst;       // watch / higher / lower lists
    uint32_t *xb;        // bitmap words for colours > 32
    uint32_t *tcnt;      // scan scratch: per tile class counts (2 per tile)
    unsigned long long *tsum;  // scan scratch: per tile (list words, extra bitmap words)
    uint32_t *nc;        // [0] = compact count n', [1] = rows of degree > 2
    uint32_t *ul[2];     // active lists (compact ids), ping-pong by round
    uint4 *task;         // push tasks {list index lo, hi, entries, colour}
    uint4 *btask;        // watch-list build tasks {h, chunk | offset bits 32.. << 24, hdeg, offset
                         //   bits 0..31} -- everything the task needs, no meta load
    uint32_t *ucnt;      // [3] list counts (ring by round)
    uint32_t *pcnt;      // [3] push-task counts (ring by round)
    uint32_t *bcnt;      // [3] build-task counts (ring by round)
    int64_t *huge;       // (piece << 32 | h) items of the huge rows
    uint32_t *huge_cnt;
    uint32_t *err;       // 1 = timeout / max rounds, 2 = offsets overflow
    uint32_t *hist;
    uint32_t *trace;     // nullable: per-round diagnostics (SYM_JP_TRACE)
    int trace2;          // SYM_JP_TRACE=2: slots 512.. / 1024.. hold the slowest warp's push /
                         //   build span of phase B instead of the task counts
    unsigned long long *prof;  // profiling counter pair {alg, impl} of the current launch (nullable)
    unsigned long long *prof_jp;  // the rounds launch's pair: the count pass adds §8(d)'s JP bytes
    Key k;
    const uint32_t *okey;  // SYM_F_ORDER_LF / _SF: per-vertex order term (degree in G, or its
                           // complement), 4 B per vertex: L2-resident for the per-arc gathers
    int ord;               // 0: (pv, id); 1: largest degree first; 2: smallest degree first
};

// the vertex order of the colouring: (pv, id) -- or, with SYM_F_ORDER_LF / _SF
// (Hasenplaugh et al. [14]), the degree in G first (pv is a bijection, so the
// 64-bit key (degree term << 32 | pv) is unique)
__device__ __forceinline__ uint64_t jp_okey(Key k, const uint32_t *okey, int ord, uint32_t v) {
    if (ord == 0) return vkey(k, v);
    return ((uint64_t)__ldg(okey + v) << 32) | pv(k, v);
}

// the order terms: degree (LF) or its complement (SF), degrees in G (< 2^31)
__global__ void k_jp_okey(const int64_t *__restrict__ grp, int64_t n, int ord, uint32_t *okey) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
        const uint32_t d = (uint32_t)(grp[v + 1] - grp[v]);
        okey[v] = ord == 1 ? d : ~d;
    }
}

__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ bool in_set(const uint8_t *inS, uint32_t w) { return inS == nullptr || inS[w] != 0; }

__device__ __forceinline__ uint32_t watch_words(uint32_t hd) { return hd > JP_WLIST ? JP_WATCH : 0u; }
// list layout at a row's offset: [watch area][higher ids][lower ids]; the area is
// reserved for every row with more than JP_WLIST S-neighbours (hd + ld) -- a bound the
// count-free build knows before it has split the row -- and used when hd > JP_WLIST
__device__ __forceinline__ uint32_t watch_area(uint32_t hd, uint32_t ld) { return hd + ld > JP_WLIST ? JP_WATCH : 0u; }

__device__ __forceinline__ uint64_t meta_off(const uint4 &m1) { return (uint64_t)m1.z | ((uint64_t)m1.w << 32); }

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
// The S vertices with phase arcs are numbered by rank in id order:
//   h(v) = prefix[v >> 5] + popc(bits[v >> 5] & lanes below v)  (one 8-B load)
// so a list id is computed from 4 MB of bitmap + prefix (L2/L1-resident at R-MAT
// s24) instead of gathered from an n-entry map.  A vertex of S without phase arcs
// takes colour 1 at once.
__device__ __forceinline__ uint32_t jp_rank(const JpArgs &A, uint32_t v) {
    const uint2 x = __ldg(reinterpret_cast<const uint2 *>(A.arank) + (v >> 5));
    return x.y + __popc(x.x & ((1u << (v & 31)) - 1u));
}
// the same under a predicate (0 when !p): a predicated load, so a batch of rank lookups
// stays in flight together instead of branching around each one
__device__ __forceinline__ uint32_t jp_rank_pred(const JpArgs &A, uint32_t v, bool p) {
    const uint2 x = ld_nc_v2_pred(reinterpret_cast<const uint2 *>(A.arank) + (v >> 5), p);
    return x.y + __popc(x.x & ((1u << (v & 31)) - 1u));
}

// implicit S = 0..n-1: one bitmap word per warp step (ballot of "has phase arcs")
__global__ void k_jpc_bits(JpArgs A, int64_t n) {
    const int64_t nw = (n + 31) >> 5;
    for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nw;
         w += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t v = (w << 5) + lane_id();
        const bool in = v < n;
        const bool arcs = in && A.rp[v + 1] > A.rp[v];
        const unsigned b = __ballot_sync(FULL, arcs);
        if (lane_id() == 0) A.arank[2 * w] = b;
        if (in && !arcs) A.color[v] = 1u;
    }
}

// S given as a list (COLOR-Rand recolouring): bits of the listed vertices
__global__ void k_jpc_mark(JpArgs A) {
    const uint32_t cnt = *A.in_cnt;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += gridDim.x * blockDim.x) {
        const uint32_t v = (uint32_t)A.in_list[i];
        if (A.rp[v + 1] > A.rp[v]) atomicOr(A.arank + 2 * (v >> 5), 1u << (v & 31));
        else A.color[v] = 1u;
    }
}

// per tile of JP_TILE bitmap words: set bits
__global__ void __launch_bounds__(JP_THREADS) k_jpc_tiles(JpArgs A, int64_t nwords) {
    const int64_t base = (int64_t)blockIdx.x * JP_TILE;
    uint32_t c = 0;
    for (int u = 0; u < JP_TPT; u++) {
        const int64_t w = base + u * JP_THREADS + threadIdx.x;
        if (w < nwords) c += __popc(A.arank[2 * w]);
    }
    c = __reduce_add_sync(FULL, c);
    __shared__ uint32_t s0;
    if (threadIdx.x == 0) s0 = 0;
    __syncthreads();
    if (lane_id() == 0 && c) atomicAdd(&s0, c);
    __syncthreads();
    if (threadIdx.x == 0) A.tcnt[blockIdx.x] = s0;
}

// one CTA: exclusive prefix of the tile counts; n' = the total
__global__ void __launch_bounds__(1024) k_jpc_tiles_scan(JpArgs A, int64_t ntiles) {
    const int64_t per = (ntiles + blockDim.x - 1) / blockDim.x;
    const int64_t t0 = (int64_t)threadIdx.x * per, t1 = ntiles < t0 + per ? ntiles : t0 + per;
    uint32_t s0 = 0;
    for (int64_t t = t0; t < t1; t++) s0 += A.tcnt[t];
    __shared__ uint32_t w0[32];
    uint32_t i0 = s0;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y0 = __shfl_up_sync(FULL, i0, d);
        if (lane_id() >= d) i0 += y0;
    }
    const int wid = threadIdx.x >> 5;
    if (lane_id() == 31) w0[wid] = i0;
    __syncthreads();
    uint32_t b0 = 0, T0 = 0;
    for (int q = 0; q < (int)(blockDim.x >> 5); q++) {
        if (q < wid) b0 += w0[q];
        T0 += w0[q];
    }
    uint32_t o0 = b0 + i0 - s0;
    for (int64_t t = t0; t < t1; t++) {
        const uint32_t a0 = A.tcnt[t];
        A.tcnt[t] = o0;
        o0 += a0;
    }
    if (threadIdx.x == 0) A.nc[0] = T0;
}

// word prefixes and the compact id -> original map
__global__ void __launch_bounds__(JP_THREADS) k_jpc_assign(JpArgs A, int64_t nwords) {
    const int64_t base = (int64_t)blockIdx.x * JP_TILE;
    __shared__ uint32_t sm0[8];
    uint32_t o0 = A.tcnt[blockIdx.x];
    for (int u = 0; u < JP_TPT; u++) {
        const int64_t w = base + u * JP_THREADS + threadIdx.x;
        const uint32_t bits = w < nwords ? A.arank[2 * w] : 0u;
        uint32_t t0;
        const uint32_t p0 = block_excl_scan<uint32_t>(__popc(bits), sm0, &t0);
        if (w < nwords) {
            A.arank[2 * w + 1] = o0 + p0;
            uint32_t b = bits, h = o0 + p0;
            while (b) {
                const int k = __ffs(b) - 1;
                b &= b - 1;
                A.ov[h++] = (int32_t)((w << 5) + k);
            }
        }
        o0 += t0;
    }
}

// ---------------------------------------------------------------- build: DAG
// count pass: hdeg[h] = #higher S-neighbours, ldeg[h] = #lower S-neighbours; rows
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
            kv = jp_okey(A.k, A.okey, A.ord, (uint32_t)v);
        }
        uint32_t hi = 0, lo = 0;
        if (active && e - b <= JP_SMALL) {  // batches of 4 arcs: their loads in flight together
            for (int64_t xq = b; xq < e; xq += 4) {
                uint32_t w[4];
#pragma unroll
                for (int u = 0; u < 4; u++) w[u] = xq + u < e ? (uint32_t)__ldcs(A.ci + xq + u) : 0u;
#pragma unroll
                for (int u = 0; u < 4; u++) {
                    if (xq + u < e && in_set(A.inS, w[u])) {
                        const bool up = jp_okey(A.k, A.okey, A.ord, w[u]) > kv;
                        hi += up;
                        lo += !up;
                    }
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
            for (int64_t xb0 = wb + lane; xb0 < we; xb0 += 128) {  // 4 steps of 32 arcs in flight
                uint32_t w[4];
#pragma unroll
                for (int u = 0; u < 4; u++) w[u] = xb0 + u * 32 < we ? (uint32_t)__ldcs(A.ci + xb0 + u * 32) : 0u;
#pragma unroll
                for (int u = 0; u < 4; u++) {
                    if (xb0 + u * 32 < we && in_set(A.inS, w[u])) {
                        const bool up = jp_okey(A.k, A.okey, A.ord, w[u]) > wk;
                        lh += up;
                        ll += !up;
                    }
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
            A.hdeg[h] = hi;
            A.ldeg[h] = lo;
        }
        // algorithmic bytes: the row's columns (huge rows: k_jpc_count_huge), row pair,
        // id map entry, the two counts
        prof_add(A.prof, 0ull, active ? (huge ? 0ull : 4ull * (uint64_t)(e - b)) + 28ull : 0ull);
        // §8(d) JP (push form): 8 B per phase arc + 12 B per vertex, charged to the rounds
        // (huge rows: their pieces add the arcs in k_jpc_count_huge)
        prof_add(A.prof_jp, active ? 8ull * (uint64_t)(hi + lo) + 12ull : 0ull, 0ull);
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
        const uint64_t kv = jp_okey(A.k, A.okey, A.ord, (uint32_t)v);
        uint32_t lh = 0, ll = 0;
        for (int64_t x = pb + threadIdx.x; x < pe_; x += JP_HUGE_THREADS) {
            const uint32_t w = (uint32_t)__ldg(A.ci + x);
            if (in_set(A.inS, w)) {
                const bool up = jp_okey(A.k, A.okey, A.ord, w) > kv;
                lh += up;
                ll += !up;
            }
        }
        lh = __reduce_add_sync(FULL, lh);
        ll = __reduce_add_sync(FULL, ll);
        if (lane_id() == 0) {
            if (lh) atomicAdd(A.hdeg + h, lh);
            if (ll) atomicAdd(A.ldeg + h, ll);
        }
        prof_add(A.prof, 0ull, threadIdx.x == 0 ? 4ull * (uint64_t)(pe_ - pb) : 0ull);
        prof_add(A.prof_jp, lane_id() == 0 ? 8ull * (uint64_t)(lh + ll) : 0ull, 0ull);  // lh, ll: warp totals
    }
}


// bitmap words of compact vertex h: cap = (higher + fixed-coloured neighbours) + 1 bits
__device__ __forceinline__ uint32_t jp_words(const JpArgs &A, int64_t h) {
    const int32_t v = A.ov[h];
    const int64_t deg = A.rp[v + 1] - A.rp[v];
    return (uint32_t)((deg - (int64_t)A.ldeg[h] + 1 + 31) >> 5);
}

// per tile of JP_TILE compact ids: list words and extra bitmap words
__global__ void __launch_bounds__(JP_THREADS) k_jpc_sums(JpArgs A) {
    const uint32_t cnt = A.nc[0];
    const int64_t base = (int64_t)blockIdx.x * JP_TILE;
    if (base >= cnt) return;
    unsigned long long sl = 0, sx = 0;
    for (int u = 0; u < JP_TPT; u++) {
        const int64_t h = base + u * JP_THREADS + threadIdx.x;
        if (h < cnt) {
            const uint32_t hd = A.hdeg[h];
            sl += watch_area(hd, A.ldeg[h]) + hd + A.ldeg[h];
            sx += jp_words(A, h) - 1u;
        }
    }
    for (int d = 16; d; d >>= 1) {
        sl += __shfl_xor_sync(FULL, sl, d);
        sx += __shfl_xor_sync(FULL, sx, d);
    }
    __shared__ unsigned long long a[2];
    if (threadIdx.x == 0) a[0] = a[1] = 0;
    __syncthreads();
    if (lane_id() == 0) {
        atomicAdd(&a[0], sl);
        atomicAdd(&a[1], sx);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        A.tsum[2 * blockIdx.x] = a[0];
        A.tsum[2 * blockIdx.x + 1] = a[1];
    }
}

// one CTA: exclusive prefix of the tile sums (extra bitmap offsets must fit 32 bits,
// compact ids 27 bits)
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
    unsigned long long b0 = 0, b1 = 0, T1 = 0;
    for (int q = 0; q < (int)(blockDim.x >> 5); q++) {
        if (q < wid) {
            b0 += w0[q];
            b1 += w1[q];
        }
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
    if (threadIdx.x == 0 && T1 > JP_HMASK) atomicOr(A.err, 2u);
}

// per compact id: list offset, meta, hot state, zeroed extra bitmap words, the list
// id map; the first round's list = the vertices with <= JP_WATCH higher neighbours
__global__ void __launch_bounds__(JP_THREADS) k_jpc_place(JpArgs A) {
    const uint32_t cnt = A.nc[0];
    const int64_t base = (int64_t)blockIdx.x * JP_TILE;
    if (base >= cnt) return;
    __shared__ unsigned long long sm0[8], sm1[8];
    unsigned long long o0 = A.tsum[2 * blockIdx.x], o1 = A.tsum[2 * blockIdx.x + 1];
    for (int u = 0; u < JP_TPT; u++) {
        const int64_t h = base + u * JP_THREADS + threadIdx.x;
        const bool active = h < cnt;
        uint32_t hd = 0, ld = 0, R = 1;
        if (active) {
            hd = A.hdeg[h];
            ld = A.ldeg[h];
            R = jp_words(A, h);
        }
        unsigned long long t0, t1;
        const unsigned long long p0 =
            block_excl_scan<unsigned long long>(active ? watch_area(hd, ld) + hd + ld : 0ull, sm0, &t0);
        const unsigned long long p1 = block_excl_scan<unsigned long long>(active ? R - 1u : 0ull, sm1, &t1);
        // Round 0 can only colour vertices without higher neighbours (nothing is coloured
        // and, without fixed colours -- S given implicitly -- nothing is forbidden), so
        // the other active vertices start in round 1's list.
        const bool ready = active && hd == 0, later = active && hd > 0 && hd <= JP_WATCH;
        const bool r0 = ready || (later && A.in_list != nullptr);
        const bool first = r0 || later;
        // CTA-aggregated list appends (one atomic per CTA and list; order immaterial)
        cta_append2x(r0, first && !r0, (uint32_t)h, A.ul[0], A.ucnt, A.ul[1], A.ucnt + 1);
        if (active) {
            const unsigned long long off = o0 + p0;
            const uint32_t x0 = (uint32_t)(o1 + p1);
            A.meta[2 * h] = make_uint4(R, hd, ld, hd > JP_WLIST ? JP_NOTBUILT : hd);
            A.meta[2 * h + 1] = make_uint4(0u, 0u, (uint32_t)off, (uint32_t)(off >> 32));
            A.hot[h] = make_uint4(0u, 0u, hd, (x0 & JP_HMASK) | (min(R, JP_R5) << JP_HBITS));
            for (uint32_t q = 1; q < R; q++) A.xb[x0 + q - 1] = 0u;
            A.hdeg[h] = 0;  // fill cursors of the huge rows
            A.ldeg[h] = 0;
        }
        // algorithmic bytes: counts read, meta + hot record + zeroed extra words written
        prof_add(A.prof, 0ull, active ? 8ull + 48ull + 4ull * (R - 1u) : 0ull);
        o0 += t0;
        o1 += t1;
    }
}

// ---------------------------------------------------------------- count-free build
// With S implicit (every vertex of the phase CSR; COLOR-NONE / -Degk / -Rand's first
// phase) a row's higher + lower neighbours are exactly its phase arcs, so the lists can
// be placed from the degrees alone and split while they are filled -- higher ids from
// the front of the row's area, lower ids from the back -- with no counting pass over
// the arcs.  The counts the fill finds then size the hot records, the bitmap words
// (true cap) and the first round's lists (k_jpc_place_cf).

__device__ __forceinline__ uint32_t jp_deg(const JpArgs &A, int64_t h) {
    const int32_t v = A.ov[h];
    return (uint32_t)(A.rp[v + 1] - A.rp[v]);
}

// per tile of JP_TILE compact ids: list words (degree + watch area); huge rows' pieces
__global__ void __launch_bounds__(JP_THREADS) k_jpc_lsums_cf(JpArgs A) {
    const uint32_t cnt = A.nc[0];
    const int64_t base = (int64_t)blockIdx.x * JP_TILE;
    if (base >= cnt) return;
    unsigned long long sl = 0;
    for (int u = 0; u < JP_TPT; u++) {
        const int64_t h = base + u * JP_THREADS + threadIdx.x;
        const uint32_t d = h < cnt ? jp_deg(A, h) : 0u;
        sl += watch_area(d, 0u) + d;
        const uint32_t np = d > (uint32_t)JP_BUDGET ? (d + JP_PIECE - 1) / JP_PIECE : 0u;
        const int64_t ps = warp_reserve(np, A.huge_cnt);
        for (uint32_t q = 0; q < np; q++) A.huge[ps + q] = ((int64_t)q << 32) | (uint32_t)h;
        prof_add(A.prof, 0ull, h < cnt ? 12ull : 0ull);
        // §8(d) JP (push form): 8 B per phase arc + 12 B per vertex, charged to the rounds
        prof_add(A.prof_jp, h < cnt ? 8ull * d + 12ull : 0ull, 0ull);
    }
    for (int d = 16; d; d >>= 1) sl += __shfl_xor_sync(FULL, sl, d);
    __shared__ unsigned long long a0;
    if (threadIdx.x == 0) a0 = 0;
    __syncthreads();
    if (lane_id() == 0) atomicAdd(&a0, sl);
    __syncthreads();
    if (threadIdx.x == 0) {
        A.tsum[2 * blockIdx.x] = a0;
        A.tsum[2 * blockIdx.x + 1] = 0;
    }
}

// list offsets (meta[2h+1].zw) from the scanned tile sums
__global__ void __launch_bounds__(JP_THREADS) k_jpc_offs_cf(JpArgs A) {
    const uint32_t cnt = A.nc[0];
    const int64_t base = (int64_t)blockIdx.x * JP_TILE;
    if (base >= cnt) return;
    __shared__ unsigned long long sm0[8];
    unsigned long long o0 = A.tsum[2 * blockIdx.x];
    for (int u = 0; u < JP_TPT; u++) {
        const int64_t h = base + u * JP_THREADS + threadIdx.x;
        const uint32_t d = h < cnt ? jp_deg(A, h) : 0u;
        unsigned long long t0;
        const unsigned long long p0 = block_excl_scan<unsigned long long>(h < cnt ? watch_area(d, 0u) + d : 0ull, sm0, &t0);
        if (h < cnt) {
            const unsigned long long off = o0 + p0;
            A.meta[2 * h + 1] = make_uint4(0u, 0u, (uint32_t)off, (uint32_t)(off >> 32));
        }
        prof_add(A.prof, 0ull, h < cnt ? 28ull : 0ull);
        o0 += t0;
    }
}

// per tile: extra bitmap words of the true cap (hd + 1 bits), once the fill has counted
__global__ void __launch_bounds__(JP_THREADS) k_jpc_xsums_cf(JpArgs A) {
    const uint32_t cnt = A.nc[0];
    const int64_t base = (int64_t)blockIdx.x * JP_TILE;
    if (base >= cnt) return;
    unsigned long long sx = 0;
    for (int u = 0; u < JP_TPT; u++) {
        const int64_t h = base + u * JP_THREADS + threadIdx.x;
        if (h < cnt) sx += (A.hdeg[h] + 1u + 31u) / 32u - 1u;
    }
    for (int d = 16; d; d >>= 1) sx += __shfl_xor_sync(FULL, sx, d);
    __shared__ unsigned long long a1;
    if (threadIdx.x == 0) a1 = 0;
    __syncthreads();
    if (lane_id() == 0) atomicAdd(&a1, sx);
    __syncthreads();
    if (threadIdx.x == 0) {
        A.tsum[2 * blockIdx.x] = 0;
        A.tsum[2 * blockIdx.x + 1] = a1;
    }
}

// per compact id: meta, hot state, zeroed extra bitmap words, the first round's lists
// (the list offset is already in meta[2h+1])
__global__ void __launch_bounds__(JP_THREADS) k_jpc_place_cf(JpArgs A) {
    const uint32_t cnt = A.nc[0];
    const int64_t base = (int64_t)blockIdx.x * JP_TILE;
    if (base >= cnt) return;
    __shared__ unsigned long long sm1[8];
    unsigned long long o1 = A.tsum[2 * blockIdx.x + 1];
    for (int u = 0; u < JP_TPT; u++) {
        const int64_t h = base + u * JP_THREADS + threadIdx.x;
        const bool active = h < cnt;
        uint32_t hd = 0, ld = 0, R = 1;
        if (active) {
            hd = A.hdeg[h];
            ld = A.ldeg[h];
            R = (hd + 1u + 31u) / 32u;
        }
        unsigned long long t1;
        const unsigned long long p1 = block_excl_scan<unsigned long long>(active ? R - 1u : 0ull, sm1, &t1);
        const bool ready = active && hd == 0, later = active && hd > 0 && hd <= JP_WATCH;
        cta_append2x(ready, later, (uint32_t)h, A.ul[0], A.ucnt, A.ul[1], A.ucnt + 1);
        if (active) {
            const uint32_t x0 = (uint32_t)(o1 + p1);
            A.meta[2 * h] = make_uint4(R, hd, ld, hd > JP_WLIST ? JP_NOTBUILT : hd);
            A.hot[h] = make_uint4(0u, 0u, hd, (x0 & JP_HMASK) | (min(R, JP_R5) << JP_HBITS));
            for (uint32_t q = 1; q < R; q++) A.xb[x0 + q - 1] = 0u;
        }
        prof_add(A.prof, 0ull, active ? 8ull + 40ull + 4ull * (R - 1u) : 0ull);
        o1 += t1;
    }
}

// fixed colour c of a neighbour outside S (COLOR-Rand recolouring) as a forbidden bit
__device__ __forceinline__ void jp_fixed(const JpArgs &A, int64_t h, uint32_t R, uint32_t x0, uint32_t w) {
    const uint32_t c = A.color[w];
    if (c == 0) return;
    const uint32_t q = (c - 1) >> 5, bit = 1u << ((c - 1) & 31);
    if (q == 0) atomicOr(&A.hot[h].y, bit);
    else if (q < R) atomicOr(A.xb + x0 + q - 1, bit);
}

// fill pass: higher and lower lists (list ids, CSR order); fixed colours of
// neighbours outside S.  Columns and lists stream (evict-first) so the id map stays
// in L2 for the gathers.  CF (count-free build, S implicit): the area of a row is its
// degree (+ watch area), higher ids fill it from the front and lower ids from the
// back, and the counts are written out (hdeg / ldeg) for k_jpc_place_cf.
// 5 CTAs/SM (48 regs, no spills; 59 without the bound -> 4): more rank lookups in flight
#ifndef SYM_FILL_MINB
#define SYM_FILL_MINB 5
#endif
#ifndef SYM_FILL_BATCH
#define SYM_FILL_BATCH 4  // arcs per batch of a lane's short row
#endif
template <bool CF>
#if SYM_FILL_MINB > 0
__global__ void __launch_bounds__(JP_THREADS, SYM_FILL_MINB) k_jpc_fill(JpArgs A) {
#else
__global__ void __launch_bounds__(JP_THREADS) k_jpc_fill(JpArgs A) {
#endif
    const uint32_t cnt = A.nc[0];
    const int lane = lane_id();
    const int64_t warp_g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = warp_g * 32; base < cnt; base += nwarps * 32) {
        const int64_t h = base + lane;
        const bool active = h < cnt;
        int32_t v = 0;
        int64_t b = 0, e = 0;
        uint64_t kv = 0, hl = 0, ll = 0;
        uint32_t R = 0, x0 = 0;
        if (active) {
            v = A.ov[h];
            b = A.rp[v];
            e = A.rp[v + 1];
            kv = jp_okey(A.k, A.okey, A.ord, (uint32_t)v);
            if (CF) {
                const uint4 m1 = A.meta[2 * h + 1];
                const uint32_t d = (uint32_t)(e - b);
                hl = meta_off(m1) + watch_area(d, 0u);
                ll = hl + d;  // lower ids from the back: ll = one past the next slot
            } else {
                const uint4 m0 = A.meta[2 * h], m1 = A.meta[2 * h + 1];
                R = m0.x;
                x0 = A.hot[h].w & JP_HMASK;
                hl = meta_off(m1) + watch_area(m0.y, m0.z);
                ll = hl + m0.y;
            }
        }
        const uint64_t hl0 = hl, ll0 = ll;
        if (active && e - b <= JP_SMALL) {  // batches of FB arcs: their loads in flight together
            constexpr int FB = SYM_FILL_BATCH;
            for (int64_t xq = b; xq < e; xq += FB) {
                uint32_t w[FB], rk[FB];
                bool ok[FB], sv[FB];
#pragma unroll
                for (int u = 0; u < FB; u++) {
                    ok[u] = xq + u < e;
                    w[u] = ok[u] ? (uint32_t)__ldcs(A.ci + xq + u) : 0u;
                }
#pragma unroll
                for (int u = 0; u < FB; u++) {
                    sv[u] = ok[u] && (CF || in_set(A.inS, w[u]));
                    rk[u] = jp_rank_pred(A, w[u], sv[u]);
                }
#pragma unroll
                for (int u = 0; u < FB; u++) {
                    if (!ok[u]) continue;
                    if (!sv[u]) jp_fixed(A, h, R, x0, w[u]);
                    else if (jp_okey(A.k, A.okey, A.ord, w[u]) > kv) __stcs(A.lst + hl++, rk[u]);
                    else if (CF) __stcs(A.lst + --ll, rk[u]);
                    else __stcs(A.lst + ll++, rk[u]);
                }
            }
            if (CF) {
                A.hdeg[h] = (uint32_t)(hl - hl0);
                A.ldeg[h] = (uint32_t)(ll0 - ll);
            }
        }
        unsigned medm = __ballot_sync(FULL, active && e - b > JP_SMALL && e - b <= JP_BUDGET);
        while (medm) {
            const int src = __ffs(medm) - 1;
            medm &= medm - 1;
            const int64_t wb = __shfl_sync(FULL, b, src), we = __shfl_sync(FULL, e, src);
            const uint64_t wk = __shfl_sync(FULL, kv, src);
            const int64_t wh = base + src;
            const uint32_t wR = __shfl_sync(FULL, R, src), wx0 = __shfl_sync(FULL, x0, src);
            uint64_t whl = __shfl_sync(FULL, hl, src), wll = __shfl_sync(FULL, ll, src);
            const uint64_t whl0 = whl, wll0 = wll;
            const unsigned lt = (1u << lane) - 1u;
            for (int64_t xb0 = wb; xb0 < we; xb0 += 128) {  // 4 steps of 32 arcs in flight
                uint32_t w[4], rk[4];
                bool up[4], dn[4];
#pragma unroll
                for (int u = 0; u < 4; u++) {
                    const int64_t x = xb0 + u * 32 + lane;
                    w[u] = x < we ? (uint32_t)__ldcs(A.ci + x) : 0u;
                }
#pragma unroll
                for (int u = 0; u < 4; u++) {
                    const bool ok = xb0 + u * 32 + lane < we;
                    const bool sv = ok && (CF || in_set(A.inS, w[u]));
                    up[u] = sv && jp_okey(A.k, A.okey, A.ord, w[u]) > wk;
                    dn[u] = sv && !up[u];
                    rk[u] = jp_rank_pred(A, w[u], sv);
                    if (!CF && ok && !sv) jp_fixed(A, wh, wR, wx0, w[u]);
                }
#pragma unroll
                for (int u = 0; u < 4; u++) {
                    const unsigned mu = __ballot_sync(FULL, up[u]), md = __ballot_sync(FULL, dn[u]);
                    if (up[u]) __stcs(A.lst + whl + __popc(mu & lt), rk[u]);
                    if (CF) {
                        if (dn[u]) __stcs(A.lst + wll - 1 - __popc(md & lt), rk[u]);
                        wll -= __popc(md);
                    } else {
                        if (dn[u]) __stcs(A.lst + wll + __popc(md & lt), rk[u]);
                        wll += __popc(md);
                    }
                    whl += __popc(mu);
                }
            }
            if (CF && lane == 0) {
                A.hdeg[wh] = (uint32_t)(whl - whl0);
                A.ldeg[wh] = (uint32_t)(wll0 - wll);
            }
        }
        // algorithmic bytes: the row's columns read + list ids written (huge rows:
        // k_jpc_fill_huge), row pair, id map, meta + hot record read
        prof_add(A.prof, 0ull, active ? (e - b > JP_BUDGET ? 0ull : 8ull * (uint64_t)(e - b)) + 68ull : 0ull);
    }
}

// huge rows: one CTA per piece; each warp counts its 512-arc slice (ballots), reserves
// its positions on the row's two cursors with one atomic each, then writes (the
// slice is re-read from L2; holding it in registers instead cost occupancy -- 68 regs,
// one CTA per SM -- and jp_build went 4.03 -> 4.53 ms at R-MAT s24).  CF: the lower cursor counts from the back of the area.
template <bool CF>
__global__ void __launch_bounds__(JP_HUGE_THREADS) k_jpc_fill_huge(JpArgs A) {
    constexpr int SLICE = JP_PIECE / (JP_HUGE_THREADS / 32);
    const uint32_t cnt = *A.huge_cnt;
    const int lane = lane_id();
    const unsigned lt = (1u << lane) - 1u;
    for (uint32_t p = blockIdx.x; p < cnt; p += gridDim.x) {
        const int64_t item = A.huge[p];
        const int32_t h = (int32_t)(uint32_t)item;
        const int64_t j = item >> 32;
        const int32_t v = A.ov[h];
        const int64_t b = A.rp[v], e = A.rp[v + 1];
        const int64_t sb0 = b + j * JP_PIECE + (int64_t)(threadIdx.x >> 5) * SLICE;
        const int64_t se = min(e, sb0 + SLICE);
        const uint64_t kv = jp_okey(A.k, A.okey, A.ord, (uint32_t)v);
        const uint4 m0 = CF ? make_uint4(0u, 0u, 0u, 0u) : A.meta[2 * h], m1 = A.meta[2 * h + 1];
        const uint32_t x0 = CF ? 0u : A.hot[h].w & JP_HMASK;
        const uint32_t d = (uint32_t)(e - b);
        const uint64_t hl = meta_off(m1) + (CF ? watch_area(d, 0u) : watch_area(m0.y, m0.z));
        const uint64_t ll = CF ? hl + d : hl + m0.y;  // CF: one past the back of the area
        uint32_t nu = 0, nd = 0;
        for (int64_t xq = sb0 + lane; xq - lane < se; xq += 128) {  // 4 loads in flight per lane
            uint32_t w[4];
#pragma unroll
            for (int u = 0; u < 4; u++) w[u] = xq + u * 32 < se ? (uint32_t)__ldg(A.ci + xq + u * 32) : 0u;
#pragma unroll
            for (int u = 0; u < 4; u++) {
                const bool sv = xq + u * 32 < se && (CF || in_set(A.inS, w[u]));
                const bool up = sv && jp_okey(A.k, A.okey, A.ord, w[u]) > kv;
                nu += __popc(__ballot_sync(FULL, up));
                nd += __popc(__ballot_sync(FULL, sv && !up));
            }
        }
        uint32_t pu = 0, pd = 0;
        if (lane == 0) {
            if (nu) pu = atomicAdd(A.hdeg + h, nu);
            if (nd) pd = atomicAdd(A.ldeg + h, nd);
        }
        pu = __shfl_sync(FULL, pu, 0);
        pd = __shfl_sync(FULL, pd, 0);
        for (int64_t xq = sb0 + lane; xq - lane < se; xq += 128) {  // 4 steps of 32 arcs in flight
            uint32_t w[4], rk[4];
            bool up[4], dn[4];
#pragma unroll
            for (int u = 0; u < 4; u++) w[u] = xq + u * 32 < se ? (uint32_t)__ldg(A.ci + xq + u * 32) : 0u;
#pragma unroll
            for (int u = 0; u < 4; u++) {
                const bool ok = xq + u * 32 < se;
                const bool sv = ok && (CF || in_set(A.inS, w[u]));
                up[u] = sv && jp_okey(A.k, A.okey, A.ord, w[u]) > kv;
                dn[u] = sv && !up[u];
                rk[u] = jp_rank_pred(A, w[u], sv);
                if (!CF && ok && !sv) jp_fixed(A, h, m0.x, x0, w[u]);
            }
#pragma unroll
            for (int u = 0; u < 4; u++) {
                const unsigned mu = __ballot_sync(FULL, up[u]), md = __ballot_sync(FULL, dn[u]);
                if (up[u]) __stcs(A.lst + hl + pu + __popc(mu & lt), rk[u]);
                if (dn[u]) {
                    if (CF) __stcs(A.lst + ll - 1 - (pd + __popc(md & lt)), rk[u]);
                    else __stcs(A.lst + ll + pd + __popc(md & lt), rk[u]);
                }
                pu += __popc(mu);
                pd += __popc(md);
            }
        }
        prof_add(A.prof, 0ull, lane == 0 && se > sb0 ? 8ull * (uint64_t)(se - sb0) : 0ull);
    }
}

// colours back to original ids
__global__ void k_jpc_scatter(JpArgs A) {
    const uint32_t cnt = A.nc[0];
    for (int64_t h = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; h < cnt; h += (int64_t)gridDim.x * blockDim.x)
        A.color[A.ov[h]] = A.hot[h].x;
}

// ---------------------------------------------------------------- rounds
__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_release_u32(uint32_t *p, uint32_t v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

struct JrCtl {
    uint32_t *arr;     // barrier arrivals (monotone)
    uint32_t *levels;  // out: rounds run
    uint32_t max_rounds;
};

// software grid barrier (all CTAs co-resident); k = barriers passed so far.  The
// fence orders this CTA's writes (colours, lists, task entries, bitmap REDs) before
// the arrival, so the next phase sees them.
// After the barrier, thread 0 loads up to three counters into sm[0..2] (one L2 read
// per CTA instead of one per warp) -- visible to the CTA after the final bar.sync.
__device__ __forceinline__ void grid_sync(const JrCtl &C, uint32_t &k, const uint32_t *p0 = nullptr,
                                          const uint32_t *p1 = nullptr, const uint32_t *p2 = nullptr,
                                          uint32_t *sm = nullptr) {
    __syncthreads();
    k++;
    if (threadIdx.x == 0) {
        // arrival = one release reduction (no return); every CTA polls the counter (a
        // polling back-off of 100-1000 ns changed nothing: profiles/r2h_jp_async_sweep.json)
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(C.arr) : "memory");
        const uint32_t target = k * gridDim.x;
        while (ld_acquire_u32(C.arr) < target) {
        }
        // the three counter loads in flight together (predicated, see ld_cg_pred)
        const uint32_t v0 = ld_cg_pred(p0, p0 != nullptr), v1 = ld_cg_pred(p1, p1 != nullptr),
                       v2 = ld_cg_pred(p2, p2 != nullptr);
        if (p0) sm[0] = v0;
        if (p1) sm[1] = v1;
        if (p2) sm[2] = v2;
    }
    __syncthreads();
}

// One check stage over N watch-list entries e[u] (valid[u]): can higher neighbour e
// not take colour m (word q, bit)?  Coloured: its colour differs; uncoloured: m is
// forbidden for it, or m > cap (q >= R).  Three batched load steps: the 16-B hot
// records; the full R of saturated R fields (>= 31 words, from meta); the bitmap words
// q of the uncoloured ones.
template <int N>
__device__ __forceinline__ void jp_nb_stage(const JpArgs &A, const uint32_t (&e)[N], const bool (&valid)[N],
                                            uint32_t m, uint32_t q, uint32_t bit, bool (&ok)[N]) {
    uint4 s[N];
    uint32_t Rf[N], wd[N];
#pragma unroll
    for (int u = 0; u < N; u++) s[u] = ld_cg_v4_pred(A.hot + e[u], valid[u]);
#pragma unroll
    for (int u = 0; u < N; u++)
        Rf[u] = ld_cg_pred(&A.meta[2 * e[u]].x, valid[u] && s[u].x == 0u && q >= JP_R5 && (s[u].w >> JP_HBITS) == JP_R5);
#pragma unroll
    for (int u = 0; u < N; u++) {
        const uint32_t R5 = s[u].w >> JP_HBITS, R = R5 < JP_R5 ? R5 : (q >= JP_R5 ? Rf[u] : JP_R5);
        wd[u] = ld_cg_pred(A.xb + (s[u].w & JP_HMASK) + q - 1, valid[u] && s[u].x == 0u && q > 0u && q < R);
        Rf[u] = R;
    }
#pragma unroll
    for (int u = 0; u < N; u++) {
        if (!valid[u]) ok[u] = true;
        else if (s[u].x != 0u) ok[u] = s[u].x != m;
        else if (q == 0u) ok[u] = (s[u].y >> bit) & 1u;
        else ok[u] = q >= Rf[u] || ((wd[u] >> bit) & 1u);  // q >= R: m > cap
    }
}

// One check of vertex h (compact id; act = the lane holds a vertex): the early-commit
// rule over its watch list (the higher neighbours that were uncoloured -- or, in the
// asynchronous tail, not yet fully pushed -- when the list was built; every other
// higher neighbour's colour is already in h's bitmap, so it cannot equal m).  The
// first JP_LANE_CHECKS entries are checked by the lane (all loads in flight), the rest
// by the whole warp, 32 per step, resuming at the last blocker when m is unchanged.
// Must be called by all lanes of the warp.
struct JpLane {
    uint32_t h, R, hd, ld, wc, pos, lm, m;
    uint64_t off;
    int state;  // 0 checking, 1 passed, 2 failed (memo pos/lm), 3 idle, 5 watch list not built
};

// SPARSE (a round with at most one vertex per warp -- the latency-bound tail): every
// step is warp-wide instead -- the extra bitmap words 32 at a time, the list 64
// entries per step (a watch list holds <= JP_WATCH = 64), no lane stage -- so a check
// is ~4 dependent loads instead of ~10.
template <bool SPARSE>
__device__ __forceinline__ void jp_check(const JpArgs &A, bool act, uint32_t h_in, JpLane &L,
                                         unsigned long long &bytes) {
    const int lane = lane_id();
    uint32_t h = h_in, R = 1, hd = 0, ld = 0, wc = 0, pos = 0, lm = 0, m = 1;
    uint32_t xwo = 0;  // SPARSE: offset of h's extra bitmap words
    uint64_t off = 0;
    int state = 3;
    if (act) {
        const uint4 m0 = __ldcg(A.meta + 2 * h), m1 = __ldcg(A.meta + 2 * h + 1);
        R = m0.x;
        hd = m0.y;
        ld = m0.z;
        wc = m0.w;
        pos = m1.x;
        lm = m1.y;
        off = meta_off(m1);
        bytes += 40;
        if (wc == JP_NOTBUILT) {
            state = 5;
        } else {
            state = 0;
            const uint4 hs = __ldcg(A.hot + h);
            const uint32_t z0 = ~hs.y;
            if (z0) {
                m = __ffs(z0);
            } else if (SPARSE) {
                m = 0;  // the warp scans the extra words below
                xwo = hs.w & JP_HMASK;
            } else {  // colours > 32: bits are only ever set, so m >= the m of the last
                      // failed check (lm) -- the scan starts at lm's word, 4 words in flight
                const uint32_t *xw = A.xb + (hs.w & JP_HMASK);
                uint32_t k = lm > 32u ? (lm - 1) >> 5 : 1u;
                for (m = 0; m == 0 && k < R; k += 4) {
                    uint32_t z[4];
#pragma unroll
                    for (int u = 0; u < 4; u++) z[u] = k + u < R ? ~__ldcg(xw + k + u - 1) : 0u;
#pragma unroll
                    for (int u = 3; u >= 0; u--)
                        if (z[u]) m = (k + u) * 32 + __ffs(z[u]);
                }
                if (m == 0) m = R * 32 + 1;  // unreachable: a zero lies within cap bits
            }
        }
    }
    if (SPARSE) {  // warp-wide mex over the extra bitmap words, 32 words per step
        unsigned need = __ballot_sync(FULL, state == 0 && m == 0);
        while (need) {
            const int src = __ffs(need) - 1;
            need &= need - 1;
            const uint32_t sR = __shfl_sync(FULL, R, src), slm = __shfl_sync(FULL, lm, src);
            const uint32_t *xw = A.xb + __shfl_sync(FULL, xwo, src);
            uint32_t k = slm > 32u ? (slm - 1) >> 5 : 1u, mm = sR * 32 + 1;  // fallback unreachable
            for (; k < sR; k += 32) {
                const uint32_t z = k + lane < sR ? ~__ldcg(xw + k + lane - 1) : 0u;
                const unsigned b = __ballot_sync(FULL, z != 0u);
                if (b) {
                    const int f = __ffs(b) - 1;
                    mm = (k + f) * 32 + __ffs(__shfl_sync(FULL, z, f));
                    break;
                }
            }
            if (lane == src) m = mm;
        }
    }
    const uint32_t q = (m - 1) >> 5, bit = (m - 1) & 31;
    uint32_t j = (lm == m && pos < wc) ? pos : 0u;  // m unchanged: resume at the last blocker
    // the list checked: the watch area (hd > JP_WLIST) or the higher list itself
    const uint64_t coff = off + (hd > JP_WLIST ? 0u : watch_area(hd, ld));
    // ---- lane: the first JP_LANE_CHECKS entries (all loads of a stage in flight)
    // (SYM_JP_LANE_ALL = 0: a lane checks its list alone only when the rest of it fits
    // the lane stage; a longer one goes straight to the warp -- one chain, not two)
    // (SYM_JP_LANE_ITERS > 1: up to that many lane batches before the warp takes over)
    for (int it = 0; it < SYM_JP_LANE_ITERS; it++)
    if (!SPARSE && state == 0 && (SYM_JP_LANE_ALL || wc - j <= (uint32_t)JP_LANE_CHECKS)) {
        uint32_t e[JP_LANE_CHECKS];
        bool valid[JP_LANE_CHECKS], ok[JP_LANE_CHECKS];
#pragma unroll
        for (int u = 0; u < JP_LANE_CHECKS; u++) {
            valid[u] = j + u < wc;
            e[u] = ld_cg_pred(A.lst + coff + j + u, valid[u]);
        }
        jp_nb_stage<JP_LANE_CHECKS>(A, e, valid, m, q, bit, ok);
#pragma unroll
        for (int u = 0; u < JP_LANE_CHECKS; u++) {
            if (state == 0) {
                if (j >= wc) {
                    state = 1;
                } else if (!ok[u]) {
                    state = 2;
                    pos = j;
                    lm = m;
                } else {
                    j++;
                }
            }
        }
        if (state == 0 && j >= wc) state = 1;
        bytes += 12ull * min(wc, (uint32_t)JP_LANE_CHECKS);
    }
    // ---- warp: the rest of a list (<= JP_WLIST entries: at most two steps)
    unsigned need = __ballot_sync(FULL, state == 0);
    while (need) {
        const int src = __ffs(need) - 1;
        need &= need - 1;
        uint32_t wj = __shfl_sync(FULL, j, src);
        const uint32_t wwc = __shfl_sync(FULL, wc, src), wm = __shfl_sync(FULL, m, src);
        const uint64_t woff = __shfl_sync(FULL, coff, src);
        const uint32_t wq = (wm - 1) >> 5, wbit = (wm - 1) & 31;
        int wstate = wj >= wwc ? 1 : 0;
        uint32_t wpos = 0;
        constexpr int S = (SPARSE || SYM_JP_WARP_S2) ? 2 : 1;  // entries per lane per step
        while (wstate == 0) {
            bool ok[S], valid[S];
            uint32_t eu[S];
#pragma unroll
            for (int u = 0; u < S; u++) {
                valid[u] = wj + u * 32 + lane < wwc;
                eu[u] = ld_cg_pred(A.lst + woff + wj + u * 32 + lane, valid[u]);
            }
            jp_nb_stage<S>(A, eu, valid, wm, wq, wbit, ok);
#pragma unroll
            for (int u = 0; u < S; u++) {
                const unsigned fails = __ballot_sync(FULL, !ok[u]);
                if (wstate == 0 && fails) {
                    wstate = 2;
                    wpos = wj + u * 32 + __ffs(fails) - 1;
                }
            }
            if (wstate == 0) {
                wj += 32 * S;
                if (wj >= wwc) wstate = 1;
            }
            bytes += lane == 0 ? 384ull * S : 0ull;
        }
        if (lane == src) {
            state = wstate;
            if (wstate == 2) {
                pos = wpos;
                lm = m;
            }
        }
    }
    L.h = h;
    L.R = R;
    L.hd = hd;
    L.ld = ld;
    L.wc = wc;
    L.pos = pos;
    L.lm = lm;
    L.m = m;
    L.off = off;
    L.state = state;
}

// Phase A of round r: every active vertex (count <= JP_WATCH) is checked (jp_check); a
// vertex whose higher list is longer than JP_WLIST asks phase B for its watch list
// first.
__device__ __forceinline__ void jp_phase_a(const JpArgs &A, uint32_t r, uint32_t cnt, int64_t warp_g,
                                           int64_t nwarps, unsigned long long &bytes) {
    const int lane = lane_id();
    const uint32_t *U = A.ul[r & 1];
    uint32_t *Un = A.ul[(r + 1) & 1];
    // a long list is read coalesced (entry it*32*nwarps + warp*32 + lane); a short one
    // spreads over all warps (entry it*32*nwarps + lane*nwarps + warp), so the
    // warp-cooperative steps of different vertices run in parallel
    const bool spread = cnt < 32 * nwarps;
    for (int64_t it = 0; it < cnt; it += nwarps * 32) {
        const int64_t i = it + (spread ? (int64_t)lane * nwarps + warp_g : warp_g * 32 + lane);
        const bool act = i < cnt;
        JpLane L;
        if (cnt <= nwarps) jp_check<true>(A, act, act ? __ldcg(U + i) : 0u, L, bytes);
        else jp_check<false>(A, act, act ? __ldcg(U + i) : 0u, L, bytes);
        const uint32_t h = L.h, hd = L.hd, ld = L.ld, pos = L.pos, lm = L.lm, m = L.m;
        const uint64_t off = L.off;
        const int state = L.state;
        // ---- outcome
        const bool pass = state == 1, stay = state == 2 || state == 5;
        if (pass) A.hot[h].x = m;
        if (state == 2) *reinterpret_cast<uint2 *>(A.meta + 2 * h + 1) = make_uint2(pos, lm);
        if (state == 5) reinterpret_cast<uint32_t *>(A.meta + 2 * h)[3] = 0u;  // filled by phase B
        // the three reservations (next list, push tasks, build tasks): warp scans, then
        // lane 0 issues the three atomics back to back (one round trip, not three)
        const uint32_t nt = pass ? (ld + JP_PUSH - 1) / JP_PUSH : 0u;
        const uint32_t nb = state == 5 ? (hd + JP_BUILD - 1) / JP_BUILD : 0u;
        uint32_t xs = stay ? 1u : 0u, xt = nt, xb_ = nb;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t ys = __shfl_up_sync(FULL, xs, d), yt = __shfl_up_sync(FULL, xt, d),
                           yb = __shfl_up_sync(FULL, xb_, d);
            if (lane >= d) {
                xs += ys;
                xt += yt;
                xb_ += yb;
            }
        }
        const uint32_t Ts = __shfl_sync(FULL, xs, 31), Tt = __shfl_sync(FULL, xt, 31), Tb = __shfl_sync(FULL, xb_, 31);
        // lanes 0, 1, 2 issue the three reservations as ONE instruction (one round trip;
        // from a single lane ptxas aggregates each uniform-address atomic separately)
        uint32_t *ra = lane == 0 ? A.ucnt + (r + 1) % 3 : (lane == 1 ? A.pcnt + r % 3 : A.bcnt + r % 3);
        const uint32_t rv = lane == 0 ? Ts : (lane == 1 ? Tt : Tb);
        const uint32_t rold = atom_add_pred(ra, rv, lane < 3 && rv != 0u);
        const int64_t slot = (int64_t)__shfl_sync(FULL, rold, 0) + xs - (stay ? 1u : 0u);
        const int64_t ts = (int64_t)__shfl_sync(FULL, rold, 1) + xt - nt;
        const int64_t bs = (int64_t)__shfl_sync(FULL, rold, 2) + xb_ - nb;
        if (stay) Un[slot] = h;
        // push tasks of a new colour
        if (nt) {
            const uint64_t l0 = off + watch_area(hd, ld) + hd;  // the lower list
            for (uint32_t t = 0; t < nt; t++) {
                const uint64_t s0 = l0 + (uint64_t)t * JP_PUSH;
                A.task[ts + t] = make_uint4((uint32_t)s0, (uint32_t)(s0 >> 32), min(JP_PUSH, ld - t * JP_PUSH), m);
            }
        }
        // watch-list build tasks, one per JP_BUILD higher entries
        for (uint32_t t = 0; t < nb; t++)
            A.btask[bs + t] = make_uint4(h, t | ((uint32_t)(off >> 32) << 24), hd, (uint32_t)off);
        bytes += (state == 2 ? 8ull : 0ull) + (stay ? 4ull : 0ull) + (pass ? 4ull + 16ull * nt : 0ull) + 8ull * nb;
    }
}

// A new colour c (word q, bit) for lower neighbours e[u] (list ids, flags act): a
// neighbour already coloured (early commit) needs nothing; otherwise its forbidden
// bit and one higher neighbour less to wait for.  The push that brings a count to
// JP_WATCH activates the neighbour (next round's list).  Each stage's loads/atomics
// are in flight together.
#ifndef SYM_JP_DIAG
#define SYM_JP_DIAG 0  // 1: compile the SYM_JP_TRACE=3/4 sub-step timers (they cost registers)
#endif
// diagnostics (SYM_JP_TRACE=4): wait for v, then read the timer
__device__ __forceinline__ uint64_t jp_stamp_after(uint32_t v, uint32_t *sink) {
    if (__ballot_sync(FULL, v == 0x7fffffe1u) == 0xffffffffu) *sink = 0u;
    return globaltimer_ns();
}

template <int K, class Activate>
__device__ __forceinline__ void jp_push(const JpArgs &A, const uint32_t (&e)[K], bool (&act)[K], uint32_t q,
                                        uint32_t bit, const Activate &activate, uint32_t *tr4 = nullptr) {
#if SYM_JP_DIAG
    const uint64_t tq0 = tr4 ? globaltimer_ns() : 0;
#endif
    uint32_t old[K], x[K];
    // the count decrement needs no filter: a coloured neighbour was activated before its
    // check (count <= JP_WATCH), so its decrement can never be the activating one -- the
    // atomics go out together with the filter loads (colours > 32: the extra-word offset)
    // (predicated PTX atomics: with `act ? atomicSub(..) : 0` the compiler branched around
    // each atomic and tested its result inside the branch, so the K returning atomics ran
    // one after another -- ~1 us each in the tail)
    // One 64-bit atomic per target: {count, xo} are adjacent in the hot record, so
    // adding -1 to the pair decrements the count (never 0 before: no borrow) and
    // returns the R field and extra-word offset with it -- no separate load.  No colour
    // filter: a bit in the bitmap of an already coloured vertex is never read (nb_ok
    // tests its colour first).
    // all K atomics first, their results read only afterwards (with the select in the
    // same loop ptxas consumed each result before issuing the next atomic: ~14 % of the
    // rounds kernel's stall samples sat on those selects)
    uint64_t o[K];
#pragma unroll
    for (int u = 0; u < K; u++) o[u] = atom_dec64_pred(reinterpret_cast<unsigned long long *>(&A.hot[e[u]].z), act[u]);
#pragma unroll
    for (int u = 0; u < K; u++) {
        old[u] = (uint32_t)o[u];
        x[u] = act[u] && q > 0 ? (uint32_t)(o[u] >> 32) : 0xffffffffu;
    }
#if SYM_JP_DIAG
    uint64_t tq1 = 0, tq2 = 0, tq3 = 0;
    if (tr4) {
        uint32_t y = 0, z = 0;
#pragma unroll
        for (int u = 0; u < K; u++) y ^= old[u], z ^= x[u];
        tq1 = jp_stamp_after(y, tr4 + 3);
        tq2 = jp_stamp_after(z, tr4 + 3);
    }
#endif
    if (q == 0) {
#pragma unroll
        for (int u = 0; u < K; u++)
            if (act[u]) atomicOr(&A.hot[e[u]].y, 1u << bit);
    } else {
        uint32_t Rf[K];  // saturated R field (>= 31 words): the full count from meta
#pragma unroll
        for (int u = 0; u < K; u++)
            Rf[u] = ld_cg_pred(&A.meta[2 * e[u]].x, act[u] && (x[u] >> JP_HBITS) == JP_R5 && q >= JP_R5);
#pragma unroll
        for (int u = 0; u < K; u++) {
            const uint32_t R5 = x[u] >> JP_HBITS;
            const bool go = act[u] && (q < R5 || (R5 == JP_R5 && q < Rf[u]));
            x[u] = go ? (x[u] & JP_HMASK) : 0xffffffffu;
        }
#pragma unroll
        for (int u = 0; u < K; u++)
            if (x[u] != 0xffffffffu) atomicOr(A.xb + x[u] + q - 1, 1u << bit);
    }
#if SYM_JP_DIAG
    if (tr4) {
        uint32_t z = 0;
#pragma unroll
        for (int u = 0; u < K; u++) z ^= x[u];
        tq3 = jp_stamp_after(z, tr4 + 3);
    }
#endif
    // activations: one warp-aggregated reservation on the next list (all lanes call)
    uint32_t na = 0;
#pragma unroll
    for (int u = 0; u < K; u++) na += (act[u] && old[u] == JP_WATCH + 1u) ? 1u : 0u;
    if (__any_sync(FULL, na != 0)) {
        const int lane = lane_id();
        uint32_t incl = na;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(FULL, incl, d);
            if (lane >= d) incl += y;
        }
        uint32_t base = 0;
        if (lane == 31) base = atomicAdd(activate.cnt, incl);
        uint32_t slot = __shfl_sync(FULL, base, 31) + incl - na;
#pragma unroll
        for (int u = 0; u < K; u++)
            if (act[u] && old[u] == JP_WATCH + 1u) activate.list[slot++] = e[u];
    }
#if SYM_JP_DIAG
    if (tr4) {
        __syncwarp();
        const uint64_t tq4 = globaltimer_ns();
        if (lane_id() == 0) {  // slowest: atomics returned, hot loads, saturated-R loads + REDs, activations
            atomicMax(tr4 + 512, (uint32_t)((tq1 - tq0) >> 5));
            atomicMax(tr4 + 1024, (uint32_t)((tq2 - tq1) >> 5));
            atomicMax(tr4 + 1536, (uint32_t)((tq4 - tq3) >> 5));
        }
    }
#endif
}

// round mode: an activated vertex joins round r+1's list
struct JpNextList {
    uint32_t *cnt, *list;
    __device__ __forceinline__ JpNextList(const JpArgs &A, uint32_t r)
        : cnt(A.ucnt + (r + 1) % 3), list(A.ul[(r + 1) & 1]) {}
};

// Phase B of round r: push the new colours; build the requested watch lists
__device__ __forceinline__ void jp_phase_b(const JpArgs &A, uint32_t r, uint32_t cnt, uint32_t nbt,
                                           int64_t warp_g, int64_t nwarps, unsigned long long &bytes) {
    const int lane = lane_id();
    const bool tr = A.trace2 && A.trace && r < 512;
    const uint64_t tp0 = tr ? globaltimer_ns() : 0;
    for (int64_t base = warp_g; base - warp_g < cnt; base += nwarps * 32) {
        const int64_t i = base + (int64_t)lane * nwarps;  // tasks spread over all warps
        uint4 tk = make_uint4(0u, 0u, 0u, 0u);
        if (i < cnt) tk = __ldcg(A.task + i);
        const uint64_t s0 = (uint64_t)tk.x | ((uint64_t)tk.y << 32);
        // one jp_push shape for both kinds: first every lane's own small task (<=
        // JP_PUSH_LANE entries), then each big task with its entries spread over the warp
        static_assert(JP_PUSH == 32 * JP_PUSH_LANE, "a big task is one warp step");
        bool small = tk.z > 0 && tk.z <= JP_PUSH_LANE;
        unsigned bigm = __ballot_sync(FULL, tk.z > JP_PUSH_LANE);
        bool pend = __any_sync(FULL, small);
        while (pend || bigm) {
            uint64_t ws;
            uint32_t wn, wc, stride, first;
            if (pend) {  // own small tasks
                ws = s0;
                wn = small ? tk.z : 0u;
                wc = tk.w;
                stride = 1;
                first = 0;
                pend = false;
                bytes += 4ull * wn;
            } else {
                const int src = __ffs(bigm) - 1;
                bigm &= bigm - 1;
                ws = __shfl_sync(FULL, s0, src);
                wn = __shfl_sync(FULL, tk.z, src);
                wc = __shfl_sync(FULL, tk.w, src);
                stride = 32;
                first = lane;
                bytes += lane == 0 ? 4ull * wn : 0ull;
            }
            const uint32_t q = (wc - 1) >> 5, bit = (wc - 1) & 31;
            uint32_t e[JP_PUSH_LANE];
            bool act[JP_PUSH_LANE];
#pragma unroll
            for (int u = 0; u < JP_PUSH_LANE; u++) {
                const uint32_t j = first + u * stride;
                act[u] = j < wn;
                e[u] = ld_cs_pred(A.lst + ws + j, act[u]);
            }
            jp_push<JP_PUSH_LANE>(A, e, act, q, bit, JpNextList(A, r),
                                  SYM_JP_DIAG && tr && A.trace2 == 4 ? A.trace + r : nullptr);
        }
    }
    const uint64_t tp1 = tr ? globaltimer_ns() : 0;
    if (tr && A.trace2 == 2 && lane == 0 && warp_g < cnt) atomicMax(A.trace + 512 + r, (uint32_t)((tp1 - tp0) >> 5));
    // (the last warps first: in a tail round the push tasks sit on the first warps, so a
    // warp holds a push OR a build and phase B is one dependent chain, not two)
    for (int64_t t = nwarps - 1 - warp_g; t < nbt; t += nwarps) {
        const uint4 bt = __ldcg(A.btask + t);
        const uint64_t wl = ((uint64_t)(bt.y >> 24) << 32) | bt.w, hl = wl + watch_words(bt.z);
        uint32_t *wcp = reinterpret_cast<uint32_t *>(A.meta + 2 * bt.x) + 3;
        const uint32_t j0 = (bt.y & 0xffffffu) * JP_BUILD, j1 = min(bt.z, j0 + JP_BUILD);
        constexpr int K = JP_BUILD / 32;
        uint32_t e[K], c[K];
#pragma unroll
        for (int u = 0; u < K; u++) e[u] = ld_cs_pred(A.lst + hl + j0 + u * 32 + lane, j0 + u * 32 + lane < j1);
#pragma unroll
        for (int u = 0; u < K; u++) c[u] = ld_cg_pred(&A.hot[e[u]].x, j0 + u * 32 + lane < j1);  // != 0 when out of range
        unsigned mk[K];
        uint32_t tot = 0;
#pragma unroll
        for (int u = 0; u < K; u++) {
            mk[u] = __ballot_sync(FULL, c[u] == 0u);
            tot += __popc(mk[u]);
        }
        uint32_t p0 = 0;
        if (tot && lane == 0) p0 = atomicAdd(wcp, tot);  // one reservation per task
        p0 = __shfl_sync(FULL, p0, 0);
#pragma unroll
        for (int u = 0; u < K; u++) {
            const uint32_t p = p0 + __popc(mk[u] & ((1u << lane) - 1u));
            if (c[u] == 0u && p < JP_WATCH) A.lst[wl + p] = e[u];
            p0 += __popc(mk[u]);
        }
        bytes += lane == 0 ? 8ull * (j1 - j0) : 0ull;
    }
    if (tr && A.trace2 == 2 && lane == 0 && nwarps - 1 - warp_g < nbt)
        atomicMax(A.trace + 1024 + r, (uint32_t)((globaltimer_ns() - tp1) >> 5));
}

#ifndef SYM_JR_THREADS
#define SYM_JR_THREADS 512
#endif
constexpr int JR_THREADS = SYM_JR_THREADS;
#ifndef SYM_JR_MINB
#define SYM_JR_MINB 2
#endif
constexpr uint64_t JR_TIMEOUT_NS = 20ull * 1000 * 1000 * 1000;

__global__ void __launch_bounds__(JR_THREADS, SYM_JR_MINB) k_jp_rounds(JpArgs A, JrCtl C) {
    // warp-in-CTA major: consecutive list entries of a warp step spread over SMs
    const int64_t warp_g = (int64_t)(threadIdx.x >> 5) * gridDim.x + blockIdx.x;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t t0 = globaltimer_ns();
    unsigned long long bytes = 0;
    uint32_t k = 0, r = 0;
    if (__ldcg(A.err) & 2u) return;  // the build overflowed the segment offsets (set before launch)
    __shared__ uint32_t s_val[3];    // counters loaded once per CTA by the barriers
    if (threadIdx.x == 0) s_val[0] = __ldcg(A.ucnt);
    __syncthreads();
    for (;; r++) {
        const uint32_t cnt = s_val[0];
        if (cnt == 0) break;
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            if (A.hist && r < 1024) {  // stats: list size and start time (32 ns units) of the first rounds
                A.hist[r] = cnt;
                A.hist[1024 + r] = (uint32_t)((globaltimer_ns() - t0) >> 5);
            }
            A.ucnt[(r + 2) % 3] = 0u;  // U_{r+2}'s counter: last read at the start of round r-1
            A.pcnt[(r + 2) % 3] = 0u;  // push tasks of round r+2: last read in round r-1
            A.bcnt[(r + 2) % 3] = 0u;
            if (r + 1 >= C.max_rounds || globaltimer_ns() - t0 > JR_TIMEOUT_NS) atomicOr(A.err, 1u);
        }
        jp_phase_a(A, r, cnt, warp_g, nwarps, bytes);
        grid_sync(C, k, A.pcnt + r % 3, A.bcnt + r % 3, A.err, s_val);
        if (s_val[2] != 0) break;  // read after the barrier: every CTA sees the same word
        const uint32_t pc = s_val[0], bc = s_val[1];
        if (A.trace && blockIdx.x == 0 && threadIdx.x == 0 && r < 512) {  // diagnostics
            A.trace[r] = (uint32_t)((globaltimer_ns() - t0) >> 5);
            if (!A.trace2) {
                A.trace[512 + r] = __ldcg(A.pcnt + r % 3);
                A.trace[1024 + r] = __ldcg(A.bcnt + r % 3);
            }
        }
        const uint64_t tb = A.trace ? globaltimer_ns() : 0;
        jp_phase_b(A, r, pc, bc, warp_g, nwarps, bytes);
        if (A.trace && A.trace2 < 3 && r < 512) {  // diagnostics: slowest CTA's phase-B work span
            __syncthreads();
            if (threadIdx.x == 0) atomicMax(A.trace + 1536 + r, (uint32_t)((globaltimer_ns() - tb) >> 5));
        }
        grid_sync(C, k, A.ucnt + (r + 1) % 3, nullptr, nullptr, s_val);
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) *C.levels = r;
    prof_add(A.prof, 0ull, bytes);
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

// COLOR-Rand (Alg 8): V' = endpoints of monochromatic cross arcs (lower != 0,
// SYM_F_LOWER_ONLY: only the lower-priority endpoint of each)
__global__ void k_color_conflicts(const int64_t *__restrict__ rp_x, const int32_t *__restrict__ ci_x, int64_t n,
                                  const uint32_t *color, uint8_t *mark, int32_t *list, uint32_t *cnt, int lower,
                                  Key k, const uint32_t *okey, int ord) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n; base += stride) {
        int64_t v = base + threadIdx.x;
        bool conf = false;
        if (v < n) {
            uint32_t cv = color[v];
            const uint64_t kv = lower ? jp_okey(k, okey, ord, (uint32_t)v) : 0;
            for (int64_t x = rp_x[v]; x < rp_x[v + 1] && !conf; x++)
                conf = color[ci_x[x]] == cv && (!lower || jp_okey(k, okey, ord, (uint32_t)ci_x[x]) > kv);
            mark[v] = conf ? 1 : 0;
        }
        cta_append2(conf, false, (int32_t)v, n, list, cnt, cnt);  // one atomic per CTA
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
    w.ov = a.take<int32_t>((size_t)n + 1);
    w.hdeg = a.take<uint32_t>((size_t)n + 1);
    w.ldeg = a.take<uint32_t>((size_t)n + 1);
    w.arank = a.take<uint32_t>(2 * ((size_t)(n + 31) / 32 + 1));
    w.hot = a.take<uint4>((size_t)n + 1);
    w.meta = a.take<uint4>(2 * (size_t)n + 2);
    w.ul[0] = a.take<uint32_t>((size_t)n + 1);
    w.ul[1] = a.take<uint32_t>((size_t)n + 1);
    // lists: one id per arc (higher or lower) + watch areas of JP_WATCH ids for the
    // rows with > JP_WLIST higher neighbours (fewer than nnz / JP_WLIST rows, so the
    // areas take < nnz words)
    static_assert(JP_WATCH <= JP_WLIST, "watch areas must fit the nnz bound");
    w.lst_words = std::min<int64_t>((int64_t)JP_WATCH * n, nnz) + nnz + 2;
    w.lst = a.take<uint32_t>((size_t)w.lst_words);
    // extra bitmap words: sum of ceil(cap/32) - 1 <= (nnz + n)/32
    w.xb = a.take<uint32_t>((size_t)((nnz + n) / 32 + 2));
    w.tcnt = a.take<uint32_t>(2 * (size_t)ntiles);
    w.tsum = a.take<unsigned long long>(2 * (size_t)ntiles);
    w.ntiles = ntiles;
    w.task_cap = n + nnz / JP_PUSH + 2;  // tasks of one round <= all tasks
    w.task = a.take<uint4>((size_t)w.task_cap);
    w.btask = a.take<uint4>((size_t)w.task_cap);
    w.vlist = a.take<int32_t>((size_t)n + 1);
    w.mark = a.take<uint8_t>((size_t)n + 1);
    w.okey = a.take<uint32_t>((size_t)n + 1);
    w.queue = a.take<int64_t>((size_t)(nnz / JP_BUDGET + 2));  // huge-row pieces (<= nnz/JP_BUDGET)
    w.sync = a.take<uint32_t>(64);  // rounds kernel: barrier / counters / error words
}

// SYM_F_ORDER_LF -> 1, SYM_F_ORDER_SF -> 2, else 0 (the (pv, id) order)
static int jp_order(const FlowArgs &f) {
    return (f.p.flags & SYM_F_ORDER_LF) ? 1 : ((f.p.flags & SYM_F_ORDER_SF) ? 2 : 0);
}

// Build: compact ids, hot state, meta, higher and lower lists, the first round's
// list.  sync words: [0] barrier arrivals, [1] barrier generation, [4..6] list
// counts, [8..10] push-task counts, [12..14] build-task counts, [32] error, [33]
// rounds, [40..41] compact counts.
// the fill passes (one resident wave of each grid-stride kernel, see mis.cu round_grid)
template <bool CF>
static int jp_launch_fill(JpArgs &A, cudaStream_t s) {
    {
        int per = 2048 / JP_THREADS;
#if SYM_ROUND_ONE_WAVE
        int x = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&x, k_jpc_fill<CF>, JP_THREADS, 0) == cudaSuccess && x > 0)
            per = std::min(per, x);
#endif
        k_jpc_fill<CF><<<num_sms() * per, JP_THREADS, 0, s>>>(A);
    }
    SYM_LAUNCH_CHECK();
    {
        // block-strided pieces: one resident wave (40 regs x 512 threads -> 3 CTAs/SM, not 4)
        int per = 4;
#if SYM_ROUND_ONE_WAVE
        int x = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&x, k_jpc_fill_huge<CF>, JP_HUGE_THREADS, 0) == cudaSuccess &&
            x > 0)
            per = std::min(per, x);
#endif
        k_jpc_fill_huge<CF><<<num_sms() * per, JP_HUGE_THREADS, 0, s>>>(A);
    }
    SYM_LAUNCH_CHECK();
    return SYM_OK;
}

static bool getenv_flag(const char *name) {
    const char *e = getenv(name);
    return e && *e && *e != '0';
}

static int jp_build(const FlowArgs &f, ColorWs &w, JpArgs &A, uint32_t *color, const int64_t *rp,
                    const int32_t *ci, const uint8_t *inS, const int32_t *list0, const uint32_t *cnt0,
                    int64_t implicit_n, unsigned long long *rounds_ctr) {
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
    const int64_t n = f.g.n;
    SYM_CUDA(cudaMemsetAsync(ctl->huge, 0, sizeof(ctl->huge), s));
    SYM_CUDA(cudaMemsetAsync(w.sync, 0, 64 * sizeof(uint32_t), s));
    A.rp = rp;
    A.ci = ci;
    A.inS = inS;
    A.color = color;
    A.in_list = list0;
    A.in_cnt = cnt0;
    A.implicit_n = implicit_n;
    A.ov = w.ov;
    A.hdeg = w.hdeg;
    A.ldeg = w.ldeg;
    A.arank = w.arank;
    A.hot = w.hot;
    A.meta = w.meta;
    A.lst = w.lst;
    A.xb = w.xb;
    A.tcnt = w.tcnt;
    A.tsum = w.tsum;
    A.nc = w.sync + 40;
    A.ul[0] = w.ul[0];
    A.ul[1] = w.ul[1];
    A.task = w.task;
    A.ucnt = w.sync + 4;
    A.pcnt = w.sync + 8;
    A.bcnt = w.sync + 12;
    A.btask = w.btask;
    A.huge = w.queue;
    A.huge_cnt = &ctl->huge[1];
    A.err = w.sync + 32;
    A.hist = nullptr;
    A.trace = nullptr;
    A.trace2 = 0;
    A.prof = nullptr;
    A.prof_jp = rounds_ctr;
    A.k = stream_key(f.p.seed, TAG_VERTEX, 0);
    A.okey = w.okey;
    A.ord = jp_order(f);
    const int64_t nwords = (n + 31) / 32;
    const unsigned tiles_w = (unsigned)((nwords + JP_TILE - 1) / JP_TILE);
    const unsigned tiles_c = (unsigned)((n + JP_TILE - 1) / JP_TILE);  // compact ids <= n
    unsigned long long *ctr = prof_counter(s);  // algorithmic bytes of the build (profiling)
    A.prof = ctr;
    prof_begin("jp_build", s);
    if (list0) {
        SYM_CUDA(cudaMemsetAsync(w.arank, 0, 2 * sizeof(uint32_t) * (size_t)nwords, s));
        k_jpc_mark<<<num_sms() * 8, 256, 0, s>>>(A);
    } else {
        k_jpc_bits<<<num_sms() * 8, 256, 0, s>>>(A, implicit_n);
    }
    SYM_LAUNCH_CHECK();
    k_jpc_tiles<<<tiles_w, JP_THREADS, 0, s>>>(A, nwords);
    SYM_LAUNCH_CHECK();
    k_jpc_tiles_scan<<<1, 1024, 0, s>>>(A, tiles_w);
    SYM_LAUNCH_CHECK();
    k_jpc_assign<<<tiles_w, JP_THREADS, 0, s>>>(A, nwords);
    SYM_LAUNCH_CHECK();
    // count-free build when S is implicit (every vertex of the phase CSR): the lists are
    // placed from the degrees and split while filled; otherwise count, place, fill
    const bool cf = inS == nullptr && list0 == nullptr && !getenv_flag("SYM_JP_COUNTED");
    if (cf) {
        SYM_CUDA(cudaMemsetAsync(w.hdeg, 0, sizeof(uint32_t) * (size_t)(n + 1), s));
        SYM_CUDA(cudaMemsetAsync(w.ldeg, 0, sizeof(uint32_t) * (size_t)(n + 1), s));
        if (tiles_c) {
            k_jpc_lsums_cf<<<tiles_c, JP_THREADS, 0, s>>>(A);
            SYM_LAUNCH_CHECK();
        }
        k_jpc_sums_scan<<<1, 1024, 0, s>>>(A, tiles_c);
        SYM_LAUNCH_CHECK();
        if (tiles_c) {
            k_jpc_offs_cf<<<tiles_c, JP_THREADS, 0, s>>>(A);
            SYM_LAUNCH_CHECK();
        }
        SYM_TRY(jp_launch_fill<true>(A, s));
        if (tiles_c) {
            k_jpc_xsums_cf<<<tiles_c, JP_THREADS, 0, s>>>(A);
            SYM_LAUNCH_CHECK();
        }
        k_jpc_sums_scan<<<1, 1024, 0, s>>>(A, tiles_c);
        SYM_LAUNCH_CHECK();
        if (tiles_c) {
            k_jpc_place_cf<<<tiles_c, JP_THREADS, 0, s>>>(A);
            SYM_LAUNCH_CHECK();
        }
    } else {
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
        SYM_TRY(jp_launch_fill<false>(A, s));
    }
    prof_end_dev(s, ctr);
    A.prof = nullptr;
    A.prof_jp = nullptr;
    return SYM_OK;
}

// every round in one persistent cooperative launch
static int jp_run(const FlowArgs &f, ColorWs &w, uint32_t *color, const int64_t *rp, const int32_t *ci,
                  const uint8_t *inS, const int32_t *list0, const uint32_t *cnt0, int64_t implicit_n, int phase) {
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
    if (f.g.n == 0) return SYM_OK;
    // one resident wave of the cooperative rounds kernel, per device (-1: unsupported)
    static std::atomic<int> grid_slots[SYM_MAX_DEVICES];
    const int grid = dev_cached(grid_slots, [] {
        int coop = 0, per_sm = 0;
        const int dev = current_device();
        if (dev < 0 || cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, dev) != cudaSuccess || !coop)
            return -1;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_jp_rounds, JR_THREADS, 0) != cudaSuccess ||
            per_sm < 1)
            return -1;
        // SYM_JR_CTAS_PER_SM < the occupancy leaves SMs' register space to kernels of other
        // streams (the latency-bound rounds barely use the GPU)
        const char *e = getenv("SYM_JR_CTAS_PER_SM");
        if (e && atoi(e) > 0) per_sm = std::min(per_sm, atoi(e));
        return num_sms() * per_sm;
    });
    if (grid < 0) {
        set_error("JP needs a cooperative launch of k_jp_rounds (persistent rounds kernel) on this device");
        return SYM_ECUDA;
    }
    JpArgs A;
    unsigned long long *rounds_ctr = prof_counter(s);  // profiling: the rounds launch's byte pair
    SYM_TRY(jp_build(f, w, A, color, rp, ci, inS, list0, cnt0, implicit_n, rounds_ctr));
    JrCtl C;
    C.arr = w.sync;
    C.levels = w.sync + 33;
    C.max_rounds = f.p.max_rounds ? f.p.max_rounds : 0xffffffffu;
    // barriers (2 per round) x grid must not overflow the arrival word
    C.max_rounds = std::min<uint64_t>(C.max_rounds, 0xffffffffull / (2ull * (uint64_t)grid) - 1);
    A.hist = f.stats ? ctl->hist + phase * 2048 : nullptr;
    static const bool jp_trace = getenv("SYM_JP_TRACE") != nullptr;
    A.trace = jp_trace && f.stats && phase == 0 ? ctl->hist + 2048 : nullptr;
    static const int jp_trace2 = jp_trace ? atoi(getenv("SYM_JP_TRACE")) : 0;
    A.trace2 = jp_trace2 >= 2 ? jp_trace2 : 0;  // 2: push / build spans, 3: push sub-steps
    if (A.trace) SYM_CUDA(cudaMemsetAsync(A.trace, 0, 2048 * sizeof(uint32_t), s));
    A.prof = rounds_ctr;
    void *args[] = {&A, &C};
    prof_begin("jp_rounds", s);
    SYM_CUDA(cudaLaunchCooperativeKernel((const void *)k_jp_rounds, dim3(grid), dim3(JR_THREADS), args, 0, s));
    prof_end_dev(s, A.prof);
    k_jpc_scatter<<<num_sms() * 8, 256, 0, s>>>(A);
    SYM_LAUNCH_CHECK();
    uint32_t err = 0, levels = 0;
    SYM_TRY(read_u32(A.err, &err, s));
    if (err) {
        SYM_TRY(read_u32(C.levels, &levels, s));
        if (err & 2u) {
            set_error("JP: more than 2^27 vertices or 2^32 extra bitmap words");
            return SYM_EINVAL;
        }
        const bool rounds = f.p.max_rounds && levels + 1 >= f.p.max_rounds;
        set_error(rounds ? "JP did not converge within max_rounds" : "JP rounds kernel timed out");
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
    if (f.p.flags & (SYM_F_COLOR_EB | SYM_F_COLOR_VB)) return run_color_spec(f, w, color);  // the paper's subroutines
    SYM_CUDA(cudaMemsetAsync(color, 0, sizeof(uint32_t) * (size_t)g.n, s));
    if (jp_order(f)) {
        k_jp_okey<<<num_sms() * 8, 256, 0, s>>>(g.rp, g.n, jp_order(f), w.okey);
        SYM_LAUNCH_CHECK();
    }
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
                                                          &ctl->conflicts, (f.p.flags & SYM_F_LOWER_ONLY) ? 1 : 0,
                                                          stream_key(f.p.seed, TAG_VERTEX, 0), w.okey, jp_order(f));
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
