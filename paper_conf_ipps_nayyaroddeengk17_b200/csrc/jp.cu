// color.cu -- Jones-Plassmann colouring and the COLOR flows.
//
// JP ([18]) with fixed priorities colours v once every higher-(pv,id)
// neighbour of its phase set S is coloured, with the smallest colour >= 1 not held by
// any coloured neighbour: exactly first-fit greedy in priority order (DESIGN §3 C1).
//
// Push form with forbidden-colour bitmaps (the FORBIDDEN array of P:214/P:234, sized
// deg(v)+1 bits per vertex since mex <= deg+1; bit offset row_ptr[v] + v):
//   init   cnt[v] = #higher S-neighbours; fixed colours of neighbours outside S
//          (COLOR-Rand recolouring) are pre-set in v's bitmap; cnt == 0 -> ready
//          (a ready vertex without phase arcs takes colour 1 at once).
//   round  every ready vertex v is split into tasks of <= JP_CHUNK arcs that carry
//          v's row bounds.  A task computes colour(v) = first zero bit of v's bitmap
//          (complete: all higher neighbours pushed in earlier rounds), and for each
//          lower S-neighbour w of its chunk sets bit colour(v) in w's bitmap and
//          decrements cnt[w]; the decrement reaching 0 appends w's tasks for the
//          next round.  Rows <= JP_LANE arcs are handled by one lane, longer chunks
//          by a warp; consecutive task indices go to different warps so the chunks
//          of one hub run in parallel.
// The dependent chain per round is: task -> (arcs | bitmap) -> (row bounds of w |
// decrement) -> reservation; each arc is read twice in total (init + push).
// Rounds = the JP dependency depth (~5e3 on R-MAT scale 24), so a round is latency-
// bound: one kernel per round on a short grid.
#include <cstdlib>

#include "internal.h"

namespace sym {

constexpr int JP_SMALL = 32;
constexpr int JP_BUDGET = 4096;
constexpr int JP_THREADS = 256;
constexpr int JP_HUGE_THREADS = 512;
constexpr int JP_CHUNK = 256;  // arcs per warp task (8 per lane)
constexpr int JP_LANE = 8;     // rows with <= JP_LANE arcs are a lane task

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
    uint32_t *cnt;
    uint32_t *bits;      // forbidden-colour bitmaps
    const int32_t *in_list;    // init: vertex list (nullable = implicit)
    const uint32_t *in_cnt;
    int64_t implicit_n;
    const JpTask *tin;
    JpTask *tout;
    uint32_t *out_cnt;
    uint32_t *clear_cnt;
    int32_t *huge;
    uint32_t *huge_cnt;
    uint32_t *huge_clear;
    uint32_t *hist;
    int round;
    Key k;
};

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

__device__ __forceinline__ void set_forbidden(uint32_t *bits, int64_t B, int64_t nbits, uint32_t c) {
    if (c >= 1 && (int64_t)c <= nbits) {
        int64_t pos = B + c - 1;
        atomicOr(bits + (pos >> 5), 1u << (pos & 31));
    }
}

// first zero bit of bits[B, B+nbits) -> mex (1-based); warp-cooperative
__device__ __forceinline__ uint32_t warp_mex(const uint32_t *bits, int64_t B, int64_t nbits) {
    const int lane = lane_id();
    const int64_t end = B + nbits;
    const int64_t w0 = B >> 5, w1 = (end - 1) >> 5;
    for (int64_t k0 = w0; k0 <= w1; k0 += 32) {
        int64_t wi = k0 + lane;
        uint32_t zeros = 0;
        if (wi <= w1) {
            uint32_t word = __ldcg(bits + wi);
            int64_t lo = max(B, wi * 32) - wi * 32, hi = min(end, wi * 32 + 32) - wi * 32;
            uint32_t width = (uint32_t)(hi - lo);
            uint32_t mask = (width >= 32 ? 0xffffffffu : ((1u << width) - 1u)) << lo;
            zeros = ~word & mask;
        }
        unsigned bal = __ballot_sync(FULL, zeros != 0);
        if (bal) {
            int src = __ffs(bal) - 1;
            uint32_t z = __shfl_sync(FULL, zeros, src);
            int64_t pos = (k0 + src) * 32 + __ffs(z) - 1;
            return (uint32_t)(pos - B + 1);
        }
    }
    return (uint32_t)nbits;  // unreachable: at most nbits-1 bits can be set
}

// mex of a short bitmap (nbits <= 33) by one lane
__device__ __forceinline__ uint32_t lane_mex(const uint32_t *bits, int64_t B, int64_t nbits) {
    const int64_t w0 = B >> 5;
    const uint64_t lo = __ldcg(bits + w0), hi = __ldcg(bits + w0 + 1);
    const uint64_t word = (lo | (hi << 32)) >> (B & 31);
    const uint64_t valid = nbits >= 64 ? ~0ULL : ((1ULL << nbits) - 1ULL);
    return (uint32_t)__ffsll((long long)(~word & valid));
}

// ---------------------------------------------------------------- init
// cnt[v] = #higher S-neighbours; pre-set fixed colours of non-S neighbours; ready
// vertices enqueue their tasks for round 0.
__global__ void __launch_bounds__(JP_THREADS) k_jp_init(JpArgs A) {
    const uint32_t cnt = A.in_list ? *A.in_cnt : (uint32_t)A.implicit_n;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        *A.clear_cnt = 0;
        *A.huge_clear = 0;
    }
    const int lane = lane_id();
    const int64_t warp_g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = warp_g * 32; base < cnt; base += nwarps * 32) {
        int64_t i = base + lane;
        int32_t v = -1;
        if (i < cnt) v = A.in_list ? A.in_list[i] : (int32_t)i;
        bool active = v >= 0;
        int64_t b = 0, e = 0;
        uint64_t kv = 0;
        if (active) {
            b = A.rp[v];
            e = A.rp[v + 1];
            kv = vkey(A.k, (uint32_t)v);
        }
        uint32_t c = 0;
        if (active && e - b <= JP_SMALL) {
            for (int64_t x = b; x < e; x++) {
                uint32_t w = (uint32_t)__ldg(A.ci + x);
                if (in_set(A.inS, w)) c += vkey(A.k, w) > kv ? 1u : 0u;
                else set_forbidden(A.bits, b + v, e - b + 1, A.color[w]);
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
            for (int64_t x = wb + lane; x < we; x += 32) {
                uint32_t w = (uint32_t)__ldg(A.ci + x);
                if (in_set(A.inS, w)) lc += vkey(A.k, w) > wk ? 1u : 0u;
                else set_forbidden(A.bits, wb + wv, we - wb + 1, A.color[w]);
            }
            for (int d = 16; d; d >>= 1) lc += __shfl_xor_sync(FULL, lc, d);
            if (lane == src) c = lc;
        }
        bool huge = active && e - b > JP_BUDGET;
        if (active && !huge) A.cnt[v] = c;
        bool ready = active && !huge && c == 0;
        if (ready && e == b) {  // no phase neighbour: colour 1 now, no task
            A.color[v] = 1u;
            ready = false;
        }
        uint32_t nt = ready ? n_tasks(e - b) : 0u;
        int64_t slot = warp_reserve(nt, A.out_cnt);
        put_tasks(A.tout, slot, v, b, e, nt);
        int64_t hs = warp_append(huge, A.huge_cnt);
        if (hs >= 0) A.huge[hs] = v;
    }
}

__global__ void __launch_bounds__(JP_HUGE_THREADS) k_jp_init_huge(JpArgs A) {
    const uint32_t cnt = *A.huge_cnt;
    __shared__ uint32_t s_sum;
    __shared__ int64_t s_slot;
    for (uint32_t h = blockIdx.x; h < cnt; h += gridDim.x) {
        const int32_t v = A.huge[h];
        const int64_t b = A.rp[v], e = A.rp[v + 1];
        const uint64_t kv = vkey(A.k, (uint32_t)v);
        if (threadIdx.x == 0) s_sum = 0;
        __syncthreads();
        uint32_t lc = 0;
        for (int64_t x = b + threadIdx.x; x < e; x += JP_HUGE_THREADS) {
            uint32_t w = (uint32_t)__ldg(A.ci + x);
            if (in_set(A.inS, w)) lc += vkey(A.k, w) > kv ? 1u : 0u;
            else set_forbidden(A.bits, b + v, e - b + 1, A.color[w]);
        }
        for (int d = 16; d; d >>= 1) lc += __shfl_xor_sync(FULL, lc, d);
        if (lane_id() == 0) atomicAdd(&s_sum, lc);
        __syncthreads();
        const uint32_t nt = n_tasks(e - b);
        if (threadIdx.x == 0) {
            A.cnt[v] = s_sum;
            s_slot = (s_sum == 0) ? (int64_t)atomicAdd(A.out_cnt, nt) : -1;
        }
        __syncthreads();
        if (s_slot >= 0)
            for (uint32_t q = threadIdx.x; q < nt; q += JP_HUGE_THREADS) {
                JpTask t;
                t.b = b;
                t.e = e;
                t.v = v;
                t.j = q;
                t.pad = 0;
                A.tout[s_slot + q] = t;
            }
        __syncthreads();
    }
}

// ---------------------------------------------------------------- push rounds
// Push the colour c of a vertex to the lower S-neighbours w[0..U) (flags in low[]):
// the row bounds of w and the decrement are issued together, then the bitmap bit.
template <int U>
__device__ __forceinline__ uint32_t jp_push_arcs(const JpArgs &A, const uint32_t (&w)[U], bool (&low)[U], uint32_t c,
                                                 int64_t (&wb)[U], int64_t (&we)[U]) {
    uint32_t old[U];
#pragma unroll
    for (int u = 0; u < U; u++) {
        if (low[u]) {
            wb[u] = A.rp[w[u]];
            we[u] = A.rp[w[u] + 1];
            old[u] = atomicSub(A.cnt + w[u], 1u);
        }
    }
    uint32_t ready = 0;
#pragma unroll
    for (int u = 0; u < U; u++) {
        if (low[u]) {
            set_forbidden(A.bits, wb[u] + w[u], we[u] - wb[u] + 1, c);
            if (old[u] == 1u) ready |= 1u << u;
        }
    }
    return ready;
}

template <int U>
__device__ __forceinline__ void jp_enqueue(const JpArgs &A, const uint32_t (&w)[U], uint32_t ready,
                                           const int64_t (&wb)[U], const int64_t (&we)[U]) {
    uint32_t nt = 0;
#pragma unroll
    for (int u = 0; u < U; u++)
        if ((ready >> u) & 1u) nt += n_tasks(we[u] - wb[u]);
    int64_t slot = warp_reserve(nt, A.out_cnt);
#pragma unroll
    for (int u = 0; u < U; u++) {
        if ((ready >> u) & 1u) {
            uint32_t k = n_tasks(we[u] - wb[u]);
            put_tasks(A.tout, slot, (int32_t)w[u], wb[u], we[u], k);
            slot += k;
        }
    }
}

__global__ void __launch_bounds__(JP_THREADS) k_jp_push(JpArgs A) {
    const uint32_t cnt = *A.in_cnt;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        *A.clear_cnt = 0;
        if (A.hist && A.round < 2048) A.hist[A.round] = cnt;
    }
    const int lane = lane_id();
    const int64_t warp_g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    // task index t = it*32*nwarps + lane*nwarps + warp: consecutive tasks (the chunks
    // of one hub) land on different warps
    for (int64_t base = warp_g; base - warp_g < cnt; base += nwarps * 32) {
        const int64_t t = base + (int64_t)lane * nwarps;
        int32_t v = -1;
        uint32_t j = 0;
        int64_t b = 0, e = 0;
        if (t < cnt) {
            const longlong2 *p = reinterpret_cast<const longlong2 *>(A.tin + t);
            longlong2 q0 = __ldcg(p), q1 = __ldcg(p + 1);
            b = q0.x;
            e = q0.y;
            v = (int32_t)(uint32_t)q1.x;
            j = (uint32_t)((uint64_t)q1.x >> 32);
        }
        const uint64_t kv = v >= 0 ? vkey(A.k, (uint32_t)v) : 0;
        // ---- short rows: one lane does the whole task
        const bool small = v >= 0 && e - b <= JP_LANE;
        {
            uint32_t w[JP_LANE];
            bool low[JP_LANE];
#pragma unroll
            for (int u = 0; u < JP_LANE; u++) {
                low[u] = small && b + u < e;
                w[u] = low[u] ? (uint32_t)__ldg(A.ci + b + u) : 0u;
            }
            uint32_t c = 0;
            if (small) {
                c = lane_mex(A.bits, b + v, e - b + 1);
                A.color[v] = c;
            }
#pragma unroll
            for (int u = 0; u < JP_LANE; u++) low[u] = low[u] && in_set(A.inS, w[u]) && vkey(A.k, w[u]) < kv;
            int64_t wb[JP_LANE], we[JP_LANE];
            uint32_t ready = jp_push_arcs<JP_LANE>(A, w, low, c, wb, we);
            jp_enqueue<JP_LANE>(A, w, ready, wb, we);
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
                int64_t x = cb + u * 32 + lane;
                low[u] = x < te;
                w[u] = low[u] ? (uint32_t)__ldg(A.ci + x) : 0u;
            }
            const uint32_t c = warp_mex(A.bits, tb + tv, te - tb + 1);
            if (tj == 0 && lane == 0) A.color[tv] = c;
#pragma unroll
            for (int u = 0; u < U; u++) low[u] = low[u] && in_set(A.inS, w[u]) && vkey(A.k, w[u]) < tk;
            int64_t wb[U], we[U];
            uint32_t ready = jp_push_arcs<U>(A, w, low, c, wb, we);
            jp_enqueue<U>(A, w, ready, wb, we);
        }
    }
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
    w.cnt = a.take<uint32_t>((size_t)n + 1);
    w.bits = a.take<uint32_t>((size_t)((nnz + n) / 32 + 2));
    w.bits_words = (nnz + n) / 32 + 2;
    w.queue_cap = n + nnz / JP_CHUNK + 2;  // tasks in one round <= all tasks
    w.task = a.take<int64_t>(2 * (size_t)w.queue_cap * (sizeof(JpTask) / sizeof(int64_t)));
    w.vlist = a.take<int32_t>((size_t)n + 1);
    w.mark = a.take<uint8_t>((size_t)n + 1);
    w.queue = a.take<int32_t>((size_t)(nnz / JP_BUDGET + 2));  // deferred init rows
}

// JP over (rp, ci) for the vertex set S (list/implicit) with membership inS; the
// bitmap layout follows this CSR (offset rp[v] + v, deg+1 bits).
// ---------------------------------------------------------------- asynchronous JP
// No global rounds: a persistent grid of warps colours vertices as soon as they are
// ready.  A lane that makes a short-row vertex (deg <= JP_LANE) ready colours it
// itself next (per-lane continuation stack, no queue hop); longer rows are split into
// JP_CHUNK-arc tasks appended to one global queue that idle warps claim.  Pushes set
// the forbidden bit, fence, then decrement; the decrement that reaches 0 is followed
// by a fence before the bitmap is read, so every higher neighbour's colour is seen.
// Termination: an exact count of coloured vertices (flushed before a warp waits).
// A warp waiting on an empty queue slot also watches the count, an error flag and a
// %globaltimer deadline, so a bug cannot hang the device.
constexpr int JA_STACK = 16;
constexpr uint64_t JA_TIMEOUT_NS = 20ull * 1000 * 1000 * 1000;

struct JaArgs {
    const int64_t *rp;
    const int32_t *ci;
    const uint8_t *inS;
    uint32_t *color;
    uint32_t *cnt;
    uint32_t *bits;
    JpTask *q;
    int64_t qcap;
    uint32_t *head, *tail, *done, *err;
    const uint32_t *target;  // vertices to colour by tasks
    Key k;
};

__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ int32_t ld_volatile_i32(const int32_t *p) {
    int32_t v;
    asm volatile("ld.volatile.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_volatile_i32(int32_t *p, int32_t v) {
    asm volatile("st.volatile.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// lane-level enqueue of all chunk tasks of vertex w (flag field v written last)
__device__ __forceinline__ void ja_enqueue(const JaArgs &A, int32_t w, int64_t wb, int64_t we) {
    const uint32_t nt = n_tasks(we - wb);
    const uint32_t slot = atomicAdd(A.tail, nt);
    for (uint32_t q = 0; q < nt; q++) {
        JpTask *t = A.q + slot + q;
        t->b = wb;
        t->e = we;
        t->j = q;
    }
    __threadfence();
    for (uint32_t q = 0; q < nt; q++) st_volatile_i32(&A.q[slot + q].v, w);
}

struct JaStack {
    int32_t v[JA_STACK];
    int64_t b[JA_STACK], e[JA_STACK];
    int sp;
};

__device__ __forceinline__ void ja_ready(const JaArgs &A, JaStack &st, int32_t w, int64_t wb, int64_t we) {
    if (we - wb <= JP_LANE && st.sp < JA_STACK) {
        st.v[st.sp] = w;
        st.b[st.sp] = wb;
        st.e[st.sp] = we;
        st.sp++;
    } else {
        ja_enqueue(A, w, wb, we);
    }
}

// colour a short-row vertex and push to its lower S-neighbours (one lane)
__device__ __forceinline__ void ja_lane_vertex(const JaArgs &A, JaStack &st, int32_t v, int64_t b, int64_t e,
                                               uint32_t &ncol) {
    const uint64_t kv = vkey(A.k, (uint32_t)v);
    __threadfence();  // acquire: the decrement that made v ready precedes these reads
    const uint32_t c = lane_mex(A.bits, b + v, e - b + 1);
    A.color[v] = c;
    ncol++;
    uint32_t w[JP_LANE];
    bool low[JP_LANE];
    int64_t wb[JP_LANE], we[JP_LANE];
#pragma unroll
    for (int u = 0; u < JP_LANE; u++) {
        low[u] = b + u < e;
        w[u] = low[u] ? (uint32_t)__ldg(A.ci + b + u) : 0u;
    }
#pragma unroll
    for (int u = 0; u < JP_LANE; u++) {
        low[u] = low[u] && in_set(A.inS, w[u]) && vkey(A.k, w[u]) < kv;
        if (low[u]) {
            wb[u] = A.rp[w[u]];
            we[u] = A.rp[w[u] + 1];
        }
    }
#pragma unroll
    for (int u = 0; u < JP_LANE; u++)
        if (low[u]) set_forbidden(A.bits, wb[u] + w[u], we[u] - wb[u] + 1, c);
    __threadfence();  // release: the forbidden bits precede the decrements
#pragma unroll
    for (int u = 0; u < JP_LANE; u++)
        if (low[u] && atomicSub(A.cnt + w[u], 1u) == 1u) ja_ready(A, st, (int32_t)w[u], wb[u], we[u]);
}

__global__ void __launch_bounds__(JP_THREADS) k_jp_async(JaArgs A) {
    const int lane = lane_id();
    JaStack st;
    st.sp = 0;
    uint32_t ncol = 0;
    const uint64_t t0 = globaltimer_ns();
    const uint32_t target = *A.target;
    for (;;) {
        // 1. drain the lanes' continuation stacks
        while (__any_sync(FULL, st.sp > 0)) {
            if (st.sp > 0) {
                st.sp--;
                ja_lane_vertex(A, st, st.v[st.sp], st.b[st.sp], st.e[st.sp], ncol);
            }
        }
        // 2. flush the coloured count, then claim one queued task for the warp
        uint32_t sum = ncol;
        for (int d = 16; d; d >>= 1) sum += __shfl_xor_sync(FULL, sum, d);
        ncol = 0;
        int32_t tv = -1;
        uint32_t idx = 0;
        bool quit = false;
        if (lane == 0) {
            if (sum) atomicAdd(A.done, sum);
            idx = atomicAdd(A.head, 1u);
            uint32_t spins = 0;
            for (;;) {
                tv = idx < A.qcap ? ld_volatile_i32(&A.q[idx].v) : -1;
                if (tv >= 0) break;
                if ((++spins & 63u) == 0) {
                    if (ld_volatile_u32(A.done) >= target || ld_volatile_u32(A.err)) {
                        quit = true;
                        break;
                    }
                    if (globaltimer_ns() - t0 > JA_TIMEOUT_NS) {
                        atomicExch(A.err, 1u);
                        quit = true;
                        break;
                    }
                }
                __nanosleep(64);
            }
        }
        quit = __shfl_sync(FULL, quit, 0);
        if (quit) return;
        tv = __shfl_sync(FULL, tv, 0);
        idx = __shfl_sync(FULL, idx, 0);
        __threadfence();
        const int64_t tb = __ldcg(&A.q[idx].b), te = __ldcg(&A.q[idx].e);
        const uint32_t tj = __ldcg(&A.q[idx].j);
        // 3. process the chunk with the whole warp
        const uint64_t tk = vkey(A.k, (uint32_t)tv);
        const int64_t cb = tb + (int64_t)tj * JP_CHUNK;
        constexpr int U = JP_CHUNK / 32;
        uint32_t w[U];
        bool low[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            int64_t x = cb + u * 32 + lane;
            low[u] = x < te;
            w[u] = low[u] ? (uint32_t)__ldg(A.ci + x) : 0u;
        }
        const uint32_t c = warp_mex(A.bits, tb + tv, te - tb + 1);
        if (tj == 0 && lane == 0) {
            A.color[tv] = c;
            ncol++;
        }
        int64_t wb[U], we[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            low[u] = low[u] && in_set(A.inS, w[u]) && vkey(A.k, w[u]) < tk;
            if (low[u]) {
                wb[u] = A.rp[w[u]];
                we[u] = A.rp[w[u] + 1];
            }
        }
#pragma unroll
        for (int u = 0; u < U; u++)
            if (low[u]) set_forbidden(A.bits, wb[u] + w[u], we[u] - wb[u] + 1, c);
        __threadfence();
#pragma unroll
        for (int u = 0; u < U; u++)
            if (low[u] && atomicSub(A.cnt + w[u], 1u) == 1u) ja_ready(A, st, (int32_t)w[u], wb[u], we[u]);
    }
}

// target = #S vertices with phase arcs (the others were coloured by the init pass)
__global__ void k_jp_count_targets(const int64_t *__restrict__ rp, const int32_t *list, const uint32_t *list_cnt,
                                   int64_t implicit_n, uint32_t *target) {
    const uint32_t cnt = list ? *list_cnt : (uint32_t)implicit_n;
    uint32_t local = 0;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += gridDim.x * blockDim.x) {
        int64_t v = list ? list[i] : (int64_t)i;
        local += rp[v + 1] > rp[v] ? 1u : 0u;
    }
    for (int d = 16; d; d >>= 1) local += __shfl_xor_sync(FULL, local, d);
    if (lane_id() == 0 && local) atomicAdd(target, local);
}

static int jp_run_async(const FlowArgs &f, ColorWs &w, uint32_t *color, const int64_t *rp, const int32_t *ci,
                        const uint8_t *inS, const int32_t *list0, const uint32_t *cnt0, int64_t implicit_n,
                        int phase) {
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
    const Key k = stream_key(f.p.seed, TAG_VERTEX, 0);
    JpTask *q = reinterpret_cast<JpTask *>(w.task);
    const int64_t qcap = 2 * w.queue_cap;
    // counters: ring[0] = tail (init writes the first ready tasks there), ring[1] =
    // head, ring[2] = done, flag = error, q_head = target
    SYM_CUDA(cudaMemsetAsync(ctl->ring, 0, sizeof(ctl->ring) + sizeof(ctl->huge), s));
    SYM_CUDA(cudaMemsetAsync(&ctl->flag, 0, sizeof(uint32_t), s));
    SYM_CUDA(cudaMemsetAsync(&ctl->q_head, 0, sizeof(uint32_t), s));
    SYM_CUDA(cudaMemsetAsync(w.bits, 0, sizeof(uint32_t) * (size_t)w.bits_words, s));
    SYM_CUDA(cudaMemsetAsync(q, 0xff, sizeof(JpTask) * (size_t)qcap, s));
    prof_begin("jp_init", s);
    JpArgs A;
    A.rp = rp;
    A.ci = ci;
    A.inS = inS;
    A.color = color;
    A.cnt = w.cnt;
    A.bits = w.bits;
    A.k = k;
    A.huge = w.queue;
    A.hist = nullptr;
    A.in_list = list0;
    A.in_cnt = cnt0;
    A.implicit_n = implicit_n;
    A.tin = nullptr;
    A.tout = q;
    A.out_cnt = &ctl->ring[0];
    A.clear_cnt = &ctl->ring[3];
    A.huge_cnt = &ctl->huge[1];
    A.huge_clear = &ctl->huge[0];
    A.round = 0;
    k_jp_init<<<num_sms() * (2048 / JP_THREADS), JP_THREADS, 0, s>>>(A);
    SYM_LAUNCH_CHECK();
    k_jp_init_huge<<<num_sms() * 2, JP_HUGE_THREADS, 0, s>>>(A);
    SYM_LAUNCH_CHECK();
    k_jp_count_targets<<<num_sms() * 4, 256, 0, s>>>(rp, list0, cnt0, implicit_n, &ctl->q_head);
    prof_end(s, -1);
    SYM_LAUNCH_CHECK();
    JaArgs J;
    J.rp = rp;
    J.ci = ci;
    J.inS = inS;
    J.color = color;
    J.cnt = w.cnt;
    J.bits = w.bits;
    J.q = q;
    J.qcap = qcap;
    J.tail = &ctl->ring[0];
    J.head = &ctl->ring[1];
    J.done = &ctl->ring[2];
    J.err = &ctl->flag;
    J.target = &ctl->q_head;
    J.k = k;
    int per_sm = 0;
    SYM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_jp_async, JP_THREADS, 0));
    if (per_sm < 1) per_sm = 1;
    // algorithmic bytes of the asynchronous pass: every arc of the phase
    // CSR read once (4 B) + per vertex the row bounds of the task (8 B) and the
    // colour write (4 B); counter/bitmap atomics are L2 traffic
    const int64_t phase_nnz = rp == f.g.rp ? f.g.nnz : (rp == f.split.rp_in ? f.split.nnz_in : -1);
    const double jp_bytes = phase_nnz >= 0 ? 4.0 * (double)phase_nnz + 12.0 * (double)f.g.n : -1.0;
    prof_begin("jp_async", s);
    k_jp_async<<<num_sms() * per_sm, JP_THREADS, 0, s>>>(J);
    prof_end(s, jp_bytes);
    SYM_LAUNCH_CHECK();
    uint32_t err = 0;
    SYM_TRY(read_u32(&ctl->flag, &err, s));
    if (err) {
        set_error("asynchronous JP stalled (device timeout)");
        return SYM_ECUDA;
    }
    if (f.stats) f.stats->rounds[phase] = 0;
    return SYM_OK;
}

static int jp_run(const FlowArgs &f, ColorWs &w, uint32_t *color, const int64_t *rp, const int32_t *ci,
                  const uint8_t *inS, const int32_t *list0, const uint32_t *cnt0, int64_t implicit_n, int phase) {
    if (!getenv("SYM_JP_ROUNDS")) return jp_run_async(f, w, color, rp, ci, inS, list0, cnt0, implicit_n, phase);
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
    const Key k = stream_key(f.p.seed, TAG_VERTEX, 0);
    JpTask *tq[2] = {reinterpret_cast<JpTask *>(w.task), reinterpret_cast<JpTask *>(w.task) + w.queue_cap};
    SYM_CUDA(cudaMemsetAsync(ctl->ring, 0, sizeof(ctl->ring) + sizeof(ctl->huge), s));
    SYM_CUDA(cudaMemsetAsync(w.bits, 0, sizeof(uint32_t) * (size_t)w.bits_words, s));
    JpArgs A;
    A.rp = rp;
    A.ci = ci;
    A.inS = inS;
    A.color = color;
    A.cnt = w.cnt;
    A.bits = w.bits;
    A.k = k;
    A.huge = w.queue;
    A.hist = ctl->hist + phase * 2048;
    A.in_list = list0;
    A.in_cnt = cnt0;
    A.implicit_n = implicit_n;
    A.tin = nullptr;
    A.tout = tq[0];
    A.out_cnt = &ctl->ring[0];
    A.clear_cnt = &ctl->ring[2];
    A.huge_cnt = &ctl->huge[1];
    A.huge_clear = &ctl->huge[0];
    A.round = 0;
    prof_begin("jp_init", s);
    k_jp_init<<<num_sms() * (2048 / JP_THREADS), JP_THREADS, 0, s>>>(A);
    SYM_LAUNCH_CHECK();
    k_jp_init_huge<<<num_sms() * 2, JP_HUGE_THREADS, 0, s>>>(A);
    prof_end(s, -1);
    SYM_LAUNCH_CHECK();
    const uint32_t maxr = f.p.max_rounds ? f.p.max_rounds : 0xffffffffu;
    const int grid = num_sms() * 2;  // frontiers are small: a short grid launches and drains fast
    int r = 0, batch = 8;
    for (;;) {
        for (int bb = 0; bb < batch; bb++, r++) {
            A.tin = tq[r & 1];
            A.in_cnt = &ctl->ring[r % 3];
            A.tout = tq[(r + 1) & 1];
            A.out_cnt = &ctl->ring[(r + 1) % 3];
            A.clear_cnt = &ctl->ring[(r + 2) % 3];
            A.round = r < 2048 ? r : 2047;
            prof_begin("jp_push", s);
            k_jp_push<<<grid, JP_THREADS, 0, s>>>(A);
            prof_end(s, -1);
            SYM_LAUNCH_CHECK();
        }
        uint32_t left = 0;
        SYM_TRY(read_u32(&ctl->ring[r % 3], &left, s));
        if (left == 0) break;
        if ((uint32_t)r >= maxr) {
            set_error("JP did not converge within max_rounds");
            return SYM_EROUNDS;
        }
        if (batch < 256) batch *= 2;
    }
    if (f.stats) f.stats->rounds[phase] = (uint32_t)r;
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
