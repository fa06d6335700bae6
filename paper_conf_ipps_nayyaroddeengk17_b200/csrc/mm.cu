// mm.cu -- handshake (LMAX) matching rounds and the MM flows.
//
// Round r, for every vertex u of the frontier (Birn et al. [5]):
//   resolve: if u picked p in round r-1 and p picked u, the edge is matched
//            (both endpoints write their own mate; "mutual picks are matched");
//   pick:    otherwise u picks the heaviest edge (pe(u,w), w) to a neighbour w that is
//            still unmatched in the phase graph; no such neighbour => u is dead.
// Picks are double-buffered (pick[r&1] written in round r, pick[(r+1)&1] read), so the
// mutual test always compares round r-1 picks.  A vertex that matches or dies writes
// -1 as its current pick, so stale picks never pair with it.  mate only moves
// -1 -> partner, so reading it in place (stale) can only add dead candidates; every
// mutual pick is then locally heaviest among truly live edges, which is the greedy
// (GM) order with the same fixed priorities ([6]).
//
// Round 0 of the first phase specialises away the mate gathers (nothing is matched
// yet): a pure streaming pass over col_idx with the edge hash computed on the fly.
// A vertex whose previous pick is still unmatched keeps it without rescanning its row
// (the live set only shrinks and the keys are fixed, so it is still the heaviest); if
// the pick is matched but the second-heaviest neighbour of the last scan (alt) is
// not, that one is now the heaviest -- again no rescan.  Liveness is one bit of the
// matched bitmap (2 MB at s24, L2-resident), gathered in predicated batches.
// Rows: one lane up to MM_SMALL arcs (batches of 8), a warp up to MM_BUDGET, a CTA
// beyond (k_mm_huge).
#include "internal.h"

namespace sym {

#ifndef SYM_MM_SMALL
#define SYM_MM_SMALL 32  // one lane per row up to 32 arcs (batches of 8): MM-Rand4 4.32 -> 3.99 ms with 5 CTAs/SM
#endif
constexpr int MM_SMALL = SYM_MM_SMALL;  // rows up to MM_SMALL arcs are scanned by one lane
#ifndef SYM_MM_WSTEP
#define SYM_MM_WSTEP 4
#endif
#ifndef SYM_MM_BUDGET
#define SYM_MM_BUDGET 1024  // 4096 -> 1024: MM-Rand4 3.95 -> 3.89 ms (a 4096-arc row was 32 serial warp steps)
#endif
constexpr int MM_BUDGET = SYM_MM_BUDGET;  // rows longer than this go to the CTA kernel
constexpr int MM_THREADS = 256;
constexpr int MM_HUGE_THREADS = 512;

struct MmRoundArgs {
    const int64_t *rp, *rp2;  // dual mode: hbits[u] ? (rp2, ci2) : (rp, ci)
    const int32_t *ci, *ci2;
    const uint32_t *hbits;
    int dual;
    int32_t *mate;
    uint32_t *mbits;  // matched bitmap (1 bit per vertex, L2-resident): the liveness gathers
    const int32_t *pick_prev;
    int32_t *pick_cur;
    int32_t *alt;     // nullable: u's second-heaviest believed-live neighbour at its last scan (-1: none)
    const int32_t *in_list;
    int in_rev;
    const uint32_t *in_cnt;
    int64_t implicit_n;
    int32_t *out_list;
    uint32_t *out_cnt;
    uint32_t *clear_cnt;
    int32_t *huge;
    uint32_t *huge_cnt;
    uint32_t *huge_clear;
    uint32_t *hist;
    int round;
    Key k;
    unsigned long long *prof;  // profiling: algorithmic bytes of this launch (nullable)
    int64_t row_base;          // global id of local row 0 (sharded path; 0 otherwise)
};
// algorithmic bytes: 4 B per column word loaded; per active vertex the
// row_ptr pair (16 B) and the pick write (4 B); per resolved vertex the two pick
// reads (8 B) and, if matched, the mate write (4 B).  Neighbour liveness is one bit of
// the matched bitmap (n/8 bytes: 2 MB at R-MAT s24, L2-resident; the 4-B mate array is
// 67 MB) and counts 0 HBM bytes.

__device__ __forceinline__ bool mm_matched(const uint32_t *mbits, uint32_t v) { return (mbits[v >> 5] >> (v & 31)) & 1u; }
__device__ __forceinline__ void mm_set_matched(uint32_t *mbits, uint32_t v) { atomicOr(mbits + (v >> 5), 1u << (v & 31)); }

// top-2 of keys offset by one (0 = none; a key's low word is an id < 2^31, so +1 never
// carries): merge (a1 > a2) with (b1 > b2)
__device__ __forceinline__ void top2_merge(uint64_t &a1, uint64_t &a2, uint64_t b1, uint64_t b2) {
    const uint64_t lo = a1 < b1 ? a1 : b1, hi2 = a1 > b1 ? a2 : b2;
    a1 = a1 > b1 ? a1 : b1;
    a2 = lo > hi2 ? lo : hi2;
}
__device__ __forceinline__ void top2_add(uint64_t &a1, uint64_t &a2, uint64_t k) {
    if (k > a1) {
        a2 = a1;
        a1 = k;
    } else if (k > a2) {
        a2 = k;
    }
}

__device__ __forceinline__ void mm_row(const MmRoundArgs &A, int32_t u, int64_t &b, int64_t &e, const int32_t *&ci) {
    if (A.dual && ((A.hbits[u >> 5] >> (u & 31)) & 1u)) {
        b = A.rp2[u - A.row_base];
        e = A.rp2[u - A.row_base + 1];
        ci = A.ci2;
    } else {
        b = A.rp[u - A.row_base];
        e = A.rp[u - A.row_base + 1];
        ci = A.ci;
    }
}

#ifndef SYM_MM_ALT
#define SYM_MM_ALT 1
#endif
// 5 CTAs/SM (48 regs, no spills; 6 CTAs at 40 regs spilled once the lane path took rows of
// up to 32 arcs and the liveness gathers became one predicated batch)
#ifndef SYM_MM_MINB
#define SYM_MM_MINB 5
#endif
#if SYM_MM_MINB > 0
#define MM_ROUND_BOUNDS __launch_bounds__(MM_THREADS, SYM_MM_MINB)
#else
#define MM_ROUND_BOUNDS __launch_bounds__(MM_THREADS)
#endif
template <bool RESOLVE, bool MATE>
__global__ void MM_ROUND_BOUNDS k_mm_round(MmRoundArgs A) {
    const uint32_t cnt = A.in_list ? *A.in_cnt : (uint32_t)A.implicit_n;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        *A.clear_cnt = 0;
        *A.huge_clear = 0;
        if (A.hist && A.round < 2048) A.hist[A.round] = cnt;
    }
    const int lane = lane_id();
    const int64_t warp_g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = warp_g * 32; base < cnt; base += nwarps * 32) {
        int64_t i = base + lane;
        int32_t u = -1;
        if (i < cnt) u = A.in_list ? (A.in_rev ? A.in_list[-1 - i] : A.in_list[i]) : (int32_t)i;
        bool active = u >= 0;
        const bool listed = active;
        unsigned long long nb = 0, colb = 0;  // implementation bytes beyond the column words; column words
        int32_t p = -1;
        bool reuse = false;
        if (RESOLVE && active) {
            p = A.pick_prev[u];
            nb += 8;
            if (p >= 0 && A.pick_prev[p] == u) {
                A.mate[u] = p;
                mm_set_matched(A.mbits, (uint32_t)u);
                A.pick_cur[u] = -1;
                active = false;
                nb += 4;
            } else if (mm_matched(A.mbits, (uint32_t)u)) {  // defensive: never re-pick a matched vertex
                // (the matched bitmap, 2 MB and L2-resident, not the 67 MB mate array)
                A.pick_cur[u] = -1;
                active = false;
            } else if (MATE && p >= 0 && !mm_matched(A.mbits, (uint32_t)p)) {
                // u's pick is still unmatched: the live set only shrinks and the keys are
                // fixed, so it is still u's heaviest live edge -- no rescan.  A stale read
                // (p matched in this very round) keeps a dead pick one more round, as a
                // stale mate read in a rescan would; more rounds (32 vs 24 at R-MAT s24
                // MM-Rand4) but far fewer row scans: 5.52 -> 4.93 ms (checking whether p
                // is matching right now: 25 rounds, 5.10 ms)
                reuse = true;
                nb += 4;
            } else if (MATE && p >= 0 && A.alt) {
                // p is matched: u's second-heaviest neighbour at its last scan, if still
                // unmatched, is now its heaviest live one (every other heavier neighbour
                // was already matched then) -- no rescan
                const int32_t q = A.alt[u];
                nb += 4;
                if (q >= 0 && !mm_matched(A.mbits, (uint32_t)q)) {
                    reuse = true;
                    p = q;
                    A.alt[u] = -1;
                    nb += 8;
                }
            }
        }
        const bool scan = active && !reuse;
        int64_t b = 0, e = 0;
        const int32_t *ci = A.ci;
        if (scan) mm_row(A, u, b, e, ci);
        const int64_t d = e - b;
        nb += scan ? 20 : 0;
        uint64_t best = 0, sec = 0;  // sec: second-heaviest key + 1 (0 = none)
        bool has = false;
        if (scan && d <= MM_SMALL) {
            // short row by one lane, in batches of 8: all column loads (streamed,
            // evict-first so the gathered bitmap stays in L2), then all liveness gathers,
            // then the top-2
            colb += 4 * (unsigned long long)d;
            uint64_t b1 = 0;
            for (int64_t xq = b; xq < e; xq += 8) {
                uint32_t w[8], mw[8];  // columns, their matched-bitmap words
                bool live[8];
#pragma unroll
                for (int q = 0; q < 8; q++) w[q] = (xq + q < e) ? (uint32_t)__ldcs(ci + xq + q) : 0u;
#pragma unroll
                for (int q = 0; q < 8; q++) mw[q] = MATE ? ld_cg_pred(A.mbits + (w[q] >> 5), xq + q < e) : 0u;
#pragma unroll
                for (int q = 0; q < 8; q++) live[q] = (xq + q < e) && !((mw[q] >> (w[q] & 31)) & 1u);
#pragma unroll
                for (int q = 0; q < 8; q++)
                    if (live[q]) top2_add(b1, sec, ekey(A.k, (uint32_t)u, w[q]) + 1);
            }
            has = b1 != 0;
            best = b1 - 1;
        }
        // warp-cooperative argmax for medium rows
        unsigned medm = __ballot_sync(FULL, scan && d > MM_SMALL && d <= MM_BUDGET);
        while (medm) {
            const int src = __ffs(medm) - 1;
            medm &= medm - 1;
            const int64_t wb = __shfl_sync(FULL, b, src), we = __shfl_sync(FULL, e, src);
            const int32_t wu = __shfl_sync(FULL, u, src);
            const int32_t *wci = (const int32_t *)__shfl_sync(FULL, (unsigned long long)ci, src);
            uint64_t lb = 0, l2 = 0;  // top-2 keys + 1 (0 = none)
            constexpr int WS = SYM_MM_WSTEP;  // arcs per lane per warp step, all loads in flight
            for (int64_t x = wb; x < we; x += 32 * WS) {
                uint32_t w[WS];
                bool ok[WS];
#pragma unroll
                for (int q = 0; q < WS; q++) {
                    int64_t y = x + q * 32 + lane;
                    ok[q] = y < we;
                    w[q] = ok[q] ? (uint32_t)__ldcs(wci + y) : 0u;
                    colb += ok[q] ? 4 : 0;
                }
                uint32_t mw[WS];  // the liveness gathers in flight together (predicated loads)
#pragma unroll
                for (int q = 0; q < WS; q++) mw[q] = MATE ? ld_cg_pred(A.mbits + (w[q] >> 5), ok[q]) : 0u;
#pragma unroll
                for (int q = 0; q < WS; q++)
                    if (ok[q] && !((mw[q] >> (w[q] & 31)) & 1u)) top2_add(lb, l2, ekey(A.k, (uint32_t)wu, w[q]) + 1);
            }
#pragma unroll
            for (int dd = 16; dd; dd >>= 1) {
                const uint64_t o1 = __shfl_xor_sync(FULL, lb, dd), o2 = __shfl_xor_sync(FULL, l2, dd);
                top2_merge(lb, l2, o1, o2);
            }
            if (lane == src) {
                best = lb - 1;
                has = lb != 0;
                sec = l2;
            }
        }
        if (reuse) has = true;
        bool defer = scan && d > MM_BUDGET;
        if (active && !defer) A.pick_cur[u] = reuse ? p : (has ? (int32_t)(uint32_t)best : -1);
        if (A.alt && scan && !defer) A.alt[u] = sec ? (int32_t)(uint32_t)(sec - 1) : -1;
        int64_t slot = warp_append(active && !defer && has, A.out_cnt);
        if (slot >= 0) A.out_list[slot] = u;
        int64_t hs = warp_append(defer, A.huge_cnt);
        if (hs >= 0) A.huge[hs] = u;
        // §8(d): 4 B per scanned arc + 9 B per active vertex (row_ptr pair, pick)
        prof_add(A.prof, colb + (listed ? 9 : 0), colb + nb);
    }
}

// rows longer than MM_BUDGET: one CTA per vertex, block top-2 (argmax + the alternate)
template <bool MATE>
__global__ void __launch_bounds__(MM_HUGE_THREADS) k_mm_huge(MmRoundArgs A) {
    const uint32_t cnt = *A.huge_cnt;
    __shared__ unsigned long long s_b1[MM_HUGE_THREADS / 32], s_b2[MM_HUGE_THREADS / 32];
    const int lane = lane_id(), warp = threadIdx.x >> 5;
    for (uint32_t h = blockIdx.x; h < cnt; h += gridDim.x) {
        const int32_t u = A.huge[h];
        int64_t b, e;
        const int32_t *ci;
        mm_row(A, u, b, e, ci);
        uint64_t l1 = 0, l2 = 0;  // top-2 keys + 1 (0 = none)
        unsigned long long nb = 0;
        for (int64_t x = b; x < e; x += 4 * MM_HUGE_THREADS) {
            uint32_t w[4];
            bool ok[4];
#pragma unroll
            for (int q = 0; q < 4; q++) {
                int64_t y = x + q * MM_HUGE_THREADS + threadIdx.x;
                ok[q] = y < e;
                w[q] = ok[q] ? (uint32_t)__ldcs(ci + y) : 0u;
                nb += ok[q] ? 4 : 0;
            }
            uint32_t mw[4];
#pragma unroll
            for (int q = 0; q < 4; q++) mw[q] = MATE ? ld_cg_pred(A.mbits + (w[q] >> 5), ok[q]) : 0u;
#pragma unroll
            for (int q = 0; q < 4; q++)
                if (ok[q] && !((mw[q] >> (w[q] & 31)) & 1u)) top2_add(l1, l2, ekey(A.k, (uint32_t)u, w[q]) + 1);
        }
#pragma unroll
        for (int dd = 16; dd; dd >>= 1) {
            const uint64_t o1 = __shfl_xor_sync(FULL, l1, dd), o2 = __shfl_xor_sync(FULL, l2, dd);
            top2_merge(l1, l2, o1, o2);
        }
        prof_add(A.prof, nb, nb);
        if (lane == 0) {
            s_b1[warp] = l1;
            s_b2[warp] = l2;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            uint64_t b1 = 0, b2 = 0;
            for (int q = 0; q < MM_HUGE_THREADS / 32; q++) top2_merge(b1, b2, s_b1[q], s_b2[q]);
            A.pick_cur[u] = b1 ? (int32_t)(uint32_t)(b1 - 1) : -1;
            if (A.alt) A.alt[u] = b2 ? (int32_t)(uint32_t)(b2 - 1) : -1;
            if (b1) {
                uint32_t slot = atomicAdd(A.out_cnt, 1u);
                A.out_list[slot] = u;
            }
        }
        __syncthreads();
    }
}

// phase-2 frontier: unmatched vertices that have phase-2 arcs (CTA-aggregated appends:
// per-warp appends serialised at the counter, 0.38 ms at R-MAT s24)
__global__ void k_mm_phase2_list(const int64_t *__restrict__ rp, const int64_t *__restrict__ rp2,
                                 const uint32_t *__restrict__ hbits, int dual, int64_t n, const int32_t *mate,
                                 int32_t *list, uint32_t *cnt) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n; base += stride) {
        int64_t v = base + threadIdx.x;
        bool take = false;
        if (v < n && mate[v] < 0) {
            bool useX = dual ? ((hbits[v >> 5] >> (v & 31)) & 1u) : true;
            const int64_t *r = useX ? rp2 : rp;
            take = r[v + 1] > r[v];
        }
        cta_append2(take, false, (int32_t)v, n, list, cnt, cnt);  // one atomic per CTA (order immaterial)
    }
}

__global__ void k_mm_count(const int32_t *mate, int64_t n, unsigned long long *count) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    uint32_t local = 0;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) local += mate[v] > v;
    for (int d = 16; d; d >>= 1) local += __shfl_xor_sync(FULL, local, d);
    if (lane_id() == 0 && local) atomicAdd(count, (unsigned long long)local);
}

// ------------------------------------------------------------------ host side
void carve_mm_ws(Arena &a, int64_t n, int64_t nnz, MmWs &w) {
    w.pick[0] = a.take<int32_t>((size_t)n + 1);
    w.pick[1] = a.take<int32_t>((size_t)n + 1);
    w.vlist = a.take<int32_t>((size_t)n + 1);
    w.fr[0] = a.take<int32_t>((size_t)n + 1);
    w.fr[1] = a.take<int32_t>((size_t)n + 1);
    w.huge_cap = nnz / MM_BUDGET + 2;
    w.huge = reinterpret_cast<int64_t *>(a.take<int32_t>((size_t)w.huge_cap));
    w.gmax = a.take<unsigned long long>((size_t)n + 1);
    w.mbits = a.take<uint32_t>((size_t)(n + 31) / 32 + 1);
    w.alt = a.take<int32_t>((size_t)n + 1);
}

struct MmPhase {
    const int64_t *rp, *rp2;
    const int32_t *ci, *ci2;
    int dual;
    const int32_t *list0;
    int rev0;
    const uint32_t *cnt0;
    int64_t implicit_n;
    bool first;  // no vertex matched yet: round 0 skips the mate gathers
    int64_t nnz = -1;  // arcs of the phase CSR when known on the host (profiling only)
};

// One resident wave of the grid-stride round kernel (see mis.cu round_grid).
static int mm_round_grid() {
#if SYM_ROUND_ONE_WAVE
    static std::atomic<int> slots[SYM_MAX_DEVICES];
    return dev_cached(slots, [] {
        int per = 2048 / MM_THREADS, x = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&x, k_mm_round<false, false>, MM_THREADS, 0) == cudaSuccess && x > 0)
            per = std::min(per, x);
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&x, k_mm_round<false, true>, MM_THREADS, 0) == cudaSuccess && x > 0)
            per = std::min(per, x);
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&x, k_mm_round<true, true>, MM_THREADS, 0) == cudaSuccess && x > 0)
            per = std::min(per, x);
        return num_sms() * per;
    });
#else
    return num_sms() * (2048 / MM_THREADS);
#endif
}

static int mm_phase(const FlowArgs &f, MmWs &w, int32_t *mate, const MmPhase &ph, int phase) {
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
    SYM_CUDA(cudaMemsetAsync(ctl->ring, 0, sizeof(ctl->ring) + sizeof(ctl->huge), s));
    const Key k = stream_key(f.p.seed, TAG_EDGE, 0);
    const uint32_t maxr = f.p.max_rounds ? f.p.max_rounds : 0xffffffffu;
    const int full_grid = mm_round_grid();
    int grid = full_grid;
    int r = 0;
    // no alternates yet (the streaming round 0 finds the heaviest arc only: tracking a
    // second there cost more than it saved -- 1.7 -> 2.9 ms round 0 at R-MAT s24 MM-NONE)
    SYM_CUDA(cudaMemsetAsync(w.alt, 0xff, sizeof(int32_t) * (size_t)(f.g.n + 1), s));
    const int batch = SYM_POLL_BATCH;  // rounds launched per host poll of the frontier count
    if (ph.first && !ph.dual) {
        // round 0 as one streaming pass: every phase vertex picks its heaviest arc;
        // the vertices with a pick form round 1's frontier (fr[1], ring[1])
        int64_t nnz = 0;
        SYM_TRY(phase_arcs(f, ph.rp, &nnz));
        if (nnz > 0) {
            SYM_TRY(run_round0(1, Graph{f.g.n, nnz, ph.rp, ph.ci}, f.first_row, (nnz + SPLIT_TILE - 1) / SPLIT_TILE, k,
                               w.gmax, nullptr, w.pick[0], ph.list0 ? f.hbits : nullptr, w.fr[1], &ctl->ring[1], s));
            r = 1;
        }
    }
    for (;;) {
        for (int bb = 0; bb < batch && (uint32_t)r < maxr; bb++, r++) {  // never past the cap
            MmRoundArgs A{};
            A.rp = ph.rp;
            A.rp2 = ph.rp2;
            A.ci = ph.ci;
            A.ci2 = ph.ci2;
            A.hbits = f.hbits;
            A.dual = ph.dual;
            A.mate = mate;
            A.mbits = w.mbits;
            A.pick_prev = w.pick[(r + 1) & 1];
            A.pick_cur = w.pick[r & 1];
            A.alt = SYM_MM_ALT ? w.alt : nullptr;
            if (r == 0) {
                A.in_list = ph.list0;
                A.in_rev = ph.rev0;
                A.in_cnt = ph.cnt0;
            } else {
                A.in_list = w.fr[r & 1];
                A.in_rev = 0;
                A.in_cnt = &ctl->ring[r % 3];
            }
            A.implicit_n = ph.implicit_n;
            A.out_list = w.fr[(r + 1) & 1];
            A.out_cnt = &ctl->ring[(r + 1) % 3];
            A.clear_cnt = &ctl->ring[(r + 2) % 3];
            A.huge = reinterpret_cast<int32_t *>(w.huge);
            A.huge_cnt = &ctl->huge[r & 1];
            A.huge_clear = &ctl->huge[(r + 1) & 1];
            A.hist = ctl->hist + phase * 2048;
            A.round = r < 2048 ? r : 2047;
            A.k = k;
            A.row_base = 0;
            // round 0 of a phase has nothing to resolve (its pick buffers hold stale or
            // uninitialised values); round 0 of the first phase has nothing matched yet
            // profiling byte counters are accumulated by the kernels
            if (r == 0 && ph.first) {
                A.prof = prof_counter(s);
                prof_begin("mm_round0", s);
                k_mm_round<false, false><<<grid, MM_THREADS, 0, s>>>(A);
                prof_end_dev(s, A.prof);
                SYM_LAUNCH_CHECK();
                A.prof = prof_counter(s);
                prof_begin("mm_huge", s);
                k_mm_huge<false><<<num_sms() * 2, MM_HUGE_THREADS, 0, s>>>(A);
                prof_end_dev(s, A.prof);
            } else if (r == 0) {
                A.prof = prof_counter(s);
                prof_begin("mm_round", s);
                k_mm_round<false, true><<<grid, MM_THREADS, 0, s>>>(A);
                prof_end_dev(s, A.prof);
                SYM_LAUNCH_CHECK();
                A.prof = prof_counter(s);
                prof_begin("mm_huge", s);
                k_mm_huge<true><<<num_sms() * 2, MM_HUGE_THREADS, 0, s>>>(A);
                prof_end_dev(s, A.prof);
            } else {
                A.prof = prof_counter(s);
                prof_begin("mm_round", s);
                k_mm_round<true, true><<<grid, MM_THREADS, 0, s>>>(A);
                prof_end_dev(s, A.prof);
                SYM_LAUNCH_CHECK();
                A.prof = prof_counter(s);
                prof_begin("mm_huge", s);
                k_mm_huge<true><<<num_sms() * 2, MM_HUGE_THREADS, 0, s>>>(A);
                prof_end_dev(s, A.prof);
            }
            SYM_LAUNCH_CHECK();
        }
        uint32_t left = 0;
        SYM_TRY(read_u32(&ctl->ring[r % 3], &left, s));
        if (left == 0) break;
        if ((uint32_t)r >= maxr) {
            set_error("MM phase did not converge within max_rounds");
            return SYM_EROUNDS;
        }
        // frontiers only shrink: size the next launches for `left` vertices
        const int64_t need = ((int64_t)left + MM_THREADS - 1) / MM_THREADS;
        grid = (int)(need < full_grid ? (need > 0 ? need : 1) : full_grid);
    }
    if (f.stats) f.stats->rounds[phase] = (uint32_t)r;
    return SYM_OK;
}

int run_mm(const FlowArgs &f, MmWs &w, int32_t *mate) {
    const Graph &g = f.g;
    cudaStream_t s = f.stream;
    Ctl *ctl = f.ctl;
    SYM_CUDA(cudaMemsetAsync(mate, 0xff, sizeof(int32_t) * (size_t)g.n, s));
    SYM_CUDA(cudaMemsetAsync(w.mbits, 0, sizeof(uint32_t) * ((size_t)(g.n + 31) / 32 + 1), s));
    const int kind = f.p.kind;
    MmPhase ph{};
    if (kind == SYM_DECOMP_NONE) {
        ph = MmPhase{g.rp, nullptr, g.ci, nullptr, 0, nullptr, 0, nullptr, g.n, true};
        ph.nnz = g.nnz;
        SYM_TRY(mm_phase(f, w, mate, ph, 0));
    } else {
        // phase 1: M_IS = MM(union G_i) (RAND, Alg 5 l.5; BRIDGE, Alg 4: the 2-edge-connected
        // components) / M_H = MM(G_H) (DEGk, Alg 6 l.5)
        if (kind == SYM_DECOMP_RAND || kind == SYM_DECOMP_BRIDGE) {
            ph = MmPhase{f.split.rp_in, nullptr, f.split.ci_in, nullptr, 0, nullptr, 0, nullptr, g.n, true};
            ph.nnz = f.split.nnz_in;
        } else {
            SYM_CUDA(cudaMemsetAsync(&ctl->cnt_front, 0, 2 * sizeof(uint32_t), s));
            SYM_TRY(launch_classify_degk(g, f.p.param, f.hbits, w.vlist, ctl, s));
            ph = MmPhase{f.split.rp_in, nullptr, f.split.ci_in, nullptr, 0, w.vlist + g.n, 1, &ctl->cnt_back, 0,
                         true};
        }
        SYM_TRY(mm_phase(f, w, mate, ph, 0));
        // phase 2: V' = unmatched; MM(G_{k+1}[V']) (Alg 5 l.6-7) / MM(G_LC[V']) (Alg 6 l.6-7)
        const int dual = kind == SYM_DECOMP_DEGK;
        SYM_CUDA(cudaMemsetAsync(&ctl->cnt_front, 0, sizeof(uint32_t), s));
        k_mm_phase2_list<<<num_sms() * 8, 256, 0, s>>>(g.rp, f.split.rp_x, f.hbits, dual, g.n, mate, w.vlist,
                                                         &ctl->cnt_front);
        SYM_LAUNCH_CHECK();
        if (dual) ph = MmPhase{g.rp, f.split.rp_x, g.ci, f.split.ci_x, 1, w.vlist, 0, &ctl->cnt_front, 0, false};
        else ph = MmPhase{f.split.rp_x, nullptr, f.split.ci_x, nullptr, 0, w.vlist, 0, &ctl->cnt_front, 0, false};
        SYM_TRY(mm_phase(f, w, mate, ph, 1));
    }
    if (f.stats) {
        uint32_t hist[4096];
        SYM_CUDA(cudaMemcpyAsync(hist, ctl->hist, sizeof(hist), cudaMemcpyDeviceToHost, s));
        SYM_CUDA(cudaStreamSynchronize(s));
        for (int ph2 = 0; ph2 < 2; ph2++) {
            uint32_t rr = 0;
            for (int i = 0; i < 2048 && i < (int)f.stats->rounds[ph2]; i++) rr += hist[ph2 * 2048 + i] ? 1 : 0;
            f.stats->rounds[ph2] = rr;
            f.stats->phase_vertices[ph2] = hist[ph2 * 2048];
        }
        if (f.p.flags & SYM_F_STATS) {
            SYM_CUDA(cudaMemsetAsync(&ctl->result, 0, sizeof(uint64_t), s));
            k_mm_count<<<num_sms() * 8, 256, 0, s>>>(mate, g.n, (unsigned long long *)&ctl->result);
            SYM_LAUNCH_CHECK();
            uint64_t c = 0;
            SYM_TRY(read_u64(&ctl->result, &c, s));
            f.stats->result_size = (int64_t)c;
        }
    }
    return SYM_OK;
}

// ------------------------------------------------------------------ sharded MM (C-ABI below)
// owned vertices [v0, v1) with mate[v] < 0 and at least one arc in the local phase CSR
__global__ void k_shard_mm_frontier(const int64_t *__restrict__ rp, int64_t v0, int64_t v1, const int32_t *mate,
                                    int32_t *list, uint32_t *cnt) {
    const int64_t n = v1 - v0, stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n; base += stride) {
        const int64_t i = base + threadIdx.x;
        const bool take = i < n && mate[v0 + i] < 0 && rp[i + 1] > rp[i];
        const int64_t s = warp_append(take, cnt);
        if (s >= 0) list[s] = (int32_t)(v0 + i);
    }
}

// ---- deltas of the sharded flow (shard.cu): every pick / match an owned boundary
// vertex wrote in this round, {id | matched << 31, pick} (8 B)
__global__ void k_sh_delta_mm(const int32_t *__restrict__ list, const uint32_t *cnt, const int32_t *mate,
                              const int32_t *pick_cur, const uint32_t *__restrict__ bnd, int64_t v0, uint2 *send,
                              uint32_t *dcnt) {
    const int64_t c = *cnt, stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < c; base += stride) {
        const int64_t i = base + threadIdx.x;
        const int32_t u = i < c ? list[i] : -1;
        const bool b = u >= 0 && ((bnd[(u - v0) >> 5] >> ((u - v0) & 31)) & 1u);
        const int64_t slot = warp_append(b, dcnt);
        if (slot >= 0) send[slot] = make_uint2((uint32_t)u | (mate[u] >= 0 ? 0x80000000u : 0u), (uint32_t)pick_cur[u]);
    }
}

// the owned mates (global ids) -> the caller's output
__global__ void k_sh_mm_out(const int32_t *mate, int64_t v0, int64_t v1, int32_t *out) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = v0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < v1; v += stride) out[v - v0] = mate[v];
}

}  // namespace sym

using namespace sym;

// ------------------------------------------------------------------ sharded MM (C-ABI)
struct MmShardWs {
    int32_t *mate = nullptr, *pick[2] = {nullptr, nullptr}, *huge = nullptr;
    uint32_t *mbits = nullptr;
    SplitWs sw;
    int64_t *rp_in = nullptr, *rp_x = nullptr;
    int32_t *ci_in = nullptr, *ci_x = nullptr;
};

static void carve_mm_sharded(Arena &a, const ShardPlan &P, const sym_params *p, ShardCtx &x, MmShardWs &w) {
    carve_shard_common(a, P, sizeof(uint2), x);
    const size_t pad = (size_t)P.N * (size_t)P.B;
    w.mate = a.take<int32_t>(pad);
    w.pick[0] = a.take<int32_t>(pad);
    w.pick[1] = a.take<int32_t>(pad);
    w.huge = a.take<int32_t>((size_t)(P.nnz / MM_BUDGET + 2));
    w.mbits = a.take<uint32_t>(pad / 32 + 1);
    if (p->kind == SYM_DECOMP_RAND) {  // the owned rows' RAND decomposition (Alg 2, local)
        carve_split_ws(a, P.nl, P.nnz, w.sw);
        w.rp_in = a.take<int64_t>((size_t)P.nl + 1);
        w.rp_x = a.take<int64_t>((size_t)P.nl + 1);
        w.ci_in = a.take<int32_t>((size_t)P.nnz + 1);
        w.ci_x = a.take<int32_t>((size_t)P.nnz + 1);
    }
}

namespace sym {
void carve_mm_sharded_dry(Arena &a, const ShardPlan &P, const sym_params *p, ShardCtx &x) {
    MmShardWs w;
    carve_mm_sharded(a, P, p, x, w);
}
}  // namespace sym

static int mm_shard_grid(int64_t items) {
    int64_t want = (items + 255) / 256, cap = (int64_t)num_sms() * 8;
    return (int)(want < 1 ? 1 : (want < cap ? want : cap));
}

// handshake rounds of one phase (phase CSR rp/ci over the owned rows, global ids)
static int mm_sharded_phase(const ShardPlan &P, ShardCtx &x, const sym_params *p, MmShardWs &w, const int64_t *rp,
                            const int32_t *ci, uint32_t *rounds) {
    cudaStream_t s = x.s;
    SYM_CUDA(cudaMemsetAsync(x.cnt_in(0), 0, sizeof(uint32_t), s));
    if (P.nl > 0) {
        k_shard_mm_frontier<<<mm_shard_grid(P.nl), 256, 0, s>>>(rp, P.v0, P.v1, w.mate, x.list_in(0), x.cnt_in(0));
        SYM_LAUNCH_CHECK();
    }
    const uint32_t maxr = p->max_rounds ? p->max_rounds : 0xffffffffu;
    const Key k = stream_key(p->seed, TAG_EDGE, 0);
    int64_t local = P.nl;
    for (int r = 0;; r++) {
        if ((uint32_t)r >= maxr) {
            set_error("sharded MM phase did not converge within max_rounds");
            return SYM_EROUNDS;
        }
        SYM_CUDA(cudaMemsetAsync(x.dcnt(r), 0, 2 * sizeof(uint32_t), s));
        SYM_CUDA(cudaMemsetAsync(x.scratch, 0, 4 * sizeof(uint32_t), s));
        if (local > 0) {
            MmRoundArgs A{};
            A.rp = rp;
            A.rp2 = nullptr;
            A.ci = ci;
            A.ci2 = nullptr;
            A.hbits = nullptr;
            A.dual = 0;
            A.mate = w.mate;
            A.mbits = w.mbits;
            A.pick_prev = w.pick[(r + 1) & 1];
            A.pick_cur = w.pick[r & 1];
            A.in_list = x.list_in(r);
            A.in_rev = 0;
            A.in_cnt = x.cnt_in(r);
            A.implicit_n = 0;
            A.out_list = x.list_out(r);
            A.out_cnt = x.cnt_out(r);
            A.clear_cnt = x.scratch + 1;
            A.huge = w.huge;
            A.huge_cnt = x.scratch;
            A.huge_clear = x.scratch + 2;
            A.hist = nullptr;
            A.round = 0;
            A.k = k;
            A.prof = nullptr;
            A.row_base = P.v0;
            const int grid = (int)std::min<int64_t>(mm_round_grid(), mm_shard_grid(local));
            if (r == 0) k_mm_round<false, true><<<grid, MM_THREADS, 0, s>>>(A);  // round 0: nothing to resolve
            else k_mm_round<true, true><<<grid, MM_THREADS, 0, s>>>(A);
            SYM_LAUNCH_CHECK();
            k_mm_huge<true><<<num_sms() * 2, MM_HUGE_THREADS, 0, s>>>(A);
            SYM_LAUNCH_CHECK();
            k_sh_delta_mm<<<mm_shard_grid(local), 256, 0, s>>>(x.list_in(r), x.cnt_in(r), w.mate, A.pick_cur, x.bnd,
                                                              P.v0, (uint2 *)x.send, x.dcnt(r));
            SYM_LAUNCH_CHECK();
        }
        uint64_t front = 0;
        SYM_TRY(shard_exchange(P, x, r & 1, SH_MM, nullptr, w.mate, w.pick[r & 1], w.mbits, &front));
        local = x.host_all[2 * P.rank + 1];
        if (front == 0) {
            *rounds = (uint32_t)(r + 1);
            return SYM_OK;
        }
    }
}

extern "C" int sym_mm_sharded(const sym_graph_shard *g, const sym_params *p, sym_comm *c, void *ws, size_t ws_bytes,
                              int32_t *mate, sym_shard_stats *stats, sym_stream_t stream) {
    ShardPlan P;
    SYM_TRY(shard_check(g, p, c, &P));
    if (p->kind == SYM_DECOMP_DEGK) {
        set_error("sharded MM supports the NONE and RAND decompositions");
        return SYM_EINVAL;
    }
    if (P.nl > 0 && !mate) { set_error("mate is NULL"); return SYM_EINVAL; }
    ShardCtx x;
    MmShardWs w;
    SYM_TRY(shard_carve_ws(ws, ws_bytes, [&](Arena &a) {
        x = ShardCtx();
        w = MmShardWs();
        carve_mm_sharded(a, P, p, x, w);
    }));
    x.c = c;
    x.s = (cudaStream_t)stream;
    cudaStream_t s = x.s;
    if (stats) memset(stats, 0, sizeof(*stats));
    const size_t pad = (size_t)P.N * (size_t)P.B;
    SYM_CUDA(cudaMemsetAsync(w.mate, 0xff, sizeof(int32_t) * pad, s));
    SYM_CUDA(cudaMemsetAsync(w.mbits, 0, sizeof(uint32_t) * (pad / 32 + 1), s));
    SYM_CUDA(cudaMemsetAsync(w.pick[0], 0xff, sizeof(int32_t) * pad, s));
    SYM_CUDA(cudaMemsetAsync(w.pick[1], 0xff, sizeof(int32_t) * pad, s));
    SYM_CUDA(cudaMemsetAsync(x.pair, 0, 8 * sizeof(uint32_t), s));
    SYM_TRY(shard_boundary(P, x, s));
    uint32_t rounds[3] = {0, 0, 0};
    if (p->kind == SYM_DECOMP_NONE) {
        SYM_TRY(mm_sharded_phase(P, x, p, w, P.rp, P.ci, &rounds[0]));  // LMAX on G
    } else {
        // labels hash the GLOBAL id (row_base), so the parts equal the single-GPU ones
        SYM_TRY(run_split(Graph{P.nl, P.nnz, P.rp, P.ci}, p->kind, p->param, p->seed, w.sw, nullptr, w.rp_in, w.ci_in,
                          w.rp_x, w.ci_x, nullptr, s, P.v0));
        SYM_TRY(mm_sharded_phase(P, x, p, w, w.rp_in, w.ci_in, &rounds[0]));  // M_IS on the parts (Alg 5 l.5)
        SYM_TRY(mm_sharded_phase(P, x, p, w, w.rp_x, w.ci_x, &rounds[1]));    // cross edges among unmatched (l.6-7)
    }
    if (P.nl > 0) {
        k_sh_mm_out<<<mm_shard_grid(P.nl), 256, 0, s>>>(w.mate, P.v0, P.v1, mate);
        SYM_LAUNCH_CHECK();
    }
    if (stats) {
        memcpy(stats->rounds, rounds, sizeof(rounds));
        shard_stats_out(x, stats);
        SYM_TRY(shard_count_boundary(P, x, &stats->boundary));
    }
    return SYM_OK;
}
