// mis.cu -- Luby local-maximum rounds and the MIS flows.
//
// Round rule (P:272-274 with fixed priorities, DESIGN §3 M1): an undecided vertex v
//   -> OUT  if some phase neighbour is IN,
//   -> IN   if no undecided phase neighbour has a larger (pv, id) key,
//   else stays undecided and is appended to the next frontier.
// Only HIGHER neighbours' statuses are gathered: a lower neighbour w turns In only when
// every higher neighbour of w -- v among them -- is Out, so none is In while v is
// undecided (this halves the status gathers).
// Status moves only UNDEC -> {IN, OUT}, and v turns IN only when every higher
// neighbour is final-OUT, so decisions may be taken in place and read by other
// threads of the same round: any interleaving yields the lexicographically-first
// MIS (Blelloch et al. [6]).  Neighbours marked INACTIVE are not
// in the current phase and are ignored.
//
// Push-Out: a vertex that turns IN marks its undecided phase neighbours OUT at once, so
// a blocked vertex only waits at its first undecided higher neighbour and resumes there
// next round (resume memo, out_pos parallel to the frontier list).
//
// Load balance for power-law rows (R-MAT: max degree ~4e5 at scale 24):
//   every row               : one lane checks the window of MIS_SMALL arcs at its resume
//                             position (all loads in flight); most rows block or decide there;
//   rows past their window  : the warp scans 4x32 arcs per step (ballot early exit)
//                             for up to MIS_BUDGET arcs;
//   rows still undecided    : deferred (v, resume offset) to k_mis_huge, where a
//                             whole CTA scans the rest with __syncthreads_or exits.
// MIS-Deg2's classification (k_mis_degk_classify) decides the V_L vertices without G_L
// arcs directly (In, and their V_H neighbours Out).
#include <algorithm>

#include "internal.h"

namespace sym {

#ifndef SYM_MIS_SMALL
#define SYM_MIS_SMALL 8
#endif
constexpr int MIS_SMALL = SYM_MIS_SMALL;  // arcs per lane window
#ifndef SYM_MIS_BUDGET
#define SYM_MIS_BUDGET 4096
#endif
constexpr int MIS_BUDGET = SYM_MIS_BUDGET;
constexpr int MIS_THREADS = 256;
constexpr int MIS_HUGE_THREADS = 512;

enum { R_NONE = 0, R_IN = 1, R_OUT = 2, R_BLK = 3, R_DEFER = 4 };

struct MisRoundArgs {
    const int64_t *rp;
    const int32_t *ci;
    uint8_t *st;
    const int32_t *in_list;  // nullptr => implicit list [0, implicit_n)
    int in_rev;              // list stored backwards: v = in_list[-1 - i]
    const int32_t *in_pos;   // nullable: resume offset (from the row start) of in_list[i]
    int32_t *out_pos;        // nullable: resume offsets of the blocked vertices, parallel to out_list
    int push_out;            // an In vertex marks its undecided neighbours Out (not in shard mode)
    const uint32_t *in_cnt;
    int64_t implicit_n;
    int32_t *out_list;
    uint32_t *out_cnt;
    uint32_t *clear_cnt;
    int64_t *huge;
    uint32_t *huge_cnt;
    uint32_t *huge_clear;
    uint32_t *hist;
    int round;
    Key k;
    unsigned long long *prof;  // profiling: algorithmic bytes of this launch (nullable)
    // sharded mode: rows are local (row of vertex v is v - row_base); neighbours whose
    // class bit in `nfilter` differs from `ncls` are not in the phase (ncls < 0: none)
    int64_t row_base;
    const uint32_t *nfilter;
    int ncls;
};

// statuses of neighbours w[u] with want[u] (ST_OUT otherwise -- no effect on the
// rule), restricted to the phase set: the filter words, then the statuses, each step's
// loads in flight together
template <int K>
__device__ __forceinline__ void mis_gather(const MisRoundArgs &A, const uint32_t (&w)[K], const bool (&want)[K],
                                           uint8_t (&s)[K]) {
    bool go[K];
    if (A.ncls >= 0) {
        uint32_t fw[K];
#pragma unroll
        for (int u = 0; u < K; u++) fw[u] = ld_nc_pred(A.nfilter + (w[u] >> 5), want[u]);
#pragma unroll
        for (int u = 0; u < K; u++) go[u] = want[u] && (int)((fw[u] >> (w[u] & 31)) & 1u) == A.ncls;
    } else {
#pragma unroll
        for (int u = 0; u < K; u++) go[u] = want[u];
    }
#pragma unroll
    for (int u = 0; u < K; u++) s[u] = ld_u8_pred(A.st + w[u], go[u], ST_OUT);
}

// bytes: §8(d) algorithmic = 4 B per column word the kernel loads + 9 B
// per active vertex (row_ptr pair + status); the implementation's own count adds the
// list entry, the resume offset and the status read (9 B more per active vertex) and 1 B
// per decided status write.  Neighbour-status gathers hit the L2-resident status
// array: 0 HBM bytes.
// Lane stage: one lane scans the window [x, x + MIS_SMALL) of its row -- all column
// loads, then all status gathers, then the rule (the order of the arcs does not matter:
// any In neighbour -> Out, else any higher undecided neighbour -> blocked at the first
// one).  Column words are streamed with evict-first loads so the gathered status stays
// in L2.  R_NONE: the window holds neither (the row continues past it, or v is In).
__device__ __forceinline__ int mis_scan_window(const MisRoundArgs &A, int64_t x, int64_t e, uint64_t kv,
                                               int64_t &pos, unsigned long long &lb, uint32_t (&w)[MIS_SMALL]) {
    uint8_t s[MIS_SMALL];
#pragma unroll
    for (int u = 0; u < MIS_SMALL; u++) w[u] = (x + u < e) ? (uint32_t)__ldcs(A.ci + x + u) : 0u;
    // only higher neighbours can decide v: a lower neighbour turns In only once every
    // higher neighbour of it -- v included -- is Out, so while v is undecided none is In
    // two batched load steps (predicated, no branch per arc): the phase-filter words of
    // the higher neighbours, then their statuses
    bool hi[MIS_SMALL];
#pragma unroll
    for (int u = 0; u < MIS_SMALL; u++) hi[u] = x + u < e && vkey(A.k, w[u]) > kv;
    mis_gather(A, w, hi, s);
    bool in = false;
    int fb = MIS_SMALL;
#pragma unroll
    for (int u = MIS_SMALL - 1; u >= 0; u--) {
        in |= s[u] == ST_IN;
        if (s[u] == ST_UNDEC) fb = u;
    }
    lb += 4 * (unsigned long long)min(e - x, (int64_t)MIS_SMALL);
    if (in) return R_OUT;
    if (fb < MIS_SMALL) {
        pos = x + fb;
        return R_BLK;
    }
    return R_NONE;
}

// push-Out of 4 arcs x, x+S, x+2S, x+3S (< e): the column loads, then the status loads,
// then the stores, each step's accesses in flight together
template <int S>
__device__ __forceinline__ void mis_push4(const MisRoundArgs &A, int64_t x, int64_t e) {
    uint32_t w[4];
    uint8_t sv[4];
#pragma unroll
    for (int u = 0; u < 4; u++) w[u] = x + u * S < e ? (uint32_t)__ldcs(A.ci + x + u * S) : 0u;
#pragma unroll
    for (int u = 0; u < 4; u++) sv[u] = ld_u8_pred(A.st + w[u], x + u * S < e, ST_OUT);
#pragma unroll
    for (int u = 0; u < 4; u++)
        if (sv[u] == ST_UNDEC) A.st[w[u]] = ST_OUT;
}

// Resume memo: a blocked vertex records where its scan stopped (the first undecided
// higher neighbour, or the start of the warp step that found one); every arc before it
// is a lower neighbour or a final-Out higher one, so the next round resumes there.
#ifndef SYM_MIS_LANE_ITERS
#define SYM_MIS_LANE_ITERS 2  // MIS-Deg2 1.13 -> 1.06 ms (MIS-NONE unchanged; 4 windows: slower)
#endif
#ifndef SYM_MIS_MINB
#define SYM_MIS_MINB 5  // 48 regs, 5 CTAs/SM: 1.46 -> 1.39 ms MIS-NONE at R-MAT s24 (62 regs unbounded)
#endif
#if SYM_MIS_MINB > 0
__global__ void __launch_bounds__(MIS_THREADS, SYM_MIS_MINB) k_mis_round(MisRoundArgs A) {
#else
__global__ void __launch_bounds__(MIS_THREADS) k_mis_round(MisRoundArgs A) {
#endif
    const uint32_t cnt = A.in_list ? *A.in_cnt : (uint32_t)A.implicit_n;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        *A.clear_cnt = 0;
        *A.huge_clear = 0;
        if (A.hist && A.round < (1 << 12)) A.hist[A.round] = cnt;
    }
    const int lane = lane_id();
    const int64_t warp_g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = warp_g * 32; base < cnt; base += nwarps * 32) {
        int64_t i = base + lane;
        int32_t v = -1;
        if (i < cnt) v = A.in_list ? (A.in_rev ? A.in_list[-1 - i] : A.in_list[i]) : (int32_t)i;
        bool active = v >= 0 && A.st[v] == ST_UNDEC;
        int64_t b = 0, e = 0, x0 = 0;
        uint64_t kv = 0;
        if (active) {
            b = A.rp[v - A.row_base];
            e = A.rp[v - A.row_base + 1];
            x0 = b + (A.in_pos ? A.in_pos[i] : 0);
            kv = vkey(A.k, (uint32_t)v);
        }
        int res = R_NONE;
        int64_t resume = 0, pos = 0;
        unsigned long long lb = 0;  // column words loaded (4 B each)
        // lane stage: the first MIS_SMALL arcs of every row (a long row of an R-MAT graph
        // is almost always decided or blocked within them)
        uint32_t wv[MIS_SMALL];
        int64_t xw = x0 + MIS_SMALL;  // where the warp stage starts
        if (active) {
            res = mis_scan_window(A, x0, e, kv, pos, lb, wv);
            // (SYM_MIS_LANE_ITERS > 1: more lane windows before the warp stage)
            for (int it = 1; it < SYM_MIS_LANE_ITERS && res == R_NONE && xw < e; it++, xw += MIS_SMALL) {
                uint32_t wt[MIS_SMALL];
                res = mis_scan_window(A, xw, e, kv, pos, lb, wt);
            }
            if (res == R_NONE && xw >= e) res = R_IN;
        }
        unsigned longm = __ballot_sync(FULL, active && res == R_NONE);
        while (longm) {
            const int src = __ffs(longm) - 1;
            longm &= longm - 1;
            const int64_t wb = __shfl_sync(FULL, xw, src), we = __shfl_sync(FULL, e, src);
            const uint64_t wk = __shfl_sync(FULL, kv, src);
            const int64_t lim = min(we, wb + MIS_BUDGET);
            int r = R_IN;
            int64_t wpos = 0;
            for (int64_t x = wb; x < lim; x += 128) {
                uint32_t w[4];
                bool ok[4];
#pragma unroll
                for (int u = 0; u < 4; u++) {
                    int64_t y = x + u * 32 + lane;
                    ok[u] = y < lim;
                    w[u] = ok[u] ? (uint32_t)__ldcs(A.ci + y) : 0u;
                    lb += ok[u] ? 4 : 0;
                }
                bool fin = false, fblk = false, hi[4];
                uint8_t sw[4];
#pragma unroll
                for (int u = 0; u < 4; u++) hi[u] = ok[u] && vkey(A.k, w[u]) > wk;  // higher neighbours only
                mis_gather(A, w, hi, sw);
#pragma unroll
                for (int u = 0; u < 4; u++) {
                    fin |= sw[u] == ST_IN;
                    fblk |= sw[u] == ST_UNDEC;
                }
                if (__any_sync(FULL, fin)) { r = R_OUT; break; }
                if (__any_sync(FULL, fblk)) { r = R_BLK; wpos = x; break; }
            }
            if (r == R_IN && lim < we) r = R_DEFER;
            if (lane == src) {
                res = r;
                resume = lim;
                pos = wpos;
            }
        }
        // push-Out: a new In vertex marks its undecided neighbours Out (only undecided
        // ones: INACTIVE vertices are outside the phase), so a blocked vertex waits at
        // its first undecided higher neighbour and never rescans its row for an In one
        // (none of those neighbours can turn In meanwhile: each has v above it)
        if (A.push_out) {
            const bool lanepush = res == R_IN && x0 == b && e - b <= MIS_SMALL;
            if (lanepush) {
                uint8_t sv[MIS_SMALL];
#pragma unroll
                for (int u = 0; u < MIS_SMALL; u++) sv[u] = ld_u8_pred(A.st + wv[u], b + u < e, ST_OUT);
#pragma unroll
                for (int u = 0; u < MIS_SMALL; u++)
                    if (sv[u] == ST_UNDEC) A.st[wv[u]] = ST_OUT;
            }
            unsigned pm = __ballot_sync(FULL, res == R_IN && !lanepush);
            while (pm) {
                const int src = __ffs(pm) - 1;
                pm &= pm - 1;
                const int64_t wb = __shfl_sync(FULL, b, src), we = __shfl_sync(FULL, e, src);
                for (int64_t x = wb + lane; x < we; x += 128) mis_push4<32>(A, x, we);
                prof_add(A.prof, lane == 0 ? 4ull * (we - wb) : 0ull, lane == 0 ? 4ull * (we - wb) : 0ull);  // row re-read
            }
        }
        if (res == R_IN) A.st[v] = ST_IN;
        else if (res == R_OUT) A.st[v] = ST_OUT;
        // §8(d): 4 B per scanned arc + 9 B per active vertex; the implementation also
        // reads the list entry and the status (5 B) and writes decided statuses
        prof_add(A.prof, lb + (active ? 9 : 0), lb + (active ? 18 : 0) + ((res == R_IN || res == R_OUT) ? 1 : 0));
        int64_t slot = warp_append(res == R_BLK, A.out_cnt);
        if (slot >= 0) {
            A.out_list[slot] = v;
            if (A.out_pos) A.out_pos[slot] = (int32_t)(pos - b);
        }
        int64_t hs = warp_append(res == R_DEFER, A.huge_cnt);
        if (hs >= 0) {
            A.huge[2 * hs] = v;
            A.huge[2 * hs + 1] = resume;
        }
    }
}

// deferred long rows: one CTA per vertex, scanning the remainder of its row
__global__ void __launch_bounds__(MIS_HUGE_THREADS) k_mis_huge(MisRoundArgs A) {
    const uint32_t cnt = *A.huge_cnt;
    for (uint32_t h = blockIdx.x; h < cnt; h += gridDim.x) {
        const int32_t v = (int32_t)A.huge[2 * h];
        const int64_t b = A.huge[2 * h + 1], e = A.rp[v - A.row_base + 1];
        const uint64_t kv = vkey(A.k, (uint32_t)v);
        int r = R_IN;
        int64_t bpos = b;
        unsigned long long lb = 0;  // column words (the vertex was counted active by k_mis_round)
        for (int64_t x = b; x < e; x += 4 * MIS_HUGE_THREADS) {
            bool fin = false, fblk = false;
            uint32_t w[4];
            bool ok[4], hi[4];
            uint8_t sw[4];
#pragma unroll
            for (int u = 0; u < 4; u++) {
                int64_t y = x + u * MIS_HUGE_THREADS + threadIdx.x;
                ok[u] = y < e;
                w[u] = ok[u] ? (uint32_t)__ldcs(A.ci + y) : 0u;
                lb += ok[u] ? 4 : 0;
            }
#pragma unroll
            for (int u = 0; u < 4; u++) hi[u] = ok[u] && vkey(A.k, w[u]) > kv;  // higher neighbours only
            mis_gather(A, w, hi, sw);
#pragma unroll
            for (int u = 0; u < 4; u++) {
                fin |= sw[u] == ST_IN;
                fblk |= sw[u] == ST_UNDEC;
            }
            if (__syncthreads_or(fin)) { r = R_OUT; break; }
            if (__syncthreads_or(fblk)) { r = R_BLK; bpos = x; break; }
        }
        if (r == R_IN && A.push_out) {  // push-Out over the whole row (see k_mis_round)
            const int64_t rb = A.rp[v - A.row_base];
            for (int64_t x = rb + threadIdx.x; x < e; x += 4 * MIS_HUGE_THREADS) mis_push4<MIS_HUGE_THREADS>(A, x, e);
            prof_add(A.prof, threadIdx.x == 0 ? 4ull * (e - rb) : 0ull, threadIdx.x == 0 ? 4ull * (e - rb) : 0ull);
        }
        if (threadIdx.x == 0) {
            if (r == R_IN) A.st[v] = ST_IN;
            else if (r == R_OUT) A.st[v] = ST_OUT;
            else {
                uint32_t slot = atomicAdd(A.out_cnt, 1u);
                A.out_list[slot] = v;
                if (A.out_pos) A.out_pos[slot] = (int32_t)(bpos - A.rp[v - A.row_base]);
            }
        }
        prof_add(A.prof, lb, lb + (threadIdx.x == 0 ? 9 : 0));  // impl: + row end + status write
        __syncthreads();
    }
}

// MIS-Deg2 fix-up: every cross neighbour of I_L leaves the remaining graph
__global__ void k_mis_kill_cross(const int64_t *__restrict__ rp_x, const int32_t *__restrict__ ci_x,
                                 const int32_t *__restrict__ list, const uint32_t *cnt, uint8_t *st) {
    const uint32_t c = *cnt;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < c; i += gridDim.x * blockDim.x) {
        int32_t v = list[i];
        if (st[v] != ST_IN) continue;
        for (int64_t x = rp_x[v]; x < rp_x[v + 1]; x++) st[ci_x[x]] = ST_OUT;
    }
}

// MIS-Deg2 classification fused with the trivial part of phase L: V_H -> back of vlist
// (undecided); a V_L vertex without G_L arcs is its own component of G_L, so it is in
// I_L at once and every neighbour of it (all in V_H: it has no G_L arcs) leaves the
// remaining graph (the fix-up of P:288 for it); the other V_L vertices -> front of vlist
// for phase L.  Status must be all undecided on entry.
__global__ void k_mis_degk_classify(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci,
                                    const int64_t *__restrict__ rp_in, int64_t n, uint32_t k, uint8_t *st,
                                    int32_t *vlist, uint32_t *cnt_front, uint32_t *cnt_back) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n; base += stride) {
        const int64_t v = base + threadIdx.x;
        bool h = false, lo = false;
        if (v < n) {
            const int64_t b = rp[v], e = rp[v + 1];
            h = e - b > (int64_t)k;
            if (!h) {
                if (rp_in[v + 1] == rp_in[v]) {  // isolated in G_L
                    st[v] = ST_IN;
                    for (int64_t x = b; x < e; x++) st[ci[x]] = ST_OUT;  // <= k arcs, all to V_H
                } else {
                    lo = true;
                }
            }
        }
        cta_append2(lo, h, (int32_t)v, n, vlist, cnt_front, cnt_back);
    }
}

// MIS-Rand: classify by cross degree: interior (front list, UNDEC) / boundary B
// (back list, INACTIVE during phase A)
__global__ void k_mis_classify_cross(const int64_t *__restrict__ rp_x, int64_t n, uint8_t *st, int32_t *vlist,
                                     uint32_t *cnt_front, uint32_t *cnt_back) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n; base += stride) {
        int64_t v = base + threadIdx.x;
        bool valid = v < n;
        bool bnd = valid && (rp_x[v + 1] > rp_x[v]);
        if (valid) st[v] = bnd ? ST_INACTIVE : ST_UNDEC;
        cta_append2(valid && !bnd, bnd, (int32_t)v, n, vlist, cnt_front, cnt_back);
    }
}

// MIS-Rand fix-up: remove N(I_A) (all arcs of interior vertices are intra)
__global__ void k_mis_kill_all(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci,
                               const int32_t *__restrict__ list, const uint32_t *cnt, uint8_t *st) {
    const uint32_t c = *cnt;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < c; i += gridDim.x * blockDim.x) {
        int32_t v = list[i];
        if (st[v] != ST_IN) continue;
        for (int64_t x = rp[v]; x < rp[v + 1]; x++) st[ci[x]] = ST_OUT;
    }
}

__global__ void k_mis_reactivate(const int32_t *__restrict__ list_end, const uint32_t *cnt, uint8_t *st) {
    const uint32_t c = *cnt;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < c; i += gridDim.x * blockDim.x) {
        int32_t v = list_end[-1 - (int64_t)i];
        if (st[v] == ST_INACTIVE) st[v] = ST_UNDEC;
    }
}

__global__ void k_mis_finish(uint8_t *st, int64_t n, unsigned long long *count) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    uint32_t local = 0;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
        uint8_t s = st[v];
        uint8_t o = (s == ST_IN) ? 1 : 0;
        st[v] = o;
        local += o;
    }
    if (count) {
        for (int d = 16; d; d >>= 1) local += __shfl_xor_sync(FULL, local, d);
        if (lane_id() == 0 && local) atomicAdd(count, (unsigned long long)local);
    }
}

// ------------------------------------------------------------------ f1 variants
// SYM_F_PER_ROUND -- LubyMIS as Luby states it: every round r draws fresh
// priorities from K(seed, VERTEX, r) (phase-local r), and is two synchronous steps:
// step 1, the undecided frontier vertices that beat every undecided phase neighbour
// become candidates; step 2, candidates join I and undecided vertices with a candidate
// (now In) neighbour leave.  With re-drawn priorities the result depends on the round
// structure, so both steps run as separate kernels (warp per vertex).
constexpr uint8_t ST_CAND = 4;

__device__ __forceinline__ int32_t mis_list_at(const int32_t *list, int rev, int64_t i) {
    return list ? (rev ? list[-1 - i] : list[i]) : (int32_t)i;
}

__global__ void k_luby_select(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci, uint8_t *st,
                              const int32_t *list, int rev, const uint32_t *cnt, int64_t implicit_n, Key k) {
    const int lane = lane_id();
    const int64_t c = list ? (int64_t)*cnt : implicit_n;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < c; i += nw) {
        const int32_t v = mis_list_at(list, rev, i);
        if (st[v] != ST_UNDEC) continue;
        const uint64_t kv = vkey(k, (uint32_t)v);
        const int64_t e = rp[v + 1];
        bool beaten = false;
        for (int64_t x = rp[v] + lane; x - lane < e && !beaten; x += 32) {
            bool b = false;
            if (x < e) {
                const uint32_t w = (uint32_t)ci[x];
                const uint8_t sw = st[w];
                b = (sw == ST_UNDEC || sw == ST_CAND) && vkey(k, w) > kv;
            }
            beaten = __any_sync(FULL, b);
        }
        if (!beaten && lane == 0) st[v] = ST_CAND;
    }
}

__global__ void k_luby_resolve(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci, uint8_t *st,
                               const int32_t *list, int rev, const uint32_t *cnt, int64_t implicit_n, int32_t *out,
                               uint32_t *out_cnt) {
    const int lane = lane_id();
    const int64_t c = list ? (int64_t)*cnt : implicit_n;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < c; i += nw) {
        const int32_t v = mis_list_at(list, rev, i);
        const uint8_t sv = st[v];
        if (sv == ST_CAND) {
            if (lane == 0) st[v] = ST_IN;
            continue;
        }
        if (sv != ST_UNDEC) continue;
        const int64_t e = rp[v + 1];
        bool hit = false;
        for (int64_t x = rp[v] + lane; x - lane < e && !hit; x += 32) {
            bool b = false;
            if (x < e) {
                const uint8_t sw = st[ci[x]];
                b = sw == ST_CAND || sw == ST_IN;  // joined I in this round (no older In neighbour exists)
            }
            hit = __any_sync(FULL, b);
        }
        if (lane == 0) {
            if (hit) st[v] = ST_OUT;
            else out[atomicAdd(out_cnt, 1u)] = v;
        }
    }
}

// SYM_F_CONFLICT_DROP (MIS-Rand, reading G10 i): In vertices with a higher-priority In
// cross neighbour are dropped (mark), then I' = In \ dropped and everything else is
// undecided again (warp per vertex over the cross CSR)
__global__ void k_mis_drop_mark(const int64_t *__restrict__ rp_x, const int32_t *__restrict__ ci_x, const uint8_t *st,
                                int64_t n, Key k, uint8_t *mark) {
    const int lane = lane_id();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; v < n; v += nw) {
        if (st[v] != ST_IN) {
            if (lane == 0) mark[v] = 0;
            continue;
        }
        const uint64_t kv = vkey(k, (uint32_t)v);
        const int64_t e = rp_x[v + 1];
        bool hit = false;
        for (int64_t x = rp_x[v] + lane; x - lane < e && !hit; x += 32) {
            const bool b = x < e && st[ci_x[x]] == ST_IN && vkey(k, (uint32_t)ci_x[x]) > kv;
            hit = __any_sync(FULL, b);
        }
        if (lane == 0) mark[v] = hit ? 1 : 0;
    }
}

__global__ void k_mis_drop_apply(uint8_t *st, const uint8_t *mark, int64_t n) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
        st[v] = (st[v] == ST_IN && !mark[v]) ? ST_IN : ST_UNDEC;
}

// undecided vertices with an In neighbour leave ("remove from G vertices that are in I
// or have a neighbour in I"); the rest -> list (warp per vertex)
__global__ void k_mis_kill_pull(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci, uint8_t *st, int64_t n,
                                int32_t *list, uint32_t *cnt) {
    const int lane = lane_id();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; v < n; v += nw) {
        if (st[v] != ST_UNDEC) continue;
        const int64_t e = rp[v + 1];
        bool hit = false;
        for (int64_t x = rp[v] + lane; x - lane < e && !hit; x += 32) hit = __any_sync(FULL, x < e && st[ci[x]] == ST_IN);
        if (lane == 0) {
            if (hit) st[v] = ST_OUT;
            else list[atomicAdd(cnt, 1u)] = (int32_t)v;
        }
    }
}

// SYM_F_SPARSER_FIRST: the boundary first -- B undecided (back of vlist), the interior
// INACTIVE (front)
__global__ void k_mis_classify_bfirst(const int64_t *__restrict__ rp_x, int64_t n, uint8_t *st, int32_t *vlist,
                                      uint32_t *cnt_front, uint32_t *cnt_back) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n; base += stride) {
        int64_t v = base + threadIdx.x;
        bool valid = v < n;
        bool bnd = valid && (rp_x[v + 1] > rp_x[v]);
        if (valid) st[v] = bnd ? ST_UNDEC : ST_INACTIVE;
        cta_append2(valid && !bnd, bnd, (int32_t)v, n, vlist, cnt_front, cnt_back);
    }
}

// In vertices of a (possibly reversed) list remove their neighbours; then the
// INACTIVE vertices of another list become undecided
__global__ void k_mis_kill_list(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci, const int32_t *list,
                                int rev, const uint32_t *cnt, uint8_t *st) {
    const uint32_t c = *cnt;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < c; i += gridDim.x * blockDim.x) {
        const int32_t v = mis_list_at(list, rev, i);
        if (st[v] != ST_IN) continue;
        for (int64_t x = rp[v]; x < rp[v + 1]; x++) st[ci[x]] = ST_OUT;
    }
}

__global__ void k_mis_wake_list(const int32_t *list, int rev, const uint32_t *cnt, uint8_t *st) {
    const uint32_t c = *cnt;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < c; i += gridDim.x * blockDim.x) {
        const int32_t v = mis_list_at(list, rev, i);
        if (st[v] == ST_INACTIVE) st[v] = ST_UNDEC;
    }
}

// ------------------------------------------------------------------ host side
void carve_mis_ws(Arena &a, int64_t n, int64_t nnz, MisWs &w) {
    w.vlist = a.take<int32_t>((size_t)n + 1);
    w.fr[0] = a.take<int32_t>((size_t)n + 1);
    w.fr[1] = a.take<int32_t>((size_t)n + 1);
    w.fp[0] = a.take<int32_t>((size_t)n + 1);
    w.fp[1] = a.take<int32_t>((size_t)n + 1);
    w.huge_cap = nnz / MIS_BUDGET + 2;
    w.huge = a.take<int64_t>((size_t)(2 * w.huge_cap));
    w.gmax = a.take<unsigned long long>((size_t)n + 1);
    w.mark = a.take<uint8_t>((size_t)n + 1);
}

// One resident wave: the grid-stride round kernels lose ~20 % to a partial second wave
// when the grid asks for more CTAs than fit (8 requested, 6 resident at 40 regs).
static int round_grid() {
#if SYM_ROUND_ONE_WAVE
    static std::atomic<int> slots[SYM_MAX_DEVICES];
    return dev_cached(slots, [] {
        int per = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_mis_round, MIS_THREADS, 0) != cudaSuccess || per < 1)
            per = 2048 / MIS_THREADS;
        return num_sms() * per;
    });
#else
    return num_sms() * (2048 / MIS_THREADS);
#endif
}

// SYM_F_PER_ROUND: classic Luby rounds of one phase (round r draws K(seed, VERTEX, r));
// the host reads the frontier count after every round
static int mis_phase_per_round(const FlowArgs &f, MisWs &w, uint8_t *st, const int64_t *rp, const int32_t *ci,
                               const int32_t *list0, int rev0, const uint32_t *cnt0, int64_t implicit_n, int phase) {
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
    const uint32_t maxr = f.p.max_rounds ? f.p.max_rounds : 0xffffffffu;
    const int32_t *list = list0;
    int rev = rev0;
    const uint32_t *cnt = cnt0;
    int64_t len = list0 ? (int64_t)num_sms() * 8 * 8 : implicit_n;  // host view of the list length (grid size)
    uint32_t r = 0;
    for (;; r++) {
        if (r >= maxr) {
            set_error("MIS phase did not converge within max_rounds");
            return SYM_EROUNDS;
        }
        const Key k = stream_key(f.p.seed, TAG_VERTEX, r);
        uint32_t *out_cnt = &ctl->ring[(r + 1) % 2];
        int32_t *out = w.fr[(r + 1) & 1];
        SYM_CUDA(cudaMemsetAsync(out_cnt, 0, sizeof(uint32_t), s));
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((int64_t)num_sms() * 8, (len * 32 + 255) / 256));
        k_luby_select<<<grid, 256, 0, s>>>(rp, ci, st, list, rev, cnt, implicit_n, k);
        SYM_LAUNCH_CHECK();
        k_luby_resolve<<<grid, 256, 0, s>>>(rp, ci, st, list, rev, cnt, implicit_n, out, out_cnt);
        SYM_LAUNCH_CHECK();
        uint32_t left = 0;
        SYM_TRY(read_u32(out_cnt, &left, s));
        if (f.stats && r < 2048) f.stats->rounds[phase] = r + 1;
        if (left == 0) break;
        list = out;
        rev = 0;
        cnt = out_cnt;
        len = left;
    }
    return SYM_OK;
}

// Run Luby rounds of one phase until the frontier is empty.  Round 0 reads
// (list0, rev0, cnt0) -- or the implicit range [0, implicit_n) when list0 == nullptr.
static int mis_phase(const FlowArgs &f, MisWs &w, uint8_t *st, const int64_t *rp, const int32_t *ci,
                     const int32_t *list0, int rev0, const uint32_t *cnt0, int64_t implicit_n, int phase,
                     bool stream_round0 = false) {
    // stream_round0: round 0 as a gather-free streaming pass (round0.cu).  Measured at
    // R-MAT s24 it is slower than the early-exit frontier kernel, whose
    // round 0 reads only ~30 % of the arcs, so it is off by default for MIS.
    if (f.p.flags & SYM_F_PER_ROUND)
        return mis_phase_per_round(f, w, st, rp, ci, list0, rev0, cnt0, implicit_n, phase);
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
    SYM_CUDA(cudaMemsetAsync(ctl->ring, 0, sizeof(ctl->ring) + sizeof(ctl->huge), s));
    const Key k = stream_key(f.p.seed, TAG_VERTEX, 0);
    if (stream_round0) {
        // round 0 as one streaming pass: every local maximum of the phase joins I
        int64_t nnz = 0;
        SYM_TRY(phase_arcs(f, rp, &nnz));
        if (nnz > 0)
            SYM_TRY(run_round0(0, Graph{f.g.n, nnz, rp, ci}, f.first_row, (nnz + SPLIT_TILE - 1) / SPLIT_TILE, k,
                               w.gmax, st, nullptr, nullptr, nullptr, nullptr, s));
    }
    const uint32_t maxr = f.p.max_rounds ? f.p.max_rounds : 0xffffffffu;
    int grid = round_grid();
    int r = 0;
    const int batch = SYM_POLL_BATCH;  // rounds launched per host poll of the frontier count
    for (;;) {
        for (int b = 0; b < batch && (uint32_t)r < maxr; b++, r++) {  // never past the cap
            MisRoundArgs A{};
            A.rp = rp;
            A.ci = ci;
            A.st = st;
            if (r == 0) {
                A.in_list = list0;
                A.in_rev = rev0;
                A.in_cnt = cnt0;
                A.in_pos = nullptr;
            } else {
                A.in_list = w.fr[r & 1];
                A.in_rev = 0;
                A.in_cnt = &ctl->ring[r % 3];
                A.in_pos = w.fp[r & 1];
            }
            A.implicit_n = implicit_n;
            A.out_list = w.fr[(r + 1) & 1];
            A.out_pos = w.fp[(r + 1) & 1];
            A.push_out = 1;
            A.out_cnt = &ctl->ring[(r + 1) % 3];
            A.clear_cnt = &ctl->ring[(r + 2) % 3];
            A.huge = w.huge;
            A.huge_cnt = &ctl->huge[r & 1];
            A.huge_clear = &ctl->huge[(r + 1) & 1];
            A.hist = (phase == 0) ? ctl->hist : ctl->hist + 2048;
            A.round = r < 2048 ? r : 2047;
            A.k = k;
            A.row_base = 0;
            A.nfilter = nullptr;
            A.ncls = -1;
            A.prof = prof_counter(s);
            prof_begin("mis_round", s);
            k_mis_round<<<grid, MIS_THREADS, 0, s>>>(A);
            prof_end_dev(s, A.prof);
            SYM_LAUNCH_CHECK();
            A.prof = prof_counter(s);
            prof_begin("mis_huge", s);
            k_mis_huge<<<num_sms() * 2, MIS_HUGE_THREADS, 0, s>>>(A);
            prof_end_dev(s, A.prof);
            SYM_LAUNCH_CHECK();
        }
        uint32_t left = 0;
        SYM_TRY(read_u32(&ctl->ring[r % 3], &left, s));
        if (left == 0) break;
        if ((uint32_t)r >= maxr) {
            set_error("MIS phase did not converge within max_rounds");
            return SYM_EROUNDS;
        }
        // frontiers only shrink: size the next launches for `left` vertices
        const int64_t need = ((int64_t)left + MIS_THREADS - 1) / MIS_THREADS;
        grid = (int)std::min<int64_t>(round_grid(), std::max<int64_t>(need, 1));
    }
    if (f.stats) f.stats->rounds[phase] = (uint32_t)r;  // refined from hist below
    return SYM_OK;
}

// SYM_F_SPARSER_FIRST: does G_{k+1} have fewer arcs than the union of the parts?
static bool mis_cross_sparser(const FlowArgs &f) {
    int64_t nin = 0;
    if (phase_arcs(f, f.split.rp_in, &nin) != SYM_OK) return false;
    return f.g.nnz - nin < nin;
}

int run_mis(const FlowArgs &f, MisWs &w, uint8_t *st) {
    const Graph &g = f.g;
    cudaStream_t s = f.stream;
    Ctl *ctl = f.ctl;
    const int kind = f.p.kind;
    if (kind == SYM_DECOMP_NONE) {
        SYM_CUDA(cudaMemsetAsync(st, ST_UNDEC, (size_t)g.n, s));
        SYM_TRY(mis_phase(f, w, st, g.rp, g.ci, nullptr, 0, nullptr, g.n, 0));
        if (f.stats) f.stats->phase_vertices[0] = g.n;
    } else if (kind == SYM_DECOMP_DEGK) {
        // lists V_L (front) and V_H (back); status all undecided
        SYM_CUDA(cudaMemsetAsync(st, ST_UNDEC, (size_t)g.n, s));
        SYM_CUDA(cudaMemsetAsync(&ctl->cnt_front, 0, 2 * sizeof(uint32_t), s));
        k_mis_degk_classify<<<num_sms() * 8, 256, 0, s>>>(g.rp, g.ci, f.split.rp_in, g.n, f.p.param, st, w.vlist,
                                                          &ctl->cnt_front, &ctl->cnt_back);
        SYM_LAUNCH_CHECK();
        // phase L: I_L = MIS(G_L) on the intra CSR restricted to V_L (tiny: the rows
        // of V_H in the same CSR are not in this phase, so no streaming round 0)
        SYM_TRY(mis_phase(f, w, st, f.split.rp_in, f.split.ci_in, w.vlist, 0, &ctl->cnt_front, 0, 0, false));
        // fix-up: remove N(I_L) from V_H through the cross arcs G_C
        k_mis_kill_cross<<<num_sms() * 4, 256, 0, s>>>(f.split.rp_x, f.split.ci_x, w.vlist, &ctl->cnt_front, st);
        SYM_LAUNCH_CHECK();
        // phase R: MIS of the remaining V_H on G_H
        SYM_TRY(mis_phase(f, w, st, f.split.rp_in, f.split.ci_in, w.vlist + g.n, 1, &ctl->cnt_back, 0, 1));
    } else if (f.p.flags & SYM_F_CONFLICT_DROP) {
        // reading G10 (i): I_P = MIS of the parts (every vertex, intra arcs); I' = I_P
        // minus the lower In end of every In-In cross arc; then the MIS of V \ N[I'] on G
        SYM_CUDA(cudaMemsetAsync(st, ST_UNDEC, (size_t)g.n, s));
        SYM_TRY(mis_phase(f, w, st, f.split.rp_in, f.split.ci_in, nullptr, 0, nullptr, g.n, 0));
        k_mis_drop_mark<<<num_sms() * 8, 256, 0, s>>>(f.split.rp_x, f.split.ci_x, st, g.n,
                                                      stream_key(f.p.seed, TAG_VERTEX, 0), w.mark);
        SYM_LAUNCH_CHECK();
        k_mis_drop_apply<<<num_sms() * 8, 256, 0, s>>>(st, w.mark, g.n);
        SYM_LAUNCH_CHECK();
        SYM_CUDA(cudaMemsetAsync(&ctl->cnt_front, 0, sizeof(uint32_t), s));
        k_mis_kill_pull<<<num_sms() * 8, 256, 0, s>>>(g.rp, g.ci, st, g.n, w.vlist, &ctl->cnt_front);
        SYM_LAUNCH_CHECK();
        SYM_TRY(mis_phase(f, w, st, g.rp, g.ci, w.vlist, 0, &ctl->cnt_front, 0, 1));
    } else if ((f.p.flags & SYM_F_SPARSER_FIRST) && mis_cross_sparser(f)) {
        // P:284/P:286 (reading G10 ii): G_{k+1} is sparser than the parts -> the
        // boundary's MIS first (all arcs among B), then the interior not adjacent to it
        SYM_CUDA(cudaMemsetAsync(&ctl->cnt_front, 0, 2 * sizeof(uint32_t), s));
        k_mis_classify_bfirst<<<num_sms() * 8, 256, 0, s>>>(f.split.rp_x, g.n, st, w.vlist, &ctl->cnt_front,
                                                            &ctl->cnt_back);
        SYM_LAUNCH_CHECK();
        SYM_TRY(mis_phase(f, w, st, g.rp, g.ci, w.vlist + g.n, 1, &ctl->cnt_back, 0, 0));  // I_1 = MIS(G[B])
        k_mis_kill_list<<<num_sms() * 4, 256, 0, s>>>(g.rp, g.ci, w.vlist + g.n, 1, &ctl->cnt_back, st);
        SYM_LAUNCH_CHECK();
        k_mis_wake_list<<<num_sms() * 4, 256, 0, s>>>(w.vlist, 0, &ctl->cnt_front, st);
        SYM_LAUNCH_CHECK();
        SYM_TRY(mis_phase(f, w, st, g.rp, g.ci, w.vlist, 0, &ctl->cnt_front, 0, 1));  // I_2 on the interior
    } else {
        SYM_CUDA(cudaMemsetAsync(&ctl->cnt_front, 0, 2 * sizeof(uint32_t), s));
        k_mis_classify_cross<<<num_sms() * 8, 256, 0, s>>>(f.split.rp_x, g.n, st, w.vlist, &ctl->cnt_front,
                                                           &ctl->cnt_back);
        SYM_LAUNCH_CHECK();
        // phase A: I_A = MIS of the partition interiors (boundary vertices INACTIVE)
        SYM_TRY(mis_phase(f, w, st, f.split.rp_in, f.split.ci_in, w.vlist, 0, &ctl->cnt_front, 0, 0));
        // R = G - N[I_A]
        k_mis_kill_all<<<num_sms() * 4, 256, 0, s>>>(f.split.rp_in, f.split.ci_in, w.vlist, &ctl->cnt_front, st);
        SYM_LAUNCH_CHECK();
        k_mis_reactivate<<<num_sms() * 4, 256, 0, s>>>(w.vlist + g.n, &ctl->cnt_back, st);
        SYM_LAUNCH_CHECK();
        // phase B: I_B = MIS(R) on G
        SYM_TRY(mis_phase(f, w, st, g.rp, g.ci, w.vlist + g.n, 1, &ctl->cnt_back, 0, 1));
    }
    unsigned long long *cnt = (f.p.flags & SYM_F_STATS) ? (unsigned long long *)&ctl->result : nullptr;
    if (cnt) SYM_CUDA(cudaMemsetAsync(cnt, 0, sizeof(uint64_t), s));
    k_mis_finish<<<num_sms() * 8, 256, 0, s>>>(st, g.n, cnt);
    SYM_LAUNCH_CHECK();
    if (f.stats) {
        uint32_t hist[4096];
        SYM_CUDA(cudaMemcpyAsync(hist, ctl->hist, sizeof(hist), cudaMemcpyDeviceToHost, s));
        SYM_CUDA(cudaStreamSynchronize(s));
        for (int ph = 0; ph < 2; ph++) {
            uint32_t rr = 0;
            for (int i = 0; i < 2048 && i < (int)f.stats->rounds[ph]; i++) rr += hist[ph * 2048 + i] ? 1 : 0;
            f.stats->rounds[ph] = rr;
            f.stats->phase_vertices[ph] = hist[ph * 2048];
        }
        if (cnt) {
            uint64_t c = 0;
            SYM_TRY(read_u64(&ctl->result, &c, s));
            f.stats->result_size = (int64_t)c;
        }
    }
    return SYM_OK;
}

// ------------------------------------------------------------------ sharded MIS
// A rank owns rows [v_begin, v_end) (global ids, v_begin % 32 == 0) stored with global
// column ids and keeps a full replica of the status array; after every round the
// caller all-gathers the owned status segments (torch.distributed / NCCL over NVLink)
// and all-reduces the frontier counts.  DEGk is applied as a class predicate on the
// owned rows (the global class bitmap is all-gathered once): phase L runs on V_L with
// V_H neighbours ignored, the fix-up turns every owned V_H vertex with an In V_L
// neighbour Out, phase R runs on V_H with V_L neighbours ignored.

__global__ void k_shard_classify(const int64_t *__restrict__ rp, int64_t v0, int64_t v1, uint32_t k,
                                 uint32_t *__restrict__ hbits) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = v0 + (int64_t)blockIdx.x * blockDim.x; base < v1; base += stride) {
        const int64_t v = base + threadIdx.x;  // base is a multiple of 32 (v0 % 32 == 0)
        const bool h = v < v1 && (rp[v - v0 + 1] - rp[v - v0]) > (int64_t)k;
        const unsigned word = __ballot_sync(FULL, h);
        if (lane_id() == 0 && base + (threadIdx.x & ~31) < v1) hbits[v >> 5] = word;
    }
}

__global__ void k_shard_frontier(const uint32_t *__restrict__ hbits, int cls, const uint8_t *__restrict__ st,
                                 int64_t v0, int64_t v1, int32_t *list, uint32_t *count) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = v0 + (int64_t)blockIdx.x * blockDim.x; base < v1; base += stride) {
        const int64_t v = base + threadIdx.x;
        bool take = v < v1 && st[v] == ST_UNDEC && (cls < 0 || (int)((hbits[v >> 5] >> (v & 31)) & 1u) == cls);
        int64_t slot = warp_append(take, count);
        if (slot >= 0) list[slot] = (int32_t)v;
    }
}

__global__ void k_shard_finish(const uint8_t *__restrict__ st, int64_t v0, int64_t v1, uint8_t *__restrict__ out) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = v0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < v1; v += stride)
        out[v - v0] = st[v] == ST_IN ? 1 : 0;
}

// ---- deltas of the sharded flow (shard.cu): owned boundary vertices whose status
// changed, packed id << 2 | status (4 B)
__device__ __forceinline__ bool sh_bnd(const uint32_t *bnd, int64_t i) { return (bnd[i >> 5] >> (i & 31)) & 1u; }

// decided in this round: the round's input list entries (all undecided at its start)
// that are now In / Out
__global__ void k_sh_delta_mis(const int32_t *__restrict__ list, const uint32_t *cnt, const uint8_t *st,
                               const uint32_t *__restrict__ bnd, int64_t v0, uint32_t *send, uint32_t *dcnt) {
    const int64_t c = *cnt, stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < c; base += stride) {
        const int64_t i = base + threadIdx.x;
        const int32_t v = i < c ? list[i] : -1;
        const uint8_t sv = v >= 0 ? st[v] : (uint8_t)ST_UNDEC;
        const int64_t slot = warp_append(v >= 0 && sv != ST_UNDEC && sh_bnd(bnd, v - v0), dcnt);
        if (slot >= 0) send[slot] = ((uint32_t)v << 2) | sv;
    }
}

// MIS-Deg2 fix-up, pull form with deltas: an owned undecided V_H vertex with
// an In V_L neighbour leaves the remaining graph (warp per vertex)
__global__ void k_sh_kill_degk(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci,
                               const uint32_t *__restrict__ hbits, uint8_t *st, int64_t v0, int64_t v1,
                               const uint32_t *__restrict__ bnd, uint32_t *send, uint32_t *dcnt) {
    const int lane = lane_id();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = v0 + (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5); v < v1; v += nw) {
        if (!((hbits[v >> 5] >> (v & 31)) & 1u) || st[v] != ST_UNDEC) continue;
        const int64_t b = rp[v - v0], e = rp[v - v0 + 1];
        bool hit = false;
        for (int64_t x = b; x < e && !hit; x += 32) {
            bool h = false;
            if (x + lane < e) {
                const uint32_t w = (uint32_t)__ldcs(ci + x + lane);
                h = !((hbits[w >> 5] >> (w & 31)) & 1u) && st[w] == ST_IN;
            }
            hit = __any_sync(FULL, h);
        }
        if (hit && lane == 0) {
            st[v] = ST_OUT;
            if (sh_bnd(bnd, v - v0)) send[atomicAdd(dcnt, 1u)] = ((uint32_t)v << 2) | ST_OUT;
        }
    }
}

// MIS-Rand (reading G10): B = owned vertices with a cross arc (RAND labels
// differ) are not in phase A: INACTIVE (warp per vertex)
__global__ void k_sh_rand_inactive(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci, Key kr,
                                   uint32_t p, uint8_t *st, int64_t v0, int64_t v1, const uint32_t *__restrict__ bnd,
                                   uint32_t *send, uint32_t *dcnt) {
    const int lane = lane_id();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = v0 + (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5); v < v1; v += nw) {
        const uint32_t lv = rand_label(kr, (uint32_t)v, p);
        const int64_t b = rp[v - v0], e = rp[v - v0 + 1];
        bool hit = false;
        for (int64_t x = b; x < e && !hit; x += 32) {
            const bool h = x + lane < e && rand_label(kr, (uint32_t)ci[x + lane], p) != lv;
            hit = __any_sync(FULL, h);
        }
        if (hit && lane == 0) {
            st[v] = ST_INACTIVE;
            if (sh_bnd(bnd, v - v0)) send[atomicAdd(dcnt, 1u)] = ((uint32_t)v << 2) | ST_INACTIVE;
        }
    }
}

// MIS-Rand fix-up: an owned B vertex with an In neighbour (an interior vertex of I_A)
// is removed (Out); the others enter phase B (undecided)
__global__ void k_sh_rand_release(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci, uint8_t *st,
                                  int64_t v0, int64_t v1, const uint32_t *__restrict__ bnd, uint32_t *send,
                                  uint32_t *dcnt) {
    const int lane = lane_id();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = v0 + (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5); v < v1; v += nw) {
        if (st[v] != ST_INACTIVE) continue;
        const int64_t b = rp[v - v0], e = rp[v - v0 + 1];
        bool hit = false;
        for (int64_t x = b; x < e && !hit; x += 32) {
            const bool h = x + lane < e && st[ci[x + lane]] == ST_IN;
            hit = __any_sync(FULL, h);
        }
        if (lane == 0) {
            const uint8_t ns = hit ? ST_OUT : ST_UNDEC;
            st[v] = ns;
            if (sh_bnd(bnd, v - v0)) send[atomicAdd(dcnt, 1u)] = ((uint32_t)v << 2) | ns;
        }
    }
}

}  // namespace sym

using namespace sym;

// ------------------------------------------------------------------ sharded MIS (C-ABI)
static void carve_mis_sharded(Arena &a, const ShardPlan &P, ShardCtx &x, uint8_t *&st, int64_t *&huge) {
    carve_shard_common(a, P, sizeof(uint32_t), x);
    st = a.take<uint8_t>((size_t)P.N * (size_t)P.B);
    huge = a.take<int64_t>(2 * (size_t)(P.nnz / MIS_BUDGET + 2));
}

static int shard_grid(int64_t items) {
    int64_t want = (items + 255) / 256, cap = (int64_t)num_sms() * 8;
    return (int)(want < 1 ? 1 : (want < cap ? want : cap));
}

// Luby rounds of one phase over the owned frontier (class cls of the DEGk bitmap, -1:
// all), exchanging the boundary decisions after every round.  *rounds = rounds run.
static int mis_sharded_phase(const ShardPlan &P, ShardCtx &x, const sym_params *p, uint8_t *st, int64_t *huge, int cls,
                             uint32_t *rounds) {
    cudaStream_t s = x.s;
    SYM_CUDA(cudaMemsetAsync(x.cnt_in(0), 0, sizeof(uint32_t), s));
    if (P.nl > 0) {
        k_shard_frontier<<<shard_grid(P.nl), 256, 0, s>>>(x.hbits, cls, st, P.v0, P.v1, x.list_in(0), x.cnt_in(0));
        SYM_LAUNCH_CHECK();
    }
    const uint32_t maxr = p->max_rounds ? p->max_rounds : 0xffffffffu;
    const Key k = stream_key(p->seed, TAG_VERTEX, 0);
    int64_t local = P.nl;  // this rank's frontier length (host view, sizes the grid)
    for (int r = 0;; r++) {
        if ((uint32_t)r >= maxr) {
            set_error("sharded MIS phase did not converge within max_rounds");
            return SYM_EROUNDS;
        }
        SYM_CUDA(cudaMemsetAsync(x.dcnt(r), 0, 2 * sizeof(uint32_t), s));
        SYM_CUDA(cudaMemsetAsync(x.scratch, 0, 4 * sizeof(uint32_t), s));
        if (local > 0) {
            MisRoundArgs A{};
            A.rp = P.rp;
            A.ci = P.ci;
            A.st = st;
            A.in_list = x.list_in(r);
            A.in_rev = 0;
            A.in_cnt = x.cnt_in(r);
            A.implicit_n = 0;
            A.out_list = x.list_out(r);
            A.out_cnt = x.cnt_out(r);
            A.clear_cnt = x.scratch + 1;
            A.huge = huge;
            A.huge_cnt = x.scratch;
            A.huge_clear = x.scratch + 2;
            A.hist = nullptr;
            A.round = 0;
            A.k = k;
            A.prof = nullptr;
            A.row_base = P.v0;
            A.nfilter = x.hbits;
            A.ncls = cls;
            k_mis_round<<<std::min<int64_t>(round_grid(), shard_grid(local)), MIS_THREADS, 0, s>>>(A);
            SYM_LAUNCH_CHECK();
            k_mis_huge<<<num_sms() * 2, MIS_HUGE_THREADS, 0, s>>>(A);
            SYM_LAUNCH_CHECK();
            k_sh_delta_mis<<<shard_grid(local), 256, 0, s>>>(x.list_in(r), x.cnt_in(r), st, x.bnd, P.v0,
                                                             (uint32_t *)x.send, x.dcnt(r));
            SYM_LAUNCH_CHECK();
        }
        uint64_t front = 0;
        SYM_TRY(shard_exchange(P, x, r & 1, SH_MIS, st, nullptr, nullptr, nullptr, &front));
        local = x.host_all[2 * P.rank + 1];
        if (front == 0) {
            *rounds = (uint32_t)(r + 1);
            return SYM_OK;
        }
    }
}

extern "C" {

size_t sym_sharded_workspace_bytes(const sym_graph_shard *g, const sym_params *p, const sym_comm *c, int problem) {
    ShardPlan P;
    if (shard_check(g, p, c, &P) != SYM_OK) return 0;
    Arena a;
    ShardCtx x;
    if (problem == SYM_PROBLEM_MIS) {
        uint8_t *st;
        int64_t *huge;
        carve_mis_sharded(a, P, x, st, huge);
    } else if (problem == SYM_PROBLEM_MM) {
        carve_mm_sharded_dry(a, P, p, x);
    } else if (problem == SYM_PROBLEM_COLOR) {
        carve_color_sharded_dry(a, P, x);
    } else {
        return 0;
    }
    return a.used + 256;
}

int sym_mis_sharded(const sym_graph_shard *g, const sym_params *p, sym_comm *c, void *ws, size_t ws_bytes,
                    uint8_t *in_set, sym_shard_stats *stats, sym_stream_t stream) {
    ShardPlan P;
    SYM_TRY(shard_check(g, p, c, &P));
    if (P.nl > 0 && !in_set) { set_error("in_set is NULL"); return SYM_EINVAL; }
    ShardCtx x;
    uint8_t *st = nullptr;
    int64_t *huge = nullptr;
    SYM_TRY(shard_carve_ws(ws, ws_bytes, [&](Arena &a) {
        x = ShardCtx();
        carve_mis_sharded(a, P, x, st, huge);
    }));
    x.c = c;
    x.s = (cudaStream_t)stream;
    cudaStream_t s = x.s;
    if (stats) memset(stats, 0, sizeof(*stats));
    SYM_CUDA(cudaMemsetAsync(st, ST_UNDEC, (size_t)P.N * (size_t)P.B, s));
    SYM_CUDA(cudaMemsetAsync(x.pair, 0, 8 * sizeof(uint32_t), s));
    SYM_TRY(shard_boundary(P, x, s));
    uint32_t rounds[3] = {0, 0, 0};
    uint64_t front = 0;
    if (p->kind == SYM_DECOMP_NONE) {
        SYM_TRY(mis_sharded_phase(P, x, p, st, huge, -1, &rounds[0]));
    } else if (p->kind == SYM_DECOMP_DEGK) {
        // V_H bitmap: owned words, then all-gathered once
        if (P.nl > 0) {
            k_shard_classify<<<shard_grid(P.nl), 256, 0, s>>>(P.rp, P.v0, P.v1, p->param, x.hbits);
            SYM_LAUNCH_CHECK();
        }
        SYM_TRY(shard_gather_hbits(P, x));
        SYM_TRY(mis_sharded_phase(P, x, p, st, huge, 0, &rounds[0]));  // I_L = MIS(G_L)
        SYM_CUDA(cudaMemsetAsync(x.pair, 0, 2 * sizeof(uint32_t), s));
        if (P.nl > 0) {
            k_sh_kill_degk<<<num_sms() * 8, 256, 0, s>>>(P.rp, P.ci, x.hbits, st, P.v0, P.v1, x.bnd,
                                                         (uint32_t *)x.send, x.pair);
            SYM_LAUNCH_CHECK();
        }
        SYM_TRY(shard_exchange(P, x, 0, SH_MIS, st, nullptr, nullptr, nullptr, &front));
        SYM_TRY(mis_sharded_phase(P, x, p, st, huge, 1, &rounds[1]));  // I_R on the remaining V_H
    } else {
        const Key kr = stream_key(p->seed, TAG_RAND, 0);
        SYM_CUDA(cudaMemsetAsync(x.pair, 0, 2 * sizeof(uint32_t), s));
        if (P.nl > 0) {
            k_sh_rand_inactive<<<num_sms() * 8, 256, 0, s>>>(P.rp, P.ci, kr, p->param, st, P.v0, P.v1, x.bnd,
                                                             (uint32_t *)x.send, x.pair);
            SYM_LAUNCH_CHECK();
        }
        SYM_TRY(shard_exchange(P, x, 0, SH_MIS, st, nullptr, nullptr, nullptr, &front));
        SYM_TRY(mis_sharded_phase(P, x, p, st, huge, -1, &rounds[0]));  // I_A on the interiors
        SYM_CUDA(cudaMemsetAsync(x.pair, 0, 2 * sizeof(uint32_t), s));
        if (P.nl > 0) {
            k_sh_rand_release<<<num_sms() * 8, 256, 0, s>>>(P.rp, P.ci, st, P.v0, P.v1, x.bnd, (uint32_t *)x.send,
                                                            x.pair);
            SYM_LAUNCH_CHECK();
        }
        SYM_TRY(shard_exchange(P, x, 0, SH_MIS, st, nullptr, nullptr, nullptr, &front));
        SYM_TRY(mis_sharded_phase(P, x, p, st, huge, -1, &rounds[1]));  // I_B on G - N[I_A]
    }
    if (P.nl > 0) {
        k_shard_finish<<<shard_grid(P.nl), 256, 0, s>>>(st, P.v0, P.v1, in_set);
        SYM_LAUNCH_CHECK();
    }
    if (stats) {
        memcpy(stats->rounds, rounds, sizeof(rounds));
        shard_stats_out(x, stats);
        SYM_TRY(shard_count_boundary(P, x, &stats->boundary));
    }
    return SYM_OK;
}

}  // extern "C"
