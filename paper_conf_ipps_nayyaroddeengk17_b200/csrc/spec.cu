// spec.cu -- the paper's own colouring subroutines (include/sym.h
// SYM_F_COLOR_EB / SYM_F_COLOR_VB): speculative colouring as P:216-218 describes
// Deveci et al. [10], and COLOR-Degk's literal (k+1)-slot G_L loop (Alg 9 l.6).
//
// Speculative rounds on the admitted arcs (all / same class / both in V_H), with a
// colour window of W colours per vertex (EB: a 32-bit mask; VB: a FORBIDDEN
// array of the average degree of the graph being coloured):
//   1. every uncoloured vertex takes the smallest colour of [base, base + W) no admitted
//      neighbour holds; if none is free, base += W ("OFFSET") and it waits a round;
//   2. every admitted edge whose ends share a colour resets its LOWER-id end.
// The steps are separate kernels over frozen snapshots (tentative colours T, reset
// flags R), so the result is a deterministic function of the graph -- bit-identical
// to oracle/oracle.c or_color_spec.  Conflicts can only involve a vertex coloured in
// the round, so step 2 scans the rows of those vertices only; a lower-id neighbour it
// resets may be an older one, which then rejoins the uncoloured list.
#include "internal.h"

namespace sym {

constexpr int SP_THREADS = 256, SP_WARPS = SP_THREADS / 32, SP_WIN = 1024;
constexpr int SP_BUDGET = 2048;       // rows longer than this are scanned by a whole CTA
constexpr int SP_HUGE_THREADS = 512;
enum { SP_ALL = 0, SP_SAME = 1, SP_HH = 3 };

struct SpecArgs {
    const int64_t *rp;
    const int32_t *ci;
    int admit;             // SP_ALL / SP_SAME / SP_HH
    int kind;              // class function: RAND label hash, DEGk bitmap, NONE
    uint32_t param;
    Key kr;
    const uint32_t *hbits;
    uint32_t W;            // colour window (<= SP_WIN)
    uint32_t *C;           // colours (0 = uncoloured)
    uint32_t *T;           // tentative colours of step 1
    uint32_t *base;        // window start per vertex
    uint8_t *R;            // reset flags of step 2
};

__device__ __forceinline__ uint32_t sp_class(const SpecArgs &A, uint32_t v) {
    if (A.kind == SYM_DECOMP_RAND) return rand_label(A.kr, v, A.param);
    if (A.kind == SYM_DECOMP_DEGK) return (A.hbits[v >> 5] >> (v & 31)) & 1u;
    return 0u;
}

__device__ __forceinline__ bool sp_admitted(const SpecArgs &A, uint32_t cv, uint32_t w) {
    if (A.admit == SP_ALL) return true;
    const uint32_t cw = sp_class(A, w);
    return A.admit == SP_SAME ? cw == cv : (cv == 1u && cw == 1u);
}

// step 1 (warp per listed uncoloured vertex): T[v] = smallest free colour of the window
__global__ void __launch_bounds__(SP_THREADS) k_spec_assign(SpecArgs A, const uint32_t *__restrict__ list,
                                                            const uint32_t *cnt, uint32_t *hlist, uint32_t *hcnt) {
    __shared__ uint32_t s_mask[SP_WARPS][SP_WIN / 32];
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    const int64_t c = *cnt, nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < c; i += nw) {
        const uint32_t v = list[i];
        if (A.rp[v + 1] - A.rp[v] > SP_BUDGET) {  // a hub: k_spec_assign_huge
            if (lane == 0) hlist[atomicAdd(hcnt, 1u)] = v;
            continue;
        }
        const uint32_t b0 = A.base[v], cv = sp_class(A, v);
        for (int q = lane; q < SP_WIN / 32; q += 32) s_mask[wib][q] = 0u;
        __syncwarp();
        for (int64_t x = A.rp[v] + lane; x < A.rp[v + 1]; x += 32) {
            const uint32_t w = (uint32_t)A.ci[x];
            if (!sp_admitted(A, cv, w)) continue;
            const uint32_t cw = A.C[w];
            if (cw >= b0 && cw - b0 < A.W) atomicOr(&s_mask[wib][(cw - b0) >> 5], 1u << ((cw - b0) & 31));
        }
        __syncwarp();
        // first zero bit below W
        uint32_t first = 0xffffffffu;
        for (uint32_t q = lane; q * 32 < A.W; q += 32) {
            uint32_t free = ~s_mask[wib][q];
            const uint32_t lim = A.W - q * 32;
            if (lim < 32) free &= (1u << lim) - 1u;
            if (free) first = min(first, q * 32 + (uint32_t)(__ffs(free) - 1));
        }
        for (int d = 16; d; d >>= 1) first = min(first, __shfl_xor_sync(FULL, first, d));
        if (lane == 0) {
            if (first != 0xffffffffu) {
                A.T[v] = b0 + first;
            } else {
                A.T[v] = 0u;
                A.base[v] = b0 + A.W;  // "OFFSET": the next window, next round
            }
        }
        __syncwarp();
    }
}

// step 1 for the hubs (one CTA per vertex, the window mask in shared memory)
__global__ void __launch_bounds__(SP_HUGE_THREADS) k_spec_assign_huge(SpecArgs A, const uint32_t *__restrict__ hlist,
                                                                      const uint32_t *hcnt) {
    __shared__ uint32_t s_mask[SP_WIN / 32];
    __shared__ uint32_t s_first;
    const uint32_t c = *hcnt;
    for (uint32_t h = blockIdx.x; h < c; h += gridDim.x) {
        const uint32_t v = hlist[h];
        const uint32_t b0 = A.base[v], cv = sp_class(A, v);
        if (threadIdx.x < SP_WIN / 32) s_mask[threadIdx.x] = 0u;
        if (threadIdx.x == 0) s_first = 0xffffffffu;
        __syncthreads();
        for (int64_t x = A.rp[v] + threadIdx.x; x < A.rp[v + 1]; x += blockDim.x) {
            const uint32_t w = (uint32_t)A.ci[x];
            if (!sp_admitted(A, cv, w)) continue;
            const uint32_t cw = A.C[w];
            if (cw >= b0 && cw - b0 < A.W) atomicOr(&s_mask[(cw - b0) >> 5], 1u << ((cw - b0) & 31));
        }
        __syncthreads();
        if (threadIdx.x < SP_WIN / 32 && threadIdx.x * 32 < A.W) {
            uint32_t free = ~s_mask[threadIdx.x];
            const uint32_t lim = A.W - threadIdx.x * 32;
            if (lim < 32) free &= (1u << lim) - 1u;
            if (free) atomicMin(&s_first, threadIdx.x * 32 + (uint32_t)(__ffs(free) - 1));
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            if (s_first != 0xffffffffu) {
                A.T[v] = b0 + s_first;
            } else {
                A.T[v] = 0u;
                A.base[v] = b0 + A.W;
            }
        }
        __syncthreads();
    }
}

// commit the tentative colours (after every step-1 read of the snapshot)
__global__ void k_spec_commit(SpecArgs A, const uint32_t *__restrict__ list, const uint32_t *cnt) {
    const int64_t c = *cnt;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < c; i += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t v = list[i];
        A.C[v] = A.T[v];
    }
}

// step 2 (warp per listed vertex coloured this round): the lower-id end of every
// conflicting admitted edge is flagged; the first flag of a vertex appends it to the
// reset list
__device__ __forceinline__ void sp_flag(const SpecArgs &A, uint32_t u, uint32_t *rlist, uint32_t *rcnt) {
    // byte flags, claimed with a CAS on the containing 32-bit word (R is 256-B aligned)
    unsigned int *word = reinterpret_cast<unsigned int *>(A.R + (u & ~3u));
    const unsigned int sh = 8u * (u & 3u);
    unsigned int old = *reinterpret_cast<volatile unsigned int *>(word);
    while (!((old >> sh) & 0xffu)) {
        const unsigned int prev = atomicCAS(word, old, old | (1u << sh));
        if (prev == old) {
            rlist[atomicAdd(rcnt, 1u)] = u;
            return;
        }
        old = prev;
    }
}

__global__ void __launch_bounds__(SP_THREADS) k_spec_detect(SpecArgs A, const uint32_t *__restrict__ list,
                                                            const uint32_t *cnt, uint32_t *rlist, uint32_t *rcnt) {
    const int lane = lane_id();
    const int64_t c = *cnt, nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < c; i += nw) {
        const uint32_t v = list[i];
        const uint32_t col = A.C[v];
        if (col == 0u) continue;  // waited (window full)
        if (A.rp[v + 1] - A.rp[v] > SP_BUDGET) continue;  // a hub: k_spec_detect_huge
        const uint32_t cv = sp_class(A, v);
        bool self = false;
        for (int64_t x = A.rp[v] + lane; x < A.rp[v + 1]; x += 32) {
            const uint32_t w = (uint32_t)A.ci[x];
            if (A.C[w] != col || !sp_admitted(A, cv, w)) continue;
            if (w > v) self = true;
            else sp_flag(A, w, rlist, rcnt);  // a lower (maybe older) end
        }
        if (__any_sync(FULL, self) && lane == 0) sp_flag(A, v, rlist, rcnt);
    }
}

// step 2 for the hubs (one CTA per vertex of the hub list)
__global__ void __launch_bounds__(SP_HUGE_THREADS) k_spec_detect_huge(SpecArgs A, const uint32_t *__restrict__ hlist,
                                                                      const uint32_t *hcnt, uint32_t *rlist,
                                                                      uint32_t *rcnt) {
    const uint32_t c = *hcnt;
    for (uint32_t h = blockIdx.x; h < c; h += gridDim.x) {
        const uint32_t v = hlist[h];
        const uint32_t col = A.C[v];
        if (col == 0u) continue;  // uniform across the CTA
        const uint32_t cv = sp_class(A, v);
        bool self = false;
        for (int64_t x = A.rp[v] + threadIdx.x; x < A.rp[v + 1]; x += blockDim.x) {
            const uint32_t w = (uint32_t)A.ci[x];
            if (A.C[w] != col || !sp_admitted(A, cv, w)) continue;
            if (w > v) self = true;
            else sp_flag(A, w, rlist, rcnt);
        }
        if (__syncthreads_or(self) && threadIdx.x == 0) sp_flag(A, v, rlist, rcnt);
    }
}

// the next round's uncoloured list: the vertices that waited (window full; C == 0,
// never flagged) ...
__global__ void k_spec_next_wait(SpecArgs A, const uint32_t *__restrict__ list, const uint32_t *cnt, uint32_t *next,
                                 uint32_t *ncnt) {
    const int64_t c = *cnt, stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < c; base += stride) {
        const int64_t i = base + threadIdx.x;
        const uint32_t v = i < c ? list[i] : 0u;
        const int64_t slot = warp_append(i < c && A.C[v] == 0u, ncnt);
        if (slot >= 0) next[slot] = v;
    }
}

// ... and the reset ones (after the waiting ones were collected)
__global__ void k_spec_next_reset(SpecArgs A, const uint32_t *__restrict__ rlist, const uint32_t *rcnt, uint32_t *next,
                                  uint32_t *ncnt) {
    const int64_t c = *rcnt, stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < c; base += stride) {
        const int64_t i = base + threadIdx.x;
        const uint32_t v = i < c ? rlist[i] : 0u;
        if (i < c) {
            A.C[v] = 0u;
            A.R[v] = 0;
        }
        const int64_t slot = warp_append(i < c, ncnt);
        if (slot >= 0) next[slot] = v;
    }
}

// ---- COLOR-Degk's literal G_L loop (Alg 9 l.6): V_L starts at M+1; the lower-id end
// of every same-colour G_L edge moves to the smallest free slot of M+1 .. M+k+1
__global__ void k_gl_init(const uint32_t *__restrict__ hbits, int64_t n, const uint32_t *M, uint32_t *C) {
    const uint32_t m1 = *M + 1u;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
        if (!((hbits[v >> 5] >> (v & 31)) & 1u)) C[v] = m1;
}

__global__ void k_gl_round(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci,
                           const uint32_t *__restrict__ hbits, const int32_t *__restrict__ vlist, const uint32_t *cnt,
                           uint32_t k, const uint32_t *M, const uint32_t *C, uint32_t *T, uint32_t *moved) {
    const uint32_t m = *M;
    const int64_t c = *cnt, stride = (int64_t)gridDim.x * blockDim.x;
    uint32_t mv = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < c; i += stride) {
        const uint32_t v = (uint32_t)vlist[i];  // V_L vertex: degree <= k, one thread
        const uint32_t cv = C[v];
        bool conf = false;
        uint64_t used = 0;  // slots 1..k+1 (k + 1 <= 63)
        for (int64_t x = rp[v]; x < rp[v + 1]; x++) {
            const uint32_t w = (uint32_t)ci[x];
            if ((hbits[w >> 5] >> (w & 31)) & 1u) continue;  // G_L arcs only
            const uint32_t cw = C[w];
            conf |= w > v && cw == cv;
            if (cw > m && cw - m <= k + 1) used |= 1ull << (cw - m);
        }
        uint32_t t = cv;
        if (conf) {
            uint32_t s = 1;
            while (s <= k + 1 && ((used >> s) & 1ull)) s++;
            t = m + s;
            mv++;
        }
        T[v] = t;
    }
    mv = __reduce_add_sync(FULL, mv);
    if (lane_id() == 0 && mv) atomicAdd(moved, mv);
}

__global__ void k_gl_commit(const int32_t *__restrict__ vlist, const uint32_t *cnt, const uint32_t *T, uint32_t *C) {
    const int64_t c = *cnt;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < c; i += (int64_t)gridDim.x * blockDim.x)
        C[vlist[i]] = T[vlist[i]];
}

// uncoloured (C == 0) vertices -> list (the start of a speculative phase)
__global__ void k_spec_list(const uint32_t *C, int64_t n, uint32_t *list, uint32_t *cnt) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n; base += stride) {
        const int64_t v = base + threadIdx.x;
        cta_append2x(v < n && C[v] == 0u, false, (uint32_t)v, list, cnt, list, cnt);
    }
}

__global__ void k_spec_fill(uint32_t *a, int64_t n, uint32_t val) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) a[v] = val;
}

// admitted arcs (VB window = their number / n)
__global__ void k_spec_arcs(SpecArgs A, int64_t n, unsigned long long *out) {
    unsigned long long local = 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
        if (A.admit == SP_ALL) {
            local += (unsigned long long)(A.rp[v + 1] - A.rp[v]);
            continue;
        }
        const uint32_t cv = sp_class(A, (uint32_t)v);
        for (int64_t x = A.rp[v]; x < A.rp[v + 1]; x++) local += sp_admitted(A, cv, (uint32_t)A.ci[x]);
    }
    for (int d = 16; d; d >>= 1) local += __shfl_xor_sync(FULL, local, d);
    if (lane_id() == 0 && local) atomicAdd(out, local);
}

// ------------------------------------------------------------------ host side
// fix-up kernels of jp.cu
__global__ void k_color_max_h(const uint32_t *color, const uint32_t *hbits, int64_t n, uint32_t *mx);
__global__ void k_color_conflicts(const int64_t *__restrict__ rp_x, const int32_t *__restrict__ ci_x, int64_t n,
                                  const uint32_t *color, uint8_t *mark, int32_t *list, uint32_t *cnt, int lower,
                                  Key k, const uint32_t *okey, int ord);
__global__ void k_color_reset(const int32_t *list, const uint32_t *cnt, uint32_t *color);
__global__ void k_color_max(const uint32_t *color, int64_t n, uint32_t *mx);

static int sp_grid(int64_t items, int per_cta) {
    int64_t want = (items + per_cta - 1) / per_cta, cap = (int64_t)num_sms() * 8;
    return (int)(want < 1 ? 1 : (want < cap ? want : cap));
}

// one speculative phase: every vertex with C == 0 is coloured
static int spec_phase(const FlowArgs &f, ColorWs &w, SpecArgs A, int vb, int phase) {
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
    const int64_t n = f.g.n;
    A.W = 32;
    if (vb) {  // VB: the FORBIDDEN window = the average degree of the graph being coloured
        SYM_CUDA(cudaMemsetAsync(&ctl->result, 0, sizeof(uint64_t), s));
        k_spec_arcs<<<num_sms() * 8, 256, 0, s>>>(A, n, (unsigned long long *)&ctl->result);
        SYM_LAUNCH_CHECK();
        uint64_t arcs = 0;
        SYM_TRY(read_u64(&ctl->result, &arcs, s));
        const int64_t avg = n > 0 ? (int64_t)arcs / n : 1;
        A.W = (uint32_t)std::min<int64_t>(SP_WIN, std::max<int64_t>(1, avg));
    }
    k_spec_fill<<<num_sms() * 8, 256, 0, s>>>(A.base, n, 1u);
    SYM_LAUNCH_CHECK();
    SYM_CUDA(cudaMemsetAsync(A.R, 0, (size_t)n + 1, s));
    uint32_t *cnt[2] = {&ctl->ring[0], &ctl->ring[1]};
    uint32_t *rcnt = &ctl->ring[2];
    SYM_CUDA(cudaMemsetAsync(cnt[0], 0, sizeof(uint32_t), s));
    k_spec_list<<<num_sms() * 8, 256, 0, s>>>(A.C, n, w.ul[0], cnt[0]);
    SYM_LAUNCH_CHECK();
    uint32_t left = 0;
    SYM_TRY(read_u32(cnt[0], &left, s));
    const uint32_t maxr = f.p.max_rounds ? f.p.max_rounds : 0xffffffffu;
    uint32_t r = 0;
    for (; left > 0; r++) {
        if (r >= maxr) {
            set_error("speculative colouring did not converge within max_rounds");
            return SYM_EROUNDS;
        }
        uint32_t *list = w.ul[r & 1], *next = w.ul[(r + 1) & 1];
        SYM_CUDA(cudaMemsetAsync(cnt[(r + 1) & 1], 0, sizeof(uint32_t), s));
        SYM_CUDA(cudaMemsetAsync(rcnt, 0, sizeof(uint32_t), s));
        uint32_t *hlist = reinterpret_cast<uint32_t *>(w.queue), *hcnt = &ctl->huge[0];
        SYM_CUDA(cudaMemsetAsync(hcnt, 0, sizeof(uint32_t), s));
        k_spec_assign<<<sp_grid(left, SP_WARPS), SP_THREADS, 0, s>>>(A, list, cnt[r & 1], hlist, hcnt);
        SYM_LAUNCH_CHECK();
        k_spec_assign_huge<<<num_sms() * 2, SP_HUGE_THREADS, 0, s>>>(A, hlist, hcnt);
        SYM_LAUNCH_CHECK();
        k_spec_commit<<<sp_grid(left, 256), 256, 0, s>>>(A, list, cnt[r & 1]);
        SYM_LAUNCH_CHECK();
        k_spec_detect<<<sp_grid(left, SP_WARPS), SP_THREADS, 0, s>>>(A, list, cnt[r & 1],
                                                                     reinterpret_cast<uint32_t *>(w.ov), rcnt);
        SYM_LAUNCH_CHECK();
        k_spec_detect_huge<<<num_sms() * 2, SP_HUGE_THREADS, 0, s>>>(A, hlist, hcnt, reinterpret_cast<uint32_t *>(w.ov),
                                                                    rcnt);
        SYM_LAUNCH_CHECK();
        k_spec_next_wait<<<sp_grid(left, 256), 256, 0, s>>>(A, list, cnt[r & 1], next, cnt[(r + 1) & 1]);
        SYM_LAUNCH_CHECK();
        k_spec_next_reset<<<num_sms() * 4, 256, 0, s>>>(A, reinterpret_cast<uint32_t *>(w.ov), rcnt, next,
                                                        cnt[(r + 1) & 1]);
        SYM_LAUNCH_CHECK();
        SYM_TRY(read_u32(cnt[(r + 1) & 1], &left, s));
    }
    if (f.stats && phase < 3) f.stats->rounds[phase] = r;
    return SYM_OK;
}

int run_color_spec(const FlowArgs &f, ColorWs &w, uint32_t *color) {
    const Graph &g = f.g;
    cudaStream_t s = f.stream;
    Ctl *ctl = f.ctl;
    const int kind = f.p.kind;
    const int vb = (f.p.flags & SYM_F_COLOR_VB) ? 1 : 0;
    SpecArgs A;
    A.rp = g.rp;
    A.ci = g.ci;
    A.admit = SP_ALL;
    A.kind = kind;
    A.param = f.p.param;
    A.kr = stream_key(f.p.seed, TAG_RAND, 0);
    A.hbits = f.hbits;
    A.W = 32;
    A.C = color;
    A.T = w.hdeg;
    A.base = w.ldeg;
    A.R = w.mark;
    SYM_CUDA(cudaMemsetAsync(color, 0, sizeof(uint32_t) * (size_t)g.n, s));
    if (kind == SYM_DECOMP_NONE) {
        SYM_TRY(spec_phase(f, w, A, vb, 0));
    } else if (kind == SYM_DECOMP_DEGK) {
        // C_H on G_H (V_L parked at a non-zero colour: not in the H rounds' lists, and the
        // H rounds admit H-H arcs only), then the G_L loop.  V_L list at the front of vlist.
        SYM_CUDA(cudaMemsetAsync(&ctl->cnt_front, 0, 2 * sizeof(uint32_t), s));
        SYM_TRY(launch_classify_degk(g, f.p.param, f.hbits, w.vlist, ctl, s));
        SYM_CUDA(cudaMemsetAsync(&ctl->max_color, 0, sizeof(uint32_t), s));
        k_gl_init<<<num_sms() * 8, 256, 0, s>>>(f.hbits, g.n, &ctl->max_color, color);  // park V_L at 0 + 1
        SYM_LAUNCH_CHECK();
        A.admit = SP_HH;
        SYM_TRY(spec_phase(f, w, A, vb, 0));
        SYM_CUDA(cudaMemsetAsync(&ctl->max_color, 0, sizeof(uint32_t), s));
        k_color_max_h<<<num_sms() * 8, 256, 0, s>>>(color, f.hbits, g.n, &ctl->max_color);
        SYM_LAUNCH_CHECK();
        k_gl_init<<<num_sms() * 8, 256, 0, s>>>(f.hbits, g.n, &ctl->max_color, color);
        SYM_LAUNCH_CHECK();
        uint32_t nl = 0;
        SYM_TRY(read_u32(&ctl->cnt_front, &nl, s));
        uint32_t r = 0;
        for (; nl > 0; r++) {
            if (f.p.max_rounds && r >= f.p.max_rounds) {
                set_error("the G_L loop did not converge within max_rounds");
                return SYM_EROUNDS;
            }
            SYM_CUDA(cudaMemsetAsync(&ctl->conflicts, 0, sizeof(uint32_t), s));
            k_gl_round<<<sp_grid(nl, 256), 256, 0, s>>>(g.rp, g.ci, f.hbits, w.vlist, &ctl->cnt_front, f.p.param,
                                                       &ctl->max_color, color, w.hdeg, &ctl->conflicts);
            SYM_LAUNCH_CHECK();
            uint32_t moved = 0;
            SYM_TRY(read_u32(&ctl->conflicts, &moved, s));
            if (!moved) break;
            k_gl_commit<<<sp_grid(nl, 256), 256, 0, s>>>(w.vlist, &ctl->cnt_front, w.hdeg, color);
            SYM_LAUNCH_CHECK();
        }
        if (f.stats) f.stats->rounds[1] = r;
    } else {
        // C_IS on the parts; V' (both ends, or the lower ends); recolour against G
        A.admit = SP_SAME;
        SYM_TRY(spec_phase(f, w, A, vb, 0));
        SYM_CUDA(cudaMemsetAsync(&ctl->conflicts, 0, sizeof(uint32_t), s));
        k_color_conflicts<<<num_sms() * 8, 256, 0, s>>>(f.split.rp_x, f.split.ci_x, g.n, color, w.mark, w.vlist,
                                                          &ctl->conflicts, (f.p.flags & SYM_F_LOWER_ONLY) ? 1 : 0,
                                                          stream_key(f.p.seed, TAG_VERTEX, 0), nullptr, 0);
        SYM_LAUNCH_CHECK();
        k_color_reset<<<num_sms() * 4, 256, 0, s>>>(w.vlist, &ctl->conflicts, color);
        SYM_LAUNCH_CHECK();
        A.admit = SP_ALL;
        SYM_TRY(spec_phase(f, w, A, vb, 1));
    }
    if (f.stats) {
        SYM_CUDA(cudaMemsetAsync(&ctl->flag, 0, sizeof(uint32_t), s));
        k_color_max<<<num_sms() * 8, 256, 0, s>>>(color, g.n, &ctl->flag);
        SYM_LAUNCH_CHECK();
        uint32_t mx = 0, conf = 0;
        SYM_TRY(read_u32(&ctl->flag, &mx, s));
        f.stats->max_color = mx;
        f.stats->result_size = mx;
        if (kind == SYM_DECOMP_RAND) {
            SYM_TRY(read_u32(&ctl->conflicts, &conf, s));
            f.stats->conflicts = conf;
        }
    }
    return SYM_OK;
}

}  // namespace sym
