// color.cu -- Jones-Plassmann colouring and the COLOR flows.
//
// JP ([18]) with fixed priorities colours v once every higher-(pv,id)
// neighbour of its phase set S is coloured, with the smallest colour >= 1 not held by
// any coloured neighbour: exactly first-fit greedy in priority order (DESIGN §3 C1).
// Work-efficient push form:
//   init   cnt[v] = #higher neighbours of v in S; cnt == 0 -> ready frontier F_0
//   round  for v in F_r: one pass over v's row: gather neighbour colours for the mex
//          (lower S-neighbours are still uncoloured; vertices outside S are fixed
//          constraints), and decrement cnt[w] of every lower S-neighbour w; the
//          decrement that reaches 0 appends w to F_{r+1}.
// Each arc is read twice in total (init + colouring pass).  Rows: lane-serial up
// to JP_SMALL arcs (one 64-bit colour window suffices since mex <= deg+1), warp with
// a (deg+1)-bit shared-memory bitmap up to JP_BUDGET, CTA kernel beyond.
#include "internal.h"

namespace sym {

constexpr int JP_SMALL = 32;
constexpr int JP_BUDGET = 4096;
constexpr int JP_THREADS = 256;
constexpr int JP_HUGE_THREADS = 512;
constexpr int JP_WARP_WORDS = (JP_BUDGET + 1 + 31) / 32 + 1;  // bitmap words per warp
constexpr int JP_HUGE_WORDS = 16384 / 32;                      // CTA window (colours)

struct JpArgs {
    const int64_t *rp;
    const int32_t *ci;
    const uint8_t *inS;  // nullable: S = all vertices
    uint32_t *color;
    uint32_t *cnt;
    const int32_t *in_list;
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
};

__device__ __forceinline__ bool in_set(const uint8_t *inS, uint32_t w) { return inS == nullptr || inS[w] != 0; }

// ---------------------------------------------------------------- init: pending counts
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
                c += (in_set(A.inS, w) && vkey(A.k, w) > kv) ? 1u : 0u;
            }
        }
        unsigned medm = __ballot_sync(FULL, active && e - b > JP_SMALL && e - b <= JP_BUDGET);
        while (medm) {
            const int src = __ffs(medm) - 1;
            medm &= medm - 1;
            const int64_t wb = __shfl_sync(FULL, b, src), we = __shfl_sync(FULL, e, src);
            const uint64_t wk = __shfl_sync(FULL, kv, src);
            uint32_t lc = 0;
            for (int64_t x = wb + lane; x < we; x += 32) {
                uint32_t w = (uint32_t)__ldg(A.ci + x);
                lc += (in_set(A.inS, w) && vkey(A.k, w) > wk) ? 1u : 0u;
            }
            for (int d = 16; d; d >>= 1) lc += __shfl_xor_sync(FULL, lc, d);
            if (lane == src) c = lc;
        }
        bool huge = active && e - b > JP_BUDGET;
        if (active && !huge) A.cnt[v] = c;
        int64_t slot = warp_append(active && !huge && c == 0, A.out_cnt);
        if (slot >= 0) A.out_list[slot] = v;
        int64_t hs = warp_append(huge, A.huge_cnt);
        if (hs >= 0) A.huge[hs] = v;
    }
}

__global__ void __launch_bounds__(JP_HUGE_THREADS) k_jp_init_huge(JpArgs A) {
    const uint32_t cnt = *A.huge_cnt;
    __shared__ uint32_t s_sum;
    for (uint32_t h = blockIdx.x; h < cnt; h += gridDim.x) {
        const int32_t v = A.huge[h];
        const int64_t b = A.rp[v], e = A.rp[v + 1];
        const uint64_t kv = vkey(A.k, (uint32_t)v);
        if (threadIdx.x == 0) s_sum = 0;
        __syncthreads();
        uint32_t lc = 0;
        for (int64_t x = b + threadIdx.x; x < e; x += JP_HUGE_THREADS) {
            uint32_t w = (uint32_t)__ldg(A.ci + x);
            lc += (in_set(A.inS, w) && vkey(A.k, w) > kv) ? 1u : 0u;
        }
        for (int d = 16; d; d >>= 1) lc += __shfl_xor_sync(FULL, lc, d);
        if (lane_id() == 0) atomicAdd(&s_sum, lc);
        __syncthreads();
        if (threadIdx.x == 0) {
            A.cnt[v] = s_sum;
            if (s_sum == 0) {
                uint32_t slot = atomicAdd(A.out_cnt, 1u);
                A.out_list[slot] = v;
            }
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------- colouring rounds
__device__ __forceinline__ void jp_push(const JpArgs &A, uint32_t w, uint64_t kv, bool &ready) {
    ready = false;
    if (in_set(A.inS, w) && vkey(A.k, w) < kv) ready = atomicSub(&A.cnt[w], 1u) == 1u;
}

__global__ void __launch_bounds__(JP_THREADS) k_jp_round(JpArgs A) {
    __shared__ uint32_t s_bits[JP_THREADS / 32][JP_WARP_WORDS];
    const uint32_t cnt = *A.in_cnt;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        *A.clear_cnt = 0;
        *A.huge_clear = 0;
        if (A.hist && A.round < 2048) A.hist[A.round] = cnt;
    }
    const int lane = lane_id(), warp = threadIdx.x >> 5;
    uint32_t *bits = s_bits[warp];
    const int64_t warp_g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = warp_g * 32; base < cnt; base += nwarps * 32) {
        int64_t i = base + lane;
        int32_t v = -1;
        if (i < cnt) v = A.in_list[i];
        bool active = v >= 0;
        int64_t b = 0, e = 0;
        uint64_t kv = 0;
        if (active) {
            b = A.rp[v];
            e = A.rp[v + 1];
            kv = vkey(A.k, (uint32_t)v);
        }
        // lane-serial: colours 1..64 window (mex <= deg + 1 <= 33)
        if (active && e - b <= JP_SMALL) {
            uint64_t used = 0;
            for (int64_t x = b; x < e; x++) {
                uint32_t w = (uint32_t)__ldg(A.ci + x);
                uint32_t c = A.color[w];
                if (c >= 1 && c <= 64) used |= 1ULL << (c - 1);
                bool ready;
                jp_push(A, w, kv, ready);
                if (ready) {
                    // rare enough to append one by one (frontier order is irrelevant)
                    uint32_t slot = atomicAdd(A.out_cnt, 1u);
                    A.out_list[slot] = (int32_t)w;
                }
            }
            A.color[v] = (uint32_t)__ffsll((long long)~used);
        }
        // warp-cooperative: (deg+1)-bit bitmap in shared memory
        unsigned medm = __ballot_sync(FULL, active && e - b > JP_SMALL && e - b <= JP_BUDGET);
        while (medm) {
            const int src = __ffs(medm) - 1;
            medm &= medm - 1;
            const int64_t wb = __shfl_sync(FULL, b, src), we = __shfl_sync(FULL, e, src);
            const uint64_t wk = __shfl_sync(FULL, kv, src);
            const int32_t wv = __shfl_sync(FULL, v, src);
            const int nwords = (int)((we - wb + 1 + 31) / 32) + 1;
            for (int q = lane; q < nwords; q += 32) bits[q] = 0;
            __syncwarp();
            const uint32_t cap = (uint32_t)(we - wb + 1);
            for (int64_t x = wb; x < we; x += 32) {
                int64_t y = x + lane;
                bool ready = false;
                uint32_t w = 0;
                if (y < we) {
                    w = (uint32_t)__ldg(A.ci + y);
                    uint32_t c = A.color[w];
                    if (c >= 1 && c <= cap) atomicOr(&bits[(c - 1) >> 5], 1u << ((c - 1) & 31));
                    jp_push(A, w, wk, ready);
                }
                int64_t slot = warp_append(ready, A.out_cnt);
                if (slot >= 0) A.out_list[slot] = (int32_t)w;
            }
            __syncwarp();
            // mex: first zero bit
            uint32_t mex = 0;
            for (int q0 = 0; q0 < nwords && !mex; q0 += 32) {
                int q = q0 + lane;
                uint32_t word = (q < nwords) ? bits[q] : 0u;
                unsigned nf = __ballot_sync(FULL, word != 0xffffffffu);
                if (nf) {
                    int ql = __ffs(nf) - 1;
                    uint32_t wd = __shfl_sync(FULL, word, ql);
                    mex = (uint32_t)(q0 + ql) * 32 + (uint32_t)__ffs(~wd);
                }
            }
            if (lane == 0) A.color[wv] = mex;
            __syncwarp();
        }
        int64_t hs = warp_append(active && e - b > JP_BUDGET, A.huge_cnt);
        if (hs >= 0) A.huge[hs] = v;
    }
}

__global__ void __launch_bounds__(JP_HUGE_THREADS) k_jp_round_huge(JpArgs A) {
    __shared__ uint32_t s_bits[JP_HUGE_WORDS];
    __shared__ uint32_t s_mex;
    const uint32_t cnt = *A.huge_cnt;
    for (uint32_t h = blockIdx.x; h < cnt; h += gridDim.x) {
        const int32_t v = A.huge[h];
        const int64_t b = A.rp[v], e = A.rp[v + 1];
        const uint64_t kv = vkey(A.k, (uint32_t)v);
        // pass 1: decrements of lower S-neighbours (independent of the colour)
        for (int64_t x0 = b; x0 < e; x0 += JP_HUGE_THREADS) {  // uniform trip count for warp_append
            int64_t x = x0 + threadIdx.x;
            uint32_t w = 0;
            bool ready = false;
            if (x < e) {
                w = (uint32_t)__ldg(A.ci + x);
                jp_push(A, w, kv, ready);
            }
            int64_t slot = warp_append(ready, A.out_cnt);
            if (slot >= 0) A.out_list[slot] = (int32_t)w;
        }
        // pass 2: mex in windows of JP_HUGE_WORDS*32 colours
        uint32_t c0 = 1;
        for (;;) {
            for (int q = threadIdx.x; q < JP_HUGE_WORDS; q += JP_HUGE_THREADS) s_bits[q] = 0;
            if (threadIdx.x == 0) s_mex = 0;
            __syncthreads();
            for (int64_t x = b + threadIdx.x; x < e; x += JP_HUGE_THREADS) {
                uint32_t c = A.color[__ldg(A.ci + x)];
                if (c >= c0 && c < c0 + JP_HUGE_WORDS * 32) {
                    uint32_t o = c - c0;
                    atomicOr(&s_bits[o >> 5], 1u << (o & 31));
                }
            }
            __syncthreads();
            if (threadIdx.x == 0) {
                uint32_t m = 0;
                for (int q = 0; q < JP_HUGE_WORDS; q++)
                    if (s_bits[q] != 0xffffffffu) {
                        m = c0 + (uint32_t)q * 32 + (uint32_t)__ffs(~s_bits[q]) - 1;
                        break;
                    }
                s_mex = m;
            }
            __syncthreads();
            uint32_t m = s_mex;
            __syncthreads();
            if (m) {
                if (threadIdx.x == 0) A.color[v] = m;
                break;
            }
            c0 += JP_HUGE_WORDS * 32;
        }
        __syncthreads();
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
    w.queue = a.take<int32_t>(2 * ((size_t)n + 1));  // frontier ping-pong
    w.vlist = a.take<int32_t>((size_t)n + 1);
    w.mark = a.take<uint8_t>((size_t)n + 1);
    w.task = a.take<int64_t>((size_t)(nnz / JP_BUDGET + 2));
    w.queue_cap = n + 1;
}

// JP over (rp, ci) for the vertex set S (list/implicit) with membership inS
static int jp_run(const FlowArgs &f, ColorWs &w, uint32_t *color, const int64_t *rp, const int32_t *ci,
                  const uint8_t *inS, const int32_t *list0, const uint32_t *cnt0, int64_t implicit_n, int phase) {
    Ctl *ctl = f.ctl;
    cudaStream_t s = f.stream;
    const Key k = stream_key(f.p.seed, TAG_VERTEX, 0);
    int32_t *fr[2] = {w.queue, w.queue + w.queue_cap};
    int32_t *huge = reinterpret_cast<int32_t *>(w.task);
    SYM_CUDA(cudaMemsetAsync(ctl->ring, 0, sizeof(ctl->ring) + sizeof(ctl->huge), s));
    const int grid = num_sms() * (2048 / JP_THREADS);
    JpArgs A;
    A.rp = rp;
    A.ci = ci;
    A.inS = inS;
    A.color = color;
    A.cnt = w.cnt;
    A.k = k;
    A.huge = huge;
    A.hist = ctl->hist + phase * 2048;
    // init: round index -1 writes F_0 into fr[0] with count ring[0]
    A.in_list = list0;
    A.in_cnt = cnt0;
    A.implicit_n = implicit_n;
    A.out_list = fr[0];
    A.out_cnt = &ctl->ring[0];
    A.clear_cnt = &ctl->ring[2];
    A.huge_cnt = &ctl->huge[1];
    A.huge_clear = &ctl->huge[0];
    A.round = 0;
    prof_begin("jp_init", s);
    k_jp_init<<<grid, JP_THREADS, 0, s>>>(A);
    SYM_LAUNCH_CHECK();
    k_jp_init_huge<<<num_sms() * 2, JP_HUGE_THREADS, 0, s>>>(A);
    prof_end(s, -1);
    SYM_LAUNCH_CHECK();
    const uint32_t maxr = f.p.max_rounds ? f.p.max_rounds : 0xffffffffu;
    int r = 0, batch = 8;
    for (;;) {
        for (int bb = 0; bb < batch; bb++, r++) {
            A.in_list = fr[r & 1];
            A.in_cnt = &ctl->ring[r % 3];
            A.out_list = fr[(r + 1) & 1];
            A.out_cnt = &ctl->ring[(r + 1) % 3];
            A.clear_cnt = &ctl->ring[(r + 2) % 3];
            A.huge_cnt = &ctl->huge[r & 1];
            A.huge_clear = &ctl->huge[(r + 1) & 1];
            A.round = r < 2048 ? r : 2047;
            prof_begin("jp_round", s);
            k_jp_round<<<grid, JP_THREADS, 0, s>>>(A);
            prof_end(s, -1);
            SYM_LAUNCH_CHECK();
            prof_begin("jp_huge", s);
            k_jp_round_huge<<<num_sms() * 2, JP_HUGE_THREADS, 0, s>>>(A);
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
