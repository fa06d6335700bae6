// bridge.cu -- the BRIDGE decomposition (Alg 1; SURVEY §8(f) f4;
// include/sym.h SYM_DECOMP_BRIDGE).
//
//   1. a BFS forest T (Alg 1 l.2, "we take an arbitrary vertex r as root and perform a
//      parallel BFS"): one root per connected component -- its smallest id, from a
//      hook-and-compress connected-components pass -- and level-synchronous BFS from
//      all roots at once; P(v) = the smallest-id neighbour one level up (deterministic);
//   2. for every non-tree edge {x, y}, the tree edges on the paths from x and y up to
//      their least common ancestor are marked (l.3-4: "walking up the tree towards the
//      root from x and y in parallel");
//   3. the unmarked tree edges are the bridges B (l.6-7); G_1, G_2, .. (l.8) are what
//      remains: the split puts the non-bridge arcs in the intra CSR and the bridges in
//      the cross CSR (two passes: per-row counts, a scan, a scatter), so MM-Bridge (Alg 4),
// COLOR-Bridge (Alg 7) and MIS-Bridge (Alg 10) run as the RAND flows on it.  Every
// output is a function of the graph only (BFS levels and the min-id parent / component
// rules are schedule-independent) -- bit-identical to the oracle's bridges / classes.
#include "internal.h"

namespace sym {

constexpr int BR_THREADS = 256;

__device__ __forceinline__ int32_t cc_find(int32_t *p, int32_t v) {
    while (true) {  // path halving (pointers only move towards the root)
        const int32_t q = p[v];
        if (q == v) return v;
        const int32_t g = p[q];
        p[v] = g;
        v = g;
    }
}

// the arc (u, w) is a bridge: the tree edge of u's parent or of w's parent, unmarked
__device__ __forceinline__ bool br_is_bridge(const int32_t *par, const uint8_t *mark, int32_t u, int32_t w) {
    return (par[u] == w && !mark[u]) || (par[w] == u && !mark[w]);
}

// hook: for every arc u < w the larger root points to the smaller one (so each
// component's root ends as its smallest id)
__global__ void __launch_bounds__(BR_THREADS) k_cc_hook(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci,
                                                        int64_t n, int32_t *p, uint32_t *changed) {
    const int lane = lane_id();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    bool ch = false;
    for (int64_t u = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; u < n; u += nw) {
        for (int64_t x = rp[u] + lane; x < rp[u + 1]; x += 32) {
            const int32_t w = ci[x];
            if (w <= u) continue;
            while (true) {
                int32_t ru = cc_find(p, (int32_t)u), rw = cc_find(p, w);
                if (ru == rw) break;
                const int32_t hi = max(ru, rw), lo = min(ru, rw);
                if (atomicCAS(p + hi, hi, lo) == hi) {
                    ch = true;
                    break;
                }
            }
        }
    }
    if (__any_sync(FULL, ch) && lane == 0) *changed = 1u;
}

__global__ void k_cc_compress(int32_t *p, int64_t n) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) p[v] = cc_find(p, (int32_t)v);
}

__global__ void k_cc_init(int32_t *p, int64_t n) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) p[v] = (int32_t)v;
}

// BFS roots: the smallest id of every component with an edge (level 0)
__global__ void k_br_roots(const int64_t *__restrict__ rp, const int32_t *__restrict__ cc, int64_t n, int32_t *level,
                           int32_t *list, uint32_t *cnt) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n; base += stride) {
        const int64_t v = base + threadIdx.x;
        bool root = false;
        if (v < n) {
            root = cc[v] == (int32_t)v && rp[v + 1] > rp[v];
            level[v] = root ? 0 : -1;
        }
        const int64_t slot = warp_append(root, cnt);
        if (slot >= 0) list[slot] = (int32_t)v;
    }
}

// one BFS level (warp per frontier vertex): unvisited neighbours get level L + 1
__global__ void __launch_bounds__(BR_THREADS) k_br_bfs(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci,
                                                       const int32_t *__restrict__ list, const uint32_t *cnt, int32_t L,
                                                       int32_t *level, int32_t *next, uint32_t *ncnt) {
    const int lane = lane_id();
    const int64_t c = *cnt, nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < c; i += nw) {
        const int32_t u = list[i];
        const int64_t e = rp[u + 1];
        for (int64_t x0 = rp[u]; x0 < e; x0 += 32) {
            const int64_t x = x0 + lane;
            bool take = false;
            int32_t w = 0;
            if (x < e) {
                w = ci[x];
                take = level[w] == -1 && atomicCAS(level + w, -1, L + 1) == -1;
            }
            const int64_t slot = warp_append(take, ncnt);
            if (slot >= 0) next[slot] = w;
        }
    }
}

// P(v) = the smallest-id neighbour one level up (roots and isolated vertices: -1)
__global__ void __launch_bounds__(BR_THREADS) k_br_parent(const int64_t *__restrict__ rp,
                                                          const int32_t *__restrict__ ci, int64_t n,
                                                          const int32_t *__restrict__ level, int32_t *par,
                                                          uint8_t *mark) {
    const int lane = lane_id();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; v < n; v += nw) {
        const int32_t lv = level[v];
        int32_t best = 0x7fffffff;
        if (lv > 0)
            for (int64_t x = rp[v] + lane; x < rp[v + 1]; x += 32) {
                const int32_t w = ci[x];
                if (level[w] == lv - 1) best = min(best, w);
            }
        for (int d = 16; d; d >>= 1) best = min(best, __shfl_xor_sync(FULL, best, d));
        if (lane == 0) {
            par[v] = best == 0x7fffffff ? -1 : best;
            mark[v] = 0;
        }
    }
}

// Alg 1 l.3-4: every non-tree edge {x, y} (x < y) marks the tree edges up to the LCA
// (mark[v] = 1: the tree edge (v, P(v)) lies on a cycle)
__global__ void __launch_bounds__(BR_THREADS) k_br_mark(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci,
                                                        int64_t n, const int32_t *__restrict__ level,
                                                        const int32_t *__restrict__ par, uint8_t *mark) {
    const int lane = lane_id();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t u = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; u < n; u += nw) {
        for (int64_t xx = rp[u] + lane; xx < rp[u + 1]; xx += 32) {
            int32_t y = ci[xx], x = (int32_t)u;
            if (y <= x || par[x] == y || par[y] == x) continue;  // each non-tree edge once
            while (x != y) {
                const int32_t lx = level[x], ly = level[y];
                if (lx >= ly) {
                    mark[x] = 1;
                    x = par[x];
                }
                if (ly >= lx) {
                    mark[y] = 1;
                    y = par[y];
                }
            }
        }
    }
}

// ---- the split (two passes): per-row intra counts -> scan -> scatter
__global__ void __launch_bounds__(BR_THREADS) k_br_count(const int64_t *__restrict__ rp,
                                                         const int32_t *__restrict__ ci, int64_t n,
                                                         const int32_t *__restrict__ par,
                                                         const uint8_t *__restrict__ mark, int64_t *cnt) {
    const int lane = lane_id();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; v < n; v += nw) {
        int64_t c = 0;
        for (int64_t x = rp[v] + lane; x < rp[v + 1]; x += 32) c += !br_is_bridge(par, mark, (int32_t)v, ci[x]);
        for (int d = 16; d; d >>= 1) c += __shfl_xor_sync(FULL, c, d);
        if (lane == 0) cnt[v] = c;
    }
}

// exclusive scan of n int64 counts in place into out[0..n] (out[n] = total): per-block
// sums, one block scanning the sums, then the blocks' own scans
constexpr int BR_SCAN = 1024;
__global__ void __launch_bounds__(BR_SCAN) k_br_scan_blocks(const int64_t *in, int64_t n, int64_t *bsum) {
    __shared__ int64_t sm[32];
    const int64_t i = (int64_t)blockIdx.x * BR_SCAN + threadIdx.x;
    int64_t x = i < n ? in[i] : 0;
    for (int d = 16; d; d >>= 1) x += __shfl_xor_sync(FULL, x, d);
    if (lane_id() == 0) sm[threadIdx.x >> 5] = x;
    __syncthreads();
    if (threadIdx.x == 0) {
        int64_t t = 0;
        for (int q = 0; q < BR_SCAN / 32; q++) t += sm[q];
        bsum[blockIdx.x] = t;
    }
}

__global__ void __launch_bounds__(BR_SCAN) k_br_scan_sums(int64_t *bsum, int64_t nb) {
    __shared__ int64_t sm[32];
    const int64_t per = (nb + BR_SCAN - 1) / BR_SCAN;
    const int64_t b0 = (int64_t)threadIdx.x * per, b1 = min(nb, b0 + per);
    int64_t s = 0;
    for (int64_t b = b0; b < b1; b++) s += bsum[b];
    int64_t incl = s;
    for (int d = 1; d < 32; d <<= 1) {
        const int64_t y = __shfl_up_sync(FULL, incl, d);
        if (lane_id() >= d) incl += y;
    }
    if (lane_id() == 31) sm[threadIdx.x >> 5] = incl;
    __syncthreads();
    int64_t before = 0;
    for (int q = 0; q < (int)(threadIdx.x >> 5); q++) before += sm[q];
    int64_t o = before + incl - s;
    for (int64_t b = b0; b < b1; b++) {
        const int64_t a = bsum[b];
        bsum[b] = o;
        o += a;
    }
}

__global__ void __launch_bounds__(BR_SCAN) k_br_scan_apply(int64_t *io, int64_t n, const int64_t *bsum) {
    __shared__ int64_t sm[32];
    const int64_t i = (int64_t)blockIdx.x * BR_SCAN + threadIdx.x;
    const int64_t x = i < n ? io[i] : 0;
    int64_t incl = x;
    for (int d = 1; d < 32; d <<= 1) {
        const int64_t y = __shfl_up_sync(FULL, incl, d);
        if (lane_id() >= d) incl += y;
    }
    if (lane_id() == 31) sm[threadIdx.x >> 5] = incl;
    __syncthreads();
    int64_t before = 0;
    for (int q = 0; q < (int)(threadIdx.x >> 5); q++) before += sm[q];
    const int64_t excl = bsum[blockIdx.x] + before + incl - x;
    __syncthreads();
    if (i < n) io[i] = excl;
    if (i == n - 1) io[n] = excl + x;
}

// scatter: row v's non-bridge arcs to ci_in[rp_in[v]..], bridges to ci_x[rp_x[v]..]
// (rp_x[v] = rp[v] - rp_in[v]), both in input order
__global__ void __launch_bounds__(BR_THREADS) k_br_scatter(const int64_t *__restrict__ rp,
                                                           const int32_t *__restrict__ ci, int64_t n,
                                                           const int32_t *__restrict__ par,
                                                           const uint8_t *__restrict__ mark,
                                                           const int64_t *__restrict__ rp_in, int32_t *ci_in,
                                                           int64_t *rp_x, int32_t *ci_x) {
    const int lane = lane_id();
    const unsigned lt = (1u << lane) - 1u;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; v <= n; v += nw) {
        if (v == n) {
            if (lane == 0) rp_x[n] = rp[n] - rp_in[n];
            continue;
        }
        int64_t oi = rp_in[v], ox = rp[v] - rp_in[v];
        if (lane == 0) rp_x[v] = ox;
        for (int64_t x0 = rp[v]; x0 < rp[v + 1]; x0 += 32) {
            const int64_t x = x0 + lane;
            const bool ok = x < rp[v + 1];
            const int32_t w = ok ? ci[x] : 0;
            const bool intra = ok && !br_is_bridge(par, mark, (int32_t)v, w);
            const unsigned mi = __ballot_sync(FULL, intra), mx = __ballot_sync(FULL, ok && !intra);
            if (intra) ci_in[oi + __popc(mi & lt)] = w;
            else if (ok) ci_x[ox + __popc(mx & lt)] = w;
            oi += __popc(mi);
            ox += __popc(mx);
        }
    }
}

// optional label output: 1 for the endpoints of a bridge, else 0 (the component ids
// of G - B do not fit 16 bits)
__global__ void __launch_bounds__(BR_THREADS) k_br_labels(const int64_t *__restrict__ rp_x, int64_t n,
                                                          uint16_t *label) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
        label[v] = rp_x[v + 1] > rp_x[v] ? 1 : 0;
}

// ------------------------------------------------------------------ host side
void carve_bridge_ws(Arena &a, int64_t n, BridgeWs &w) {
    w.cc = a.take<int32_t>((size_t)n + 1);
    w.level = a.take<int32_t>((size_t)n + 1);
    w.par = a.take<int32_t>((size_t)n + 1);
    w.mark = a.take<uint8_t>((size_t)n + 1);
    w.fr[0] = a.take<int32_t>((size_t)n + 1);
    w.fr[1] = a.take<int32_t>((size_t)n + 1);
    w.bsum = a.take<int64_t>((size_t)(n / BR_SCAN + 2));
    w.ctr = a.take<uint32_t>(8);
}

static int br_grid(int64_t items, int per) {
    int64_t want = (items + per - 1) / per, cap = (int64_t)num_sms() * 8;
    return (int)(want < 1 ? 1 : (want < cap ? want : cap));
}

// hook-and-compress connected components into w.cc (label = the smallest id)
static int br_components(const Graph &g, const BridgeWs &w, cudaStream_t s) {
    k_cc_init<<<br_grid(g.n, 256), 256, 0, s>>>(w.cc, g.n);
    SYM_LAUNCH_CHECK();
    for (int it = 0; it < 64; it++) {
        SYM_CUDA(cudaMemsetAsync(w.ctr, 0, sizeof(uint32_t), s));
        k_cc_hook<<<br_grid(g.n * 32, BR_THREADS), BR_THREADS, 0, s>>>(g.rp, g.ci, g.n, w.cc, w.ctr);
        SYM_LAUNCH_CHECK();
        k_cc_compress<<<br_grid(g.n, 256), 256, 0, s>>>(w.cc, g.n);
        SYM_LAUNCH_CHECK();
        uint32_t ch = 0;
        SYM_TRY(read_u32(w.ctr, &ch, s));
        if (!ch) return SYM_OK;
    }
    set_error("connected components did not converge");
    return SYM_ECUDA;
}

int run_bridge_split(const Graph &g, const BridgeWs &w, int64_t *rp_in, int32_t *ci_in, int64_t *rp_x, int32_t *ci_x,
                     uint16_t *label, cudaStream_t s) {
    if (g.n == 0) return SYM_OK;
    prof_begin("split_bridge", s);
    // 1. components -> roots -> BFS forest -> min-id parents
    SYM_TRY(br_components(g, w, s));
    SYM_CUDA(cudaMemsetAsync(w.ctr + 1, 0, 2 * sizeof(uint32_t), s));
    k_br_roots<<<br_grid(g.n, 256), 256, 0, s>>>(g.rp, w.cc, g.n, w.level, w.fr[0], w.ctr + 1);
    SYM_LAUNCH_CHECK();
    uint32_t cnt = 0;
    SYM_TRY(read_u32(w.ctr + 1, &cnt, s));
    for (int32_t L = 0; cnt > 0; L++) {
        uint32_t *cin = w.ctr + 1 + (L & 1), *cout = w.ctr + 1 + ((L + 1) & 1);
        SYM_CUDA(cudaMemsetAsync(cout, 0, sizeof(uint32_t), s));
        k_br_bfs<<<br_grid((int64_t)cnt * 32, BR_THREADS), BR_THREADS, 0, s>>>(g.rp, g.ci, w.fr[L & 1], cin, L,
                                                                               w.level, w.fr[(L + 1) & 1], cout);
        SYM_LAUNCH_CHECK();
        SYM_TRY(read_u32(cout, &cnt, s));
    }
    k_br_parent<<<br_grid(g.n * 32, BR_THREADS), BR_THREADS, 0, s>>>(g.rp, g.ci, g.n, w.level, w.par, w.mark);
    SYM_LAUNCH_CHECK();
    // 2. LCA walks of the non-tree edges
    k_br_mark<<<br_grid(g.n * 32, BR_THREADS), BR_THREADS, 0, s>>>(g.rp, g.ci, g.n, w.level, w.par, w.mark);
    SYM_LAUNCH_CHECK();
    // 3. the split by the bridges
    k_br_count<<<br_grid(g.n * 32, BR_THREADS), BR_THREADS, 0, s>>>(g.rp, g.ci, g.n, w.par, w.mark, rp_in);
    SYM_LAUNCH_CHECK();
    const int64_t nb = (g.n + BR_SCAN - 1) / BR_SCAN;
    k_br_scan_blocks<<<(unsigned)nb, BR_SCAN, 0, s>>>(rp_in, g.n, w.bsum);
    SYM_LAUNCH_CHECK();
    k_br_scan_sums<<<1, BR_SCAN, 0, s>>>(w.bsum, nb);
    SYM_LAUNCH_CHECK();
    k_br_scan_apply<<<(unsigned)nb, BR_SCAN, 0, s>>>(rp_in, g.n, w.bsum);
    SYM_LAUNCH_CHECK();
    k_br_scatter<<<br_grid((g.n + 1) * 32, BR_THREADS), BR_THREADS, 0, s>>>(g.rp, g.ci, g.n, w.par, w.mark, rp_in,
                                                                            ci_in, rp_x, ci_x);
    SYM_LAUNCH_CHECK();
    if (label) {
        k_br_labels<<<br_grid(g.n, 256), 256, 0, s>>>(rp_x, g.n, label);
        SYM_LAUNCH_CHECK();
    }
    prof_end(s, -1.0, -1.0);
    return SYM_OK;
}

}  // namespace sym
