// decompose.cu -- RAND / DEGk decomposition kernels.
//
//   k_classify_degk  Alg 3 l.4-8: V_H = {deg(v) > k} as a bitmap (L2-resident,
//                    n/8 bytes) plus vertex lists (V_L from the front, V_H from the back).
//   k_first_row      per arc tile, the first row whose arcs start in the tile.
//   k_split          ONE streaming pass over col_idx: every arc (v,w) is intra iff
//                    class(v) == class(w) (RAND: label by hash, Alg 2 l.3 P:76; DEGk:
//                    bitmap).  The intra CSR (G[V_i] / G_L u G_H) is the
//                    stable compaction of the flat arc array, and the cross CSR
//                    (G_{k+1} / G_C) its complement, so a tile only needs
//                    its global intra prefix: decoupled look-back over tiles of 2048
//                    arcs (dynamic tile ids), block scan of the intra flags, compaction
//                    staged in shared memory, coalesced stores.  row_ptr_in[r] is the
//                    intra prefix at row r's first arc; row_ptr_x[r] = row_ptr[r] -
//                    row_ptr_in[r].  Bytes: 8 B/arc (read + write col) + 24 B/vertex.
#include "internal.h"

namespace sym {

enum { KIND_NONE = 0, KIND_RAND = 1, KIND_DEGK = 2 };
// DEGk: the V_H-bitmap word of each neighbour is gathered inside the flag loop, one
// dependent L2 access per arc.  Issuing a thread's 16 gathers as one batch -- right
// after the column loads, or just before the flag loop -- measured slower (3.31 ->
// 3.59 / 3.75 ms at R-MAT s24): the kernel sits at ~51 % of L2 throughput and the
// bursts only add contention.

// ------------------------------------------------------------------ classification
__global__ void k_classify_degk(const int64_t *__restrict__ rp, int64_t n, uint32_t k, uint32_t *__restrict__ hbits,
                                int32_t *__restrict__ vlist, uint32_t *cnt_front, uint32_t *cnt_back) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n; base += stride) {
        int64_t v = base + threadIdx.x;
        bool valid = v < n;
        bool h = false;
        if (valid) h = (rp[v + 1] - rp[v]) > (int64_t)k;
        unsigned word = __ballot_sync(FULL, h);
        if (lane_id() == 0 && valid) hbits[v >> 5] = word;
        if (vlist) cta_append2(valid && !h, h, (int32_t)v, n, vlist, cnt_front, cnt_back);
    }
}

// optional per-vertex class output (uint16): RAND part or DEGk class
__global__ void k_labels(const int64_t *__restrict__ rp, int64_t n, int kind, uint32_t param, Key kr,
                         uint16_t *__restrict__ label) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
        uint16_t c = 0;
        if (kind == KIND_RAND) c = (uint16_t)rand_label(kr, (uint32_t)v, param);
        else if (kind == KIND_DEGK) c = (rp[v + 1] - rp[v]) > (int64_t)param ? 1 : 0;
        label[v] = c;
    }
}

// ------------------------------------------------------------------ tile -> first row
// first_row[t] = smallest r in [0, n] with rp[r] >= t * TILE
__global__ void k_first_row(const int64_t *__restrict__ rp, int64_t n, int64_t ntiles, int64_t *__restrict__ first_row) {
    int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= ntiles) return;
    int64_t target = t * SPLIT_TILE;
    int64_t lo = 0, hi = n;  // answer in [0, n]; rp[n] = nnz > target for t < ntiles
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (rp[mid] >= target) hi = mid;
        else lo = mid + 1;
    }
    first_row[t] = lo;
}

// ------------------------------------------------------------------ block scan helpers
template <class T, class Op>
__device__ __forceinline__ T warp_incl_scan(T x, Op op) {
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        T y = __shfl_up_sync(FULL, x, d);
        if (lane_id() >= d) x = op(x, y);
    }
    return x;
}

// ------------------------------------------------------------------ the split
constexpr uint64_t LB_AGG = 1ULL << 62, LB_INC = 2ULL << 62, LB_VAL = (1ULL << 62) - 1;

// One tile = SPLIT_TILE consecutive arcs = SPLIT_PER_THREAD per thread (blocked).
// Tile id = blockIdx.x: CUDA dispatches blocks in index order, so every predecessor
// of a tile is resident or finished when the tile looks back (as CUB's single-pass
// scans rely on).
template <int KIND, bool VEC>
__device__ __forceinline__ void split_tile(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci, int64_t n,
                                           int64_t nnz, const int64_t *__restrict__ first_row, int64_t ntiles,
                                           const uint32_t *__restrict__ hbits, Key kr, uint32_t p,
                                           uint64_t *tile_state, int64_t *__restrict__ rp_in,
                                           int32_t *__restrict__ ci_in, int64_t *__restrict__ rp_x,
                                           int32_t *__restrict__ ci_x, int64_t row_base) {
    constexpr int T = SPLIT_TILE, V = SPLIT_PER_THREAD, NT = SPLIT_THREADS, NW = NT / 32;
    static_assert(V % 4 == 0 && T < 32768, "tile layout");
    __shared__ __align__(16) int16_t s_head[T];   // head position of the row owning each arc, or -1
    __shared__ __align__(16) uint16_t s_cls[T];   // class of the row whose head is at this position
    __shared__ __align__(16) int32_t s_out[T];    // compacted tile: intra then cross
    __shared__ __align__(16) uint16_t s_excl[T + 8];
    __shared__ int32_t s_wsum[NW];
    __shared__ int64_t s_prefix;
    __shared__ uint32_t s_cls0;

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int64_t t = blockIdx.x;
    const int64_t a = t * T;
    const int len = (int)min((int64_t)T, nnz - a);
    const int j0 = tid * V;

    // 1. issue this thread's column loads first (streaming, 128-bit)
    int32_t dst[V];
    if (VEC && j0 + V <= len) {
        const int4 *p4 = reinterpret_cast<const int4 *>(ci + a + j0);
#pragma unroll
        for (int q = 0; q < V / 4; q++) {
            int4 x = __ldcs(p4 + q);
            dst[4 * q] = x.x;
            dst[4 * q + 1] = x.y;
            dst[4 * q + 2] = x.z;
            dst[4 * q + 3] = x.w;
        }
    } else {
#pragma unroll
        for (int i = 0; i < V; i++) dst[i] = (j0 + i < len) ? __ldcs(ci + a + j0 + i) : 0;
    }
    const int64_t r_begin = first_row[t];
    const int64_t r_end = (t + 1 < ntiles) ? first_row[t + 1] : n + 1;

    auto vclass = [&](uint32_t v) -> uint32_t {
        if (KIND == KIND_RAND) return rand_label(kr, v, p);
        if (KIND == KIND_DEGK) return (hbits[v >> 5] >> (v & 31)) & 1u;
        return 0u;
    };

    // 2. heads of the non-empty rows starting in this tile
    {
        int4 m1 = make_int4(-1, -1, -1, -1);
        for (int j = tid * 8; j < T; j += NT * 8) *reinterpret_cast<int4 *>(s_head + j) = m1;
    }
    if (tid == 0) s_cls0 = (r_begin > 0) ? vclass((uint32_t)(row_base + r_begin - 1)) : 0u;
    __syncthreads();
    for (int64_t r = r_begin + tid; r < r_end; r += NT) {
        if (r >= n) continue;
        int64_t s = rp[r], e = rp[r + 1];
        if (e > s) {
            int j = (int)(s - a);
            s_head[j] = (int16_t)j;
            s_cls[j] = (uint16_t)vclass((uint32_t)(row_base + r));
        }
    }
    __syncthreads();

    // 3. the source row of each arc = last head at or before it: thread-local max,
    //    block exclusive max-scan, then the intra flags
    int hmax = -1;
#pragma unroll
    for (int q = 0; q < V / 8; q++) {
        int4 h = *reinterpret_cast<const int4 *>(s_head + j0 + 8 * q);
        const int16_t *hh = reinterpret_cast<const int16_t *>(&h);
#pragma unroll
        for (int i = 0; i < 8; i++) hmax = max(hmax, (int)hh[i]);
    }
    int carry;
    {
        int incl = hmax;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            int y = __shfl_up_sync(FULL, incl, d);
            if (lane >= d) incl = max(incl, y);
        }
        if (lane == 31) s_wsum[warp] = incl;
        int excl_w = __shfl_up_sync(FULL, incl, 1);
        if (lane == 0) excl_w = -1;
        __syncthreads();
        int wcarry = -1;
        for (int w = 0; w < warp; w++) wcarry = max(wcarry, s_wsum[w]);
        carry = max(excl_w, wcarry);
    }
    uint32_t flags = 0;
    int cnt = 0;
    {
        int h = carry;
#pragma unroll
        for (int q = 0; q < V / 8; q++) {
            int4 hv = *reinterpret_cast<const int4 *>(s_head + j0 + 8 * q);
            const int16_t *hh = reinterpret_cast<const int16_t *>(&hv);
#pragma unroll
            for (int i = 0; i < 8; i++) {
                const int k = 8 * q + i;
                h = max(h, (int)hh[i]);
                if (j0 + k < len) {
                    uint32_t cs = (h >= 0) ? (uint32_t)s_cls[h] : s_cls0;
                    bool intra = (KIND == KIND_NONE) ? true : (vclass((uint32_t)dst[k]) == cs);
                    flags |= (intra ? 1u : 0u) << k;
                    cnt += intra;
                }
            }
        }
    }
    __syncthreads();  // s_wsum reuse
    // 4. block exclusive sum of the intra counts
    int excl, total;
    {
        int incl = cnt;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            int y = __shfl_up_sync(FULL, incl, d);
            if (lane >= d) incl += y;
        }
        if (lane == 31) s_wsum[warp] = incl;
        __syncthreads();
        int wbase = 0;
        total = 0;
#pragma unroll
        for (int w = 0; w < NW; w++) {
            int sv = s_wsum[w];
            wbase += (w < warp) ? sv : 0;
            total += sv;
        }
        excl = wbase + incl - cnt;
    }
    // 5. decoupled look-back for the tile's global intra prefix, by the whole CTA:
    //    NT predecessors per step (a one-warp look-back walks ~tiles_in_flight/32
    //    dependent L2 reads per tile, which caps the kernel near 2 TB/s)
    if (t == 0) {
        if (tid == 0) {
            atomicExch((unsigned long long *)&tile_state[0], (unsigned long long)(LB_INC | (uint64_t)total));
            s_prefix = 0;
        }
    } else {
        __shared__ int s_upto[NW];
        __shared__ long long s_part[NW];
        if (tid == 0) atomicExch((unsigned long long *)&tile_state[t], (unsigned long long)(LB_AGG | (uint64_t)total));
        int64_t prefix = 0;
        int64_t pos = t - 1;
        for (;;) {
            const int64_t idx = pos - tid;  // tid 0 = nearest predecessor
            uint64_t sv = LB_INC;           // idx < 0 acts as an inclusive zero
            if (idx >= 0) {
                do {
                    sv = ld_volatile_u64(&tile_state[idx]);
                } while ((sv >> 62) == 0);
            }
            const unsigned inc = __ballot_sync(FULL, (sv >> 62) == 2);
            if (lane == 0) s_upto[warp] = inc ? warp * 32 + __ffs(inc) - 1 : NT;
            __syncthreads();
            int upto = NT;
#pragma unroll
            for (int w = 0; w < NW; w++) upto = min(upto, s_upto[w]);
            long long contrib = (tid <= upto) ? (long long)(sv & LB_VAL) : 0;
#pragma unroll
            for (int d = 16; d; d >>= 1) contrib += __shfl_xor_sync(FULL, contrib, d);
            if (lane == 0) s_part[warp] = contrib;
            __syncthreads();
#pragma unroll
            for (int w = 0; w < NW; w++) prefix += s_part[w];
            __syncthreads();
            if (upto < NT) break;
            pos -= NT;
        }
        if (tid == 0) {
            atomicExch((unsigned long long *)&tile_state[t], (unsigned long long)(LB_INC | (uint64_t)(prefix + total)));
            s_prefix = prefix;
        }
    }
    // 6. stage the compacted tile and the per-position intra prefix in shared memory
    {
        int o = excl;
        uint16_t ex[V];
#pragma unroll
        for (int i = 0; i < V; i++) {
            ex[i] = (uint16_t)o;
            int j = j0 + i;
            if (j < len) {
                if ((flags >> i) & 1u) s_out[o] = dst[i];
                else s_out[total + (j - o)] = dst[i];
            }
            o += (flags >> i) & 1u;
        }
#pragma unroll
        for (int q = 0; q < V / 8; q++) {
            uint4 pk;
            pk.x = (uint32_t)ex[8 * q + 0] | ((uint32_t)ex[8 * q + 1] << 16);
            pk.y = (uint32_t)ex[8 * q + 2] | ((uint32_t)ex[8 * q + 3] << 16);
            pk.z = (uint32_t)ex[8 * q + 4] | ((uint32_t)ex[8 * q + 5] << 16);
            pk.w = (uint32_t)ex[8 * q + 6] | ((uint32_t)ex[8 * q + 7] << 16);
            *reinterpret_cast<uint4 *>(s_excl + j0 + 8 * q) = pk;
        }
    }
    __syncthreads();
    if (tid == 0) s_excl[len] = (uint16_t)total;  // position len (last tile: rows starting at nnz)
    __syncthreads();
    const int64_t P = s_prefix;
    // 7. coalesced stores of the two compacted streams
    for (int i = tid; i < total; i += NT) ci_in[P + i] = s_out[i];
    const int64_t X = a - P;
    for (int i = tid; i < len - total; i += NT) ci_x[X + i] = s_out[total + i];
    // 8. row pointers of rows whose first arc lies in this tile (and, in the last
    //    tile, the rows starting at nnz including the sentinel r = n)
    for (int64_t r = r_begin + tid; r < r_end; r += NT) {
        int64_t s = rp[r];
        int j = (int)(s - a);
        int64_t v_in = P + (int64_t)s_excl[j];
        rp_in[r] = v_in;
        rp_x[r] = s - v_in;
    }
}

#define SPLIT_PARAMS                                                                                             \
    const int64_t *__restrict__ rp, const int32_t *__restrict__ ci, int64_t n, int64_t nnz,                      \
        const int64_t *__restrict__ first_row, int64_t ntiles, const uint32_t *__restrict__ hbits, Key kr,       \
        uint32_t p, uint64_t *tile_state, int64_t *__restrict__ rp_in, int32_t *__restrict__ ci_in,              \
        int64_t *__restrict__ rp_x, int32_t *__restrict__ ci_x, int64_t row_base
#define SPLIT_FWD rp, ci, n, nnz, first_row, ntiles, hbits, kr, p, tile_state, rp_in, ci_in, rp_x, ci_x, row_base

// DEGk / NONE: 4 CTAs/SM at the compiler's register choice.  RAND (hash labels, no
// class gathers) gains from a 5th CTA per SM (<= 51 regs, 40 KB smem each): 2.0 ->
// 1.8 ms at R-MAT s24 p = 4; the same bound made the DEGk split slower (3.4 -> 5.0 ms).
template <int KIND, bool VEC>
__global__ void __launch_bounds__(SPLIT_THREADS) k_split(SPLIT_PARAMS) {
    split_tile<KIND, VEC>(SPLIT_FWD);
}
template <bool VEC>
__global__ void __launch_bounds__(SPLIT_THREADS, 5) k_split_rand(SPLIT_PARAMS) {
    split_tile<KIND_RAND, VEC>(SPLIT_FWD);
}

// ------------------------------------------------------------------ host side
void carve_split_ws(Arena &a, int64_t n, int64_t nnz, SplitWs &w) {
    int64_t ntiles = (nnz + SPLIT_TILE - 1) / SPLIT_TILE;
    w.ntiles = ntiles;
    w.hbits = a.take<uint32_t>((size_t)((n + 31) / 32 + 1));
    w.first_row = a.take<int64_t>((size_t)ntiles + 1);
    w.tile_state = a.take<uint64_t>((size_t)ntiles + 1);
}

static int grid_for(int64_t items, int threads, int per_sm = 8) {
    int64_t want = (items + threads - 1) / threads;
    int64_t cap = (int64_t)num_sms() * per_sm;
    if (want < 1) want = 1;
    return (int)(want < cap ? want : cap);
}

int launch_classify_degk(const Graph &g, uint32_t k, uint32_t *hbits, int32_t *vlist, Ctl *ctl, cudaStream_t s) {
    if (g.n == 0) return SYM_OK;
    k_classify_degk<<<grid_for(g.n, 256), 256, 0, s>>>(g.rp, g.n, k, hbits, vlist, &ctl->cnt_front,
                                                          &ctl->cnt_back);
    SYM_LAUNCH_CHECK();
    return SYM_OK;
}

int run_split(const Graph &g, int kind, uint32_t param, uint64_t seed, const SplitWs &w, Ctl *ctl, int64_t *rp_in,
              int32_t *ci_in, int64_t *rp_x, int32_t *ci_x, uint16_t *label, cudaStream_t s, int64_t row_base) {
    if (kind == SYM_DECOMP_BRIDGE) return run_bridge_split(g, w.br, rp_in, ci_in, rp_x, ci_x, label, s);  // bridge.cu
    Key kr = stream_key(seed, TAG_RAND, 0);
    if (label && g.n > 0) {
        k_labels<<<grid_for(g.n, 256), 256, 0, s>>>(g.rp, g.n, kind, param, kr, label);
        SYM_LAUNCH_CHECK();
    }
    if (g.nnz == 0) {
        SYM_CUDA(cudaMemsetAsync(rp_in, 0, sizeof(int64_t) * (size_t)(g.n + 1), s));
        SYM_CUDA(cudaMemsetAsync(rp_x, 0, sizeof(int64_t) * (size_t)(g.n + 1), s));
        return SYM_OK;
    }
    if (kind == KIND_DEGK) SYM_TRY(launch_classify_degk(g, param, w.hbits, nullptr, ctl, s));
    SYM_CUDA(cudaMemsetAsync(w.tile_state, 0, sizeof(uint64_t) * (size_t)w.ntiles, s));
    k_first_row<<<(unsigned)((w.ntiles + 255) / 256), 256, 0, s>>>(g.rp, g.n, w.ntiles, w.first_row);
    SYM_LAUNCH_CHECK();
    bool vec = ((uintptr_t)g.ci & 15) == 0;
    dim3 grid((unsigned)w.ntiles);
    prof_begin(kind == SYM_DECOMP_DEGK ? "split_degk" : (kind == SYM_DECOMP_RAND ? "split_rand" : "split_none"), s);
#define SPLIT_ARGS                                                                                          \
    g.rp, g.ci, g.n, g.nnz, w.first_row, w.ntiles, w.hbits, kr, param, w.tile_state, rp_in, \
        ci_in, rp_x, ci_x, row_base
    if (kind == KIND_RAND) {
        if (vec) k_split_rand<true><<<grid, SPLIT_THREADS, 0, s>>>(SPLIT_ARGS);
        else k_split_rand<false><<<grid, SPLIT_THREADS, 0, s>>>(SPLIT_ARGS);
    } else if (kind == KIND_DEGK) {
        if (vec) k_split<KIND_DEGK, true><<<grid, SPLIT_THREADS, 0, s>>>(SPLIT_ARGS);
        else k_split<KIND_DEGK, false><<<grid, SPLIT_THREADS, 0, s>>>(SPLIT_ARGS);
    } else {
        if (vec) k_split<KIND_NONE, true><<<grid, SPLIT_THREADS, 0, s>>>(SPLIT_ARGS);
        else k_split<KIND_NONE, false><<<grid, SPLIT_THREADS, 0, s>>>(SPLIT_ARGS);
    }
#undef SPLIT_ARGS
    // algorithmic bytes: read + write every arc (8 B), read row_ptr, write both row
    // pointer arrays (24 B per row pointer)
    // 8 B/arc (column read + written) + 24 B/row pointer (read + two written)
    prof_end(s, 8.0 * (double)g.nnz + 24.0 * (double)(g.n + 1), 8.0 * (double)g.nnz + 24.0 * (double)(g.n + 1));
    SYM_LAUNCH_CHECK();
    return SYM_OK;
}

}  // namespace sym

