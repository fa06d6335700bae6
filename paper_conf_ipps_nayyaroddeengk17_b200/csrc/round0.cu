// round0.cu -- the first round of a MIS or MM phase as one HBM-streaming pass.
//
// In round 0 of a phase every phase vertex is undecided (MIS) / unmatched (MM), and
// treating a neighbour that is already Out / matched as live is conservative: it can
// only keep a vertex undecided (MIS) or make it pick a dead edge (MM), which the next
// round repairs.  So round 0 needs NO neighbour-state gathers:
//   MIS  v joins I iff every phase neighbour w has vkey(w) < vkey(v)
//   MM   pick(u) = argmax_w (pe(u,w), w) over u's phase arcs
// i.e. a segmented max over the CSR rows.  It runs on flat tiles of SPLIT_TILE arcs
// (the decomposition's tiling, so power-law rows cost nothing extra): 128-bit
// evict-first column loads, row heads and the row of every arc from the same
// head/max-scan scheme as k_split, per-row maxima by shared-memory atomics, rows
// that cross a tile boundary combined through a global atomicMax.
// Algorithmic bytes: 4 B/arc + 16 B/row (+ 4 B pick / 1 B status written).
#include "internal.h"

namespace sym {

enum { R0_MIS = 0, R0_MM = 1 };

struct Round0Args {
    const int64_t *rp;
    const int32_t *ci;
    int64_t n, nnz;
    const int64_t *first_row;
    int64_t ntiles;
    Key k;
    unsigned long long *gmax;  // per-row partial maxima of rows crossing tiles
    // MIS
    uint8_t *st;
    // MM
    int32_t *pick;
    const uint32_t *hfilter;   // MM: only rows with this class bit set emit (nullable)
    int32_t *out_list;
    uint32_t *out_cnt;
};

template <int MODE>
__device__ __forceinline__ uint64_t r0_key(const Round0Args &A, uint32_t u, uint32_t w) {
    if (MODE == R0_MIS) return vkey(A.k, w);
    return ekey(A.k, u, w);
}

// the decision for row u given the max key over its arcs (nonempty = has arcs);
// returns true if u joins the next frontier (MM) -- caller appends
template <int MODE>
__device__ __forceinline__ bool r0_emit(const Round0Args &A, uint32_t u, uint64_t m, bool nonempty) {
    if (MODE == R0_MIS) {
        if (A.st[u] == ST_UNDEC && (!nonempty || m < vkey(A.k, u))) A.st[u] = ST_IN;
        return false;
    }
    if (A.hfilter && !((A.hfilter[u >> 5] >> (u & 31)) & 1u)) return false;
    A.pick[u] = nonempty ? (int32_t)(uint32_t)m : -1;
    return nonempty;
}

// rows crossing a tile boundary: zero their global partial maxima
__global__ void k_r0_span_init(Round0Args A) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x + 1;
    if (t >= A.ntiles) return;
    const int64_t f = A.first_row[t];
    if (A.rp[f] != t * SPLIT_TILE) A.gmax[f - 1] = 0;  // row f-1 contains arc t*TILE
}

// rows crossing a tile boundary: emit once, from the first boundary they cross
template <int MODE>
__global__ void k_r0_span_emit(Round0Args A) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x + 1;
    bool take = false;
    uint32_t u = 0;
    if (t < A.ntiles) {
        const int64_t f = A.first_row[t];
        const int64_t bnd = t * SPLIT_TILE;
        if (A.rp[f] != bnd) {
            const int64_t r = f - 1;
            if (A.rp[r] >= bnd - SPLIT_TILE) {  // the row starts in tile t-1
                u = (uint32_t)r;
                take = r0_emit<MODE>(A, u, A.gmax[r], true);
            }
        }
    }
    if (MODE == R0_MM) {
        int64_t slot = warp_append(take, A.out_cnt);
        if (slot >= 0) A.out_list[slot] = (int32_t)u;
    }
}

constexpr int R0_SMEM = SPLIT_TILE * 2 + SPLIT_TILE * 4 + (SPLIT_TILE + 1) * 8;

template <int MODE>
__global__ void __launch_bounds__(SPLIT_THREADS) k_round0(Round0Args A) {
    constexpr int T = SPLIT_TILE, V = SPLIT_PER_THREAD, NT = SPLIT_THREADS, NW = NT / 32;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    int16_t *s_head = reinterpret_cast<int16_t *>(smem_raw);                        // [T]
    int32_t *s_row = reinterpret_cast<int32_t *>(s_head + T);                      // [T]
    unsigned long long *s_max = reinterpret_cast<unsigned long long *>(s_row + T);  // [T+1]
    __shared__ int s_wmax[NW];

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int j0 = tid * V;
    const int64_t G = gridDim.x;
    // persistent CTAs walk tiles t = blockIdx.x + i*G; the next tile's columns are
    // prefetched into registers while the current tile is processed
    auto load_cols = [&](int64_t tt, uint32_t(&out)[V]) {
        const int64_t aa = tt * T;
        const int ll = (int)min((int64_t)T, A.nnz - aa);
        if (j0 + V <= ll && (((uintptr_t)(A.ci + aa + j0)) & 15) == 0) {
            const int4 *p4 = reinterpret_cast<const int4 *>(A.ci + aa + j0);
#pragma unroll
            for (int q = 0; q < V / 4; q++) {
                int4 x = __ldcs(p4 + q);
                out[4 * q] = (uint32_t)x.x;
                out[4 * q + 1] = (uint32_t)x.y;
                out[4 * q + 2] = (uint32_t)x.z;
                out[4 * q + 3] = (uint32_t)x.w;
            }
        } else {
#pragma unroll
            for (int i = 0; i < V; i++) out[i] = (j0 + i < ll) ? (uint32_t)__ldcs(A.ci + aa + j0 + i) : 0u;
        }
    };
    uint32_t nxt[V];
    if ((int64_t)blockIdx.x < A.ntiles) load_cols(blockIdx.x, nxt);
    for (int64_t t = blockIdx.x; t < A.ntiles; t += G) {
    const int64_t a = t * T;
    const int len = (int)min((int64_t)T, A.nnz - a);
    // 1. this thread's columns (prefetched), and the next tile's prefetch
    uint32_t dst[V];
#pragma unroll
    for (int i = 0; i < V; i++) dst[i] = nxt[i];
    if (t + G < A.ntiles) load_cols(t + G, nxt);
    const int64_t r_begin = A.first_row[t];
    const int64_t r_end = (t + 1 < A.ntiles) ? A.first_row[t + 1] : A.n + 1;

    // 2. heads of the non-empty rows starting in this tile
    for (int j = tid * 8; j < T; j += NT * 8) *reinterpret_cast<int4 *>(s_head + j) = make_int4(-1, -1, -1, -1);
    if (tid == 0) s_max[T] = 0;
    __syncthreads();
    for (int64_t r = r_begin + tid; r < r_end; r += NT) {
        if (r >= A.n) continue;
        int64_t s = A.rp[r], e = A.rp[r + 1];
        if (e > s) {
            int j = (int)(s - a);
            s_head[j] = (int16_t)j;
            s_row[j] = (int32_t)r;
            s_max[j] = 0;
        }
    }
    __syncthreads();
    // 3. head position of every arc: thread-local max, block exclusive max-scan
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
        if (lane == 31) s_wmax[warp] = incl;
        int excl_w = __shfl_up_sync(FULL, incl, 1);
        if (lane == 0) excl_w = -1;
        __syncthreads();
        int wcarry = -1;
        for (int w = 0; w < warp; w++) wcarry = max(wcarry, s_wmax[w]);
        carry = max(excl_w, wcarry);
    }
    // 4. per-row maxima: run-length reduce inside the thread, flush to shared memory
    {
        const uint32_t r_c = (uint32_t)(r_begin > 0 ? r_begin - 1 : 0);  // row carried into the tile
        int h = carry, cur = -2, f_cur = -2;
        unsigned long long m = 0, f_m = 0;
#pragma unroll
        for (int q = 0; q < V / 8; q++) {
            int4 hv = *reinterpret_cast<const int4 *>(s_head + j0 + 8 * q);
            const int16_t *hh = reinterpret_cast<const int16_t *>(&hv);
#pragma unroll
            for (int i = 0; i < 8; i++) {
                const int kx = 8 * q + i;
                h = max(h, (int)hh[i]);
                if (j0 + kx < len) {
                    if (h != cur) {
                        // a run that started inside this thread's arcs and ended before its
                        // last one is the whole row: a plain store (sm_100 has no 64-bit
                        // shared atomicMax -- each one is a CAS loop); only the first and
                        // the last run of a thread can be shared with its neighbours
                        if (cur >= j0) {
                            s_max[cur] = m;
                        } else if (cur != -2) {  // the first run: merged after the loop
                            f_cur = cur;
                            f_m = m;
                        }
                        cur = h;
                        m = 0;
                    }
                    const uint32_t u = (h >= 0) ? (uint32_t)s_row[h] : r_c;
                    const unsigned long long key = r0_key<MODE>(A, u, dst[kx]);
                    m = key > m ? key : m;
                }
            }
        }
        if (f_cur != -2) atomicMax(&s_max[f_cur < 0 ? T : f_cur], f_m);
        if (cur != -2) atomicMax(&s_max[cur < 0 ? T : cur], m);
    }
    __syncthreads();
    // 5. decisions for rows starting here; partial maxima of rows crossing tiles
    for (int64_t base = r_begin; base < r_end; base += NT) {
        const int64_t r = base + tid;
        bool take = false;
        if (r < r_end && r < A.n) {
            const int64_t s = A.rp[r], e = A.rp[r + 1];
            if (e == s) {
                take = r0_emit<MODE>(A, (uint32_t)r, 0, false);
            } else {
                const unsigned long long m = s_max[s - a];
                if (e <= a + len) take = r0_emit<MODE>(A, (uint32_t)r, m, true);
                else atomicMax(A.gmax + r, m);
            }
        }
        if (MODE == R0_MM) {
            int64_t slot = warp_append(take, A.out_cnt);
            if (slot >= 0) A.out_list[slot] = (int32_t)r;
        }
    }
    if (tid == 0 && s_head[0] < 0 && len > 0 && r_begin > 0) atomicMax(A.gmax + (r_begin - 1), s_max[T]);
    __syncthreads();  // shared arrays are reused by the next tile
    }
}

// arcs of a phase CSR (G, or the intra/cross CSR of the decomposition): known on the
// host or read back once from row_ptr[n]
int phase_arcs(const FlowArgs &f, const int64_t *rp, int64_t *out) {
    if (rp == f.g.rp) {
        *out = f.g.nnz;
        return SYM_OK;
    }
    if (rp == f.split.rp_in && f.split.nnz_in >= 0) {
        *out = f.split.nnz_in;
        return SYM_OK;
    }
    if (rp == f.split.rp_x && f.split.nnz_x >= 0) {
        *out = f.split.nnz_x;
        return SYM_OK;
    }
    uint64_t v = 0;
    SYM_TRY(read_u64(reinterpret_cast<const uint64_t *>(rp + f.g.n), &v, f.stream));
    *out = (int64_t)v;
    return SYM_OK;
}

int launch_first_row(const Graph &g, int64_t ntiles, int64_t *first_row, cudaStream_t s) {
    k_first_row<<<(unsigned)((ntiles + 255) / 256), 256, 0, s>>>(g.rp, g.n, ntiles, first_row);
    SYM_LAUNCH_CHECK();
    return SYM_OK;
}

int run_round0(int mode, const Graph &g, const int64_t *first_row, int64_t ntiles, Key k,
               unsigned long long *gmax, uint8_t *st, int32_t *pick, const uint32_t *hfilter, int32_t *out_list,
               uint32_t *out_cnt, cudaStream_t s) {
    if (g.n == 0) return SYM_OK;
    Round0Args A;
    A.rp = g.rp;
    A.ci = g.ci;
    A.n = g.n;
    A.nnz = g.nnz;
    A.first_row = first_row;
    A.ntiles = ntiles;
    A.k = k;
    A.gmax = gmax;
    A.st = st;
    A.pick = pick;
    A.hfilter = hfilter;
    A.out_list = out_list;
    A.out_cnt = out_cnt;
    // function attributes are per device context: set once per device
    static std::atomic<int> attr[SYM_MAX_DEVICES];
    const int ok = dev_cached(attr, [] {
        if (cudaFuncSetAttribute(k_round0<R0_MIS>, cudaFuncAttributeMaxDynamicSharedMemorySize, R0_SMEM) !=
                cudaSuccess ||
            cudaFuncSetAttribute(k_round0<R0_MM>, cudaFuncAttributeMaxDynamicSharedMemorySize, R0_SMEM) != cudaSuccess)
            return -1;
        return 1;
    });
    if (ok != 1) SYM_CUDA(cudaGetLastError());
    if (g.nnz <= 0 || ntiles <= 0) return SYM_EINVAL;  // caller uses the frontier kernel instead
    SYM_TRY(launch_first_row(g, ntiles, const_cast<int64_t *>(first_row), s));
    if (ntiles > 1) {
        k_r0_span_init<<<(unsigned)((ntiles + 255) / 256), 256, 0, s>>>(A);
        SYM_LAUNCH_CHECK();
    }
    static std::atomic<int> per_slots[SYM_MAX_DEVICES];
    const int per_sm = dev_cached(per_slots, [] {
        int x = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&x, k_round0<R0_MM>, SPLIT_THREADS, R0_SMEM) != cudaSuccess)
            return 1;
        return x > 0 ? x : 1;
    });
    const int64_t want = (int64_t)num_sms() * per_sm;
    const unsigned grid = (unsigned)(want < ntiles ? want : ntiles);
    prof_begin(mode == R0_MIS ? "mis_round0" : "mm_round0", s);
    if (mode == R0_MIS) k_round0<R0_MIS><<<grid, SPLIT_THREADS, R0_SMEM, s>>>(A);
    else k_round0<R0_MM><<<grid, SPLIT_THREADS, R0_SMEM, s>>>(A);
    // §8(d): 4 B/arc + 9 B/vertex (every row is active in round 0); the kernel reads
    // 4 B/arc + 16 B/row (row pointers) and writes the decision (1 B status / 4 B pick +
    // 4 B frontier entry)
    prof_end(s, 4.0 * (double)g.nnz + 9.0 * (double)g.n,
             4.0 * (double)g.nnz + 16.0 * (double)g.n + (mode == R0_MIS ? 1.0 : 8.0) * (double)g.n);
    SYM_LAUNCH_CHECK();
    if (ntiles > 1) {
        if (mode == R0_MIS) k_r0_span_emit<R0_MIS><<<(unsigned)((ntiles + 255) / 256), 256, 0, s>>>(A);
        else k_r0_span_emit<R0_MM><<<(unsigned)((ntiles + 255) / 256), 256, 0, s>>>(A);
        SYM_LAUNCH_CHECK();
    }
    return SYM_OK;
}

}  // namespace sym
