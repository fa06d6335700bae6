// color_shard.cu -- sharded COLOR (include/sym.h `sym_shard_color_*`).
//
// A rank owns rows [v_begin, v_end) (global ids) with global column ids and keeps a
// full replica of the colour array (u32[n_global], 0 = uncoloured).  One call of
// k_shard_jp_round is one Jones-Plassmann round ([18]) over the owned frontier:
// an uncoloured v whose admitted higher-priority neighbours are all coloured takes the
// smallest colour >= 1 not held by a coloured admitted neighbour (mex).  After every
// round the caller all-gathers the owned colour segments (NCCL over NVLink) and
// all-reduces the frontier counts.
//   admit = 0: every arc (COLOR-NONE; COLOR-Rand's recolouring of V' against G),
//   admit = 1: arcs whose endpoints share a class (DEGk: the V_H bitmap; RAND: the
//              hash label of Alg 2 l.3) -- G_H and G_L coloured at once (Alg 9,
//              P:234), or the induced subgraphs G[V_i] with one palette (Alg 8).
// Why any schedule gives the greedy colouring in priority order: v is coloured only
// when every admitted higher neighbour holds its final colour, and no admitted lower
// neighbour in the phase set can be coloured before v; neighbours outside the phase
// set are fixed.  A stale (not yet all-gathered) 0 only delays v by a round.  Colour
// words are read with volatile loads (L1 bypass) because this round's own writes on
// other SMs may make a vertex ready mid-round.
#include "internal.h"

namespace sym {

constexpr int CS_THREADS = 256, CS_WARPS = CS_THREADS / 32, CS_WIN = 1024;

struct ShardColorArgs {
    const int64_t *rp;
    const int32_t *ci;
    int64_t v0, v1;
    int kind;            // SYM_DECOMP_NONE / RAND / DEGK (class function)
    uint32_t param;      // RAND p
    Key kr;              // RAND label key
    Key kv;              // vertex priority key
    const uint32_t *hbits;
    int admit;
};

__device__ __forceinline__ uint32_t cs_class(const ShardColorArgs &A, uint32_t v) {
    if (A.kind == SYM_DECOMP_RAND) return rand_label(A.kr, v, A.param);
    if (A.kind == SYM_DECOMP_DEGK) return (A.hbits[v >> 5] >> (v & 31)) & 1u;
    return 0u;
}

__device__ __forceinline__ uint32_t cs_colour(const uint32_t *c, uint32_t w) { return ld_volatile_u32(c + w); }

__device__ __forceinline__ void st_volatile_u32(uint32_t *p, uint32_t v) {
    asm volatile("st.volatile.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// warp per frontier vertex: readiness scan, then the mex in windows of 1024 colours
// (colours of an admitted neighbour set of size d never exceed d + 1)
__global__ void __launch_bounds__(CS_THREADS)
    k_shard_jp_round(ShardColorArgs A, uint32_t *color, const int32_t *__restrict__ list, const uint32_t *count,
                     int32_t *next, uint32_t *next_count) {
    __shared__ uint32_t s_mask[CS_WARPS][CS_WIN / 32];
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t cnt = *count;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < cnt; i += nw) {
        const uint32_t v = (uint32_t)list[i];
        if (cs_colour(color, v) != 0) continue;
        const uint32_t cv = cs_class(A, v);
        const uint64_t kv = vkey(A.kv, v);
        const int64_t b = A.rp[v - A.v0], e = A.rp[v - A.v0 + 1];
        bool blocked = false;
        for (int64_t x = b; x < e && !blocked; x += 32) {
            bool blk = false;
            if (x + lane < e) {
                const uint32_t w = (uint32_t)A.ci[x + lane];
                const bool adm = A.admit == 0 || cs_class(A, w) == cv;
                blk = adm && vkey(A.kv, w) > kv && cs_colour(color, w) == 0;
            }
            blocked = __any_sync(FULL, blk);
        }
        if (blocked) {
            if (lane == 0) next[atomicAdd(next_count, 1u)] = (int32_t)v;
            continue;
        }
        uint32_t c = 0;
        for (uint32_t base = 1; c == 0; base += CS_WIN) {
            s_mask[wib][lane] = 0;
            __syncwarp();
            for (int64_t x = b + lane; x < e; x += 32) {
                const uint32_t w = (uint32_t)A.ci[x];
                if (A.admit != 0 && cs_class(A, w) != cv) continue;
                const uint32_t cw = cs_colour(color, w);
                if (cw >= base && cw - base < (uint32_t)CS_WIN)
                    atomicOr(&s_mask[wib][(cw - base) >> 5], 1u << ((cw - base) & 31));
            }
            __syncwarp();
            const uint32_t freew = ~s_mask[wib][lane];
            const unsigned has = __ballot_sync(FULL, freew != 0);
            if (has) {
                const int l = __ffs(has) - 1;
                const uint32_t fw = __shfl_sync(FULL, freew, l);
                c = base + 32u * (uint32_t)l + (uint32_t)(__ffs(fw) - 1);
            }
            __syncwarp();
        }
        if (lane == 0) st_volatile_u32(color + v, c);
    }
}

// owned uncoloured vertices -> list
__global__ void k_shard_color_frontier(const uint32_t *color, int64_t v0, int64_t v1, int32_t *list,
                                       uint32_t *count) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = v0 + (int64_t)blockIdx.x * blockDim.x; base < v1; base += stride) {
        const int64_t v = base + threadIdx.x;
        const int64_t slot = warp_append(v < v1 && color[v] == 0, count);
        if (slot >= 0) list[slot] = (int32_t)v;
    }
}

// COLOR-Rand fix-up, step 1 (Alg 8): V' = owned endpoints of a cross arc
// (classes differ) whose endpoints share a colour -> list (warp per vertex)
__global__ void k_shard_color_conflicts(ShardColorArgs A, const uint32_t *__restrict__ color, int32_t *list,
                                        uint32_t *count) {
    const int lane = lane_id();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t v = A.v0 + (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5); v < A.v1; v += nw) {
        const uint32_t cv = cs_class(A, (uint32_t)v), col = color[v];
        const int64_t b = A.rp[v - A.v0], e = A.rp[v - A.v0 + 1];
        bool hit = false;
        for (int64_t x = b; x < e && !hit; x += 32) {
            bool h = false;
            if (x + lane < e) {
                const uint32_t w = (uint32_t)A.ci[x + lane];
                h = cs_class(A, w) != cv && color[w] == col;
            }
            hit = __any_sync(FULL, h);
        }
        if (hit && lane == 0) list[atomicAdd(count, 1u)] = (int32_t)v;
    }
}

__global__ void k_shard_color_clear(uint32_t *color, const int32_t *__restrict__ list, const uint32_t *count) {
    const int64_t cnt = *count, stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += stride) color[list[i]] = 0;
}

// COLOR-Degk (Alg 9): max colour over owned V_H (atomicMax into *out)
__global__ void k_shard_color_maxh(const uint32_t *__restrict__ hbits, const uint32_t *__restrict__ color, int64_t v0,
                                   int64_t v1, uint32_t *out) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    uint32_t m = 0;
    for (int64_t v = v0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < v1; v += stride)
        if ((hbits[v >> 5] >> (v & 31)) & 1u) m = max(m, color[v]);
#pragma unroll
    for (int d = 16; d; d >>= 1) m = max(m, __shfl_xor_sync(FULL, m, d));
    if (lane_id() == 0 && m) atomicMax(out, m);
}

// COLOR-Degk: owned V_L colours += M ("additional k+1 colours max(C_H)+1 ..")
__global__ void k_shard_color_shift(const uint32_t *__restrict__ hbits, uint32_t *color, int64_t v0, int64_t v1,
                                    uint32_t M) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = v0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < v1; v += stride)
        if (!((hbits[v >> 5] >> (v & 31)) & 1u)) color[v] += M;
}

}  // namespace sym

using namespace sym;

static int cs_check(const sym_graph_shard *g) {
    if (!g) { set_error("shard is NULL"); return SYM_EINVAL; }
    if (g->n_global < 0 || g->n_global >= ((int64_t)1 << 31) - 1 || g->v_begin < 0 || g->v_end < g->v_begin ||
        g->v_end > g->n_global || g->nnz < 0) {
        set_error("bad shard range: need 0 <= v_begin <= v_end <= n_global < 2^31 - 1, nnz >= 0");
        return SYM_EINVAL;
    }
    if (g->v_end > g->v_begin && !g->row_ptr) { set_error("row_ptr is NULL"); return SYM_EINVAL; }
    if (g->nnz > 0 && !g->col_idx) { set_error("col_idx is NULL"); return SYM_EINVAL; }
    return SYM_OK;
}

static int cs_args(const sym_graph_shard *g, const sym_params *p, const uint32_t *hbits, int admit,
                   ShardColorArgs *A) {
    if (!p) { set_error("params is NULL"); return SYM_EINVAL; }
    if (p->kind != SYM_DECOMP_NONE && p->kind != SYM_DECOMP_RAND && p->kind != SYM_DECOMP_DEGK) {
        set_error("unknown decomposition kind");
        return SYM_EINVAL;
    }
    if (p->kind == SYM_DECOMP_RAND && (p->param == 0 || p->param > 65535)) {
        set_error("RAND needs 1 <= p <= 65535");
        return SYM_EINVAL;
    }
    if (p->kind == SYM_DECOMP_DEGK && !hbits) { set_error("DEGk needs hbits"); return SYM_EINVAL; }
    if (admit != 0 && admit != 1) { set_error("admit must be 0 or 1"); return SYM_EINVAL; }
    A->rp = g->row_ptr;
    A->ci = g->col_idx;
    A->v0 = g->v_begin;
    A->v1 = g->v_end;
    A->kind = (int)p->kind;
    A->param = p->param;
    A->kr = stream_key(p->seed, TAG_RAND, 0);
    A->kv = stream_key(p->seed, TAG_VERTEX, 0);
    A->hbits = hbits;
    A->admit = admit;
    return SYM_OK;
}

static int cs_grid(int64_t items, int per_cta) {
    int64_t want = (items + per_cta - 1) / per_cta;
    int64_t cap = (int64_t)num_sms() * 8;
    return (int)(want < 1 ? 1 : (want < cap ? want : cap));
}

extern "C" int sym_shard_color_frontier(const sym_graph_shard *g, const uint32_t *color, int32_t *list,
                                        uint32_t *count, sym_stream_t stream) {
    SYM_TRY(cs_check(g));
    if (!color || !list || !count) { set_error("NULL argument"); return SYM_EINVAL; }
    cudaStream_t s = (cudaStream_t)stream;
    SYM_CUDA(cudaMemsetAsync(count, 0, sizeof(uint32_t), s));
    if (g->v_end == g->v_begin) return SYM_OK;
    if (g->v_begin % 32) { set_error("v_begin must be a multiple of 32"); return SYM_EINVAL; }
    k_shard_color_frontier<<<cs_grid(g->v_end - g->v_begin, 256), 256, 0, s>>>(color, g->v_begin, g->v_end, list,
                                                                               count);
    SYM_LAUNCH_CHECK();
    return SYM_OK;
}

extern "C" int sym_shard_jp_round(const sym_graph_shard *g, const sym_params *p, const uint32_t *hbits, int admit,
                                  uint32_t *color, const int32_t *frontier, const uint32_t *count, int32_t *next,
                                  uint32_t *next_count, sym_stream_t stream) {
    SYM_TRY(cs_check(g));
    if (!color || !frontier || !count || !next || !next_count) { set_error("NULL argument"); return SYM_EINVAL; }
    ShardColorArgs A;
    SYM_TRY(cs_args(g, p, hbits, admit, &A));
    cudaStream_t s = (cudaStream_t)stream;
    SYM_CUDA(cudaMemsetAsync(next_count, 0, sizeof(uint32_t), s));
    if (g->v_end == g->v_begin) return SYM_OK;
    k_shard_jp_round<<<cs_grid(g->v_end - g->v_begin, CS_WARPS), CS_THREADS, 0, s>>>(A, color, frontier, count, next,
                                                                                     next_count);
    SYM_LAUNCH_CHECK();
    return SYM_OK;
}

extern "C" int sym_shard_color_conflicts(const sym_graph_shard *g, const sym_params *p, const uint32_t *hbits,
                                         const uint32_t *color, int32_t *list, uint32_t *count, sym_stream_t stream) {
    SYM_TRY(cs_check(g));
    if (!color || !list || !count) { set_error("NULL argument"); return SYM_EINVAL; }
    ShardColorArgs A;
    SYM_TRY(cs_args(g, p, hbits, 1, &A));
    cudaStream_t s = (cudaStream_t)stream;
    SYM_CUDA(cudaMemsetAsync(count, 0, sizeof(uint32_t), s));
    if (g->v_end == g->v_begin) return SYM_OK;
    k_shard_color_conflicts<<<cs_grid(g->v_end - g->v_begin, CS_WARPS), CS_THREADS, 0, s>>>(A, color, list, count);
    SYM_LAUNCH_CHECK();
    return SYM_OK;
}

extern "C" int sym_shard_color_clear(const sym_graph_shard *g, uint32_t *color, const int32_t *list,
                                     const uint32_t *count, sym_stream_t stream) {
    SYM_TRY(cs_check(g));
    if (!color || !list || !count) { set_error("NULL argument"); return SYM_EINVAL; }
    if (g->v_end == g->v_begin) return SYM_OK;
    k_shard_color_clear<<<cs_grid(g->v_end - g->v_begin, 256), 256, 0, (cudaStream_t)stream>>>(color, list, count);
    SYM_LAUNCH_CHECK();
    return SYM_OK;
}

extern "C" int sym_shard_color_maxh(const sym_graph_shard *g, const uint32_t *hbits, const uint32_t *color,
                                    uint32_t *max_out, sym_stream_t stream) {
    SYM_TRY(cs_check(g));
    if (!hbits || !color || !max_out) { set_error("NULL argument"); return SYM_EINVAL; }
    cudaStream_t s = (cudaStream_t)stream;
    SYM_CUDA(cudaMemsetAsync(max_out, 0, sizeof(uint32_t), s));
    if (g->v_end == g->v_begin) return SYM_OK;
    k_shard_color_maxh<<<cs_grid(g->v_end - g->v_begin, 256), 256, 0, s>>>(hbits, color, g->v_begin, g->v_end,
                                                                           max_out);
    SYM_LAUNCH_CHECK();
    return SYM_OK;
}

extern "C" int sym_shard_color_shift(const sym_graph_shard *g, const uint32_t *hbits, uint32_t *color, uint32_t M,
                                     sym_stream_t stream) {
    SYM_TRY(cs_check(g));
    if (!hbits || !color) { set_error("NULL argument"); return SYM_EINVAL; }
    if (g->v_end == g->v_begin) return SYM_OK;
    k_shard_color_shift<<<cs_grid(g->v_end - g->v_begin, 256), 256, 0, (cudaStream_t)stream>>>(hbits, color,
                                                                                               g->v_begin, g->v_end, M);
    SYM_LAUNCH_CHECK();
    return SYM_OK;
}
