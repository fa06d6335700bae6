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

// ---- deltas of the sharded flow (shard.cu): {id, colour} of owned boundary vertices
// coloured in this round (the round's input list entries, uncoloured at its start)
__global__ void k_sh_delta_col(const int32_t *__restrict__ list, const uint32_t *cnt, const uint32_t *color,
                               const uint32_t *__restrict__ bnd, int64_t v0, uint2 *send, uint32_t *dcnt) {
    const int64_t c = *cnt, stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < c; base += stride) {
        const int64_t i = base + threadIdx.x;
        const int32_t v = i < c ? list[i] : -1;
        const uint32_t cv = v >= 0 ? color[v] : 0u;
        const bool b = cv != 0 && ((bnd[(v - v0) >> 5] >> ((v - v0) & 31)) & 1u);
        const int64_t slot = warp_append(b, dcnt);
        if (slot >= 0) send[slot] = make_uint2((uint32_t)v, cv);
    }
}

// COLOR-Rand fix-up, step 2: uncolour V' (the conflicts list), boundary ones as deltas
__global__ void k_sh_clear_col(const int32_t *__restrict__ list, const uint32_t *cnt, uint32_t *color,
                               const uint32_t *__restrict__ bnd, int64_t v0, uint2 *send, uint32_t *dcnt) {
    const int64_t c = *cnt, stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < c; base += stride) {
        const int64_t i = base + threadIdx.x;
        const int32_t v = i < c ? list[i] : -1;
        if (v >= 0) color[v] = 0u;
        const bool b = v >= 0 && ((bnd[(v - v0) >> 5] >> ((v - v0) & 31)) & 1u);
        const int64_t slot = warp_append(b, dcnt);
        if (slot >= 0) send[slot] = make_uint2((uint32_t)v, 0u);
    }
}

__global__ void k_sh_col_out(const uint32_t *color, int64_t v0, int64_t v1, uint32_t *out) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = v0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < v1; v += stride) out[v - v0] = color[v];
}

// DEGk class bits of the owned rows (deg > k, Alg 3), mis.cu
__global__ void k_shard_classify(const int64_t *__restrict__ rp, int64_t v0, int64_t v1, uint32_t k,
                                 uint32_t *__restrict__ hbits);

}  // namespace sym

using namespace sym;

// ------------------------------------------------------------------ sharded COLOR (C-ABI)
static int cs_grid(int64_t items, int per_cta) {
    int64_t want = (items + per_cta - 1) / per_cta;
    int64_t cap = (int64_t)num_sms() * 8;
    return (int)(want < 1 ? 1 : (want < cap ? want : cap));
}

static void carve_color_sharded(Arena &a, const ShardPlan &P, ShardCtx &x, uint32_t *&color) {
    carve_shard_common(a, P, sizeof(uint2), x);
    color = a.take<uint32_t>((size_t)P.N * (size_t)P.B);
}

namespace sym {
void carve_color_sharded_dry(Arena &a, const ShardPlan &P, ShardCtx &x) {
    uint32_t *c;
    carve_color_sharded(a, P, x, c);
}
}  // namespace sym

// Jones-Plassmann rounds over the owned list fr[0] / pair[3] (filled by the
// caller), exchanging the boundary colours after every round
static int color_sharded_phase(const ShardPlan &P, ShardCtx &x, const sym_params *p, const ShardColorArgs &A,
                               uint32_t *color, uint32_t *rounds) {
    cudaStream_t s = x.s;
    const uint32_t maxr = p->max_rounds ? p->max_rounds : 0xffffffffu;
    int64_t local = P.nl;
    for (int r = 0;; r++) {
        if ((uint32_t)r >= maxr) {
            set_error("sharded COLOR phase did not converge within max_rounds");
            return SYM_EROUNDS;
        }
        SYM_CUDA(cudaMemsetAsync(x.dcnt(r), 0, 2 * sizeof(uint32_t), s));
        if (local > 0) {
            k_shard_jp_round<<<cs_grid(local, CS_WARPS), CS_THREADS, 0, s>>>(A, color, x.list_in(r), x.cnt_in(r),
                                                                            x.list_out(r), x.cnt_out(r));
            SYM_LAUNCH_CHECK();
            k_sh_delta_col<<<cs_grid(local, 256), 256, 0, s>>>(x.list_in(r), x.cnt_in(r), color, x.bnd, P.v0,
                                                               (uint2 *)x.send, x.dcnt(r));
            SYM_LAUNCH_CHECK();
        }
        uint64_t front = 0;
        SYM_TRY(shard_exchange(P, x, r & 1, SH_COLOR, nullptr, nullptr, nullptr, color, &front));
        local = x.host_all[2 * P.rank + 1];
        if (front == 0) {
            *rounds = (uint32_t)(r + 1);
            return SYM_OK;
        }
    }
}

extern "C" int sym_color_sharded(const sym_graph_shard *g, const sym_params *p, sym_comm *c, void *ws,
                                 size_t ws_bytes, uint32_t *color_out, sym_shard_stats *stats, sym_stream_t stream) {
    ShardPlan P;
    SYM_TRY(shard_check(g, p, c, &P));
    if (P.nl > 0 && !color_out) { set_error("color is NULL"); return SYM_EINVAL; }
    ShardCtx x;
    uint32_t *color = nullptr;
    SYM_TRY(shard_carve_ws(ws, ws_bytes, [&](Arena &a) {
        x = ShardCtx();
        carve_color_sharded(a, P, x, color);
    }));
    x.c = c;
    x.s = (cudaStream_t)stream;
    cudaStream_t s = x.s;
    if (stats) memset(stats, 0, sizeof(*stats));
    SYM_CUDA(cudaMemsetAsync(color, 0, sizeof(uint32_t) * (size_t)P.N * (size_t)P.B, s));
    SYM_CUDA(cudaMemsetAsync(x.pair, 0, 8 * sizeof(uint32_t), s));
    SYM_TRY(shard_boundary(P, x, s));
    ShardColorArgs A;
    A.rp = P.rp;
    A.ci = P.ci;
    A.v0 = P.v0;
    A.v1 = P.v1;
    A.kind = p->kind;
    A.param = p->param;
    A.kr = stream_key(p->seed, TAG_RAND, 0);
    A.kv = stream_key(p->seed, TAG_VERTEX, 0);
    A.hbits = x.hbits;
    A.admit = p->kind == SYM_DECOMP_NONE ? 0 : 1;
    if (p->kind == SYM_DECOMP_DEGK) {
        if (P.nl > 0) {
            k_shard_classify<<<cs_grid(P.nl, 256), 256, 0, s>>>(P.rp, P.v0, P.v1, p->param, x.hbits);
            SYM_LAUNCH_CHECK();
        }
        SYM_TRY(shard_gather_hbits(P, x));
    }
    uint32_t rounds[3] = {0, 0, 0};
    // phase 1: every owned vertex (NONE: on G; DEGk: G_H and G_L at once; RAND: the parts)
    SYM_CUDA(cudaMemsetAsync(x.cnt_in(0), 0, sizeof(uint32_t), s));
    if (P.nl > 0) {
        k_shard_color_frontier<<<cs_grid(P.nl, 256), 256, 0, s>>>(color, P.v0, P.v1, x.list_in(0), x.cnt_in(0));
        SYM_LAUNCH_CHECK();
    }
    SYM_TRY(color_sharded_phase(P, x, p, A, color, &rounds[0]));
    uint64_t front = 0;
    if (p->kind == SYM_DECOMP_DEGK) {
        // Alg 9: M = max C_H over all ranks; V_L colours += M (owned only: nothing
        // reads a remote colour after this)
        SYM_CUDA(cudaMemsetAsync(x.pair + 4, 0, sizeof(uint32_t), s));
        if (P.nl > 0) {
            k_shard_color_maxh<<<cs_grid(P.nl, 256), 256, 0, s>>>(x.hbits, color, P.v0, P.v1, x.pair + 4);
            SYM_LAUNCH_CHECK();
        }
        uint32_t M = 0;
        SYM_TRY(shard_allmax(P, x, &M));
        if (P.nl > 0) {
            k_shard_color_shift<<<cs_grid(P.nl, 256), 256, 0, s>>>(x.hbits, color, P.v0, P.v1, M);
            SYM_LAUNCH_CHECK();
        }
    } else if (p->kind == SYM_DECOMP_RAND) {
        // Alg 8: V' = owned endpoints of monochromatic cross arcs -> fr[0] /
        // pair[3]; uncolour them (boundary ones exchanged); recolour V' against G
        SYM_CUDA(cudaMemsetAsync(x.pair, 0, 4 * sizeof(uint32_t), s));
        if (P.nl > 0) {
            k_shard_color_conflicts<<<cs_grid(P.nl, CS_WARPS), CS_THREADS, 0, s>>>(A, color, x.list_in(0),
                                                                                   x.cnt_in(0));
            SYM_LAUNCH_CHECK();
            k_sh_clear_col<<<cs_grid(P.nl, 256), 256, 0, s>>>(x.list_in(0), x.cnt_in(0), color, x.bnd, P.v0,
                                                              (uint2 *)x.send, x.pair);
            SYM_LAUNCH_CHECK();
        }
        SYM_TRY(shard_exchange(P, x, 0, SH_COLOR, nullptr, nullptr, nullptr, color, &front));
        ShardColorArgs A2 = A;
        A2.admit = 0;
        SYM_TRY(color_sharded_phase(P, x, p, A2, color, &rounds[1]));
    }
    if (P.nl > 0) {
        k_sh_col_out<<<cs_grid(P.nl, 256), 256, 0, s>>>(color, P.v0, P.v1, color_out);
        SYM_LAUNCH_CHECK();
    }
    if (stats) {
        memcpy(stats->rounds, rounds, sizeof(rounds));
        shard_stats_out(x, stats);
        SYM_TRY(shard_count_boundary(P, x, &stats->boundary));
    }
    return SYM_OK;
}
