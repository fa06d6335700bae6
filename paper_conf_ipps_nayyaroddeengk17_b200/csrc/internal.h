// internal.h -- host-side internals of libsym (not part of the C-ABI).
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include <algorithm>
#include <atomic>
#include <string>
#include <vector>

// round kernels (MIS, MM) launch one resident wave instead of 8 CTAs per SM
#ifndef SYM_ROUND_ONE_WAVE
#define SYM_ROUND_ONE_WAVE 1
#endif

#include "../../include/sym.h"
#include "common.cuh"

namespace sym {

// ------------------------------------------------------------------ errors
void set_error(const std::string &msg);
int cuda_fail(cudaError_t e, const char *what, const char *file, int line);

#define SYM_CUDA(call)                                                          \
    do {                                                                        \
        cudaError_t e_ = (call);                                                \
        if (e_ != cudaSuccess) return ::sym::cuda_fail(e_, #call, __FILE__, __LINE__); \
    } while (0)
#define SYM_LAUNCH_CHECK() SYM_CUDA(cudaGetLastError())
#define SYM_TRY(expr)               \
    do {                            \
        int rc_ = (expr);           \
        if (rc_ != SYM_OK) return rc_; \
    } while (0)

// ------------------------------------------------------------------ workspace carving
// A bump allocator over the caller's workspace.  In "dry" mode (base == nullptr) it
// only counts bytes, so sym_workspace_bytes and the real carving share one code path.
struct Arena {
    char *base = nullptr;
    size_t cap = 0, used = 0;
    bool dry() const { return base == nullptr; }
    template <class T>
    T *take(size_t count) {
        size_t off = (used + 255) & ~(size_t)255;
        used = off + count * sizeof(T) + 0;
        if (dry()) return nullptr;
        return reinterpret_cast<T *>(base + off);
    }
};

// device control block: counters used by the round loops
struct Ctl {
    uint32_t ring[4];       // frontier counts (ring of 3)
    uint32_t huge[2];       // deferred long-row counts (ring of 2)
    uint32_t cnt_front;     // class list: front count
    uint32_t cnt_back;      // class list: back count
    uint32_t tile_counter;  // dynamic tile ids for the look-back split
    uint32_t flag;          // generic flag / error word
    uint32_t max_color;     // COLOR
    uint32_t conflicts;     // COLOR-RAND |V'|
    uint32_t done;          // JP: coloured count
    uint32_t q_head, q_tail;
    uint32_t pad[15];
    uint64_t result;        // reductions
    uint64_t scanned;       // SYM_F_STATS: arcs inspected
    uint32_t hist[1 << 12]; // per-round frontier sizes (stats)
};

// decomposition view used by the flows (device pointers)
struct Split {
    const int64_t *rp_in = nullptr, *rp_x = nullptr;
    const int32_t *ci_in = nullptr, *ci_x = nullptr;
    int64_t nnz_in = -1;  // known on the host only for a caller-supplied decomposition
    int64_t nnz_x = -1;
};

struct Graph {
    int64_t n, nnz;
    const int64_t *rp;
    const int32_t *ci;
};

// ------------------------------------------------------------------ decomposition (decompose.cu)
#ifndef SYM_POLL_BATCH
#define SYM_POLL_BATCH 4  // MIS / MM rounds launched per host poll of the frontier count
#endif
#ifndef SYM_SPLIT_THREADS
#define SYM_SPLIT_THREADS 256
#endif
constexpr int SPLIT_THREADS = SYM_SPLIT_THREADS;
constexpr int SPLIT_PER_THREAD = 4096 / SPLIT_THREADS;  // tiles of 4096 arcs
constexpr int SPLIT_TILE = SPLIT_THREADS * SPLIT_PER_THREAD;  // arcs per tile

// BRIDGE decomposition scratch (bridge.cu; carved only for SYM_DECOMP_BRIDGE)
struct BridgeWs {
    int32_t *cc = nullptr, *level = nullptr, *par = nullptr;
    uint8_t *mark = nullptr;
    int32_t *fr[2] = {nullptr, nullptr};
    int64_t *bsum = nullptr;
    uint32_t *ctr = nullptr;
};
void carve_bridge_ws(Arena &a, int64_t n, BridgeWs &w);
int run_bridge_split(const Graph &g, const BridgeWs &w, int64_t *rp_in, int32_t *ci_in, int64_t *rp_x, int32_t *ci_x,
                     uint16_t *label, cudaStream_t s);

struct SplitWs {
    uint32_t *hbits = nullptr;   // DEGk V_H bitmap [ceil(n/32)]
    int64_t *first_row = nullptr;
    uint64_t *tile_state = nullptr;
    int64_t ntiles = 0;
    BridgeWs br;                 // SYM_DECOMP_BRIDGE only
};
void carve_split_ws(Arena &a, int64_t n, int64_t nnz, SplitWs &w);

// class bitmap (+ optional vertex lists: class-0 from the front, class-1 from the back)
int launch_classify_degk(const Graph &g, uint32_t k, uint32_t *hbits, int32_t *vlist, Ctl *ctl,
                         cudaStream_t s);
// first_row[t] = first row whose arcs start at or after t*SPLIT_TILE (split.cu)
__global__ void k_first_row(const int64_t *__restrict__ rp, int64_t n, int64_t ntiles, int64_t *__restrict__ first_row);
int launch_first_row(const Graph &g, int64_t ntiles, int64_t *first_row, cudaStream_t s);

// round 0 of a MIS (mode 0) or MM (mode 1) phase as one streaming segmented max
// (round0.cu); returns SYM_EINVAL without launching when the phase CSR is empty
int run_round0(int mode, const Graph &g, const int64_t *first_row, int64_t ntiles, Key k,
               unsigned long long *gmax, uint8_t *st, int32_t *pick, const uint32_t *hfilter, int32_t *out_list,
               uint32_t *out_cnt, cudaStream_t s);

// decompose into caller buffers (rp_in, ci_in, rp_x, ci_x) ; kind in {NONE,RAND,DEGK}.
// row_base = global id of local row 0 (a shard's row block; RAND/NONE only, since the
// DEGk bitmap is indexed by local row)
int run_split(const Graph &g, int kind, uint32_t param, uint64_t seed, const SplitWs &w, Ctl *ctl,
              int64_t *rp_in, int32_t *ci_in, int64_t *rp_x, int32_t *ci_x, uint16_t *label, cudaStream_t s,
              int64_t row_base = 0);

// ------------------------------------------------------------------ profiling hook (profile.cu)
// Every hot launch may record a CUDA event pair on its stream plus two byte counts:
// alg  = SURVEY §8(d)'s algorithmic bytes (what the method must move: rounds 4 B per
//        scanned arc + 9 B per active vertex; split 8 B/arc + 24 B/row pointer; JP
//        8 B/arc + 12 B/vertex), and
// impl = what this implementation's kernel moves (its own HBM/L2 words: lists,
//        records, counters).
bool prof_on();
void prof_begin(const char *cls, cudaStream_t s);
void prof_end(cudaStream_t s, double alg_bytes, double impl_bytes);  // < 0: unknown on the host
// a zeroed device counter pair {alg, impl} (nullptr unless profiling) that kernels
// accumulate into; prof_end_dev closes the event pair and reads it at collect
unsigned long long *prof_counter(cudaStream_t s);
void prof_end_dev(cudaStream_t s, unsigned long long *ctr);

// warp-aggregated add of per-lane byte counts into a profiling counter pair (nullable)
__device__ __forceinline__ void prof_add(unsigned long long *ctr, unsigned long long alg, unsigned long long impl) {
    if (ctr == nullptr) return;
    for (int d = 16; d; d >>= 1) {
        alg += __shfl_xor_sync(0xffffffffu, alg, d);
        impl += __shfl_xor_sync(0xffffffffu, impl, d);
    }
    if ((threadIdx.x & 31) == 0) {
        if (alg) atomicAdd(ctr, alg);
        if (impl) atomicAdd(ctr + 1, impl);
    }
}

// ------------------------------------------------------------------ helpers (api.cu)
int read_u32(const uint32_t *dev, uint32_t *host, cudaStream_t s);
int read_u64(const uint64_t *dev, uint64_t *host, cudaStream_t s);
int num_sms();
int current_device();

// A value cached per CUDA device (grid sizes from occupancy queries, function
// attributes): computed lazily by `compute` on the first call on each device.  A
// process may drive several GPUs from several host threads; the slots are atomics
// (a racing first call computes the same value twice, which is harmless).
constexpr int SYM_MAX_DEVICES = 64;
template <class F>
int dev_cached(std::atomic<int> *slots, F compute) {
    const int d = current_device();
    if (d < 0 || d >= SYM_MAX_DEVICES) return compute();
    int v = slots[d].load(std::memory_order_relaxed);
    if (v == 0) {
        v = compute();
        slots[d].store(v, std::memory_order_relaxed);
    }
    return v;
}

// ------------------------------------------------------------------ flows
struct FlowArgs {
    Graph g;
    sym_params p;
    Split split;                // valid when p.kind != NONE
    uint32_t *hbits;            // DEGk bitmap workspace
    int64_t *first_row;         // tile -> first row table (capacity first_row_cap tiles)
    int64_t first_row_cap;
    Ctl *ctl;
    sym_stats *stats;
    cudaStream_t stream;
};

struct MisWs {
    uint8_t *st = nullptr;
    int32_t *vlist = nullptr;          // class lists (front / back)
    int32_t *fr[2] = {nullptr, nullptr};  // frontier ping-pong
    int32_t *fp[2] = {nullptr, nullptr};  // resume offsets, parallel to fr
    int64_t *huge = nullptr;           // deferred (v, resume) pairs
    int64_t huge_cap = 0;
    unsigned long long *gmax = nullptr;  // round 0: maxima of rows crossing tiles
    uint8_t *mark = nullptr;             // SYM_F_CONFLICT_DROP: dropped In vertices
};

struct MmWs {
    int32_t *pick[2] = {nullptr, nullptr};
    int32_t *vlist = nullptr;
    int32_t *fr[2] = {nullptr, nullptr};
    int64_t *huge = nullptr;
    unsigned long long *huge_best = nullptr;
    int64_t huge_cap = 0;
    unsigned long long *gmax = nullptr;  // round 0: maxima of rows crossing tiles
    uint32_t *mbits = nullptr;           // matched bitmap
    int32_t *alt = nullptr;  // second-heaviest believed-live neighbour at the last scan (-1: none)
};

struct ColorWs {
    int32_t *ov = nullptr;         // compact id -> original
    uint32_t *hdeg = nullptr;      // higher / lower degrees (build), fill cursors
    uint32_t *ldeg = nullptr;
    uint32_t *arank = nullptr;     // per 32 ids {bitmap of S vertices with phase arcs,
                                   //   exclusive popcount prefix}: compact id = rank
    uint4 *hot = nullptr;          // hot per-vertex state {colour, count, bitmap word 0,
                                   //   offset of the extra bitmap words}
    uint4 *meta = nullptr;         // per-vertex own data (2 x 16 B)
    uint32_t *ul[2] = {nullptr, nullptr};  // active lists (ping-pong by round)
    uint32_t *lst = nullptr;       // watch / higher / lower lists
    int64_t lst_words = 0;
    uint32_t *xb = nullptr;        // bitmap words for colours > 32
    uint32_t *tcnt = nullptr;      // build scan scratch (per tile)
    unsigned long long *tsum = nullptr;
    int64_t ntiles = 0;
    uint4 *task = nullptr;         // push tasks of one round
    uint4 *btask = nullptr;        // watch-list build tasks of one round
    int64_t task_cap = 0;
    int64_t *queue = nullptr;      // build: (piece << 32 | h) items of the huge rows
    int32_t *vlist = nullptr;
    uint8_t *mark = nullptr;       // COLOR-RAND V'
    uint32_t *okey = nullptr;      // SYM_F_ORDER_LF / _SF order terms
    uint32_t *sync = nullptr;      // rounds kernel: barrier / counter / error words
};

int phase_arcs(const FlowArgs &f, const int64_t *rp, int64_t *out);  // round0.cu

void carve_mis_ws(Arena &a, int64_t n, int64_t nnz, MisWs &w);
int run_mis(const FlowArgs &f, MisWs &w, uint8_t *in_set);

void carve_mm_ws(Arena &a, int64_t n, int64_t nnz, MmWs &w);
int run_mm(const FlowArgs &f, MmWs &w, int32_t *mate);

void carve_color_ws(Arena &a, int64_t n, int64_t nnz, ColorWs &w);
int run_color(const FlowArgs &f, ColorWs &w, uint32_t *color);
int run_color_spec(const FlowArgs &f, ColorWs &w, uint32_t *color);  // spec.cu (SYM_F_COLOR_EB / _VB)

// ------------------------------------------------------------------ multi-GPU (shard.cu)
enum { SH_MIS = 0, SH_MM = 1, SH_COLOR = 2 };

// a rank's block of the shard plan (shard.cu header): rows [v0, v1) with global ids
struct ShardPlan {
    int N = 1, rank = 0;
    int64_t B = 0, n = 0, v0 = 0, v1 = 0, nl = 0, nnz = 0;
    const int64_t *rp = nullptr;
    const int32_t *ci = nullptr;
};

// per-call state of a sharded flow (device buffers carved from the workspace)
struct ShardCtx {
    sym_comm *c = nullptr;
    cudaStream_t s = nullptr;
    uint32_t *pair = nullptr;     // [2 parities] x {delta count, frontier count}, [4] all-max value
    uint32_t *all = nullptr;      // gathered pairs [2N]
    uint32_t *scratch = nullptr;  // round-kernel counters (zeroed per round)
    uint32_t *bnd = nullptr;      // owned boundary bitmap
    uint32_t *hbits = nullptr;    // DEGk class bitmap replica [N*B/32]
    int32_t *fr[2] = {nullptr, nullptr};
    size_t entry = 0;             // delta entry bytes
    void *send = nullptr, *recv = nullptr;
    std::vector<uint32_t> host_all;
    uint32_t exchanges = 0;
    int64_t sent_bytes = 0, gathered_bytes = 0, max_exchange = 0;
    // round r reads list fr[r & 1] with its count in pair[2 ((r + 1) & 1) + 1] and
    // writes the next list fr[(r + 1) & 1], its count pair[2 (r & 1) + 1] and its
    // delta count pair[2 (r & 1)]; a phase's frontier kernel fills fr[0] / pair[3]
    int32_t *list_in(int r) const { return fr[r & 1]; }
    int32_t *list_out(int r) const { return fr[(r + 1) & 1]; }
    uint32_t *cnt_in(int r) const { return pair + 2 * ((r + 1) & 1) + 1; }
    uint32_t *cnt_out(int r) const { return pair + 2 * (r & 1) + 1; }
    uint32_t *dcnt(int r) const { return pair + 2 * (r & 1); }
};

int64_t shard_block(int64_t n, int nranks);
int shard_check(const sym_graph_shard *g, const sym_params *p, const sym_comm *c, ShardPlan *plan);
void carve_shard_common(Arena &a, const ShardPlan &P, size_t entry, ShardCtx &x);
int shard_boundary(const ShardPlan &P, ShardCtx &x, cudaStream_t s);
// (SH_MIS: st; SH_MM: mate, pick and, in `color`, the matched bitmap; SH_COLOR: color)
int shard_exchange(const ShardPlan &P, ShardCtx &x, int par, int problem, uint8_t *st, int32_t *mate, int32_t *pick,
                   uint32_t *color, uint64_t *front);
int shard_gather_hbits(const ShardPlan &P, ShardCtx &x);
int shard_allmax(const ShardPlan &P, ShardCtx &x, uint32_t *out);
int shard_count_boundary(const ShardPlan &P, const ShardCtx &x, int64_t *out);
void shard_stats_out(const ShardCtx &x, sym_shard_stats *st);
// workspace layouts of the sharded MM / COLOR calls (mm.cu, color_shard.cu)
void carve_mm_sharded_dry(Arena &a, const ShardPlan &P, const sym_params *p, ShardCtx &x);
void carve_color_sharded_dry(Arena &a, const ShardPlan &P, ShardCtx &x);

// the workspace of a sharded call: carve into a dry arena (sizes) or the real one
template <class F>
int shard_carve_ws(void *ws, size_t ws_bytes, F carve) {
    Arena dry;
    carve(dry);
    const size_t need = dry.used + 256;
    if (!ws || ws_bytes < need) {
        set_error("sharded workspace too small: need " + std::to_string(need) + " bytes");
        return SYM_EWORKSPACE;
    }
    Arena a;
    a.base = (char *)(((uintptr_t)ws + 255) & ~(uintptr_t)255);
    a.cap = ws_bytes;
    carve(a);
    return SYM_OK;
}

}  // namespace sym
