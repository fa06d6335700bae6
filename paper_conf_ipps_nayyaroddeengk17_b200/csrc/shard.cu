// shard.cu -- the multi-GPU exchange layer (include/sym.h
// `sym_comm_*`, `sym_*_sharded`).
//
// One process (or host thread) per rank.  A rank owns the vertex block
// [rank*B, min(n, (rank+1)*B)), B = ceil(n/N) rounded up to 32, stores those rows
// with GLOBAL column ids, and keeps replicas of the per-vertex state the round
// kernels read (MIS status, MM mate/pick, colour).  The whole round loop runs inside
// the library (mis.cu / mm.cu / color_shard.cu: sym_{mis,mm,color}_sharded); after
// each round this file's exchange() moves ONLY the state changes of BOUNDARY
// vertices (owned vertices with a remote neighbour -- the only owned entries another
// rank's kernels can read):
//   1. all-gather of {delta count, next-frontier count} (8 B per rank);
//   2. all-gather of the delta lists, padded to the largest count (4 B entries for
//      MIS: id << 2 | status; 8 B for MM {id | matched << 31, pick} and COLOR {id,
//      colour});
//   3. a scatter kernel applies the other ranks' entries to the local replicas.
// The global frontier count comes with step 1, so termination needs no extra
// collective.  Results equal the single-GPU calls bit for bit: the
// replicas of every entry a kernel reads are exactly the owner's values after each
// exchange, and FIXED priorities make any schedule reach the same result.
//
// Transports (sym_comm):
//   NCCL  -- ncclAllGather on the caller's stream (NVLink / NVSwitch between GPUs);
//   local -- N ranks driven by N host threads of ONE process (one or several
//            devices): device-to-device copies ordered by CUDA events and a host
//            barrier.  Used to run the multi-rank path on a single GPU (tests).
#include <nccl.h>

#include <chrono>
#include <condition_variable>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <vector>

#include "internal.h"

// ------------------------------------------------------------------ communicators
struct sym_comm {
    int nranks = 1, rank = 0;
    virtual ~sym_comm() {}
    // recv[q * bytes .. (q + 1) * bytes) = rank q's send[0 .. bytes), stream-ordered on s
    virtual int allgather(const void *send, void *recv, size_t bytes, cudaStream_t s) = 0;
};

namespace sym {

static int nccl_fail(ncclResult_t r, const char *what) {
    set_error(std::string("NCCL error in ") + what + ": " + ncclGetErrorString(r));
    return SYM_ENCCL;
}

struct NcclComm : sym_comm {
    ncclComm_t comm = nullptr;
    ~NcclComm() override {
        if (comm) ncclCommDestroy(comm);
    }
    int allgather(const void *send, void *recv, size_t bytes, cudaStream_t s) override {
        if (bytes == 0) return SYM_OK;
        const ncclResult_t r = ncclAllGather(send, recv, bytes, ncclUint8, comm, s);
        return r == ncclSuccess ? SYM_OK : nccl_fail(r, "ncclAllGather");
    }
};

// N ranks in one process: a rendezvous per collective (host barrier), copies issued
// by each receiver on its own stream after the senders' data-ready events, and a
// second rendezvous so no sender reuses its buffer before every reader's copy ran.
struct LocalGroup {
    int n;
    std::mutex mu;
    std::condition_variable cv;
    int arrived = 0;
    uint64_t gen = 0;
    std::vector<const void *> send;
    std::vector<cudaEvent_t> ready, done;
    explicit LocalGroup(int n_) : n(n_), send(n_), ready(n_), done(n_) {}
    // false if the other ranks did not arrive within 10 minutes (a rank failed)
    bool barrier() {
        std::unique_lock<std::mutex> lk(mu);
        const uint64_t g = gen;
        if (++arrived == n) {
            arrived = 0;
            gen++;
            cv.notify_all();
            return true;
        }
        return cv.wait_for(lk, std::chrono::minutes(10), [&] { return gen != g; });
    }
};

static std::mutex g_groups_mu;
static std::map<uint64_t, std::weak_ptr<LocalGroup>> g_groups;

struct LocalComm : sym_comm {
    static int timeout() {
        set_error("local communicator: the other ranks did not reach the collective (a rank failed?)");
        return SYM_ECUDA;
    }
    std::shared_ptr<LocalGroup> g;
    cudaEvent_t ev_ready = nullptr, ev_done = nullptr;
    ~LocalComm() override {
        if (ev_ready) cudaEventDestroy(ev_ready);
        if (ev_done) cudaEventDestroy(ev_done);
    }
    int allgather(const void *send, void *recv, size_t bytes, cudaStream_t s) override {
        if (bytes == 0) return SYM_OK;
        SYM_CUDA(cudaEventRecord(ev_ready, s));
        {
            std::lock_guard<std::mutex> lk(g->mu);
            g->send[rank] = send;
            g->ready[rank] = ev_ready;
            g->done[rank] = ev_done;
        }
        if (!g->barrier()) return timeout();
        char *out = static_cast<char *>(recv);
        for (int q = 0; q < nranks; q++) {
            if (q == rank) {
                if (send != out + (size_t)q * bytes)
                    SYM_CUDA(cudaMemcpyAsync(out + (size_t)q * bytes, send, bytes, cudaMemcpyDefault, s));
                continue;
            }
            SYM_CUDA(cudaStreamWaitEvent(s, g->ready[q], 0));
            SYM_CUDA(cudaMemcpyAsync(out + (size_t)q * bytes, g->send[q], bytes, cudaMemcpyDefault, s));
        }
        SYM_CUDA(cudaEventRecord(ev_done, s));
        if (!g->barrier()) return timeout();
        for (int q = 0; q < nranks; q++)
            if (q != rank) SYM_CUDA(cudaStreamWaitEvent(s, g->done[q], 0));
        return SYM_OK;
    }
};

// ------------------------------------------------------------------ shard plan
int64_t shard_block(int64_t n, int nranks) {
    int64_t b = (n + nranks - 1) / nranks;
    if (b < 1) b = 1;
    return (b + 31) / 32 * 32;
}

int shard_check(const sym_graph_shard *g, const sym_params *p, const sym_comm *c, ShardPlan *plan) {
    if (!g || !p || !c) {
        set_error("NULL shard, params or communicator");
        return SYM_EINVAL;
    }
    if (g->n_global < 0 || g->n_global >= ((int64_t)1 << 30) || g->nnz < 0) {
        set_error("sharded calls need 0 <= n_global < 2^30 (MIS deltas pack id << 2 | status) and nnz >= 0");
        return SYM_EINVAL;
    }
    const int64_t B = shard_block(g->n_global, c->nranks);
    const int64_t v0 = std::min<int64_t>(g->n_global, (int64_t)c->rank * B), v1 = std::min<int64_t>(g->n_global, v0 + B);
    if (g->v_begin != v0 || g->v_end != v1) {
        set_error("shard range must be the block plan [rank*B, min(n, (rank+1)*B)), B = ceil(n/N) rounded up to 32");
        return SYM_EINVAL;
    }
    if (v1 > v0 && !g->row_ptr) { set_error("row_ptr is NULL"); return SYM_EINVAL; }
    if (g->nnz > 0 && !g->col_idx) { set_error("col_idx is NULL"); return SYM_EINVAL; }
    if (p->kind < SYM_DECOMP_NONE || p->kind > SYM_DECOMP_DEGK) { set_error("unknown decomposition kind"); return SYM_EINVAL; }
    if (p->kind == SYM_DECOMP_RAND && (p->param < 1 || p->param > 65535)) {
        set_error("RAND needs 1 <= p <= 65535");
        return SYM_EINVAL;
    }
    if (p->flags & (SYM_F_PER_ROUND | SYM_F_CONFLICT_DROP | SYM_F_SPARSER_FIRST | SYM_F_LOWER_ONLY | SYM_F_COLOR_EB |
                    SYM_F_COLOR_VB | SYM_F_ORDER_LF | SYM_F_ORDER_SF)) {
        set_error("the variant flags (f1, f3) are single-GPU only");
        return SYM_EINVAL;
    }
    plan->N = c->nranks;
    plan->rank = c->rank;
    plan->B = B;
    plan->n = g->n_global;
    plan->v0 = v0;
    plan->v1 = v1;
    plan->nl = v1 - v0;
    plan->nnz = g->nnz;
    plan->rp = g->row_ptr;
    plan->ci = g->col_idx;
    return SYM_OK;
}

// common workspace of every sharded call (the problem-specific replicas follow it)
void carve_shard_common(Arena &a, const ShardPlan &P, size_t entry, ShardCtx &x) {
    x.pair = a.take<uint32_t>(8);  // [2 parities] x {delta count, frontier count} + scratch
    x.all = a.take<uint32_t>(2 * (size_t)P.N);
    x.scratch = a.take<uint32_t>(8);
    x.bnd = a.take<uint32_t>((size_t)P.B / 32 + 1);
    x.hbits = a.take<uint32_t>((size_t)P.N * (size_t)P.B / 32 + 1);
    x.fr[0] = a.take<int32_t>((size_t)P.nl + 1);
    x.fr[1] = a.take<int32_t>((size_t)P.nl + 1);
    x.entry = entry;
    x.send = a.take<char>(entry * ((size_t)P.nl + 1));
    x.recv = a.take<char>(entry * (size_t)P.N * ((size_t)P.B + 1));
}

// ------------------------------------------------------------------ kernels
// owned vertices with at least one neighbour outside [v0, v1): bit (v - v0) of bnd
__global__ void k_sh_boundary(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci, int64_t v0, int64_t v1,
                              uint32_t *bnd) {
    const int64_t nl = v1 - v0, stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < nl; base += stride) {
        const int64_t i = base + threadIdx.x;
        bool b = false;
        if (i < nl)
            for (int64_t x = rp[i]; x < rp[i + 1] && !b; x++) {
                const int64_t w = ci[x];
                b = w < v0 || w >= v1;
            }
        const unsigned word = __ballot_sync(FULL, b);
        if (lane_id() == 0 && base + (threadIdx.x & ~31) < nl) bnd[(base + (threadIdx.x & ~31)) >> 5] = word;
    }
}

__device__ __forceinline__ int64_t sh_seg_count(const uint32_t *all, int q) { return all[2 * q]; }

// apply the other ranks' delta entries (segment q: recv[q*cap .. q*cap + count_q))
template <int P>
__global__ void k_sh_scatter(const void *recv, const uint32_t *__restrict__ all, int64_t cap, int N, int rank,
                             uint8_t *st, int32_t *mate, int32_t *pick, uint32_t *color) {
    const int64_t total = cap * N, stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total; idx += stride) {
        const int q = (int)(idx / cap);
        const int64_t i = idx - (int64_t)q * cap;
        if (q == rank || i >= sh_seg_count(all, q)) continue;
        if (P == SH_MIS) {
            const uint32_t e = static_cast<const uint32_t *>(recv)[idx];
            st[e >> 2] = (uint8_t)(e & 3u);
        } else if (P == SH_MM) {
            const uint2 e = static_cast<const uint2 *>(recv)[idx];
            const uint32_t u = e.x & 0x7fffffffu;
            pick[u] = (int32_t)e.y;
            if (e.x >> 31) {  // remote entries: only "matched" is read (sign / bitmap)
                mate[u] = (int32_t)u;
                atomicOr(color + (u >> 5), 1u << (u & 31));  // SH_MM: `color` is the matched bitmap
            }
        } else {
            const uint2 e = static_cast<const uint2 *>(recv)[idx];
            color[e.x] = e.y;
        }
    }
}

static int grid_items(int64_t items, int threads) {
    int64_t want = (items + threads - 1) / threads, cap = (int64_t)num_sms() * 8;
    return (int)(want < 1 ? 1 : (want < cap ? want : cap));
}

int shard_boundary(const ShardPlan &P, ShardCtx &x, cudaStream_t s) {
    SYM_CUDA(cudaMemsetAsync(x.bnd, 0, sizeof(uint32_t) * ((size_t)P.B / 32 + 1), s));
    if (P.nl > 0) {
        k_sh_boundary<<<grid_items(P.nl, 256), 256, 0, s>>>(P.rp, P.ci, P.v0, P.v1, x.bnd);
        SYM_LAUNCH_CHECK();
    }
    return SYM_OK;
}

// One exchange (file header): gathers the {delta count, frontier count} pair of
// parity `par`, then the padded delta lists, and applies them.  *front = the global
// frontier count.
int shard_exchange(const ShardPlan &P, ShardCtx &x, int par, int problem, uint8_t *st, int32_t *mate, int32_t *pick,
                   uint32_t *color, uint64_t *front) {
    cudaStream_t s = x.s;
    SYM_TRY(x.c->allgather(x.pair + 2 * par, x.all, 2 * sizeof(uint32_t), s));
    x.host_all.resize(2 * (size_t)P.N);
    SYM_CUDA(cudaMemcpyAsync(x.host_all.data(), x.all, 2 * sizeof(uint32_t) * P.N, cudaMemcpyDeviceToHost, s));
    SYM_CUDA(cudaStreamSynchronize(s));
    uint64_t f = 0, maxd = 0;
    for (int q = 0; q < P.N; q++) {
        maxd = std::max<uint64_t>(maxd, x.host_all[2 * q]);
        f += x.host_all[2 * q + 1];
    }
    x.exchanges++;
    x.sent_bytes += (int64_t)x.host_all[2 * P.rank] * (int64_t)x.entry;
    if (maxd > 0) {
        const size_t bytes = (size_t)maxd * x.entry;
        SYM_TRY(x.c->allgather(x.send, x.recv, bytes, s));
        x.gathered_bytes += (int64_t)bytes * P.N;
        x.max_exchange = std::max<int64_t>(x.max_exchange, (int64_t)bytes * P.N);
        const int grid = grid_items((int64_t)maxd * P.N, 256);
        if (problem == SH_MIS) k_sh_scatter<SH_MIS><<<grid, 256, 0, s>>>(x.recv, x.all, (int64_t)maxd, P.N, P.rank, st, mate, pick, color);
        else if (problem == SH_MM) k_sh_scatter<SH_MM><<<grid, 256, 0, s>>>(x.recv, x.all, (int64_t)maxd, P.N, P.rank, st, mate, pick, color);
        else k_sh_scatter<SH_COLOR><<<grid, 256, 0, s>>>(x.recv, x.all, (int64_t)maxd, P.N, P.rank, st, mate, pick, color);
        SYM_LAUNCH_CHECK();
    }
    *front = f;
    return SYM_OK;
}

// all-gather the owned words of the DEGk class bitmap (computed by the caller into
// hbits[rank*B/32 ..]) into the full replica
int shard_gather_hbits(const ShardPlan &P, ShardCtx &x) {
    const size_t words = (size_t)P.B / 32;
    return x.c->allgather(x.hbits + (size_t)P.rank * words, x.hbits, words * sizeof(uint32_t), x.s);
}

// max of one u32 over the ranks (device value in x.pair[4] -> host)
int shard_allmax(const ShardPlan &P, ShardCtx &x, uint32_t *out) {
    SYM_TRY(x.c->allgather(x.pair + 4, x.all, sizeof(uint32_t), x.s));
    std::vector<uint32_t> h(P.N);
    SYM_CUDA(cudaMemcpyAsync(h.data(), x.all, sizeof(uint32_t) * P.N, cudaMemcpyDeviceToHost, x.s));
    SYM_CUDA(cudaStreamSynchronize(x.s));
    uint32_t m = 0;
    for (uint32_t v : h) m = std::max(m, v);
    *out = m;
    return SYM_OK;
}

void shard_stats_out(const ShardCtx &x, sym_shard_stats *st) {
    if (!st) return;
    st->exchanges = x.exchanges;
    st->sent_bytes = x.sent_bytes;
    st->gathered_bytes = x.gathered_bytes;
    st->max_exchange_bytes = x.max_exchange;
}

int shard_count_boundary(const ShardPlan &P, const ShardCtx &x, int64_t *out) {
    std::vector<uint32_t> h((size_t)P.B / 32 + 1);
    SYM_CUDA(cudaMemcpyAsync(h.data(), x.bnd, sizeof(uint32_t) * h.size(), cudaMemcpyDeviceToHost, x.s));
    SYM_CUDA(cudaStreamSynchronize(x.s));
    int64_t c = 0;
    for (uint32_t w : h) c += __builtin_popcount(w);
    *out = c;
    return SYM_OK;
}

}  // namespace sym

using namespace sym;

extern "C" {

int sym_comm_unique_id(void *id) {
    if (!id) { set_error("id is NULL"); return SYM_EINVAL; }
    static_assert(sizeof(ncclUniqueId) == SYM_COMM_ID_BYTES, "NCCL unique id size");
    ncclUniqueId u;
    const ncclResult_t r = ncclGetUniqueId(&u);
    if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
    memcpy(id, &u, sizeof(u));
    return SYM_OK;
}

int sym_comm_create(sym_comm **out, int nranks, int rank, const void *id) {
    if (!out || !id || nranks < 1 || rank < 0 || rank >= nranks) {
        set_error("bad communicator arguments");
        return SYM_EINVAL;
    }
    *out = nullptr;
    auto *c = new NcclComm();
    c->nranks = nranks;
    c->rank = rank;
    ncclUniqueId u;
    memcpy(&u, id, sizeof(u));
    const ncclResult_t r = ncclCommInitRank(&c->comm, nranks, u, rank);
    if (r != ncclSuccess) {
        c->comm = nullptr;
        delete c;
        return nccl_fail(r, "ncclCommInitRank");
    }
    *out = c;
    return SYM_OK;
}

int sym_comm_create_local(sym_comm **out, int nranks, int rank, uint64_t group) {
    if (!out || nranks < 1 || rank < 0 || rank >= nranks) {
        set_error("bad communicator arguments");
        return SYM_EINVAL;
    }
    *out = nullptr;
    std::shared_ptr<LocalGroup> g;
    {
        std::lock_guard<std::mutex> lk(g_groups_mu);
        g = g_groups[group].lock();
        if (!g) {
            g = std::make_shared<LocalGroup>(nranks);
            g_groups[group] = g;
        } else if (g->n != nranks) {
            set_error("local group exists with a different rank count");
            return SYM_EINVAL;
        }
    }
    auto *c = new LocalComm();
    c->nranks = nranks;
    c->rank = rank;
    c->g = g;
    if (cudaEventCreateWithFlags(&c->ev_ready, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->ev_done, cudaEventDisableTiming) != cudaSuccess) {
        delete c;
        return cuda_fail(cudaGetLastError(), "cudaEventCreate", __FILE__, __LINE__);
    }
    *out = c;
    return SYM_OK;
}

int sym_comm_destroy(sym_comm *c) {
    delete c;
    return SYM_OK;
}

int sym_comm_size(const sym_comm *c, int *nranks, int *rank) {
    if (!c) { set_error("communicator is NULL"); return SYM_EINVAL; }
    if (nranks) *nranks = c->nranks;
    if (rank) *rank = c->rank;
    return SYM_OK;
}

}  // extern "C"
