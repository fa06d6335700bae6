// api.cu -- the C-ABI entry points of libsym (include/sym.h): argument checks,
// workspace carving and dispatch to the decomposition / MIS / MM / COLOR flows.
#include <cstdio>
#include <cstring>
#include <string>

#include "internal.h"

#define SYM_VERSION "symbreak-b200 0.1.0 sm_100a"

namespace sym {

static thread_local std::string g_err;

void set_error(const std::string &msg) { g_err = msg; }

int cuda_fail(cudaError_t e, const char *what, const char *file, int line) {
    char buf[768];
    snprintf(buf, sizeof(buf), "CUDA error %d (%s) in %s at %s:%d", (int)e, cudaGetErrorString(e), what, file, line);
    g_err = buf;
    return SYM_ECUDA;
}

int current_device() {
    int dev = -1;
    return cudaGetDevice(&dev) == cudaSuccess ? dev : -1;
}

int num_sms() {
    static std::atomic<int> slots[SYM_MAX_DEVICES];
    return dev_cached(slots, [] {
        int v = 0;
        const int dev = current_device();
        if (dev >= 0 && cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess && v > 0)
            return v;
        return 148;
    });
}

int read_u32(const uint32_t *dev, uint32_t *host, cudaStream_t s) {
    SYM_CUDA(cudaMemcpyAsync(host, dev, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    SYM_CUDA(cudaStreamSynchronize(s));
    return SYM_OK;
}

int read_u64(const uint64_t *dev, uint64_t *host, cudaStream_t s) {
    SYM_CUDA(cudaMemcpyAsync(host, dev, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    SYM_CUDA(cudaStreamSynchronize(s));
    return SYM_OK;
}

// ------------------------------------------------------------------ validation kernel
// warp per row: ids in range, no self-loop, strictly ascending row, symmetric arc
__global__ void k_validate(const int64_t *__restrict__ rp, const int32_t *__restrict__ ci, int64_t n, int64_t nnz,
                           unsigned long long *bad) {
    const int lane = lane_id();
    const int64_t warp_g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long local = 0;
    if (warp_g == 0 && lane == 0 && (rp[0] != 0 || rp[n] != nnz)) local++;
    for (int64_t v = warp_g; v < n; v += nw) {
        int64_t b = rp[v], e = rp[v + 1];
        if (e < b || b < 0 || e > nnz) {
            if (lane == 0) local++;
            continue;
        }
        for (int64_t x = b + lane; x < e; x += 32) {
            int32_t w = ci[x];
            bool ok = (w >= 0) && (w < n) && (w != v);
            if (ok && x + 1 < e) ok = ci[x + 1] > w;
            if (ok) {
                int64_t lo = rp[w], hi = rp[w + 1];
                if (hi < lo || lo < 0 || hi > nnz) {
                    ok = false;
                } else {
                    bool found = false;
                    while (lo < hi) {
                        int64_t mid = (lo + hi) >> 1;
                        int32_t c = ci[mid];
                        if (c == (int32_t)v) { found = true; break; }
                        if (c < (int32_t)v) lo = mid + 1;
                        else hi = mid;
                    }
                    ok = found;
                }
            }
            if (!ok) local++;
        }
    }
    for (int d = 16; d; d >>= 1) local += __shfl_xor_sync(FULL, local, d);
    if (lane == 0 && local) atomicAdd(bad, local);
}

// ------------------------------------------------------------------ workspace layout
struct Layout {
    Ctl *ctl = nullptr;
    SplitWs sw;
    int64_t *rp_in = nullptr, *rp_x = nullptr;
    int32_t *ci_in = nullptr, *ci_x = nullptr;
    MisWs mis;
    MmWs mm;
    ColorWs col;
};

static void carve(Arena &a, int64_t n, int64_t nnz, const sym_params *p, int problem, Layout &L) {
    L.ctl = a.take<Ctl>(1);
    if (problem == SYM_PROBLEM_VALIDATE) return;
    carve_split_ws(a, n, nnz, L.sw);
    if (p->kind == SYM_DECOMP_BRIDGE && (problem == SYM_PROBLEM_DECOMPOSE || !(p->flags & SYM_F_EXT_DECOMP)))
        carve_bridge_ws(a, n, L.sw.br);
    if (problem == SYM_PROBLEM_DECOMPOSE) return;
    bool internal = p->kind != SYM_DECOMP_NONE && !(p->flags & SYM_F_EXT_DECOMP);
    if (internal) {
        L.rp_in = a.take<int64_t>((size_t)n + 1);
        L.rp_x = a.take<int64_t>((size_t)n + 1);
        L.ci_in = a.take<int32_t>((size_t)nnz + 1);
        L.ci_x = a.take<int32_t>((size_t)nnz + 1);
    }
    if (problem == SYM_PROBLEM_MIS) carve_mis_ws(a, n, nnz, L.mis);
    else if (problem == SYM_PROBLEM_MM) carve_mm_ws(a, n, nnz, L.mm);
    else if (problem == SYM_PROBLEM_COLOR) carve_color_ws(a, n, nnz, L.col);
}

static int check_graph(const sym_graph *g) {
    if (!g) { set_error("graph is NULL"); return SYM_EINVAL; }
    if (g->n < 0 || g->nnz < 0) { set_error("negative n or nnz"); return SYM_EINVAL; }
    if (g->n >= ((int64_t)1 << 31) - 1) { set_error("n must be < 2^31 - 1 (int32 vertex ids)"); return SYM_EINVAL; }
    if (g->n > 0 && !g->row_ptr) { set_error("row_ptr is NULL"); return SYM_EINVAL; }
    if (g->nnz > 0 && !g->col_idx) { set_error("col_idx is NULL"); return SYM_EINVAL; }
    if (g->n == 0 && g->nnz != 0) { set_error("nnz must be 0 when n == 0"); return SYM_EINVAL; }
    return SYM_OK;
}

static int check_params(const sym_params *p) {
    if (!p) { set_error("params is NULL"); return SYM_EINVAL; }
    if (p->kind < SYM_DECOMP_NONE || p->kind > SYM_DECOMP_BRIDGE) { set_error("unknown decomposition kind"); return SYM_EINVAL; }
    if (p->kind == SYM_DECOMP_BRIDGE && (p->flags & (SYM_F_CONFLICT_DROP | SYM_F_SPARSER_FIRST | SYM_F_LOWER_ONLY |
                                                     SYM_F_COLOR_EB | SYM_F_COLOR_VB))) {
        set_error("BRIDGE supports the FIXED flows, SYM_F_PER_ROUND and the LF / SF orders only");
        return SYM_EINVAL;
    }
    if (p->kind == SYM_DECOMP_RAND && (p->param < 1 || p->param > 65535)) {
        set_error("RAND needs 1 <= p <= 65535");
        return SYM_EINVAL;
    }
    if ((p->flags & (SYM_F_COLOR_EB | SYM_F_COLOR_VB)) && p->kind == SYM_DECOMP_DEGK && p->param > 62) {
        set_error("the literal G_L loop (SYM_F_COLOR_EB / _VB with DEGk) supports k <= 62");
        return SYM_EINVAL;
    }
    if ((p->flags & SYM_F_ORDER_LF) && (p->flags & SYM_F_ORDER_SF)) {
        set_error("SYM_F_ORDER_LF and SYM_F_ORDER_SF are alternative orders");
        return SYM_EINVAL;
    }
    if ((p->flags & (SYM_F_ORDER_LF | SYM_F_ORDER_SF)) && (p->flags & (SYM_F_COLOR_EB | SYM_F_COLOR_VB))) {
        set_error("the LF / SF orders apply to Jones-Plassmann, not to the speculative subroutines");
        return SYM_EINVAL;
    }
    if ((p->flags & SYM_F_CONFLICT_DROP) && (p->flags & SYM_F_SPARSER_FIRST)) {
        set_error("SYM_F_CONFLICT_DROP and SYM_F_SPARSER_FIRST are alternative MIS-Rand flows");
        return SYM_EINVAL;
    }
    return SYM_OK;
}

static int carve_ws(const sym_graph *g, const sym_params *p, int problem, void *ws, size_t ws_bytes, Layout &L) {
    Arena dry;
    carve(dry, g->n, g->nnz, p, problem, L);
    size_t need = dry.used + 256;
    if (!ws || ws_bytes < need) {
        char buf[160];
        snprintf(buf, sizeof(buf), "workspace too small: need %zu bytes, got %zu", need, ws ? ws_bytes : (size_t)0);
        set_error(buf);
        return SYM_EWORKSPACE;
    }
    Arena a;
    a.base = (char *)(((uintptr_t)ws + 255) & ~(uintptr_t)255);
    a.cap = ws_bytes;
    L = Layout();
    carve(a, g->n, g->nnz, p, problem, L);
    return SYM_OK;
}

static int validate_impl(const sym_graph *g, Ctl *ctl, int64_t *bad_out, cudaStream_t s) {
    SYM_CUDA(cudaMemsetAsync(&ctl->result, 0, sizeof(uint64_t), s));
    if (g->n > 0) {
        k_validate<<<num_sms() * 8, 256, 0, s>>>(g->row_ptr, g->col_idx, g->n, g->nnz,
                                                  (unsigned long long *)&ctl->result);
        SYM_LAUNCH_CHECK();
    }
    uint64_t bad = 0;
    SYM_TRY(read_u64(&ctl->result, &bad, s));
    if (bad_out) *bad_out = (int64_t)bad;
    if (bad) {
        char buf[96];
        snprintf(buf, sizeof(buf), "graph violates the CSR precondition at %llu places", (unsigned long long)bad);
        set_error(buf);
        return SYM_EGRAPH;
    }
    return SYM_OK;
}

static int check_decomp(const sym_graph *g, const sym_params *p, const sym_decomp *d) {
    if (d->n != g->n || d->kind != p->kind || d->param != p->param || d->seed != p->seed) {
        set_error("decomposition does not match (n, kind, param, seed)");
        return SYM_EINVAL;
    }
    if (g->n > 0 && (!d->row_ptr_in || !d->row_ptr_x || (g->nnz > 0 && (!d->col_in || !d->col_x)))) {
        set_error("decomposition arrays are NULL");
        return SYM_EINVAL;
    }
    return SYM_OK;
}

// common prologue of the three problem entry points
static int flow_setup(const sym_graph *g, const sym_params *p, const sym_decomp *decomp, void *ws, size_t ws_bytes,
                      const void *out, int problem, sym_stats *stats, cudaStream_t s, Layout &L, FlowArgs &f) {
    SYM_TRY(check_graph(g));
    SYM_TRY(check_params(p));
    if (g->n > 0 && !out) { set_error("output array is NULL"); return SYM_EINVAL; }
    if (decomp && p->kind != SYM_DECOMP_NONE) SYM_TRY(check_decomp(g, p, decomp));
    if (!decomp && p->kind != SYM_DECOMP_NONE && (p->flags & SYM_F_EXT_DECOMP)) {
        set_error("SYM_F_EXT_DECOMP set but decomp is NULL");
        return SYM_EINVAL;
    }
    SYM_TRY(carve_ws(g, p, problem, ws, ws_bytes, L));
    if (stats) memset(stats, 0, sizeof(*stats));
    SYM_CUDA(cudaMemsetAsync(L.ctl, 0, sizeof(Ctl), s));
    if (p->flags & SYM_F_VALIDATE) SYM_TRY(validate_impl(g, L.ctl, nullptr, s));
    f.g = Graph{g->n, g->nnz, g->row_ptr, g->col_idx};
    f.p = *p;
    f.ctl = L.ctl;
    f.stats = stats;
    f.stream = s;
    f.hbits = L.sw.hbits;
    f.first_row = L.sw.first_row;
    f.first_row_cap = L.sw.ntiles + 1;
    if (p->kind != SYM_DECOMP_NONE) {
        if (decomp) {
            f.split.rp_in = decomp->row_ptr_in;
            f.split.ci_in = decomp->col_in;
            f.split.rp_x = decomp->row_ptr_x;
            f.split.ci_x = decomp->col_x;
            f.split.nnz_in = decomp->nnz_in;
            f.split.nnz_x = decomp->nnz_x;
        } else if (g->n > 0) {
            SYM_TRY(run_split(f.g, p->kind, p->param, p->seed, L.sw, L.ctl, L.rp_in, L.ci_in, L.rp_x, L.ci_x,
                              nullptr, s));
            f.split.rp_in = L.rp_in;
            f.split.ci_in = L.ci_in;
            f.split.rp_x = L.rp_x;
            f.split.ci_x = L.ci_x;
        }
    }
    return SYM_OK;
}

}  // namespace sym

using namespace sym;

extern "C" {

const char *sym_version(void) { return SYM_VERSION; }

const char *sym_error_string(int code) {
    switch (code) {
    case SYM_OK: return "success";
    case SYM_EINVAL: return "invalid argument";
    case SYM_EWORKSPACE: return "workspace too small";
    case SYM_EGRAPH: return "graph violates the CSR precondition";
    case SYM_ECUDA: return "CUDA error";
    case SYM_ENCCL: return "NCCL error";
    case SYM_EROUNDS: return "max_rounds reached";
    }
    return "unknown error code";
}

const char *sym_last_error(void) { return g_err.c_str(); }

size_t sym_workspace_bytes(const sym_graph *g, const sym_params *p, int problem) {
    if (check_graph(g) != SYM_OK) return 0;
    if (problem != SYM_PROBLEM_VALIDATE && check_params(p) != SYM_OK) return 0;
    if (problem < SYM_PROBLEM_DECOMPOSE || problem > SYM_PROBLEM_VALIDATE) return 0;
    sym_params dflt = {SYM_DECOMP_NONE, 0, 0, 0, 0};
    Layout L;
    Arena dry;
    carve(dry, g->n, g->nnz, p ? p : &dflt, problem, L);
    return dry.used + 256;
}

int sym_validate(const sym_graph *g, void *ws, size_t ws_bytes, int64_t *bad_out, sym_stream_t stream) {
    cudaStream_t s = (cudaStream_t)stream;
    SYM_TRY(check_graph(g));
    sym_params dflt = {SYM_DECOMP_NONE, 0, 0, 0, 0};
    Layout L;
    SYM_TRY(carve_ws(g, &dflt, SYM_PROBLEM_VALIDATE, ws, ws_bytes, L));
    return validate_impl(g, L.ctl, bad_out, s);
}

int sym_decompose(const sym_graph *g, const sym_params *p, void *ws, size_t ws_bytes, sym_decomp *out,
                  sym_stream_t stream) {
    cudaStream_t s = (cudaStream_t)stream;
    SYM_TRY(check_graph(g));
    SYM_TRY(check_params(p));
    if (!out) { set_error("decomp output is NULL"); return SYM_EINVAL; }
    if (g->n > 0 && (!out->row_ptr_in || !out->row_ptr_x || (g->nnz > 0 && (!out->col_in || !out->col_x)))) {
        set_error("decomposition output arrays are NULL");
        return SYM_EINVAL;
    }
    Layout L;
    SYM_TRY(carve_ws(g, p, SYM_PROBLEM_DECOMPOSE, ws, ws_bytes, L));
    out->n = g->n;
    out->kind = p->kind;
    out->param = p->param;
    out->seed = p->seed;
    out->nnz_in = out->nnz_x = 0;
    if (g->n == 0) return SYM_OK;
    SYM_CUDA(cudaMemsetAsync(L.ctl, 0, sizeof(Ctl), s));
    if (p->flags & SYM_F_VALIDATE) SYM_TRY(validate_impl(g, L.ctl, nullptr, s));
    Graph gg{g->n, g->nnz, g->row_ptr, g->col_idx};
    SYM_TRY(run_split(gg, p->kind, p->param, p->seed, L.sw, L.ctl, out->row_ptr_in, out->col_in, out->row_ptr_x,
                      out->col_x, out->label, s));
    uint64_t nin = 0;
    SYM_TRY(read_u64((const uint64_t *)(out->row_ptr_in + g->n), &nin, s));
    out->nnz_in = (int64_t)nin;
    out->nnz_x = g->nnz - (int64_t)nin;
    return SYM_OK;
}

int sym_mis(const sym_graph *g, const sym_params *p, const sym_decomp *decomp, void *ws, size_t ws_bytes,
            uint8_t *in_set, sym_stats *stats, sym_stream_t stream) {
    cudaStream_t s = (cudaStream_t)stream;
    Layout L;
    FlowArgs f;
    SYM_TRY(flow_setup(g, p, decomp, ws, ws_bytes, in_set, SYM_PROBLEM_MIS, stats, s, L, f));
    if (g->n == 0) return SYM_OK;
    return run_mis(f, L.mis, in_set);
}

int sym_mm(const sym_graph *g, const sym_params *p, const sym_decomp *decomp, void *ws, size_t ws_bytes,
           int32_t *mate, sym_stats *stats, sym_stream_t stream) {
    cudaStream_t s = (cudaStream_t)stream;
    Layout L;
    FlowArgs f;
    SYM_TRY(flow_setup(g, p, decomp, ws, ws_bytes, mate, SYM_PROBLEM_MM, stats, s, L, f));
    if (g->n == 0) return SYM_OK;
    return run_mm(f, L.mm, mate);
}

int sym_color(const sym_graph *g, const sym_params *p, const sym_decomp *decomp, void *ws, size_t ws_bytes,
              uint32_t *color, sym_stats *stats, sym_stream_t stream) {
    cudaStream_t s = (cudaStream_t)stream;
    Layout L;
    FlowArgs f;
    SYM_TRY(flow_setup(g, p, decomp, ws, ws_bytes, color, SYM_PROBLEM_COLOR, stats, s, L, f));
    if (g->n == 0) return SYM_OK;
    return run_color(f, L.col, color);
}

}  // extern "C"
