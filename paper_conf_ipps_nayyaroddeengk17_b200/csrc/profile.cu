// profile.cu -- optional per-kernel-class device timing (sym_profile_enable/collect).
// CUDA event pairs are recorded on the launching stream around each hot launch;
// collection synchronises them after the caller's timed region.
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "internal.h"

namespace sym {

namespace {
struct Rec {
    std::string cls;
    cudaEvent_t a, b;
    double alg, impl;
    int slot;  // device byte counter pair slot, or -1
};
std::atomic<bool> g_on{false};
std::atomic<bool> g_bytes{false};  // mode 1: device byte counters too; mode 2: events only
// device byte counters for launches whose algorithmic bytes depend on the frontier
// (measurement mode only; the one allocation the library makes, lazily, when
// profiling is enabled)
constexpr int DEV_SLOTS = 1 << 16;
unsigned long long *g_dev = nullptr;
int g_dev_next = 0;
std::vector<Rec> g_recs;
std::vector<cudaEvent_t> g_pool;
// pending begins, a LIFO per stream (calls on different streams / host threads nest
// independently); every global here is guarded by g_mu
std::map<cudaStream_t, std::vector<std::pair<std::string, cudaEvent_t>>> g_open;
std::mutex g_mu;

cudaEvent_t get_event() {
    if (!g_pool.empty()) {
        cudaEvent_t e = g_pool.back();
        g_pool.pop_back();
        return e;
    }
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    return e;
}
}  // namespace

bool prof_on() { return g_on; }

void prof_begin(const char *cls, cudaStream_t s) {
    if (!g_on) return;
    std::lock_guard<std::mutex> lk(g_mu);
    cudaEvent_t e = get_event();
    cudaEventRecord(e, s);
    g_open[s].emplace_back(cls, e);
}

// closes the innermost pending begin of stream s
static void close_rec(cudaStream_t s, double alg, double impl, int slot) {
    auto it = g_open.find(s);
    if (it == g_open.end() || it->second.empty()) return;
    cudaEvent_t e = get_event();
    cudaEventRecord(e, s);
    Rec r{it->second.back().first, it->second.back().second, e, alg, impl, slot};
    it->second.pop_back();
    g_recs.push_back(r);
}

void prof_end(cudaStream_t s, double alg, double impl) {
    if (!g_on) return;
    std::lock_guard<std::mutex> lk(g_mu);
    close_rec(s, alg, impl, -1);
}

unsigned long long *prof_counter(cudaStream_t s) {
    if (!g_on || !g_bytes) return nullptr;
    std::lock_guard<std::mutex> lk(g_mu);
    if (!g_dev && cudaMalloc(&g_dev, 2 * sizeof(unsigned long long) * DEV_SLOTS) != cudaSuccess) {
        g_dev = nullptr;
        return nullptr;
    }
    if (g_dev_next >= DEV_SLOTS) return nullptr;
    unsigned long long *p = g_dev + 2 * g_dev_next++;
    cudaMemsetAsync(p, 0, 2 * sizeof(unsigned long long), s);
    return p;
}

void prof_end_dev(cudaStream_t s, unsigned long long *ctr) {
    if (!g_on) return;
    std::lock_guard<std::mutex> lk(g_mu);
    close_rec(s, ctr ? 0.0 : -1.0, ctr ? 0.0 : -1.0, ctr ? (int)((ctr - g_dev) / 2) : -1);
}

}  // namespace sym

using namespace sym;

extern "C" int sym_profile_enable(int on) {
    std::lock_guard<std::mutex> lk(g_mu);
    g_on = on != 0;
    g_bytes = on == 1;
    return SYM_OK;
}

extern "C" int sym_profile_collect(sym_kernel_profile *out, int max_entries, int *count) {
    struct Acc {
        int64_t n = 0;
        double ms = 0, alg = 0, impl = 0;
        bool alg_known = true, impl_known = true;
    };
    std::lock_guard<std::mutex> lk(g_mu);
    std::map<std::string, Acc> acc;
    std::vector<std::string> order;
    std::vector<unsigned long long> dev(2 * (size_t)g_dev_next);
    if (!g_recs.empty()) {
        cudaError_t e = cudaEventSynchronize(g_recs.back().b);
        if (e != cudaSuccess) return cuda_fail(e, "cudaEventSynchronize", __FILE__, __LINE__);
    }
    if (g_dev_next > 0) {
        cudaError_t e = cudaMemcpy(dev.data(), g_dev, 2 * sizeof(unsigned long long) * g_dev_next, cudaMemcpyDeviceToHost);
        if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpy(profile counters)", __FILE__, __LINE__);
    }
    for (auto &r : g_recs) {
        cudaError_t e = cudaEventSynchronize(r.b);
        if (e != cudaSuccess) return cuda_fail(e, "cudaEventSynchronize", __FILE__, __LINE__);
        float ms = 0;
        cudaEventElapsedTime(&ms, r.a, r.b);
        if (!acc.count(r.cls)) order.push_back(r.cls);
        Acc &x = acc[r.cls];
        x.n++;
        x.ms += ms;
        const double alg = r.slot >= 0 ? (double)dev[2 * r.slot] : r.alg;
        const double impl = r.slot >= 0 ? (double)dev[2 * r.slot + 1] : r.impl;
        if (alg < 0) x.alg_known = false;
        else x.alg += alg;
        if (impl < 0) x.impl_known = false;
        else x.impl += impl;
        g_pool.push_back(r.a);
        g_pool.push_back(r.b);
    }
    g_recs.clear();
    g_dev_next = 0;
    int c = 0;
    for (auto &name : order) {
        if (out && c < max_entries) {
            Acc &x = acc[name];
            memset(&out[c], 0, sizeof(out[c]));
            strncpy(out[c].name, name.c_str(), sizeof(out[c].name) - 1);
            out[c].launches = x.n;
            out[c].ms = x.ms;
            out[c].alg_bytes = x.alg_known ? x.alg : -1.0;
            out[c].impl_bytes = x.impl_known ? x.impl : -1.0;
        }
        c++;
    }
    if (count) *count = c;
    return SYM_OK;
}
