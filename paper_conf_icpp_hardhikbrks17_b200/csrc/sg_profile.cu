// sg_profile.cu — launch accounting and optional per-launch timing with CUDA events recorded on
// the launching stream (used by bench.py for the roofline's measured kernel duration).
#include "sg_internal.cuh"
#include <atomic>
#include <mutex>
#include <vector>
#include <cstring>

namespace {
struct Rec {
    const char* name;
    cudaEvent_t a, b;
};
std::atomic<long long> g_launches{0};
std::atomic<int> g_enabled{0};
std::mutex g_mu;
std::vector<Rec> g_recs;
std::vector<cudaEvent_t> g_free;

cudaEvent_t get_event() {
    if (!g_free.empty()) { cudaEvent_t e = g_free.back(); g_free.pop_back(); return e; }
    cudaEvent_t e;
    if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
    return e;
}
}  // namespace

namespace sg {
Prof::Prof(const char* name, cudaStream_t st) : s(st), idx(-1) {
    g_launches.fetch_add(1, std::memory_order_relaxed);
    if (!g_enabled.load(std::memory_order_relaxed)) return;
    std::lock_guard<std::mutex> lk(g_mu);
    Rec r{name, get_event(), get_event()};
    if (!r.a || !r.b) return;
    cudaEventRecord(r.a, s);
    idx = (long long)g_recs.size();
    g_recs.push_back(r);
}
Prof::~Prof() {
    if (idx < 0) return;
    std::lock_guard<std::mutex> lk(g_mu);
    cudaEventRecord(g_recs[(size_t)idx].b, s);
}
}  // namespace sg

extern "C" {
void sg_profile_enable(int on) { g_enabled.store(on ? 1 : 0); }

int64_t sg_launch_count(void) { return g_launches.load(); }

int64_t sg_profile_count(void) {
    std::lock_guard<std::mutex> lk(g_mu);
    return (int64_t)g_recs.size();
}

int64_t sg_profile_read(char* names, double* ms, int64_t max) {
    std::lock_guard<std::mutex> lk(g_mu);
    int64_t n = (int64_t)g_recs.size();
    if (n > max) n = max;
    for (int64_t i = 0; i < n; ++i) {
        float t = -1.f;
        cudaEventSynchronize(g_recs[(size_t)i].b);
        if (cudaEventElapsedTime(&t, g_recs[(size_t)i].a, g_recs[(size_t)i].b) != cudaSuccess) { cudaGetLastError(); t = -1.f; }
        if (ms) ms[i] = t;
        if (names) { strncpy(names + 32 * i, g_recs[(size_t)i].name, 31); names[32 * i + 31] = 0; }
    }
    return n;
}

void sg_profile_reset(void) {
    std::lock_guard<std::mutex> lk(g_mu);
    for (auto& r : g_recs) { g_free.push_back(r.a); g_free.push_back(r.b); }
    g_recs.clear();
}
}
