// prof.cuh -- launch counter and optional per-kernel CUDA-event timing (diagnostics
// behind mp_launch_count / mp_prof_*; bench.py uses them to time the dominant
// kernel live on the stream it runs on).
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <map>
#include <mutex>
#include <string>
#include <vector>

namespace mph {

struct ProfRec {
    const char* name;
    cudaEvent_t a, b;
};

struct Prof {
    std::atomic<uint64_t> launches{0};
    std::atomic<int> enabled{0};
    std::mutex mu;
    std::vector<ProfRec> pending;
    std::vector<cudaEvent_t> pool;
    std::map<std::string, std::pair<double, int64_t>> totals;

    cudaEvent_t ev() {
        if (!pool.empty()) {
            cudaEvent_t e = pool.back();
            pool.pop_back();
            return e;
        }
        cudaEvent_t e;
        cudaEventCreate(&e);
        return e;
    }
    void drain() {  // caller holds mu
        for (auto& r : pending) {
            cudaEventSynchronize(r.b);
            float ms = 0.f;
            cudaEventElapsedTime(&ms, r.a, r.b);
            auto& t = totals[r.name];
            t.first += ms;
            t.second += 1;
            pool.push_back(r.a);
            pool.push_back(r.b);
        }
        pending.clear();
    }
};

inline Prof& prof() {
    static Prof p;
    return p;
}

struct ProfScope {
    const char* name;
    cudaStream_t st;
    cudaEvent_t a = nullptr;
    ProfScope(const char* n, cudaStream_t s) : name(n), st(s) {
        Prof& p = prof();
        p.launches.fetch_add(1, std::memory_order_relaxed);
        if (p.enabled.load(std::memory_order_relaxed)) {
            std::lock_guard<std::mutex> g(p.mu);
            a = p.ev();
            cudaEventRecord(a, st);
        }
    }
    ~ProfScope() {
        if (!a) return;
        Prof& p = prof();
        std::lock_guard<std::mutex> g(p.mu);
        cudaEvent_t b = p.ev();
        cudaEventRecord(b, st);
        p.pending.push_back({name, a, b});
        if (p.pending.size() > 4096) p.drain();
    }
};

}  // namespace mph

// Launch a kernel, counting it and (when enabled) bracketing it with events.
#define MP_LAUNCH(kern, grid, block, smem, st, ...)                  \
    do {                                                             \
        mph::ProfScope mp_prof_scope__(#kern, (st));                 \
        kern<<<(grid), (block), (smem), (st)>>>(__VA_ARGS__);        \
    } while (0)
