// libmp.cu -- the C-ABI of include/mp.h.  Single translation unit: every
// kernel lives in the headers included below.  Argument marshalling and
// launch sequencing only; every step of the path runs in those kernels.
#include <cstdarg>
#include <vector>

#include <nvtx3/nvToolsExt.h>   // header-only NVTX v3: one range per C-ABI call (no-op without a tool)

#include "push.cuh"
#include "rep2.cuh"
#include "sim.cuh"
#include "variants.cuh"
#include "micro.cuh"

static inline cudaStream_t as_stream(void* s) { return reinterpret_cast<cudaStream_t>(s); }

// NVTX range around every C-ABI entry point, named after it (nsys / ncu --nvtx timelines)
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};
#define MP_NVTX(name) NvtxRange mp_nvtx_range__(name)

extern "C" {

mp_status mp_build_dag(int32_t n_tasks, int64_t n_edges, const int32_t* d_src, const int32_t* d_dst, void* stream,
                       mp_dag** out) {
    MP_NVTX("mp_build_dag");
    return mph::build_dag(n_tasks, n_edges, d_src, d_dst, as_stream(stream), out);
}

mp_status mp_dag_rebuild(mp_dag* dag, int32_t n_tasks, int64_t n_edges, const int32_t* d_src,
                         const int32_t* d_dst, void* stream) {
    MP_NVTX("mp_dag_rebuild");
    if (!dag) return mph::fail(MP_ERR_ARG, "dag is NULL");
    return mph::build_into(dag, n_tasks, n_edges, d_src, d_dst, as_stream(stream));
}

mp_status mp_dag_get_info(const mp_dag* dag, mp_dag_info* out) {
    if (!dag || !out) return mph::fail(MP_ERR_ARG, "NULL argument");
    out->n_tasks = dag->n;
    out->n_edges = dag->E;
    out->n_levels = dag->L;
    out->max_width = dag->max_width;
    out->d_row_ptr = dag->row_ptr;
    out->d_col = dag->col;
    out->d_indeg = dag->indeg;
    out->d_level = dag->level;
    out->d_level_ptr = dag->level_ptr;
    out->d_level_order = dag->level_order;
    return MP_OK;
}

mp_status mp_bottom_level(mp_dag* dag, int32_t n_arch, const float* d_dur, const int32_t* h_workers, float* d_bl,
                          float* d_cp, float* d_nod, void* stream) {
    MP_NVTX("mp_bottom_level");
    return mph::bottom_level(dag, n_arch, d_dur, h_workers, d_bl, d_cp, d_nod, as_stream(stream));
}

mp_status mp_affinity(mp_dag* dag, int32_t n_arch, const float* d_dur, const int32_t* h_workers, float* d_gain,
                      float* d_hd, uint8_t* d_flags, void* stream) {
    MP_NVTX("mp_affinity");
    return mph::affinity(dag, n_arch, d_dur, h_workers, d_gain, d_hd, d_flags, as_stream(stream));
}

mp_status mp_score(mp_dag* dag, int32_t n_arch, mp_crit kind, const float* d_crit, const float* d_gain,
                   const uint8_t* d_flags, float* d_crit_norm, uint64_t* d_key, void* stream) {
    MP_NVTX("mp_score");
    return mph::score(dag, n_arch, (int32_t)kind, d_crit, d_gain, d_flags, d_crit_norm, d_key, as_stream(stream));
}

mp_status mp_build_queues(mp_dag* dag, int32_t n_arch, const uint64_t* d_key, const uint8_t* d_flags,
                          const float* d_dur, const uint8_t* d_done, int64_t* d_qptr, int32_t* d_qtask,
                          mp_queue_summary* d_sum, void* stream) {
    MP_NVTX("mp_build_queues");
    return mph::build_queues(dag, n_arch, d_key, d_flags, d_dur, d_done, d_qptr, d_qtask, d_sum, as_stream(stream));
}

mp_status mp_replicas_run(mp_dag* dag, int32_t n_arch, const float* d_base_dur, const int32_t* h_workers,
                          uint64_t seed, float sigma, int64_t r0, int32_t R, float* d_cp, mp_queue_summary* d_sum,
                          int32_t* d_qtask, void* stream) {
    MP_NVTX("mp_replicas_run");
    return mph::replicas_run(dag, n_arch, d_base_dur, h_workers, seed, sigma, r0, R, d_cp, d_sum, d_qtask,
                             as_stream(stream));
}

mp_status mp_ready_init(mp_dag* dag, int32_t* d_rem, void* stream) {
    MP_NVTX("mp_ready_init");
    return mph::ready_init(dag, d_rem, as_stream(stream));
}

mp_status mp_queues_push(mp_dag* dag, int32_t n_arch, const uint64_t* d_key, const uint8_t* d_flags,
                         const float* d_dur, const int32_t* d_batch, int32_t m, int32_t* d_rem,
                         const int64_t* d_qptr_in, const int32_t* d_qtask_in, int64_t* d_qptr_out,
                         int32_t* d_qtask_out, mp_queue_summary* d_sum, void* stream) {
    MP_NVTX("mp_queues_push");
    return mph::queues_push(dag, n_arch, d_key, d_flags, d_dur, d_batch, m, d_rem, d_qptr_in, d_qtask_in, d_qptr_out,
                            d_qtask_out, d_sum, as_stream(stream));
}

mp_status mp_simulate(mp_dag* dag, int32_t n_arch, const float* d_base_dur, const int32_t* h_workers,
                      uint64_t seed, float sigma, int64_t r0, int32_t R, const int32_t* d_qtask,
                      const mp_queue_summary* d_sum, int32_t max_tries, int32_t eviction, mp_sim_stats* d_stats,
                      double* d_start, int32_t* d_worker, void* stream) {
    MP_NVTX("mp_simulate");
    mp_sim_config cfg{};
    cfg.max_tries = max_tries;
    cfg.eviction = eviction;
    cfg.top_n = 1;
    cfg.eps = 0.0f;
    return mph::simulate(dag, n_arch, d_base_dur, h_workers, seed, sigma, r0, R, d_qtask, d_sum, &cfg, d_stats,
                         d_start, d_worker, as_stream(stream));
}

mp_status mp_simulate_cfg(mp_dag* dag, int32_t n_arch, const float* d_base_dur, const int32_t* h_workers,
                          uint64_t seed, float sigma, int64_t r0, int32_t R, const int32_t* d_qtask,
                          const mp_queue_summary* d_sum, const mp_sim_config* cfg, mp_sim_stats* d_stats,
                          double* d_start, int32_t* d_worker, void* stream) {
    MP_NVTX("mp_simulate_cfg");
    return mph::simulate(dag, n_arch, d_base_dur, h_workers, seed, sigma, r0, R, d_qtask, d_sum, cfg, d_stats,
                         d_start, d_worker, as_stream(stream));
}

mp_status mp_bottom_level_w(mp_dag* dag, int32_t n_arch, const float* d_dur, const int32_t* h_workers, mp_weight kind,
                            float* d_bl, float* d_cp, void* stream) {
    MP_NVTX("mp_bottom_level_w");
    return mph::bottom_level(dag, n_arch, d_dur, h_workers, d_bl, d_cp, nullptr, as_stream(stream), (int32_t)kind);
}

mp_status mp_affinity_prefix(mp_dag* dag, int32_t n_arch, const float* d_dur, const int32_t* h_workers,
                             const int32_t* d_order, float* d_gain, float* d_hd, uint8_t* d_flags, void* stream) {
    MP_NVTX("mp_affinity_prefix");
    return mph::affinity_prefix(dag, n_arch, d_dur, h_workers, d_order, d_gain, d_hd, d_flags, as_stream(stream));
}

mp_status mp_nod_remaining(mp_dag* dag, int32_t n_arch, const float* d_dur, const int32_t* h_workers,
                           const uint8_t* d_done, float* d_nod, void* stream) {
    MP_NVTX("mp_nod_remaining");
    return mph::nod_remaining(dag, n_arch, d_dur, h_workers, d_done, d_nod, as_stream(stream));
}

mp_status mp_queues_push_all(mp_dag* dag, int32_t n_arch, const int64_t* d_qptr_all, const int32_t* d_qtask_all,
                             const uint8_t* d_flags, const float* d_dur, const int32_t* d_batch, int32_t m,
                             int32_t* d_rem, uint8_t* d_done, int64_t* d_qptr_out, int32_t* d_qtask_out,
                             mp_queue_summary* d_sum, void* stream) {
    MP_NVTX("mp_queues_push_all");
    return mph::queues_push_all(dag, n_arch, d_qptr_all, d_qtask_all, d_flags, d_dur, d_batch, m, d_rem, d_done,
                                d_qptr_out, d_qtask_out, d_sum, as_stream(stream));
}

mp_status mp_check(mp_dag* dag, void* stream) {
    MP_NVTX("mp_check");
    if (!dag) return mph::fail(MP_ERR_ARG, "dag is NULL");
    cudaStream_t st = as_stream(stream);
    MP_CUDA(cudaStreamSynchronize(st));
    MP_CUDA(cudaGetLastError());
    uint32_t e = 0;
    MP_CUDA(cudaMemcpy(&e, dag->err, 4, cudaMemcpyDeviceToHost));
    if (e) MP_CUDA(cudaMemset(dag->err, 0, 4));
    if (e & mpk::ERR_DOMAIN_BIT)
        return mph::fail(MP_ERR_DOMAIN, "duration outside {+inf, 0} U [2^-41, 2^20), NaN, or no enabled arch");
    if (e & mpk::ERR_ARG_BIT) return mph::fail(MP_ERR_ARG, "device-detected argument error");
    if (e & mpk::ERR_SIM_BIT)
        return mph::fail(MP_ERR_ARG, "mp_simulate: queues do not match the DAG (ALL-mode queues required)");
    return MP_OK;
}

void mp_free(mp_dag* dag) {
    MP_NVTX("mp_free");
    if (!dag) return;
    cudaDeviceSynchronize();
    void* ptrs[] = {dag->row_ptr, dag->col,  dag->indeg, dag->level, dag->level_ptr, dag->level_order,
                    dag->qof,     dag->nodeq, dag->rowq, dag->colq,  dag->lvlq,      dag->nodep,
                    dag->rowp,    dag->colp, dag->lvlp,  dag->err,   dag->ws,        dag->sort_status,
                    dag->scan_status, dag->tickets, dag->b_rem, dag->b_f0, dag->b_f1, dag->b_counts,
                    dag->b_kout, dag->b_pof, dag->b_bar, dag->b_colr, dag->b_rrow, dag->b_rcol};
    for (void* p : ptrs)
        if (p) cudaFree(p);
    if (dag->ev_a) cudaEventDestroy(dag->ev_a);
    if (dag->ev_b) cudaEventDestroy(dag->ev_b);
    if (dag->side) cudaStreamDestroy(dag->side);
    delete dag;
}

const char* mp_status_str(mp_status s) {
    switch (s) {
        case MP_OK: return "MP_OK";
        case MP_ERR_ARG: return "MP_ERR_ARG";
        case MP_ERR_CYCLE: return "MP_ERR_CYCLE";
        case MP_ERR_DOMAIN: return "MP_ERR_DOMAIN";
        case MP_ERR_CUDA: return "MP_ERR_CUDA";
        case MP_ERR_NOMEM: return "MP_ERR_NOMEM";
    }
    return "MP_ERR_UNKNOWN";
}

const char* mp_last_error(void) { return mph::g_last_error.c_str(); }

const char* mp_build_info(void) { return "libmp 0.1 sm_100a (B200) cuda " MP_CUDA_VERSION_STR; }

mp_status mp_microbench(int32_t kind, int32_t L, int32_t arg, const uint32_t* d_next, uint32_t* d_sink,
                        void* stream) {
    using namespace mpk;
    cudaStream_t st = as_stream(stream);
    if (L < 0 || !d_sink) return mph::fail(MP_ERR_ARG, "bad microbenchmark arguments");
    switch (kind) {
        case MP_MB_SYNC: MP_LAUNCH(k_mb_sync, 1, 1024, 0, st, L, d_sink); break;
        case MP_MB_CLUSTER: {
            if (arg < 2 || arg > 8) return mph::fail(MP_ERR_ARG, "cluster size %d outside [2, 8]", arg);
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3((unsigned)arg);
            cfg.blockDim = dim3(1024);
            cfg.stream = st;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = (unsigned)arg;
            at[0].val.clusterDim.y = 1;
            at[0].val.clusterDim.z = 1;
            cfg.attrs = at;
            cfg.numAttrs = 1;
            mph::ProfScope ps("k_mb_cluster", st);
            MP_CUDA(cudaLaunchKernelEx(&cfg, k_mb_cluster, L, d_sink));
            break;
        }
        case MP_MB_GRID: {
            int dev = 0, sms = 0;
            MP_CUDA(cudaGetDevice(&dev));
            MP_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
            void* args[] = {&L, &d_sink};
            mph::ProfScope ps("k_mb_grid", st);
            MP_CUDA(cudaLaunchCooperativeKernel((const void*)k_mb_grid, dim3((unsigned)sms), dim3(1024), args, 0, st));
            break;
        }
        case MP_MB_CHAIN:
            if (!d_next) return mph::fail(MP_ERR_ARG, "pointer chain is NULL");
            MP_LAUNCH(k_mb_chain, 1, 1, 0, st, L, d_next, d_sink);
            break;
        default: return mph::fail(MP_ERR_ARG, "unknown microbenchmark %d", kind);
    }
    MP_CUDA(cudaGetLastError());
    return MP_OK;
}

uint64_t mp_launch_count(void) { return mph::prof().launches.load(); }

void mp_prof_enable(int on) { mph::prof().enabled.store(on ? 1 : 0); }

void mp_prof_reset(void) {
    auto& p = mph::prof();
    std::lock_guard<std::mutex> g(p.mu);
    p.drain();
    p.totals.clear();
}

mp_status mp_prof_query(const char* name, double* total_ms, int64_t* launches) {
    if (!name || !total_ms || !launches) return mph::fail(MP_ERR_ARG, "NULL argument");
    auto& p = mph::prof();
    std::lock_guard<std::mutex> g(p.mu);
    p.drain();
    auto it = p.totals.find(name);
    *total_ms = it == p.totals.end() ? 0.0 : it->second.first;
    *launches = it == p.totals.end() ? 0 : it->second.second;
    return MP_OK;
}

int64_t mp_prof_names(char* buf, int64_t len) {
    auto& p = mph::prof();
    std::lock_guard<std::mutex> g(p.mu);
    p.drain();
    std::string all;
    for (auto& kv : p.totals) {
        if (!all.empty()) all += ",";
        all += kv.first;
    }
    if (buf && len > 0) {
        int64_t m = std::min<int64_t>(len - 1, (int64_t)all.size());
        memcpy(buf, all.data(), (size_t)m);
        buf[m] = 0;
    }
    return (int64_t)all.size();
}

#ifdef MP_PHASES
// debug build only (tools/k2_phases.py): accumulated K2 phase cycles (thread 0 of every CTA)
int mp_debug_k2_phases(unsigned long long* h_out32, int reset) {
    MP_NVTX("mp_debug_k2_phases");
    if (cudaMemcpyFromSymbol(h_out32, mpk::g_k2_phase, 32 * sizeof(unsigned long long)) != cudaSuccess) return 1;
    if (reset) {
        static const unsigned long long z[32] = {};
        if (cudaMemcpyToSymbol(mpk::g_k2_phase, z, sizeof(z)) != cudaSuccess) return 1;
    }
    return 0;
}
#endif
}  // extern "C"
