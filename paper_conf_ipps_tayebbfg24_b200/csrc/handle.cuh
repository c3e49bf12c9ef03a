// handle.cuh -- the opaque mp_dag handle, error plumbing and scratch arenas.
#pragma once
#include <cstdio>
#include <cstring>
#include <map>
#include <string>

#include "common.cuh"
#include "scan.cuh"
#include "sort.cuh"

struct mp_dag {
    int32_t n = 0;
    int64_t E = 0;
    int32_t L = 0;
    int32_t max_width = 0;
    int32_t P = 0;              // padded positions (levels rounded up to 32)
    int device = 0;
    // canonical arrays (mp_dag_info)
    int32_t* row_ptr = nullptr;
    int32_t* col = nullptr;
    int32_t* indeg = nullptr;
    int32_t* level = nullptr;
    int32_t* level_ptr = nullptr;
    int32_t* level_order = nullptr;
    // q-space: positions in reverse level order (levels L-1 .. 0, ids ascending)
    int32_t* qof = nullptr;     // [n]   id -> q
    int32_t* nodeq = nullptr;   // [n]   q -> id
    int32_t* rowq = nullptr;    // [n+1] successor CSR in q-space
    int32_t* colq = nullptr;    // [E]   successor q
    int32_t* lvlq = nullptr;    // [L+1] q-range of reverse level r
    // padded q-space (each level rounded up to a multiple of 32 positions)
    int32_t* nodep = nullptr;   // [P]   id or -1
    int32_t* rowp = nullptr;    // [P+1]
    int32_t* colp = nullptr;    // [E]   successor padded position
    int32_t* lvlp = nullptr;    // [L+1]
    // device scalars / flags
    uint32_t* err = nullptr;    // error bits (mpk::ERR_*)
    // scratch (grow-only, owned)
    char* ws = nullptr;
    size_t ws_cap = 0;
    unsigned long long* sort_status = nullptr;
    size_t sort_status_cap = 0; // entries
    unsigned long long* scan_status = nullptr;
    size_t scan_status_cap = 0;
    uint32_t* tickets = nullptr; // [64]
    int num_sms = 148;
    // build scratch (grow-only, reused by mp_dag_rebuild)
    int32_t* b_rem = nullptr;
    int32_t* b_f0 = nullptr;
    int32_t* b_f1 = nullptr;
    int32_t* b_counts = nullptr;
    int32_t* b_kout = nullptr;
    int32_t* b_pof = nullptr;
    int32_t* b_bar = nullptr;   // grid barrier: arrivals [0], release flag [32]
    int4* b_colr = nullptr;     // one-block Kahn: per edge {target, its row start, row end, 0}
    int32_t* b_rrow = nullptr;  // k_lvl_flow: predecessor CSR offsets [n+1]
    int32_t* b_rcol = nullptr;  // k_lvl_flow: predecessor ids [E]
    std::map<const void*, size_t> caps;  // capacity (bytes) of every grow-only field
    cudaStream_t side = nullptr;         // replica path: K2's pre-sort pass beside K1
    cudaEvent_t ev_a = nullptr, ev_b = nullptr;
};

namespace mph {

inline thread_local std::string g_last_error;

inline mp_status fail(mp_status s, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    g_last_error = buf;
    return s;
}

#define MP_CUDA(call)                                                                    \
    do {                                                                                 \
        cudaError_t e__ = (call);                                                        \
        if (e__ != cudaSuccess)                                                          \
            return mph::fail(e__ == cudaErrorMemoryAllocation ? MP_ERR_NOMEM : MP_ERR_CUDA, \
                             "%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(e__)); \
    } while (0)

// side stream + two events of a handle (created on first use, on the handle's device)
inline mp_status ensure_side_stream(mp_dag* dag) {
    if (dag->side) return MP_OK;
    if (cudaStreamCreateWithFlags(&dag->side, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&dag->ev_a, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&dag->ev_b, cudaEventDisableTiming) != cudaSuccess)
        return fail(MP_ERR_CUDA, "side stream: %s", cudaGetErrorString(cudaGetLastError()));
    return MP_OK;
}

#define MP_TRY(expr)                   \
    do {                               \
        mp_status s__ = (expr);        \
        if (s__ != MP_OK) return s__;  \
    } while (0)

// Simple bump arena over the handle's grow-only scratch buffer.
struct Arena {
    char* base;
    size_t cap;
    size_t off = 0;
    template <typename T>
    T* take(size_t count) {
        size_t bytes = (count * sizeof(T) + 255) & ~size_t(255);
        T* p = reinterpret_cast<T*>(base + off);
        off += bytes;
        return p;
    }
};

// Grow-only device buffer held in a handle field (synchronises when it grows).
inline mp_status grow_buf(void** field, size_t bytes, mp_dag* dag, cudaStream_t st) {
    if (bytes == 0) bytes = 4;
    size_t& cap = dag->caps[(const void*)field];
    if (*field && cap >= bytes) return MP_OK;
    if (*field) {
        // another stream may still use the old buffer (mp.h: one stream per handle
        // at a time, but a caller may switch streams between calls): drain the device
        MP_CUDA(cudaDeviceSynchronize());
        MP_CUDA(cudaFree(*field));
        *field = nullptr;
    }
    cap = 0;
    MP_CUDA(cudaMalloc(field, bytes));
    cap = bytes;
    return MP_OK;
}

inline size_t align256(size_t b) { return (b + 255) & ~size_t(255); }

// Ensure `dag->ws` holds at least `bytes`; growing synchronises the device (kernels of
// an earlier call on another stream may still use the old scratch).
inline mp_status ensure_ws(mp_dag* dag, size_t bytes, cudaStream_t st) {
    if (bytes <= dag->ws_cap) return MP_OK;
    (void)st;
    MP_CUDA(cudaDeviceSynchronize());
    if (dag->ws) MP_CUDA(cudaFree(dag->ws));
    dag->ws = nullptr;
    dag->ws_cap = 0;
    size_t cap = bytes + bytes / 4;
    MP_CUDA(cudaMalloc(&dag->ws, cap));
    dag->ws_cap = cap;
    return MP_OK;
}

inline mp_status ensure_sort_status(mp_dag* dag, size_t entries, cudaStream_t st) {
    if (entries <= dag->sort_status_cap) return MP_OK;
    (void)st;
    MP_CUDA(cudaDeviceSynchronize());
    if (dag->sort_status) MP_CUDA(cudaFree(dag->sort_status));
    dag->sort_status = nullptr;
    size_t cap = entries + entries / 4 + 256;
    MP_CUDA(cudaMalloc(&dag->sort_status, cap * sizeof(unsigned long long)));
    MP_CUDA(cudaMemset(dag->sort_status, 0, cap * sizeof(unsigned long long)));
    dag->sort_status_cap = cap;
    return MP_OK;
}

inline mp_status ensure_scan_status(mp_dag* dag, size_t entries, cudaStream_t st) {
    if (entries <= dag->scan_status_cap) return MP_OK;
    (void)st;
    MP_CUDA(cudaDeviceSynchronize());
    if (dag->scan_status) MP_CUDA(cudaFree(dag->scan_status));
    dag->scan_status = nullptr;
    size_t cap = entries + entries / 4 + 64;
    MP_CUDA(cudaMalloc(&dag->scan_status, cap * sizeof(unsigned long long)));
    MP_CUDA(cudaMemset(dag->scan_status, 0, cap * sizeof(unsigned long long)));
    dag->scan_status_cap = cap;
    return MP_OK;
}

inline mp_status scan(mp_dag* dag, const int32_t* in, int32_t* out, int64_t n, int32_t* d_total,
                      cudaStream_t st) {
    MP_TRY(ensure_scan_status(dag, (size_t)((n + mpk::SCAN_TILE - 1) / mpk::SCAN_TILE) + 1, st));
    // the last status word is the device epoch counter (zeroed with the array)
    mpk::ScanWs w{dag->scan_status, dag->tickets + 63,
                  reinterpret_cast<uint32_t*>(dag->scan_status + dag->scan_status_cap - 1)};
    MP_CUDA(mpk::scan_excl(in, out, n, d_total, w, st));
    return MP_OK;
}

// Bytes of sort scratch (keys/vals ping-pong, plans, histograms) for nseg x seg_len.
inline size_t sort_bytes(int64_t seg_len, int32_t nseg, int npass, bool vals) {
    size_t n = (size_t)seg_len * (size_t)nseg;
    size_t b = 2 * align256(n * 8) + (vals ? 2 * align256(n * 4) : 0);
    b += align256(mpk::sort_plan_bytes(nseg)) + align256((size_t)nseg * npass * 256 * 4);
    return b;
}

struct SortBufs {
    mpk::SortArgs args;
};

inline mpk::SortArgs carve_sort(Arena& ar, mp_dag* dag, int64_t seg_len, int32_t nseg, int bit_lo, int npass,
                                bool vals) {
    mpk::SortArgs a{};
    size_t n = (size_t)seg_len * (size_t)nseg;
    a.keys[0] = ar.take<uint64_t>(n);
    a.keys[1] = ar.take<uint64_t>(n);
    a.vals[0] = vals ? ar.take<uint32_t>(n) : nullptr;
    a.vals[1] = vals ? ar.take<uint32_t>(n) : nullptr;
    a.seg_len = seg_len;
    a.nseg = nseg;
    a.bit_lo = bit_lo;
    a.npass = npass;
    a.plans = ar.take<mpk::SortPlan>((size_t)nseg);
    a.hist = ar.take<uint32_t>((size_t)nseg * npass * 256);
    a.status = dag->sort_status;
    a.tickets = dag->tickets;
    a.d_len = nullptr;
    return a;
}

inline mp_status run_sort(mp_dag* dag, mpk::SortArgs& a, cudaStream_t st) {
    int64_t tps = (a.seg_len + mpk::SORT_TILE - 1) / mpk::SORT_TILE;
    MP_TRY(ensure_sort_status(dag, (size_t)(tps * a.nseg) * 256, st));
    a.status = dag->sort_status;
    a.depoch = reinterpret_cast<uint32_t*>(dag->sort_status + dag->sort_status_cap - 1);   // zeroed with it
    MP_CUDA(mpk::sort_launch(a, st));
    return MP_OK;
}

inline uint32_t enabled_mask(int32_t A, const int32_t* h_workers) {
    uint32_t m = 0;
    for (int a = 0; a < A; a++)
        if (h_workers[a] > 0) m |= 1u << a;
    return m;
}

}  // namespace mph
