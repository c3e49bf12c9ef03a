// push.cuh -- SURVEY §8(f) N1: incremental READY-mode PUSH of a completion batch.
//
// State kept by the caller: rem[t] = predecessors of t not completed yet
// (mp_ready_init sets it to |lambda^-(t)|) and the current per-arch queues.
// A push (a) drops the batch's tasks from the queues (they were popped, Alg. 2),
// (b) decrements rem of their successors -- a task whose counter reaches 0 is
// newly ready (P:l.91) and joins every queue whose arch can run it (P:l.104,
// Alg. 1), (c) merges the newly ready run, sorted by (key, id), into each
// queue with merge-path partitions, and (d) recomputes the queue summaries.
// mp_queues_push_all is the static-order variant: it keeps the ALL-mode queues
// and a done mask instead of the current queues and needs no sort or merge.
#pragma once
#include "path.cuh"

namespace mpk {

__global__ void k_ready_init(int32_t n, const int32_t* indeg, int32_t* rem) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x)
        rem[t] = indeg[t];
}

// Validation before any state changes (both push variants): every batch id in
// [0, n), ready and not completed (rem[u] == 0; a completed task carries
// rem = -1), not done (static-order variant), and listed once (a bit per task,
// claimed with atomicOr).  Any violation sets *bad and the error flag; the
// release kernels then leave rem / done / the queues untouched.
__global__ void k_push_validate(const int32_t* batch, int32_t m, int32_t n, const int32_t* rem, const uint8_t* done,
                                uint32_t* mark, uint32_t* bad, uint32_t* err) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t u = batch[i];
        bool ok = u >= 0 && u < n;
        if (ok) ok = rem[u] == 0 && !(done && done[u]);
        if (ok) {
            const uint32_t bit = 1u << (u & 31);
            ok = (atomicOr(&mark[u >> 5], bit) & bit) == 0;     // a second copy of u in the batch
        }
        if (!ok) {
            atomicOr(bad, 1u);
            atomicOr(err, ERR_ARG_BIT);
        }
    }
}

// mark the batch (removed from the queues, rem = -1: completed) and release successors
__global__ void k_push_release(const int32_t* batch, int32_t m, const int32_t* row_ptr, const int32_t* col,
                               int32_t* rem, uint8_t* removed, int32_t* fresh, int32_t* nfresh, const uint32_t* bad) {
    if (*bad) return;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t u = batch[i];
        removed[u] = 1;
        rem[u] = -1;
        for (int32_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) {
            const int32_t s = col[e];
            if (atomicSub(&rem[s], 1) == 1) fresh[atomicAdd(nfresh, 1)] = s;
        }
    }
}

// newly ready ids as sort keys (the run must be in id order before the stable key sort)
__global__ void k_push_ids(const int32_t* fresh, const int32_t* nfresh, uint64_t* ik, int64_t* len) {
    const int32_t nf = *nfresh;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nf; i += (int64_t)gridDim.x * blockDim.x)
        ik[i] = (uint64_t)(uint32_t)fresh[i];
    if (blockIdx.x == 0 && threadIdx.x == 0) *len = nf;
}

// new entries of every arch: key' = (arch << 60 | gainc << 30 | critc), value = task (segmented sort input)
__global__ void k_push_new(const SortPlan* iplan, uint64_t* const* ikb, const int32_t* nfresh, int32_t A,
                           const uint64_t* key,
                           const uint8_t* flags, uint64_t* skey, uint32_t* sval, int32_t* cnt_new, int64_t* total) {
    const int32_t nf = *nfresh;
    const uint64_t* ids = ikb[iplan->final_sel];
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (int64_t)nf * A;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t a = (int32_t)(i % A);
        const int32_t t = (int32_t)ids[i / A];
        uint64_t k = ~0ull;   // not enabled on a: sorts after every real entry
        if (flags[(int64_t)t * A + a] & 1) {
            const uint64_t kk = key[(int64_t)t * A + a];
            k = ((uint64_t)a << 60) | ((kk >> 32) << 30) | (kk & 0xffffffffull);
            atomicAdd(&cnt_new[a], 1);
        }
        skey[i] = k;
        sval[i] = (uint32_t)t;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) *total = (int64_t)nf * A;
}

// keep[i] = queue_in entry i survives (not in the batch); per-arch survivor counts
__global__ void k_push_keep(const int64_t* qptr_in, int32_t A, const int32_t* qin, const uint8_t* removed,
                            int32_t* keep, int32_t* cnt_keep, int64_t cap) {
    const int64_t Q = qptr_in[A];
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cap; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t k = (i < Q && !removed[qin[i]]) ? 1 : 0;
        keep[i] = k;
        if (k) {
            int a = 0;
            while (a + 1 < A && qptr_in[a + 1] <= i) a++;
            atomicAdd(&cnt_keep[a], 1);
        }
    }
}

__global__ void k_push_compact(const int64_t* qptr_in, int32_t A, const int32_t* qin, const int32_t* keep,
                               const int32_t* pos, int32_t* kept) {
    const int64_t Q = qptr_in[A];
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < Q; i += (int64_t)gridDim.x * blockDim.x)
        if (keep[i]) kept[pos[i]] = qin[i];
}

// segment offsets: kept queue a = kept[koff[a] .. koff[a+1]), new run a = sortedvals[noff[a] ..), output qptr
__global__ void k_push_offsets(int32_t A, const int32_t* cnt_keep, const int32_t* cnt_new, int64_t* koff,
                               int64_t* noff, int64_t* qptr_out) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    int64_t k = 0, m = 0;
    for (int a = 0; a < A; a++) {
        koff[a] = k;
        noff[a] = m;
        qptr_out[a] = k + m;
        k += cnt_keep[a];
        m += cnt_new[a];
    }
    koff[A] = k;
    noff[A] = m;
    qptr_out[A] = k + m;
}

MP_INLINE bool push_less(const uint64_t* key, int32_t A, int32_t a, int32_t x, int32_t y) {
    const uint64_t kx = key[(int64_t)x * A + a], ky = key[(int64_t)y * A + a];
    return kx < ky || (kx == ky && x < y);
}

// merge-path: every thread emits PUSH_IPT consecutive outputs of the concatenated per-arch merges
constexpr int PUSH_IPT = 8;
__global__ void k_push_merge(int32_t A, const uint64_t* key, const int32_t* kept, const int64_t* koff,
                             const SortPlan* plan, uint32_t* const* vb, const int64_t* noff, const int64_t* qptr_out,
                             int32_t* qout) {
    const int64_t Q = qptr_out[A];
    const uint32_t* nv = vb[plan->final_sel];
    for (int64_t i0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) * PUSH_IPT; i0 < Q;
         i0 += (int64_t)gridDim.x * blockDim.x * PUSH_IPT) {
        int a = 0;
        while (a + 1 < A && qptr_out[a + 1] <= i0) a++;
        const int32_t* X = kept + koff[a];
        const int64_t nx = koff[a + 1] - koff[a];
        const uint32_t* Y = nv + noff[a];
        const int64_t ny = noff[a + 1] - noff[a];
        int64_t d = i0 - qptr_out[a];
        // diagonal search: x + y = d, X[x-1] < Y[y] and Y[y-1] < X[x]
        int64_t lo = d > ny ? d - ny : 0, hi = d < nx ? d : nx;
        while (lo < hi) {
            const int64_t x = (lo + hi) >> 1;
            const int64_t y = d - x;
            if (push_less(key, A, a, X[x], (int32_t)Y[y - 1])) lo = x + 1;
            else hi = x;
        }
        int64_t x = lo, y = d - lo;
        for (int k = 0; k < PUSH_IPT; k++) {
            const int64_t o = i0 + k;
            if (o >= Q) break;
            while (a + 1 < A && o == qptr_out[a + 1]) {   // next (possibly empty) arch segment starts here
                a++;
                X = kept + koff[a];
                Y = nv + noff[a];
                x = 0;
                y = 0;
            }
            const int64_t nxa = koff[a + 1] - koff[a], nya = noff[a + 1] - noff[a];
            bool takex;
            if (x >= nxa) takex = false;
            else if (y >= nya) takex = true;
            else takex = push_less(key, A, a, X[x], (int32_t)Y[y]);
            qout[o] = takex ? X[x++] : (int32_t)Y[y++];
        }
    }
}

// summaries over the merged queues (exact best_remaining_work)
__global__ void k_push_summary(int32_t A, const int64_t* qptr, const int32_t* q, const uint8_t* flags,
                               const float* dur, unsigned long long* brw) {
    const int a = blockIdx.y;
    const int64_t b = qptr[a], e = qptr[a + 1];
    uint64_t lo = 0, hi = 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t rounds = (e - b + stride - 1) / stride;
    for (int64_t it = 0; it < rounds; it++) {
        const int64_t i = b + it * stride + blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
        if (i < e) {
            const int32_t t = q[i];
            if (flags[(int64_t)t * A + a] & 2) {
                bool dummy = false;
                uint64_t l, h;
                fixed64(canon_dur(dur[(int64_t)t * A + a], dummy), l, h);
                add128(lo, hi, l, h);
            }
        }
    }
    warp_sum128(lo, hi);
    if ((threadIdx.x & 31) == 0) atomic_add128(brw + 2 * a, lo, hi);
}

__global__ void k_push_finish(int32_t A, const int64_t* qptr, const int32_t* q, const unsigned long long* brw,
                              mp_queue_summary* sum) {
    if (threadIdx.x >= A) return;
    const int a = threadIdx.x;
    mp_queue_summary s;
    s.count = (int32_t)(qptr[a + 1] - qptr[a]);
    s.head = s.count > 0 ? q[qptr[a]] : -1;
    s.brw_lo = brw[2 * a];
    s.brw_hi = (int64_t)brw[2 * a + 1];
    s.brw = u128_to_double_scaled(brw[2 * a], brw[2 * a + 1]);
    sum[a] = s;
}

// ---- static-order push (mp_queues_push_all) ------------------------------------------
// Scores are whole-DAG (reading c18), so every READY-mode queue is the ALL-mode
// queue restricted to the ready tasks, in the same order: a push is a release
// followed by one stream compaction of the ALL-mode queues.

// completed tasks (validated by k_push_validate): done[t] = 1, rem[t] = -1,
// successors' counters decremented
__global__ void k_pushall_release(const int32_t* batch, int32_t m, const int32_t* row_ptr, const int32_t* col,
                                  int32_t* rem, uint8_t* done, const uint32_t* bad) {
    if (*bad) return;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t u = batch[i];
        done[u] = 1;
        rem[u] = -1;
        for (int32_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) atomicSub(&rem[col[e]], 1);
    }
}

// keep[i] = 1 iff the task at ALL-mode position i is ready (not done, no pending predecessor)
__global__ void k_pushall_flag(int64_t cap, int32_t A, const int64_t* qptr_all, const int32_t* qall,
                               const int32_t* rem, const uint8_t* done, int32_t* keep) {
    const int64_t Q = qptr_all[A];
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cap; i += (int64_t)gridDim.x * blockDim.x) {
        int32_t k = 0;
        if (i < Q) {
            const int32_t t = qall[i];
            k = (!done[t] && rem[t] == 0) ? 1 : 0;
        }
        keep[i] = k;
    }
}

// scatter the kept entries (global exclusive scan = output position, arch segments
// stay contiguous) and sum best_remaining_work per arch
__global__ void k_pushall_scatter(int32_t A, const int64_t* qptr_all, const int32_t* qall, const int32_t* keep,
                                  const int32_t* pos, const uint8_t* flags, const float* dur, int32_t* qout,
                                  unsigned long long* brw) {
    const int a = blockIdx.y;
    const int64_t b = qptr_all[a], e = qptr_all[a + 1];
    uint64_t lo = 0, hi = 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t rounds = (e - b + stride - 1) / stride;
    for (int64_t it = 0; it < rounds; it++) {
        const int64_t i = b + it * stride + blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
        if (i < e && keep[i]) {
            const int32_t t = qall[i];
            qout[pos[i]] = t;
            if (flags[(int64_t)t * A + a] & 2) {
                bool dummy = false;
                uint64_t l, h;
                fixed64(canon_dur(dur[(int64_t)t * A + a], dummy), l, h);
                add128(lo, hi, l, h);
            }
        }
    }
    warp_sum128(lo, hi);
    if ((threadIdx.x & 31) == 0) atomic_add128(brw + 2 * a, lo, hi);
}

// qptr_out[a] = kept entries before arch a's segment; summaries
__global__ void k_pushall_finish(int32_t A, int64_t cap, const int64_t* qptr_all, const int32_t* pos,
                                 const int32_t* total, const int32_t* qout, const unsigned long long* brw,
                                 int64_t* qptr_out, mp_queue_summary* sum) {
    if (threadIdx.x > A) return;
    const int a = threadIdx.x;
    const int64_t s = qptr_all[a];
    const int64_t o = s < cap ? (int64_t)pos[s] : (int64_t)*total;
    qptr_out[a] = o;
    if (a == A) return;
    const int64_t s1 = qptr_all[a + 1];
    const int64_t o1 = s1 < cap ? (int64_t)pos[s1] : (int64_t)*total;
    mp_queue_summary r;
    r.count = (int32_t)(o1 - o);
    r.head = r.count > 0 ? qout[o] : -1;
    r.brw_lo = brw[2 * a];
    r.brw_hi = (int64_t)brw[2 * a + 1];
    r.brw = u128_to_double_scaled(brw[2 * a], brw[2 * a + 1]);
    sum[a] = r;
}

}  // namespace mpk

namespace mph {

inline mp_status queues_push_all(mp_dag* dag, int32_t A, const int64_t* qptr_all, const int32_t* qall,
                                 const uint8_t* flags, const float* dur, const int32_t* batch, int32_t m,
                                 int32_t* rem, uint8_t* done, int64_t* qptr_out, int32_t* qout,
                                 mp_queue_summary* sum, cudaStream_t st) {
    using namespace mpk;
    if (!dag) return fail(MP_ERR_ARG, "dag is NULL");
    if (A < 1 || A > MAX_ARCH) return fail(MP_ERR_ARG, "n_arch %d outside [1, 8]", A);
    if (m < 0 || (m > 0 && !batch)) return fail(MP_ERR_ARG, "bad batch");
    if (!qptr_all || !qptr_out || !sum || (dag->n > 0 && (!qall || !flags || !dur || !rem || !done || !qout)))
        return fail(MP_ERR_ARG, "NULL buffer");
    if (qall == qout) return fail(MP_ERR_ARG, "qtask_all and qtask_out must not alias");
    const int32_t n = dag->n;
    const int64_t cap = (int64_t)n * A > 0 ? (int64_t)n * A : 1;
    const size_t words = ((size_t)n + 31) / 32 + 1;
    MP_TRY(ensure_ws(dag, 2 * align256((size_t)cap * 4) + align256(64) + align256(16 * MAX_ARCH) +
                              align256(words * 4) + align256(4), st));
    Arena ar{dag->ws, dag->ws_cap};
    int32_t* keep = ar.take<int32_t>((size_t)cap);
    int32_t* pos = ar.take<int32_t>((size_t)cap);
    int32_t* total = ar.take<int32_t>(16);
    unsigned long long* brw = ar.take<unsigned long long>(2 * MAX_ARCH);
    uint32_t* mark = ar.take<uint32_t>(words);
    uint32_t* bad = ar.take<uint32_t>(1);
    MP_CUDA(cudaMemsetAsync(brw, 0, 16 * MAX_ARCH, st));
    MP_CUDA(cudaMemsetAsync(total, 0, 4, st));
    if (m > 0) {
        MP_CUDA(cudaMemsetAsync(mark, 0, words * 4, st));
        MP_CUDA(cudaMemsetAsync(bad, 0, 4, st));
        MP_LAUNCH(k_push_validate, grid_for(m), 256, 0, st, batch, m, n, rem, done, mark, bad, dag->err);
        MP_LAUNCH(k_pushall_release, grid_for(m), 256, 0, st, batch, m, dag->row_ptr, dag->col, rem, done, bad);
    }
    // the ALL-mode queues hold at most n*A entries; their true length is qptr_all[A] (device)
    MP_LAUNCH(k_pushall_flag, grid_for(cap), 256, 0, st, cap, A, qptr_all, qall, rem, done, keep);
    MP_TRY(scan(dag, keep, pos, cap, total, st));
    dim3 g(grid_for(cap, 256, 148 * 4), A);
    MP_LAUNCH(k_pushall_scatter, g, 256, 0, st, A, qptr_all, qall, keep, pos, flags, dur, qout, brw);
    MP_LAUNCH(k_pushall_finish, 1, 32, 0, st, A, cap, qptr_all, pos, total, qout, brw, qptr_out, sum);
    MP_CUDA(cudaGetLastError());
    return MP_OK;
}

inline mp_status ready_init(mp_dag* dag, int32_t* rem, cudaStream_t st) {
    using namespace mpk;
    if (!dag || (dag->n > 0 && !rem)) return fail(MP_ERR_ARG, "NULL argument");
    if (dag->n > 0) MP_LAUNCH(k_ready_init, grid_for(dag->n), 256, 0, st, dag->n, dag->indeg, rem);
    MP_CUDA(cudaGetLastError());
    return MP_OK;
}

inline mp_status queues_push(mp_dag* dag, int32_t A, const uint64_t* key, const uint8_t* flags, const float* dur,
                             const int32_t* batch, int32_t m, int32_t* rem, const int64_t* qptr_in,
                             const int32_t* qin, int64_t* qptr_out, int32_t* qout, mp_queue_summary* sum,
                             cudaStream_t st) {
    using namespace mpk;
    if (!dag) return fail(MP_ERR_ARG, "dag is NULL");
    if (A < 1 || A > MAX_ARCH) return fail(MP_ERR_ARG, "n_arch %d outside [1, 8]", A);
    if (m < 0 || (m > 0 && !batch)) return fail(MP_ERR_ARG, "bad batch");
    if (!qptr_in || !qptr_out || !sum || (dag->n > 0 && (!key || !flags || !dur || !rem || !qin || !qout)))
        return fail(MP_ERR_ARG, "NULL buffer");
    if (qin == qout) return fail(MP_ERR_ARG, "in-place push is not supported (qtask_in == qtask_out)");
    const int32_t n = dag->n;
    const int64_t cap = (int64_t)n * A > 0 ? (int64_t)n * A : 1;
    const int idpass = (bits_for(n > 1 ? n : 2) + 7) / 8;
    size_t bytes = sort_bytes(cap, 1, 8, true) + sort_bytes(n > 0 ? n : 1, 1, idpass, false) + align256((size_t)n + 1) +
                   4 * align256((size_t)cap * 4) + align256(64 * 8) * 4 + align256((((size_t)n + 31) / 32 + 1) * 4) +
                   align256(4);
    MP_TRY(ensure_ws(dag, bytes, st));
    Arena ar{dag->ws, dag->ws_cap};
    SortArgs sa = carve_sort(ar, dag, cap, 1, 0, 8, true);
    SortArgs si = carve_sort(ar, dag, n > 0 ? n : 1, 1, 0, idpass, false);
    uint64_t** ikb = ar.take<uint64_t*>(2);
    int64_t* ilen = ar.take<int64_t>(1);
    uint8_t* removed = ar.take<uint8_t>((size_t)n + 1);
    int32_t* fresh = ar.take<int32_t>((size_t)cap);
    int32_t* keep = ar.take<int32_t>((size_t)cap);
    int32_t* pos = ar.take<int32_t>((size_t)cap);
    int32_t* kept = ar.take<int32_t>((size_t)cap);
    int32_t* cnts = ar.take<int32_t>(64);          // [0..7] new, [8..15] keep, [16] nfresh, [17] scan total
    int64_t* offs = ar.take<int64_t>(64);          // koff [0..8], noff [16..24], dlen [32]
    unsigned long long* brw = ar.take<unsigned long long>(2 * MAX_ARCH);
    uint32_t** vb = ar.take<uint32_t*>(2);
    const size_t words = ((size_t)n + 31) / 32 + 1;
    uint32_t* mark = ar.take<uint32_t>(words);
    uint32_t* bad = ar.take<uint32_t>(1);
    int32_t* cnt_new = cnts;
    int32_t* cnt_keep = cnts + 8;
    int32_t* nfresh = cnts + 16;
    int64_t* koff = offs;
    int64_t* noff = offs + 16;
    int64_t* dlen = offs + 32;
    MP_CUDA(cudaMemsetAsync(cnts, 0, 64 * 4, st));
    MP_CUDA(cudaMemsetAsync(brw, 0, 16 * MAX_ARCH, st));
    MP_CUDA(cudaMemsetAsync(removed, 0, (size_t)n + 1, st));
    uint32_t* hv[2] = {sa.vals[0], sa.vals[1]};
    MP_CUDA(cudaMemcpyAsync(vb, hv, sizeof(hv), cudaMemcpyHostToDevice, st));
    uint64_t* hk[2] = {si.keys[0], si.keys[1]};
    MP_CUDA(cudaMemcpyAsync(ikb, hk, sizeof(hk), cudaMemcpyHostToDevice, st));
    if (m > 0) {
        MP_CUDA(cudaMemsetAsync(mark, 0, words * 4, st));
        MP_CUDA(cudaMemsetAsync(bad, 0, 4, st));
        MP_LAUNCH(k_push_validate, grid_for(m), 256, 0, st, batch, m, n, rem, nullptr, mark, bad, dag->err);
        MP_LAUNCH(k_push_release, grid_for(m), 256, 0, st, batch, m, dag->row_ptr, dag->col, rem, removed, fresh,
                  nfresh, bad);
    }
    MP_LAUNCH(k_push_ids, grid_for(n > 0 ? n : 1), 256, 0, st, fresh, nfresh, si.keys[0], ilen);
    si.d_len = ilen;
    MP_TRY(run_sort(dag, si, st));
    MP_LAUNCH(k_push_new, grid_for(cap), 256, 0, st, si.plans, ikb, nfresh, A, key, flags, sa.keys[0], sa.vals[0],
              cnt_new, dlen);
    sa.seg_len = cap;
    sa.d_len = dlen;
    MP_TRY(run_sort(dag, sa, st));
    MP_LAUNCH(k_push_keep, grid_for(cap), 256, 0, st, qptr_in, A, qin, removed, keep, cnt_keep, cap);
    MP_TRY(scan(dag, keep, pos, cap, nullptr, st));
    MP_LAUNCH(k_push_compact, grid_for(cap), 256, 0, st, qptr_in, A, qin, keep, pos, kept);
    MP_LAUNCH(k_push_offsets, 1, 32, 0, st, A, cnt_keep, cnt_new, koff, noff, qptr_out);
    MP_LAUNCH(k_push_merge, grid_for((cap + PUSH_IPT - 1) / PUSH_IPT), 256, 0, st, A, key, kept, koff, sa.plans, vb,
              noff, qptr_out, qout);
    dim3 g(grid_for(cap, 256, 148 * 4), A);
    MP_LAUNCH(k_push_summary, g, 256, 0, st, A, qptr_out, qout, flags, dur, brw);
    MP_LAUNCH(k_push_finish, 1, 32, 0, st, A, qptr_out, qout, brw, sum);
    MP_CUDA(cudaGetLastError());
    return MP_OK;
}

}  // namespace mph
