// sim.cuh -- SURVEY §8(f) N2: discrete-event simulation of MultiPrio's PUSH
// (Alg. 1, P:l.133-136) and POP (Alg. 2, P:l.140-160) with the eviction
// mechanism (pop_condition, §V-D, P:l.214-220) and duplicate handling
// (P:l.130), batched over duration-perturbed replicas (a10).
//
// One warp simulates one instance (the event chain of one schedule is
// sequential; instances are independent).  The heaps are not binary heaps
// here: a heap's entries are always a subset of that arch's ALL-mode queue
// (a8; scores are whole-DAG, reading c18), whose order is the heap order, so
// heap a is a bitmap over queue ranks with a 32-ary summary tree on top
// (every level-k bit says "word below is non-zero").  PUSH sets the bit at
// rank_a(t) (atomicOr, lanes push different tasks at once); the root is the
// first set bit -- one ballot over the top level's <= 32 words plus one
// broadcast load per level below; a removal clears one bit and propagates
// empty words up.  A popped task's duplicates are cleared from the other
// heaps at once (a bitmap deletes in place; the paper's binary heaps remove
// them lazily, P:l.130 -- a processed duplicate is skipped without counting
// as a try, reading s5, so the schedule is the same).
//
// Per instance, a per-slot record array holds for each task t, in one 32-B
// (A <= 3) sector: rem(t) (predecessors not completed), the enabled / best
// arch masks, rank_a(t) and delta_r(t,a); a release therefore costs one
// dependent load per successor and a POP one load after the root search.
// Bitmaps live in shared memory when they fit the per-warp budget, else in a
// global per-slot scratch (same code through generic pointers).
// Readings s1-s9: DESIGN.md §2.
#pragma once
#include "handle.cuh"

namespace mpk {

constexpr int SIM_MAX_WORKERS = 256;
constexpr int SIM_MAX_LEVELS = 6;
constexpr uint32_t ERR_SIM_BIT = 8u;

struct SimArgs {
    int32_t n, A, W, S;         // S = record stride in words (power of two >= 2 + 2A)
    int32_t max_tries, eviction;
    uint64_t seed;
    float sigma;
    int64_t r0;
    int32_t R;
    int32_t wcum[9];            // workers of archs < a (arch-major numbering, s2)
    uint32_t emask;             // archs with workers > 0
    const int32_t* row_ptr;
    const int32_t* col;
    const int32_t* indeg;
    const float* base;          // [n][A]
    const int32_t* qtask;       // [R][q_stride], queue a at the prefix of counts
    int64_t q_stride;
    const mp_queue_summary* sum;  // [R][A]
    // bitmap layout (identical for every arch): level k at word offset lvoff[k]
    int32_t nlev;
    int32_t lvoff[SIM_MAX_LEVELS];
    int32_t lvsize[SIM_MAX_LEVELS];
    int32_t bm_words;           // words per arch
    int32_t smem_bits;          // 1: bitmaps in shared memory
    uint32_t* gbits;            // [slots][A*bm_words] when !smem_bits
    uint32_t* rec;              // [slots][n][S]
    mp_sim_stats* stats;        // [R]
    double* start;              // [R][n] or null
    int32_t* worker;            // [R][n] or null
    uint32_t* err;
};

// record words: [0] rem, [1] enabled mask | best mask << 8, [2, 2+A) rank_a,
// [2+A, 2+2A) bits of delta_r(t,a)
constexpr int REC_REM = 0, REC_MASK = 1, REC_RANK = 2;

struct SimShared {              // per-warp counters
    unsigned long long brw[8][2];   // best_remaining_work, exact 128-bit
    unsigned long long busy[8][2];
    int32_t count[8];               // ready_tasks_count
    int32_t ran[8];
    uint32_t again[SIM_MAX_WORKERS / 32];
    int64_t qoff[8];                // queue a's offset in the instance's queues
};

MP_INLINE void sub128_atomic(unsigned long long* p, uint64_t lo, uint64_t hi) {
    // p -= (hi:lo), as the addition of the two's complement
    uint64_t nlo = ~lo + 1ull;
    uint64_t nhi = ~hi + (lo == 0 ? 1ull : 0ull);
    atomic_add128(p, nlo, nhi);
}

MP_INLINE bool gt128(uint64_t alo, uint64_t ahi, uint64_t blo, uint64_t bhi) {
    return ahi > bhi || (ahi == bhi && alo > blo);
}

// delta_r(t, a) (a10), -0 read as +0 (c20)
MP_INLINE float sim_dur(const SimArgs& g, int64_t r, int32_t t, int32_t a) {
    float d = g.base[(int64_t)t * g.A + a];
    if (g.sigma != 0.0f) {
        uint64_t c = ((uint64_t)r * (uint64_t)g.n + (uint64_t)t) * (uint64_t)g.A + (uint64_t)a + 1ull;
        d = perturb(d, g.seed, g.sigma, c);
    }
    return (f2u(d) & 0x7fffffffu) == 0u ? 0.0f : d;
}

// set bit p of heap `bm` (atomic; concurrent setters allowed)
MP_INLINE void bm_set(uint32_t* bm, const SimArgs& g, int32_t p) {
    for (int k = 0; k < g.nlev; ++k) {
        uint32_t old = atomicOr(bm + g.lvoff[k] + (p >> 5), 1u << (p & 31));
        if (old != 0u) return;
        p >>= 5;
    }
}

// clear bit p (one lane per heap; no concurrent access to the same heap)
MP_INLINE void bm_clear(uint32_t* bm, const SimArgs& g, int32_t p) {
    for (int k = 0; k < g.nlev; ++k) {
        uint32_t* w = bm + g.lvoff[k] + (p >> 5);
        uint32_t v = *w & ~(1u << (p & 31));
        *w = v;
        if (v != 0u) return;
        p >>= 5;
    }
}

MP_INLINE bool bm_test(const uint32_t* bm, int32_t p) { return (bm[p >> 5] >> (p & 31)) & 1u; }

// first set bit (the heap root's rank) or -1; whole warp, uniform result
MP_INLINE int32_t bm_first(const uint32_t* bm, const SimArgs& g, int lane) {
    int top = g.nlev - 1;
    uint32_t v = lane < g.lvsize[top] ? bm[g.lvoff[top] + lane] : 0u;
    uint32_t m = __ballot_sync(0xffffffffu, v != 0u);
    if (m == 0u) return -1;
    int l = __ffs(m) - 1;
    uint32_t w = __shfl_sync(0xffffffffu, v, l);
    int32_t idx = l * 32 + __ffs(w) - 1;
    for (int k = top - 1; k >= 0; --k) {
        w = bm[g.lvoff[k] + idx];
        idx = idx * 32 + __ffs(w) - 1;
    }
    return idx;
}

// PUSH of task s by this lane (Alg. 1): join every enabled arch's heap;
// ready_tasks_count and best_remaining_work updated exactly.  `rc` = s's record.
MP_INLINE void sim_push(const SimArgs& g, const uint32_t* rc, uint32_t* bits, SimShared& sh) {
    uint32_t masks = rc[REC_MASK];
    for (int a = 0; a < g.A; ++a) {
        if (!((masks >> a) & 1u)) continue;
        int32_t p = (int32_t)rc[REC_RANK + a];
        if (p < 0) {              // not in the ALL-mode queue a: invalid input
            atomicOr(g.err, ERR_SIM_BIT);
            continue;
        }
        bm_set(bits + a * g.bm_words, g, p);
        atomicAdd(&sh.count[a], 1);
        if ((masks >> (8 + a)) & 1u) {
            uint64_t lo, hi;
            fixed64(u2f(rc[REC_RANK + g.A + a]), lo, hi);
            atomic_add128(sh.brw[a], lo, hi);
        }
    }
}

__global__ void __launch_bounds__(32) k_sim(SimArgs g) {
    extern __shared__ __align__(16) unsigned char smem[];
    const int lane = threadIdx.x;
    const int32_t n = g.n, A = g.A, W = g.W, S = g.S;
    SimShared& sh = *reinterpret_cast<SimShared*>(smem);
    double* until = reinterpret_cast<double*>(smem + ((sizeof(SimShared) + 15) & ~size_t(15)));
    int32_t* wtask = reinterpret_cast<int32_t*>(until + W);
    uint32_t* bits = g.smem_bits ? reinterpret_cast<uint32_t*>(wtask + ((W + 3) & ~3))
                                 : g.gbits + (size_t)blockIdx.x * (size_t)(A * g.bm_words);
    uint32_t* rec = g.rec + (size_t)blockIdx.x * (size_t)n * S;

    for (int32_t rl = blockIdx.x; rl < g.R; rl += gridDim.x) {
        const int64_t r = g.r0 + rl;
        const int32_t* q = g.qtask + (int64_t)rl * g.q_stride;
        // ---- init: records (rem, masks, no rank yet, delta_r), empty heaps,
        //      idle workers, zero counters
        for (int32_t t = lane; t < n; t += 32) {
            uint32_t* rc = rec + (size_t)t * S;
            float d[8];
            float wmin = __int_as_float(0x7f800000);
            uint32_t en = 0;
            for (int a = 0; a < A; ++a) {
                float x = sim_dur(g, r, t, a);
                d[a & 7] = x;
                if (((g.emask >> a) & 1u) && !is_inf(x)) {
                    en |= 1u << a;
                    if (x < wmin) wmin = x;
                }
            }
            uint32_t best = 0;
            for (int a = 0; a < A; ++a)
                if (((en >> a) & 1u) && d[a & 7] == wmin) best |= 1u << a;   // c15
            rc[REC_REM] = (uint32_t)g.indeg[t];
            rc[REC_MASK] = en | (best << 8);
            for (int a = 0; a < A; ++a) {
                rc[REC_RANK + a] = 0xffffffffu;
                rc[REC_RANK + A + a] = f2u(d[a & 7]);
            }
        }
        for (int32_t i = lane; i < A * g.bm_words; i += 32) bits[i] = 0u;
        for (int32_t w = lane; w < W; w += 32) { until[w] = 0.0; wtask[w] = -1; }
        if (lane < 8) {
            sh.brw[lane][0] = sh.brw[lane][1] = 0ull;
            sh.busy[lane][0] = sh.busy[lane][1] = 0ull;
            sh.count[lane] = 0;
            sh.ran[lane] = 0;
        }
        __syncwarp();
        {
            int64_t o = 0;
            for (int a = 0; a < A; ++a) {
                int32_t c = g.sum[(int64_t)rl * A + a].count;
                if (lane == 0) sh.qoff[a] = o;
                const int32_t* qa = q + o;
                for (int32_t p = lane; p < c; p += 32) {
                    int32_t t = qa[p];
                    if ((uint32_t)t < (uint32_t)n) rec[(size_t)t * S + REC_RANK + a] = (uint32_t)p;
                    else atomicOr(g.err, ERR_SIM_BIT);
                }
                o += c;
            }
        }
        __syncwarp();
        // ---- time 0: the sources are ready (P:l.91)
        for (int32_t t = lane; t < n; t += 32)
            if (g.indeg[t] == 0) sim_push(g, rec + (size_t)t * S, bits, sh);
        __syncwarp();

        double T = 0.0;
        int32_t done = 0;
        int64_t pops = 0, evictions = 0, dups = 0, rounds = 0;
        for (;;) {
            // ---- dispatch (s2, s7): idle workers POP in id order; those whose
            // POP ended on MAX_TRIES poll again, round-robin, at the same T
            for (int gi = 0; gi * 32 < W; ++gi) {
                int w = gi * 32 + lane;
                uint32_t m = __ballot_sync(0xffffffffu, w < W && wtask[w] < 0);
                if (lane == 0) sh.again[gi] = m;
            }
            __syncwarp();
            // heaps only shrink during a dispatch, so once a POP finds heap a
            // empty every later POP on a in this dispatch returns nothing too
            uint32_t empty = 0;
            for (bool any = true; any;) {
                any = false;
                for (int gi = 0; gi * 32 < W; ++gi) {
                    uint32_t m = sh.again[gi];
                    while (m) {
                        int w = gi * 32 + __ffs(m) - 1;
                        m &= m - 1;
                        int a = 0;
                        while (a + 1 < A && w >= g.wcum[a + 1]) ++a;
                        if ((empty >> a) & 1u) {
                            if (lane == 0) sh.again[gi] &= ~(1u << (w & 31));
                            __syncwarp();
                            continue;
                        }
                        uint32_t* bm = bits + a * g.bm_words;
                        const int32_t* qa = q + sh.qoff[a];
                        // ---- Alg. 2 POP
                        int tries = 0;
                        bool hit = false;
                        int32_t got = -1;
                        float dgot = 0.0f;
                        for (;;) {
                            if (tries >= g.max_tries) { hit = true; break; }
                            int32_t p = bm_first(bm, g, lane);
                            if (p < 0) { empty |= 1u << a; break; }
                            int32_t t = qa[p];
                            const uint32_t* rc = rec + (size_t)t * S;
                            uint32_t masks = rc[REC_MASK];
                            // lane b < A: arch b's rank and delta
                            int32_t rk = lane < A ? (int32_t)rc[REC_RANK + lane] : -1;
                            float mine = lane < A ? u2f(rc[REC_RANK + A + lane]) : 0.0f;
                            bool best_l = lane < A && ((masks >> (8 + lane)) & 1u);
                            float da = __shfl_sync(0xffffffffu, mine, a);
                            // pop_condition (§V-D, s4)
                            bool cond = true;
                            if (g.eviction && !((masks >> (8 + a)) & 1u)) {
                                uint64_t mlo, mhi;
                                fixed64(da, mlo, mhi);
                                bool ok = !best_l || gt128(sh.brw[lane][0], sh.brw[lane][1], mlo, mhi);
                                cond = __all_sync(0xffffffffu, ok);
                            }
                            if (cond) {
                                // heaps_pop_and_update: t leaves every heap that still
                                // holds it and their counters (s5)
                                bool held = false;
                                if (lane < A && ((masks >> lane) & 1u))
                                    held = lane == a || (rk >= 0 && bm_test(bits + lane * g.bm_words, rk));
                                uint32_t hm = __ballot_sync(0xffffffffu, held);
                                if (held) {
                                    bm_clear(bits + lane * g.bm_words, g, lane == a ? p : rk);
                                    atomicSub(&sh.count[lane], 1);
                                    if (best_l) {
                                        uint64_t lo, hi;
                                        fixed64(mine, lo, hi);
                                        sub128_atomic(sh.brw[lane], lo, hi);
                                    }
                                }
                                __syncwarp();
                                dups += __popc(hm) - 1;
                                ++pops;
                                got = t;
                                dgot = da;
                                break;
                            }
                            // heaps_evict_task: t leaves this heap only (s8)
                            if (lane == 0) {
                                bm_clear(bm, g, p);
                                sh.count[a] -= 1;
                            }
                            __syncwarp();
                            ++evictions;
                            ++tries;
                        }
                        if (hit) { ++rounds; any = true; }
                        if (lane == 0) {
                            if (!hit) sh.again[gi] &= ~(1u << (w & 31));
                            if (got >= 0) {
                                until[w] = __dadd_rn(T, (double)dgot);   // s1
                                wtask[w] = got;
                                uint64_t lo, hi;
                                fixed64(dgot, lo, hi);
                                add128(*(uint64_t*)&sh.busy[a][0], *(uint64_t*)&sh.busy[a][1], lo, hi);
                                sh.ran[a] += 1;
                                if (g.start) g.start[(int64_t)rl * n + got] = T;
                                if (g.worker) g.worker[(int64_t)rl * n + got] = w;
                            }
                        }
                        __syncwarp();
                    }
                }
            }
            // ---- next event: earliest completion (s2)
            double tmin = __longlong_as_double(0x7ff0000000000000ll);
            for (int w = lane; w < W; w += 32)
                if (wtask[w] >= 0 && until[w] < tmin) tmin = until[w];
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                double x = __shfl_xor_sync(0xffffffffu, tmin, o);
                tmin = x < tmin ? x : tmin;
            }
            if (tmin == __longlong_as_double(0x7ff0000000000000ll)) break;   // nobody busy
            T = tmin;
            // ---- completions at T, in worker id order, release their
            // successors (lanes over a task's successor row; pushes commute)
            for (int gi = 0; gi * 32 < W; ++gi) {
                int w0 = gi * 32 + lane;
                bool fin = w0 < W && wtask[w0] >= 0 && until[w0] == T;
                int32_t tl = fin ? wtask[w0] : -1;
                uint32_t m = __ballot_sync(0xffffffffu, fin);
                if (fin) wtask[w0] = -1;
                __syncwarp();
                while (m) {
                    int l = __ffs(m) - 1;
                    m &= m - 1;
                    int32_t t = __shfl_sync(0xffffffffu, tl, l);
                    ++done;
                    int32_t beg = g.row_ptr[t], end = g.row_ptr[t + 1];
                    for (int32_t j0 = beg; j0 < end; j0 += 32) {
                        int32_t j = j0 + lane;
                        if (j < end) {
                            uint32_t* rc = rec + (size_t)g.col[j] * S;
                            uint32_t k = rc[REC_REM] - 1u;
                            rc[REC_REM] = k;
                            if (k == 0u) sim_push(g, rc, bits, sh);
                        }
                    }
                    __syncwarp();
                }
            }
        }
        if (lane == 0) {
            mp_sim_stats o;
            o.makespan = T;
            o.pops = pops;
            o.evictions = evictions;
            o.dups = dups;
            o.rounds = rounds;
#pragma unroll
            for (int a = 0; a < 8; ++a) {
                o.busy[a] = a < A ? u128_to_double_scaled(sh.busy[a][0], sh.busy[a][1]) : 0.0;
                o.ran[a] = a < A ? sh.ran[a] : 0;
            }
            g.stats[rl] = o;
            if (done != n) atomicOr(g.err, ERR_SIM_BIT);
        }
        __syncwarp();
    }
}

}  // namespace mpk

namespace mph {

inline mp_status simulate(mp_dag* dag, int32_t A, const float* d_base, const int32_t* h_workers, uint64_t seed,
                          float sigma, int64_t r0, int32_t R, const int32_t* d_qtask, const mp_queue_summary* d_sum,
                          int32_t max_tries, int32_t eviction, mp_sim_stats* d_stats, double* d_start,
                          int32_t* d_worker, cudaStream_t st) {
    if (!dag) return fail(MP_ERR_ARG, "dag is NULL");
    if (A < 1 || A > 8) return fail(MP_ERR_ARG, "n_arch must be in [1, 8]");
    if (!h_workers) return fail(MP_ERR_ARG, "h_workers is NULL");
    if (R < 0 || r0 < 0) return fail(MP_ERR_ARG, "R and r0 must be >= 0");
    if (max_tries < 1) return fail(MP_ERR_ARG, "max_tries must be >= 1");
    if (!(sigma >= 0.0f && sigma < 1.0f)) return fail(MP_ERR_ARG, "sigma must be in [0, 1)");
    mpk::SimArgs g{};
    g.W = 0;
    g.wcum[0] = 0;
    for (int a = 0; a < A; ++a) {
        if (h_workers[a] < 0) return fail(MP_ERR_ARG, "negative worker count");
        g.W += h_workers[a];
        g.wcum[a + 1] = g.W;
    }
    if (g.W < 1 || g.W > mpk::SIM_MAX_WORKERS) return fail(MP_ERR_ARG, "total workers must be in [1, %d]",
                                                           mpk::SIM_MAX_WORKERS);
    const int32_t n = dag->n;
    if (R == 0) return MP_OK;
    if (!d_base || !d_qtask || !d_sum || !d_stats) return fail(MP_ERR_ARG, "NULL device pointer");
    g.n = n;
    g.A = A;
    g.S = 4;
    while (g.S < 2 + 2 * A) g.S *= 2;
    g.max_tries = max_tries;
    g.eviction = eviction ? 1 : 0;
    g.seed = seed;
    g.sigma = sigma;
    g.r0 = r0;
    g.R = R;
    g.emask = enabled_mask(A, h_workers);
    g.row_ptr = dag->row_ptr;
    g.col = dag->col;
    g.indeg = dag->indeg;
    g.base = d_base;
    g.qtask = d_qtask;
    g.q_stride = (int64_t)n * A;
    g.sum = d_sum;
    g.stats = d_stats;
    g.start = d_start;
    g.worker = d_worker;
    g.err = dag->err;
    // summary-tree layout: level 0 = ceil(n/32) words, each level above 32x
    // fewer, until one level has <= 32 words (searched by one ballot)
    int32_t words = std::max<int32_t>(1, (n + 31) / 32), off = 0;
    g.nlev = 0;
    for (;;) {
        if (g.nlev >= mpk::SIM_MAX_LEVELS) return fail(MP_ERR_ARG, "DAG too large for the simulator");
        g.lvoff[g.nlev] = off;
        g.lvsize[g.nlev] = words;
        off += words;
        g.nlev++;
        if (words <= 32) break;
        words = (words + 31) / 32;
    }
    g.bm_words = off;
    size_t base_smem = ((sizeof(mpk::SimShared) + 15) & ~size_t(15)) + (size_t)g.W * 8 + (size_t)((g.W + 3) & ~3) * 4;
    size_t bits_bytes = (size_t)(A * g.bm_words) * 4;
    const size_t kSmemBudget = 48 * 1024;   // per warp: >= 4 instances per SM
    g.smem_bits = base_smem + bits_bytes <= kSmemBudget ? 1 : 0;
    size_t smem = base_smem + (g.smem_bits ? bits_bytes : 0);
    MP_CUDA(cudaFuncSetAttribute(mpk::k_sim, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    MP_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, mpk::k_sim, 32, smem));
    if (per_sm < 1) return fail(MP_ERR_ARG, "simulator does not fit on an SM");
    int64_t slots = std::min<int64_t>(R, (int64_t)per_sm * dag->num_sms);
    size_t need = align256((size_t)slots * std::max(n, 1) * g.S * 4) +
                  (g.smem_bits ? 0 : align256((size_t)slots * bits_bytes));
    MP_TRY(ensure_ws(dag, need, st));
    Arena ar{dag->ws, dag->ws_cap};
    g.rec = ar.take<uint32_t>((size_t)slots * std::max(n, 1) * g.S);
    g.gbits = g.smem_bits ? nullptr : ar.take<uint32_t>((size_t)slots * A * g.bm_words);
    MP_LAUNCH(mpk::k_sim, (unsigned)slots, 32, smem, st, g);
    MP_CUDA(cudaGetLastError());
    return MP_OK;
}

}  // namespace mph
