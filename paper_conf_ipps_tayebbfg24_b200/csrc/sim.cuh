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
//
// Row N3 (data locality, §V-C, eq. 3): when `top_n` > 1 the POP takes, among
// the first top_n heap entries whose gain is within eps of the root's, the
// one with the largest LS_SDH^2 on the worker's memory node (lane-parallel
// over candidates, then a warp argmax); per-node residency bitmaps over the
// data handles follow task starts (a read copies, a write leaves one copy),
// and non-resident bytes cost xfer_ms_per_byte.
// Readings s1-s9, l1-l6: DESIGN.md §2.
#pragma once
#include "handle.cuh"

namespace mpk {

constexpr int SIM_MAX_WORKERS = 256;
constexpr int SIM_MAX_LEVELS = 6;
constexpr uint32_t ERR_SIM_BIT = 8u;

struct SimArgs {
    int32_t n, A, W, S;         // S = record stride in words (power of two >= 2 + 2A, + A gains)
    int32_t max_tries, eviction;
    // N3 data locality
    int32_t top_n;              // candidates (<= 1: the heap root)
    float eps;
    int32_t H, M;               // handles, memory nodes
    int32_t res_words;          // residency words per node
    int32_t res_smem;           // 1: residency bitmaps in shared memory
    uint32_t* gres;             // [slots][M*res_words] when !res_smem
    const int64_t* acc_ptr;     // [n+1] or null = no data model
    const int32_t* acc_h;
    const uint8_t* acc_mode;
    const uint64_t* hsize;
    double xfer;                // ms per non-resident byte (l6)
    int32_t wnode[SIM_MAX_WORKERS];
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
// [2+A, 2+2A) bits of delta_r(t,a), [2+2A, 2+3A) bits of gain_r(t,a) (N3 only)
constexpr int REC_REM = 0, REC_MASK = 1, REC_RANK = 2;

struct SimShared {              // per-warp counters
    unsigned long long brw[8][2];   // best_remaining_work, exact 128-bit
    unsigned long long busy[8][2];
    int32_t count[8];               // ready_tasks_count
    int32_t ran[8];
    uint32_t again[SIM_MAX_WORKERS / 32];
    int64_t qoff[8];                // queue a's offset in the instance's queues
    uint32_t hd[8];                 // hd_r(a) bits (N3 gains)
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

// smallest set bit > p, or -1 (uniform across the warp)
MP_INLINE int32_t bm_next(const uint32_t* bm, const SimArgs& g, int32_t p) {
    int k = 0;
    int32_t pos = p;
    for (;;) {
        int32_t wi = pos >> 5;
        int b = pos & 31;
        uint32_t w = b == 31 ? 0u : (bm[g.lvoff[k] + wi] & (0xffffffffu << (b + 1)));
        if (w) { pos = wi * 32 + __ffs(w) - 1; break; }
        if (k + 1 == g.nlev) {                   // top level: scan its later words
            int32_t wj = wi + 1;
            while (wj < g.lvsize[k] && bm[g.lvoff[k] + wj] == 0u) ++wj;
            if (wj >= g.lvsize[k]) return -1;
            pos = wj * 32 + __ffs(bm[g.lvoff[k] + wj]) - 1;
            break;
        }
        pos = wi;
        ++k;
    }
    for (int j = k - 1; j >= 0; --j) pos = pos * 32 + __ffs(bm[g.lvoff[j] + pos]) - 1;
    return pos;
}

// eq. 3 (P:l.209): LS_SDH^2(m,t) = sum over t's data resident on node m of
// size (read) or size^2 (write; RW counts as write, l2)
MP_INLINE uint64_t ls_sdh2(const SimArgs& g, const uint32_t* res, int m, int32_t t) {
    uint64_t v = 0;
    const uint32_t* rm = res + (size_t)m * g.res_words;
    for (int64_t i = g.acc_ptr[t], e = g.acc_ptr[t + 1]; i < e; ++i) {
        int32_t h = g.acc_h[i];
        if (!((rm[h >> 5] >> (h & 31)) & 1u)) continue;
        uint64_t z = g.hsize[h];
        v += (g.acc_mode[i] & 2u) ? z * z : z;
    }
    return v;
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
    uint32_t* res = !g.acc_ptr ? nullptr
                   : g.res_smem ? (g.smem_bits ? bits + A * g.bm_words
                                               : reinterpret_cast<uint32_t*>(wtask + ((W + 3) & ~3)))
                                : g.gres + (size_t)blockIdx.x * (size_t)g.M * g.res_words;
    const bool gains = g.top_n > 1;

    for (int32_t rl = blockIdx.x; rl < g.R; rl += gridDim.x) {
        const int64_t r = g.r0 + rl;
        const int32_t* q = g.qtask + (int64_t)rl * g.q_stride;
        // ---- init: records (rem, masks, no rank yet, delta_r), empty heaps,
        //      idle workers, zero counters
        uint32_t hdl[8];
#pragma unroll
        for (int a = 0; a < 8; ++a) hdl[a] = 0u;
        for (int32_t t = lane; t < n; t += 32) {
            uint32_t* rc = rec + (size_t)t * S;
            float d[8];
            float wmin = __int_as_float(0x7f800000);
            uint32_t en = 0;
            int k = 0;
#pragma unroll
            for (int a = 0; a < 8; ++a) {
                d[a] = 0.0f;
                if (a < A) {
                    float x = sim_dur(g, r, t, a);
                    d[a] = x;
                    if (((g.emask >> a) & 1u) && !is_inf(x)) {
                        en |= 1u << a;
                        ++k;
                        if (x < wmin) wmin = x;
                    }
                }
            }
            uint32_t best = 0;
#pragma unroll
            for (int a = 0; a < 8; ++a)
                if (a < A && ((en >> a) & 1u) && d[a] == wmin) best |= 1u << a;   // c15
            rc[REC_REM] = (uint32_t)g.indeg[t];
            rc[REC_MASK] = en | (best << 8);
#pragma unroll
            for (int a = 0; a < 8; ++a) {
                if (a < A) {
                    rc[REC_RANK + a] = 0xffffffffu;
                    rc[REC_RANK + A + a] = f2u(d[a]);
                    if (gains && k >= 2 && ((en >> a) & 1u)) {   // hd_r(a), eq. 1 / c5
                        float ref = __int_as_float(0x7f800000);
#pragma unroll
                        for (int b = 0; b < 8; ++b)
                            if (b < A && b != a && ((en >> b) & 1u)) ref = d[b] < ref ? d[b] : ref;
                        uint32_t ab = f2u(fabsf(__fsub_rn(ref, d[a])));
                        hdl[a] = ab > hdl[a] ? ab : hdl[a];
                    }
                }
            }
        }
        if (gains) {
#pragma unroll
            for (int a = 0; a < 8; ++a) {
                uint32_t v = warp_max(hdl[a]);
                if (lane == a) sh.hd[a] = v;
            }
            __syncwarp();
            // gain_r(t,a) exactly as mp_affinity (eq. 1, c5-c8)
            for (int32_t t = lane; t < n; t += 32) {
                uint32_t* rc = rec + (size_t)t * S;
                uint32_t en = rc[REC_MASK] & 0xffu;
                int k = __popc(en);
                float d[8];
#pragma unroll
                for (int a = 0; a < 8; ++a) d[a] = a < A ? u2f(rc[REC_RANK + A + a]) : 0.0f;
#pragma unroll
                for (int a = 0; a < 8; ++a) {
                    if (a >= A) continue;
                    float gv = 0.0f;
                    if ((en >> a) & 1u) {
                        float h = u2f(sh.hd[a]);
                        if (k == 1) gv = 1.0f;
                        else if (h == 0.0f) gv = 0.5f;
                        else {
                            float ref = __int_as_float(0x7f800000);
#pragma unroll
                            for (int b = 0; b < 8; ++b)
                                if (b < A && b != a && ((en >> b) & 1u)) ref = d[b] < ref ? d[b] : ref;
                            gv = __fdiv_rn(__fadd_rn(__fsub_rn(ref, d[a]), h), __fadd_rn(h, h));
                        }
                    }
                    rc[REC_RANK + 2 * A + a] = f2u(gv);
                }
            }
        }
        if (res) {   // every handle starts in main memory, node 0 (l4)
            for (int32_t i = lane; i < g.M * g.res_words; i += 32) {
                uint32_t v = 0u;
                if (i < g.res_words) {
                    int32_t lo = i * 32, left = g.H - lo;
                    v = left >= 32 ? 0xffffffffu : ((1u << left) - 1u);
                }
                res[i] = v;
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
        int64_t pops = 0, evictions = 0, dups = 0, rounds = 0, moved = 0;
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
                            int32_t t;
                            if (g.top_n > 1) {
                                // get_most_local_prio_task (§V-C): lane i holds the i-th
                                // entry in heap order (l1, l3)
                                int32_t pi = -1, pc = p;
                                for (int i = 0; i < g.top_n && pc >= 0; ++i) {
                                    if (lane == i) pi = pc;
                                    if (i + 1 < g.top_n) pc = bm_next(bm, g, pc);
                                }
                                int32_t ti = pi >= 0 ? qa[pi] : -1;
                                float gi_ = ti >= 0 ? u2f(rec[(size_t)ti * S + REC_RANK + 2 * A + a]) : 0.0f;
                                float g0 = __shfl_sync(0xffffffffu, gi_, 0);
                                bool okc = ti >= 0 && (lane == 0 || __fsub_rn(g0, gi_) <= g.eps);
                                uint32_t okm = __ballot_sync(0xffffffffu, okc);
                                uint32_t pref = ~okm & (okm + 1u);          // first failing lane
                                uint32_t cm = (pref - 1u) & okm;             // prefix of candidates
                                bool cand = (cm >> lane) & 1u;
                                uint64_t v = (cand && res) ? ls_sdh2(g, res, g.wnode[w], ti) : 0ull;
                                uint64_t vm = v;
#pragma unroll
                                for (int o = 16; o > 0; o >>= 1) {
                                    uint64_t x = __shfl_xor_sync(0xffffffffu, vm, o);
                                    vm = x > vm ? x : vm;
                                }
                                int c = __ffs(__ballot_sync(0xffffffffu, cand && v == vm)) - 1;
                                p = __shfl_sync(0xffffffffu, pi, c);
                                t = __shfl_sync(0xffffffffu, ti, c);
                            } else {
                                t = qa[p];
                            }
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
                        // data of the started task moves to the worker's node; a write
                        // leaves that node the only copy (l4)
                        uint64_t gmiss = 0;
                        if (got >= 0 && res) {
                            const int m = g.wnode[w];
                            int64_t a0 = g.acc_ptr[got], a1 = g.acc_ptr[got + 1];
                            uint64_t miss = 0;
                            for (int64_t i = a0 + lane; i < a1; i += 32) {
                                int32_t h = g.acc_h[i];
                                if (!((res[(size_t)m * g.res_words + (h >> 5)] >> (h & 31)) & 1u)) miss += g.hsize[h];
                            }
#pragma unroll
                            for (int o = 16; o > 0; o >>= 1) miss += __shfl_xor_sync(0xffffffffu, miss, o);
                            gmiss = miss;
                            moved += (int64_t)miss;
                            __syncwarp();
                            for (int64_t i = a0 + lane; i < a1; i += 32) {
                                int32_t h = g.acc_h[i];
                                if (g.acc_mode[i] & 2u)
                                    for (int m2 = 0; m2 < g.M; ++m2)
                                        if (m2 != m) atomicAnd(&res[(size_t)m2 * g.res_words + (h >> 5)], ~(1u << (h & 31)));
                                atomicOr(&res[(size_t)m * g.res_words + (h >> 5)], 1u << (h & 31));
                            }
                            __syncwarp();
                        }
                        if (lane == 0) {
                            if (!hit) sh.again[gi] &= ~(1u << (w & 31));
                            if (got >= 0) {
                                until[w] = __dadd_rn(T, __dadd_rn((double)dgot, __dmul_rn((double)gmiss, g.xfer)));  // s1, l6
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
            o.moved = moved;
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
                          const mp_sim_config* cfg, mp_sim_stats* d_stats, double* d_start, int32_t* d_worker,
                          cudaStream_t st) {
    if (!dag) return fail(MP_ERR_ARG, "dag is NULL");
    if (!cfg) return fail(MP_ERR_ARG, "cfg is NULL");
    if (A < 1 || A > 8) return fail(MP_ERR_ARG, "n_arch must be in [1, 8]");
    if (!h_workers) return fail(MP_ERR_ARG, "h_workers is NULL");
    if (R < 0 || r0 < 0) return fail(MP_ERR_ARG, "R and r0 must be >= 0");
    if (cfg->max_tries < 1) return fail(MP_ERR_ARG, "max_tries must be >= 1");
    if (cfg->top_n > 32) return fail(MP_ERR_ARG, "top_n must be <= 32");
    if (!(cfg->eps >= 0.0f)) return fail(MP_ERR_ARG, "eps must be >= 0");
    if (!(cfg->xfer_ms_per_byte >= 0.0)) return fail(MP_ERR_ARG, "xfer_ms_per_byte must be >= 0");
    if (!(sigma >= 0.0f && sigma < 1.0f)) return fail(MP_ERR_ARG, "sigma must be in [0, 1)");
    const bool data = cfg->d_acc_ptr != nullptr;
    if (data && (cfg->n_handles < 0 || (cfg->n_handles > 0 && (!cfg->d_acc_handle || !cfg->d_acc_mode || !cfg->d_size))))
        return fail(MP_ERR_ARG, "incomplete data model");
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
    // memory nodes (l5): given, or arch-0 workers share node 0 (main memory)
    // and every other worker has its own node
    g.M = 1;
    for (int w = 0; w < g.W; ++w) {
        int a = 0;
        while (a + 1 < A && w >= g.wcum[a + 1]) ++a;
        int m = cfg->h_worker_node ? cfg->h_worker_node[w] : (a == 0 ? 0 : 1 + w - h_workers[0]);
        if (m < 0 || m >= 1024) return fail(MP_ERR_ARG, "worker memory node must be in [0, 1024)");
        g.wnode[w] = m;
        g.M = std::max(g.M, m + 1);
    }
    g.M = std::max(g.M, cfg->n_nodes);
    const int32_t n = dag->n;
    if (R == 0) return MP_OK;
    if (!d_base || !d_qtask || !d_sum || !d_stats) return fail(MP_ERR_ARG, "NULL device pointer");
    g.n = n;
    g.A = A;
    g.top_n = cfg->top_n;
    g.eps = cfg->eps;
    g.S = 4;
    while (g.S < 2 + (g.top_n > 1 ? 3 : 2) * A) g.S *= 2;
    g.max_tries = cfg->max_tries;
    g.eviction = cfg->eviction ? 1 : 0;
    g.H = data ? cfg->n_handles : 0;
    g.res_words = std::max<int32_t>(1, (g.H + 31) / 32);
    g.acc_ptr = data ? cfg->d_acc_ptr : nullptr;
    g.acc_h = cfg->d_acc_handle;
    g.acc_mode = cfg->d_acc_mode;
    g.hsize = cfg->d_size;
    g.xfer = cfg->xfer_ms_per_byte;
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
    size_t res_bytes = data ? (size_t)g.M * g.res_words * 4 : 0;
    const size_t kSmemBudget = 48 * 1024;   // per warp: >= 4 instances per SM
    g.smem_bits = base_smem + bits_bytes <= kSmemBudget ? 1 : 0;
    size_t smem = base_smem + (g.smem_bits ? bits_bytes : 0);
    g.res_smem = data && smem + res_bytes <= kSmemBudget ? 1 : 0;
    if (g.res_smem) smem += res_bytes;
    MP_CUDA(cudaFuncSetAttribute(mpk::k_sim, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    MP_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, mpk::k_sim, 32, smem));
    if (per_sm < 1) return fail(MP_ERR_ARG, "simulator does not fit on an SM");
    int64_t slots = std::min<int64_t>(R, (int64_t)per_sm * dag->num_sms);
    size_t need = align256((size_t)slots * std::max(n, 1) * g.S * 4) +
                  (g.smem_bits ? 0 : align256((size_t)slots * bits_bytes)) +
                  (data && !g.res_smem ? align256((size_t)slots * res_bytes) : 0);
    MP_TRY(ensure_ws(dag, need, st));
    Arena ar{dag->ws, dag->ws_cap};
    g.rec = ar.take<uint32_t>((size_t)slots * std::max(n, 1) * g.S);
    g.gbits = g.smem_bits ? nullptr : ar.take<uint32_t>((size_t)slots * A * g.bm_words);
    g.gres = data && !g.res_smem ? ar.take<uint32_t>((size_t)slots * g.M * g.res_words) : nullptr;
    MP_LAUNCH(mpk::k_sim, (unsigned)slots, 32, smem, st, g);
    MP_CUDA(cudaGetLastError());
    return MP_OK;
}

}  // namespace mph
