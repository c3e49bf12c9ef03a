// rep2.cuh -- a10 fast path: batched duration-perturbed replicas, n < 65536.
//
// K1 k_rep2_bl   -- lanes = replicas: one CTA runs 32 replicas in lock-step
//                   (same DAG, same control flow), one warp per node of the
//                   current level; successor bottom-levels of the 32 replicas
//                   are one coalesced 128-byte line ([q][32] layout, L2
//                   resident).  Each (r,t,a) duration is hashed once here and
//                   feeds the per-replica statistics (counts, hd, exact brw),
//                   bl, CP.  Epilogue: bl transposed to [r][t].
// K2 k_rep2_sort -- one CTA per replica (persistent):
//                   crit order  : stable sort of critc(t) = 1 - bits(bl/CP)
//                                 in id order  -> pi (ids by (crit desc, id))
//                   queue a     : stable sort, in pi order, of gainc_a(t)
//                                 -> (gain desc, crit desc, id asc) = a8.
//                   Both sorts: key-range buckets of <= 16384 entries are
//                   compacted (stably) into shared memory and LSD-sorted
//                   there; ranges with one key value are streamed in order.
// Bit-exact with the oracle: same RN ops as path.cuh / replicas.cuh.
#pragma once
#include <map>
#include <mutex>
#include "replicas.cuh"

namespace mpk {

constexpr int R2_THREADS = 1024;
constexpr int R2_WARPS = 32;
constexpr int R2_CAP = 16384;
constexpr int R2_NBINS = 4096;

// Optional per-phase cycle accounting of K2 (build with -DMP_PHASES; tools/k2_phases.py).
#ifdef MP_PHASES
__device__ unsigned long long g_k2_phase[32];
MP_INLINE void k2_phase(int i) {
    __shared__ long long s_t;
    __syncthreads();
    if (threadIdx.x == 0) {
        const long long t = clock64();
        if (i > 0) atomicAdd(&g_k2_phase[i], (unsigned long long)(t - s_t));
        s_t = t;
    }
    __syncthreads();
}
#define K2_PHASE(i) k2_phase(i)
#else
#define K2_PHASE(i) ((void)0)
#endif

struct Rep2Args {
    int32_t n, A, L, R;
    int64_t r0;                  // global id of replica 0 of this call
    const int32_t* lvlq;
    const int32_t* nodeq;
    const int32_t* rowq;
    const int32_t* colq;
    const int32_t* qof;
    const float* base;
    uint32_t emask;
    uint64_t seed;
    float sigma;
    float* bl32;                 // [groups][n][32] scratch
    float* blT;                  // [R][n]
    float* cp;                   // [R]
    uint32_t* hd;                // [R][A] (float bits)
    int32_t* counts;             // [R][A]
    unsigned long long* brw;     // [R][A][2]
    uint32_t* err;
    int flow;                    // K1: 1 = dataflow over the whole q range (one CTA per group)
    // K2
    uint32_t* s_key;             // [grid][2][npad] per-CTA hot scratch: D in id order, D in sorted order
    uint16_t* s_pi;              // [grid][2][npad] per-CTA hot scratch: fine-bin ids, sorted positions
    uint32_t* s_cold;            // [grid][A+1][npad] general path only: critc, gainc per arch
    unsigned char* s_geo;        // [grid][R3_GEO_BYTES] two-arch path: cached sub-bin geometry
    int32_t* qtask;              // [R][n*A] or null
    mp_queue_summary* sum;       // [R][A]
    uint32_t* ticket;
    // two archs: K2 split for overlap with K1 (rep2_launch).  mode 1 = pre-sort pass (hash +
    // sort of replicas [0, pre_R) into pp_pos / pp_ds, launched beside K1 on the SMs K1
    // leaves idle); mode 2 = the main pass, replicas < pre_R start after their sort.
    int mode;
    int32_t pre_R;
    uint16_t* pp_pos;            // [pre_R][npad] sorted positions
    uint32_t* pp_ds;             // [pre_R][npad] D in sorted order
    uint32_t* ticket_pre;
};

template <int A>
MP_INLINE void r2_durs(const Rep2Args& a, int64_t r, int32_t t, float (&x)[A], uint32_t& en, int& k, float& w,
                       bool& bad) {
    en = 0;
    k = 0;
    w = __uint_as_float(0x7f800000u);
    const uint64_t c0 = ((uint64_t)r * (uint64_t)a.n + (uint64_t)t) * (uint64_t)A + 1u;
#pragma unroll
    for (int b = 0; b < A; b++) {
        float d = perturb(__ldg(a.base + (int64_t)t * A + b), a.seed, a.sigma, c0 + b);
        d = canon_dur(d, bad);
        x[b] = d;
        if (((a.emask >> b) & 1u) && !is_inf(d)) {
            en |= 1u << b;
            k++;
            w = d < w ? d : w;
        }
    }
    if (!k) bad = true;
}

// ---------------------------------------------------------------------------------------
// K1
// ---------------------------------------------------------------------------------------
#ifndef MP_K1_PF
#define MP_K1_PF 8
#endif
constexpr int K1_PF = MP_K1_PF;   // successor-line gathers in flight per lane

template <int A>
// A 32-replica group is run by a cluster of `cs` CTAs (cs = 1 when there are enough
// groups to fill the GPU; up to 8 for small per-GPU replica counts): the nodes of a
// level are spread over the cluster's warps and levels are separated by cluster
// barriers (release/acquire at cluster scope, bl32 lines are written once and only
// read after).
__global__ void __launch_bounds__(R2_THREADS, 1) k_rep2_bl(Rep2Args a) {
    extern __shared__ __align__(16) unsigned char r2_smem[];
    const int lane = threadIdx.x & 31, w0 = threadIdx.x >> 5;
    cg::cluster_group cluster = cg::this_cluster();
    const int cs = (int)cluster.num_blocks();
    const int crank = (int)cluster.block_rank();
    const int w = crank * R2_WARPS + w0;            // warp index within the group
    const int WG = cs * R2_WARPS;                   // warps per group
    const int64_t g = blockIdx.x / cs;
    const int64_t rl = g * 32 + lane;            // replica index within this call
    const bool live = rl < a.R;
    const int64_t r = a.r0 + rl;                 // global replica id
    float* bl32 = a.bl32 + g * (int64_t)a.n * 32;
    const float* bll = bl32 + lane;              // this lane's (replica's) column
    bool bad = false;
    uint32_t hd[A];
    int32_t cnt[A];
    uint64_t blo[A], bhi[A];
#pragma unroll
    for (int q = 0; q < A; q++) { hd[q] = 0; cnt[q] = 0; blo[q] = 0; bhi[q] = 0; }
    float cpm = 0.0f;
    // Two-arch fast path, decided once per launch from the perturbation's extremes (every
    // RN op of perturb() is monotone in u, so each perturbed duration lies between its
    // values at u = 0 and u = 1 - 2^-24; K2 uses the same bound): if every task is enabled
    // on both archs and every extreme is a nonzero domain value, no perturbed duration can
    // be 0, +inf or out of the domain, so the enabled masks, the domain checks and the
    // per-arch counters (= tasks processed) drop out, hd is one |x1 - x0| per task, and if
    // the exponents span few enough binades, best_remaining_work is summed exactly in one
    // uint64 of units 2^(emin - 150) (mantissa << (e - emin)) instead of a 128-bit fixed
    // point per task; converted to the 2^-64 units at the end.
    __shared__ uint32_t s_fok, s_emin, s_emax;
    bool fast = false;
    uint32_t emin = 0;
    uint64_t acc[2] = {0ull, 0ull};
    uint32_t hdf = 0, nproc = 0;
    uint64_t cbase = 0;
    if constexpr (A == 2) {
        if (threadIdx.x == 0) {
            s_fok = (a.emask == 3u && (reinterpret_cast<uintptr_t>(a.base) & 7u) == 0u) ? 1u : 0u;
            s_emin = 255u;
            s_emax = 0u;
        }
        __syncthreads();
        bool ok = true;
        uint32_t lmin = 255u, lmax = 0u;
        for (int32_t t = threadIdx.x; t < a.n; t += R2_THREADS) {
#pragma unroll
            for (int b = 0; b < 2; b++) {
                const float bv = __ldg(a.base + 2 * (int64_t)t + b);
                const float e0 = perturb_u(bv, a.sigma, 0u), e1 = perturb_u(bv, a.sigma, 0xFFFFFFu);
                const uint32_t ul = f2u(e0 < e1 ? e0 : e1), uh = f2u(e0 < e1 ? e1 : e0);
                // both extremes in [2^-41, 2^20) (excludes 0, -0, negatives, inf, NaN)
                if (!(ul >= 0x2B000000u && ul < 0x49800000u && uh >= 0x2B000000u && uh < 0x49800000u)) ok = false;
                lmin = min(lmin, ul >> 23);
                lmax = max(lmax, uh >> 23);
            }
        }
        ok = __all_sync(0xffffffffu, ok);
        lmin = __reduce_min_sync(0xffffffffu, lmin);
        lmax = __reduce_max_sync(0xffffffffu, lmax);
        if (lane == 0) {
            if (!ok) atomicAnd(&s_fok, 0u);
            atomicMin(&s_emin, lmin);
            atomicMax(&s_emax, lmax);
        }
        __syncthreads();
        const uint32_t nb = 32u - __clz((uint32_t)a.n);   // n < 2^nb
        fast = s_fok && s_emin <= s_emax && 24u + (s_emax - s_emin) + nb <= 64u;
        emin = s_emin;
        // splitmix64 state of (r, t = 0, arch 0): seed + ((r n + t) 2 + 1) golden
        cbase = a.seed + ((uint64_t)r * (uint64_t)a.n * 2u + 1u) * SPLITMIX_GOLDEN;
    }
    // Dataflow mode (one CTA per group): no barrier per level.  The warps walk the whole
    // q range (reverse level order) with stride 32; a node's bl line is published by a
    // per-position ready byte in shared memory (data stores, __syncwarp, block fence, flag),
    // and a gather first waits for its successor's byte (a successor has a smaller q, so
    // the smallest unfinished node can always proceed: no deadlock).  Narrow levels then
    // overlap with the next ones instead of idling 32 - width warps at a barrier.
    const bool flow = a.flow != 0 && cs == 1;
    volatile uint8_t* rdy = reinterpret_cast<volatile uint8_t*>(r2_smem);
    if (flow) {
        for (int32_t i = threadIdx.x; i < (a.n + 3) / 4; i += R2_THREADS)
            reinterpret_cast<volatile uint32_t*>(r2_smem)[i] = 0u;
        __syncthreads();
    }
    const int32_t nlv = flow ? 1 : a.L;
    for (int32_t lv = 0; lv < nlv; lv++) {
        const int32_t q1 = flow ? a.n : __ldg(a.lvlq + lv + 1);
        int32_t q = (flow ? 0 : __ldg(a.lvlq + lv)) + w;
        // software pipeline: the CSR slice of the warp's next node is loaded while the
        // current node hashes its durations and gathers its successors' bottom-levels
        int32_t v = 0, e0 = 0, e1 = 0, sv = 0;
        if (q < q1) {
            v = __ldg(a.nodeq + q);
            e0 = __ldg(a.rowq + q);
            e1 = __ldg(a.rowq + q + 1);
            sv = lane < e1 - e0 ? __ldg(a.colq + e0 + lane) : 0;
        }
        while (q < q1) {
            const int32_t qn = q + WG;
            int32_t vn = 0, e0n = 0, e1n = 0, svn = 0;
            if (qn < q1) {
                vn = __ldg(a.nodeq + qn);
                e0n = __ldg(a.rowq + qn);
                e1n = __ldg(a.rowq + qn + 1);
                svn = lane < e1n - e0n ? __ldg(a.colq + e0n + lane) : 0;
            }
            float wt;
            if (A == 2 && fast) {
                const float2 bb = __ldg(reinterpret_cast<const float2*>(a.base) + v);
                const uint64_t x0s = cbase + (uint64_t)(uint32_t)v * (2u * SPLITMIX_GOLDEN);
                const float x0 = perturb_x(bb.x, x0s, a.sigma), x1 = perturb_x(bb.y, x0s + SPLITMIX_GOLDEN, a.sigma);
                wt = x1 < x0 ? x1 : x0;
                nproc++;
                const uint32_t ab = f2u(fabsf(__fsub_rn(x1, x0)));
                hdf = ab > hdf ? ab : hdf;
                const uint32_t uw = f2u(wt);
                const uint64_t term = (uint64_t)((uw & 0x7fffffu) | 0x800000u) << ((uw >> 23) - emin);
                acc[0] += x0 == wt ? term : 0ull;
                acc[1] += x1 == wt ? term : 0ull;
            } else {
            float x[A];
            uint32_t en;
            int k;
            r2_durs<A>(a, r, v, x, en, k, wt, bad);
            if (live) {
#pragma unroll
                for (int b = 0; b < A; b++) {
                    if (!((en >> b) & 1u)) continue;
                    cnt[b]++;
                    if (x[b] == wt) {
                        uint64_t l, h;
                        fixed64(x[b], l, h);
                        add128(blo[b], bhi[b], l, h);
                    }
                    if (k >= 2) {
                        float ref = __uint_as_float(0x7f800000u);
#pragma unroll
                        for (int p = 0; p < A; p++)
                            if (p != b && ((en >> p) & 1u)) ref = x[p] < ref ? x[p] : ref;
                        uint32_t ab = f2u(fabsf(__fsub_rn(ref, x[b])));
                        hd[b] = ab > hd[b] ? ab : hd[b];
                    }
                }
            }
            if (!k) wt = 0.0f;
            }
            // successors: 32 positions per coalesced load, broadcast by shuffles, gathers K1_PF at a time
            float m = 0.0f;
            for (int32_t eb = e0; eb < e1; eb += 32) {
                const int32_t cb = min(32, e1 - eb);
                const int32_t s32 = eb == e0 ? sv : (lane < cb ? __ldg(a.colq + eb + lane) : 0);
                int32_t j = 0;
                for (; j + K1_PF <= cb; j += K1_PF) {
                    float t8[K1_PF];
                    if (flow) {
#pragma unroll
                        for (int u = 0; u < K1_PF; u++) {
                            const int32_t sp = __shfl_sync(0xffffffffu, s32, j + u);
                            while (rdy[sp] == 0) {}
                        }
                        __threadfence_block();
                    }
#pragma unroll
                    for (int u = 0; u < K1_PF; u++) {
                        const int32_t sp = __shfl_sync(0xffffffffu, s32, j + u);
                        t8[u] = bll[sp * 32];
                    }
#pragma unroll
                    for (int u = 0; u < K1_PF; u++) m = fmaxf(m, t8[u]);
                }
                for (; j < cb; j++) {
                    const int32_t sp = __shfl_sync(0xffffffffu, s32, j);
                    if (flow) {
                        while (rdy[sp] == 0) {}
                        __threadfence_block();
                    }
                    m = fmaxf(m, bll[sp * 32]);
                }
            }
            const float bb = __fadd_rn(wt, m);
            bl32[(int64_t)q * 32 + lane] = bb;
            cpm = fmaxf(cpm, bb);
            if (flow) {   // publish: every lane's store, then the ready byte
                __syncwarp();
                if (lane == 0) {
                    __threadfence_block();
                    rdy[q] = 1;
                }
            }
            q = qn;
            v = vn;
            e0 = e0n;
            e1 = e1n;
            sv = svn;
        }
        if (cs == 1) __syncthreads();
        else cluster.sync();
    }
    // ---- per-replica reductions across the 32 warps (column = lane = replica) ----
    uint32_t* red = reinterpret_cast<uint32_t*>(r2_smem);                 // [32][33]
    unsigned long long* red64 = reinterpret_cast<unsigned long long*>(r2_smem + 32 * 33 * 4 + 64);  // [32][33]
    auto colmax = [&](uint32_t val) -> uint32_t {
        red[w0 * 33 + lane] = val;
        __syncthreads();
        uint32_t m = 0;
        if (w0 == 0)
            for (int i = 0; i < 32; i++) m = max(m, red[i * 33 + lane]);
        __syncthreads();
        return m;
    };
    auto colsum = [&](uint32_t val) -> uint32_t {
        red[w0 * 33 + lane] = val;
        __syncthreads();
        uint32_t m = 0;
        if (w0 == 0)
            for (int i = 0; i < 32; i++) m += red[i * 33 + lane];
        __syncthreads();
        return m;
    };
    if (A == 2 && fast) {
        const uint32_t sh = emin - 86u;   // units 2^(emin-150) -> 2^-64 (emin >= 86 in the domain)
#pragma unroll
        for (int q = 0; q < A; q++) {
            if (q >= 2) break;
            cnt[q] = (int32_t)nproc;
            hd[q] = hdf;
            if (sh < 64u) {
                blo[q] = acc[q] << sh;
                bhi[q] = sh == 0u ? 0ull : (acc[q] >> (64u - sh));
            } else {
                blo[q] = 0ull;
                bhi[q] = acc[q] << (sh - 64u);
            }
        }
    }
    const uint32_t cpb = colmax(f2u(cpm));
    uint32_t hdb[A];
    int32_t cntb[A];
#pragma unroll
    for (int q = 0; q < A; q++) {
        hdb[q] = colmax(hd[q]);
        cntb[q] = (int32_t)colsum((uint32_t)cnt[q]);
    }
    // exact 128-bit column sums: lo words (counting carries), then hi words; CTAs of a
    // cluster merge their partial statistics with atomics (zeroed by the host)
#pragma unroll
    for (int q = 0; q < A; q++) {
        red64[w0 * 33 + lane] = blo[q];
        __syncthreads();
        uint64_t lo = 0, carry = 0;
        if (w0 == 0)
            for (int i = 0; i < 32; i++) {
                const uint64_t s2 = lo + red64[i * 33 + lane];
                carry += (s2 < lo) ? 1ull : 0ull;
                lo = s2;
            }
        __syncthreads();
        red64[w0 * 33 + lane] = bhi[q];
        __syncthreads();
        if (w0 == 0) {
            uint64_t hi = carry;
            for (int i = 0; i < 32; i++) hi += red64[i * 33 + lane];
            if (live) atomic_add128(a.brw + (rl * A + q) * 2, lo, hi);
        }
        __syncthreads();
    }
    if (w0 == 0 && live) {
        atomicMax(reinterpret_cast<uint32_t*>(a.cp) + rl, cpb);
#pragma unroll
        for (int q = 0; q < A; q++) {
            atomicMax(&a.hd[rl * A + q], hdb[q]);
            atomicAdd(&a.counts[rl * A + q], cntb[q]);
        }
    }
    // only live lanes report domain errors (a lane past R stands for no replica)
    if (__any_sync(0xffffffffu, live && bad) && lane == 0) atomicOr(a.err, ERR_DOMAIN_BIT);
    // ---- transpose bl32 [q][32] -> blT [r][t] (two archs: K2 reads bl32 directly, and
    //      only for equal-gain runs) ----
    if (A == 2) return;
    float* tile = reinterpret_cast<float*>(r2_smem) + w0 * 32 * 33;
    const int32_t nchunks = (a.n + 31) / 32;
    for (int32_t c = w; c < nchunks; c += WG) {
        const int32_t t0 = c * 32;
        for (int i = 0; i < 32; i++) {
            const int32_t t = t0 + i;
            float v = 0.0f;
            if (t < a.n) v = bl32[(int64_t)__ldg(a.qof + t) * 32 + lane];
            tile[i * 33 + lane] = v;
        }
        __syncwarp();
        for (int j = 0; j < 32; j++) {
            const int64_t rj = g * 32 + j;
            if (rj < a.R && t0 + lane < a.n) a.blT[rj * a.n + t0 + lane] = tile[lane * 33 + j];
        }
        __syncwarp();
    }
}


// ---------------------------------------------------------------------------------------
// K2: per-replica sorts in shared memory
//
// Queue a of replica r = entries t sorted by the composite key
//     key_a(t) = (gainc_a(t) << 32) | critc(t),   ties by t,
// gainc = 0x3F800000 - bits(gain) (0x40000000 = not enabled: after every real
// key), critc = 0x3F800000 - bits(bl/CP) -- i.e. (gain desc, crit desc, id asc).
// (key, t) is unique, so no step needs to be stable except where noted.
//
// Sorter: a key range [lo, hi] is histogrammed into <= 16384 equal-width bins
// (one read of gainc; critc only where the bin depends on it).  Consecutive
// bins are packed into rounds of <= R3_CAP entries; a round re-reads the keys,
// places each member at (bin start + atomic cursor) in shared memory and then
// orders every bin: insertion sort (<= 32 entries) or a block-wide rank sort
// (<= 1024).  Bins with more entries become finer ranges (deferred), or, when
// a bin holds a single key value, are streamed in id order (stable).
// ---------------------------------------------------------------------------------------
constexpr int R3_NC = 4096;      // coarse bins per range
constexpr int R3_NF = 16384;     // fine bins per range (sub-bins of the coarse bins)
constexpr int R3_CAP = 14400;    // entries per round with 64-bit keys (shared memory)
constexpr int R3_RB = R3_CAP * 10;   // round buffer bytes
template <class KT>
__host__ __device__ constexpr int r3_cap() { return R3_RB / (int)(sizeof(KT) + 2); }   // 14400 (u64 keys) / 24000 (u32)
constexpr int R3_TINY = 16;      // fine bins up to this size: thread insertion sort
constexpr int R3_MID = 256;      // up to this size: warp rank sort; larger: finer range / stream
constexpr int R3_MAXS = 192;     // range stack entries (6 words each)
constexpr int R3_MAXG = 192;     // group records per range (3 words each)

struct R3Smem {
    uint32_t* starts;   // [R3_NF + 64]  fine counts -> exclusive prefixes
    uint16_t* coff;     // [R3_NC + 64]  first fine bin of each coarse bin
    uint8_t* clog;      // [R3_NC + 64]  log2(#fine bins) of each coarse bin
    unsigned char* bkraw;  // R3_RB bytes: keys (u64 x R3_CAP or u32 x R3_CAP32) then ids (u16)
    uint32_t* sc;       // [96]
    uint32_t* misc;     // [R3_MAXS*6 + R3_MAXG*3 + 8 + 512]
};

constexpr size_t r3_smem_bytes() {
    return (size_t)(R3_NF + 64) * 4 + (size_t)(R3_NC + 64) * 2 + (size_t)(R3_NC + 64) + (size_t)R3_RB + 96 * 4 + (size_t)(R3_MAXS * 6 + R3_MAXG * 3 + 8 + 512) * 4;
}

// exclusive block scan of one value per thread (1024 threads)
MP_INLINE uint32_t r3_scan(uint32_t x, uint32_t* sc, uint32_t& total) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t incl = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) sc[w] = incl;
    __syncthreads();
    if (w == 0) {
        uint32_t v = sc[lane];
        uint32_t iv = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(0xffffffffu, iv, o);
            if (lane >= o) iv += y;
        }
        sc[lane] = iv - v;
        if (lane == 31) sc[32] = iv;
    }
    __syncthreads();
    const uint32_t r = sc[w] + incl - x;
    total = sc[32];
    __syncthreads();
    return r;
}

struct R3Keys {
    const uint32_t* hi;   // gainc_a[n]
    const uint32_t* lo;   // critc[n]
    uint16_t* fb;         // [n] fine bin of each entry in the current range (scratch)
    MP_INLINE uint64_t full(int32_t t) const {
        return ((uint64_t)__ldcg(hi + t) << 32) | (lo ? __ldcg(lo + t) : 0u);   // lo == null: 32-bit keys
    }
};

struct R3Out {
    int32_t* q;       // queue destination or null
    int32_t count;    // enabled entries (positions >= count are not written)
    uint32_t* head;   // shared
    MP_INLINE void put(int32_t pos, uint32_t t, uint64_t) const {
        if (pos == 0) *head = t;
        if (q && pos < count) __stcs(q + pos, (int32_t)t);   // streaming: keep L2 for the scratch
    }
};

struct R3PosOut {      // sorted order into scratch: P[pos] = t, Dk[pos] = high key word
    uint16_t* P;
    uint32_t* Dk;
    MP_INLINE void put(int32_t pos, uint32_t t, uint64_t key) const {
        P[pos] = (uint16_t)t;
        Dk[pos] = (uint32_t)(key >> 32);
    }
};

// Range geometry: coarse bin of key k = (k >> cs) - clb (< ncb); fine bin =
// coff[c] + ((k >> (cs - clog[c])) & ((1 << clog[c]) - 1)).
struct R3Geo {
    uint64_t lo, hi, clb;
    uint32_t cs, ncb;
};

// Is t inside [lo, hi]?  Returns its coarse bin and (if want_key) its full key; reads
// critc only when the bin or the bounds depend on it (need_bits = lowest key bit used).
MP_INLINE bool r3_locate(const R3Keys& K, int32_t t, const R3Geo& g, uint32_t need_bits, uint32_t& cb,
                         uint64_t& key) {
    const uint32_t h = __ldcg(K.hi + t);
    const uint32_t lh = (uint32_t)(g.lo >> 32), hh = (uint32_t)(g.hi >> 32);
    if (h < lh || h > hh) return false;
    if (need_bits >= 32 && h != lh && h != hh) {
        key = (uint64_t)h << 32;
        cb = (uint32_t)((key >> g.cs) - g.clb);
        return true;
    }
    key = ((uint64_t)h << 32) | (K.lo ? __ldcg(K.lo + t) : 0u);
    if (key < g.lo || key > g.hi) return false;
    cb = (uint32_t)((key >> g.cs) - g.clb);
    return true;
}

// as r3_locate, with gainc already loaded; coarse bin only
MP_INLINE bool r3_locate_h(const R3Keys& K, int32_t t, uint32_t h, const R3Geo& g, uint32_t need_bits, uint32_t& cb) {
    const uint32_t lh = (uint32_t)(g.lo >> 32), hh = (uint32_t)(g.hi >> 32);
    if (h < lh || h > hh) return false;
    if (need_bits >= 32 && h != lh && h != hh) {
        cb = (uint32_t)((((uint64_t)h << 32) >> g.cs) - g.clb);
        return true;
    }
    const uint64_t key = ((uint64_t)h << 32) | (K.lo ? __ldcg(K.lo + t) : 0u);
    if (key < g.lo || key > g.hi) return false;
    cb = (uint32_t)((key >> g.cs) - g.clb);
    return true;
}
MP_INLINE bool r3_locate_hk(const R3Keys& K, int32_t t, uint32_t h, const R3Geo& g, uint32_t need_bits,
                            uint32_t& cb, uint64_t& key) {
    const uint32_t lh = (uint32_t)(g.lo >> 32), hh = (uint32_t)(g.hi >> 32);
    if (h < lh || h > hh) return false;
    if (need_bits >= 32 && h != lh && h != hh) {
        key = (uint64_t)h << 32;
        cb = (uint32_t)((key >> g.cs) - g.clb);
        return true;
    }
    key = ((uint64_t)h << 32) | (K.lo ? __ldcg(K.lo + t) : 0u);
    if (key < g.lo || key > g.hi) return false;
    cb = (uint32_t)((key >> g.cs) - g.clb);
    return true;
}

// Fine bin of a key in coarse bin cb.  64-bit keys: 2^clog[cb] power-of-two sub-bins (a
// fine bin depends only on key bits >= cs - clog, so critc is read only where needed).
// 32-bit keys: clog[cb] = m proportional sub-bins, sub = (offset * m) >> cs (monotone,
// < m), which sizes the bins to the coarse counts without power-of-two rounding.
template <class KT>
MP_INLINE uint32_t r3_fine(const R3Smem& S, const R3Geo& g, uint32_t cb, uint64_t key) {
    const uint32_t l = S.clog[cb];
    if constexpr (sizeof(KT) == 4) {
        if (g.cs >= 32) {   // the key is k << 32: all in 32 bits (offset < 2^(cs-32) <= 2^21, m < 2^8)
            const uint32_t c32 = g.cs - 32u;
            const uint32_t off = (uint32_t)(key >> 32) - (((uint32_t)g.clb + cb) << c32);
            return (uint32_t)S.coff[cb] + ((off * l) >> c32);
        }
        const uint64_t off = key - ((g.clb + cb) << g.cs);
        return (uint32_t)S.coff[cb] + (uint32_t)((off * l) >> g.cs);
    }
    const uint32_t sub = l ? (uint32_t)((key >> (g.cs - l)) & ((1ull << l) - 1ull)) : 0u;
    return (uint32_t)S.coff[cb] + sub;
}

// fine bin of a 32-bit key k (64-bit key k << 32) in range geometry g, coarse bin included
MP_INLINE uint32_t r3_bin32(const R3Smem& S, const R3Geo& g, uint32_t k) {
    if (g.cs >= 32) {
        const uint32_t c32 = g.cs - 32u;
        const uint32_t cb = (k >> c32) - (uint32_t)g.clb;
        const uint32_t off = k - ((k >> c32) << c32);
        return (uint32_t)S.coff[cb] + ((off * (uint32_t)S.clog[cb]) >> c32);
    }
    const uint64_t key = (uint64_t)k << 32;
    return r3_fine<uint32_t>(S, g, (uint32_t)((key >> g.cs) - g.clb), key);
}


// stable stream of all entries with key == k (id order) to out[ob ...]
template <class Out>
__device__ void r3_stream_equal(const R3Keys& K, const Out& out, int32_t n, uint64_t k, int32_t ob, uint32_t* sc) {
    uint32_t run = 0;
    for (int32_t b0 = 0; b0 < n; b0 += R2_THREADS) {
        const int32_t t = b0 + threadIdx.x;
        const bool sel = t < n && K.full(t) == k;
        uint32_t tot;
        const uint32_t pos = r3_scan(sel ? 1u : 0u, sc, tot);
        if (sel) out.put(ob + (int32_t)(run + pos), (uint32_t)t, k);
        run += tot;
    }
}

template <class KT>
MP_INLINE bool r3_less(KT ka, uint16_t va, KT kb, uint16_t vb) {
    return ka < kb || (ka == kb && va < vb);
}
template <class KT>
MP_INLINE KT r3_store_key(uint64_t k) { return sizeof(KT) == 8 ? (KT)k : (KT)(k >> 32); }

// One round: fine bins [b0, b1) (each <= R3_MID entries, total cnt <= R3_CAP).
// 1. members (fb[t] in [b0, b1)) are placed at (bin start + atomic cursor) in
//    shared memory -- fb is read 16 entries (two 16-byte loads) per thread;
// 2. every placed entry ranks itself inside its bin (compares against the bin's
//    other entries) and writes straight to its final output position.
template <class KT, class Out>
__device__ void r3_round(const R3Keys& K, const Out& out, int32_t n, const R3Geo& g, uint32_t b0, uint32_t b1,
                         uint32_t base, uint32_t cnt, int32_t ob, R3Smem& S) {
    constexpr int CAPK = r3_cap<KT>();
    KT* bk = reinterpret_cast<KT*>(S.bkraw);
    uint16_t* bv = reinterpret_cast<uint16_t*>(S.bkraw + (size_t)CAPK * sizeof(KT));
    const int32_t n16 = n & ~15;
    for (int32_t c0 = threadIdx.x * 16; c0 < n16; c0 += 16 * R2_THREADS) {
        const uint4 w0 = __ldcg(reinterpret_cast<const uint4*>(K.fb + c0));
        const uint4 w1 = __ldcg(reinterpret_cast<const uint4*>(K.fb + c0 + 8));
        const uint32_t wv[8] = {w0.x, w0.y, w0.z, w0.w, w1.x, w1.y, w1.z, w1.w};
        if constexpr (sizeof(KT) == 4) {
            // 32-bit keys: read them with the scan (sequential 16-byte loads) instead of gathering
            uint32_t hv[16];
#pragma unroll
            for (int u4 = 0; u4 < 4; u4++) {
                const uint4 h = __ldcg(reinterpret_cast<const uint4*>(K.hi + c0 + 4 * u4));
                hv[4 * u4] = h.x; hv[4 * u4 + 1] = h.y; hv[4 * u4 + 2] = h.z; hv[4 * u4 + 3] = h.w;
            }
#pragma unroll
            for (int u = 0; u < 16; u++) {
                const uint32_t f = (wv[u >> 1] >> ((u & 1) * 16)) & 0xFFFFu;
                if (f < b0 || f >= b1) continue;
                const uint32_t slot = atomicAdd(&S.starts[f], 1u) - base;
                bk[slot] = (KT)hv[u];
                bv[slot] = (uint16_t)(c0 + u);
            }
        } else {
#pragma unroll
            for (int u = 0; u < 16; u++) {
                const uint32_t f = (wv[u >> 1] >> ((u & 1) * 16)) & 0xFFFFu;
                if (f < b0 || f >= b1) continue;
                const int32_t t = c0 + u;
                const uint32_t slot = atomicAdd(&S.starts[f], 1u) - base;
                bk[slot] = r3_store_key<KT>(K.full(t));
                bv[slot] = (uint16_t)t;
            }
        }
    }
    for (int32_t t = n16 + threadIdx.x; t < n; t += R2_THREADS) {
        const uint32_t f = __ldcg(K.fb + t);
        if (f < b0 || f >= b1) continue;
        const uint32_t slot = atomicAdd(&S.starts[f], 1u) - base;
        bk[slot] = r3_store_key<KT>(K.full(t));
        bv[slot] = (uint16_t)t;
    }
    __syncthreads();
    K2_PHASE(13);
    for (uint32_t j = threadIdx.x; j < cnt; j += R2_THREADS) {
        const KT k = bk[j];
        const uint16_t v = bv[j];
        const uint64_t k64 = sizeof(KT) == 8 ? (uint64_t)k : ((uint64_t)k << 32);
        uint32_t f;
        if constexpr (sizeof(KT) == 4) f = r3_bin32(S, g, (uint32_t)k);
        else f = r3_fine<KT>(S, g, (uint32_t)((k64 >> g.cs) - g.clb), k64);
        const uint32_t s0 = (f == b0 ? base : S.starts[f - 1]) - base;
        const uint32_t s1 = S.starts[f] - base;
        uint32_t rank = 0;
        uint32_t i = s0;
        for (; i + 4 <= s1; i += 4) {   // 4 independent compares per trip
#pragma unroll
            for (int u = 0; u < 4; u++) rank += r3_less<KT>(bk[i + u], bv[i + u], k, v) ? 1u : 0u;
        }
        for (; i < s1; i++) rank += r3_less<KT>(bk[i], bv[i], k, v) ? 1u : 0u;
        out.put(ob + (int32_t)(s0 + rank), v, k64);
    }
    __syncthreads();
    K2_PHASE(14);
}

MP_INLINE uint32_t r3_clog2(uint32_t x) { return x <= 1 ? 0u : 32u - __clz(x - 1); }   // ceil(log2 x)

constexpr int R3_GEO_BYTES = 16384;   // coff (2 B) + clog (1 B) per coarse bin + fine-bin count

// coarse geometry of a key range: <= R3_NC bins of width 2^cs
MP_INLINE R3Geo r3_geo(uint64_t lo, uint64_t hi) {
    R3Geo g;
    g.lo = lo;
    g.hi = hi;
    const uint64_t span = hi - lo;
    const uint32_t bits = 64u - (uint32_t)__clzll((long long)span);
    constexpr uint32_t LOGNC = 31u - __builtin_clz((unsigned)R3_NC);   // NC is a power of two
    g.cs = bits > LOGNC ? bits - LOGNC : 0;
    g.clb = lo >> g.cs;
    g.ncb = (uint32_t)((hi >> g.cs) - g.clb + 1);
    while (g.ncb > (uint32_t)R3_NC) {
        g.cs++;
        g.clb = lo >> g.cs;
        g.ncb = (uint32_t)((hi >> g.cs) - g.clb + 1);
    }
    return g;
}

// pre_nfb != 0: the top range [kmin, kmax] is pre-binned by the caller -- coff/clog hold its
// sub-bin geometry (pre_nfb fine bins), starts[] its fine counts and K.fb every entry's fine
// bin -- so passes 1-2 are skipped for it.  snap != null: the top range's sub-bin geometry is
// saved there (coff, clog, fine-bin count) for a later pre-binned call on the same range.
template <class KT, class Out>
__device__ void r3_sort(const R3Keys& K, const Out& out, int32_t n, uint64_t kmin, uint64_t kmax, R3Smem& S,
                        uint32_t pre_nfb = 0, unsigned char* snap = nullptr) {
    constexpr int CAPK = r3_cap<KT>();
    if (n <= 0) return;
    uint32_t* stk = S.misc;                        // [R3_MAXS][6]
    uint32_t* grp = S.misc + R3_MAXS * 6;          // [R3_MAXG][3]: start fine bin, start prefix, kind
    uint32_t* nstk = grp + R3_MAXG * 3;
    auto push = [&](uint64_t lo, uint64_t hi, uint32_t ob, uint32_t cnt) {  // thread 0 only
        uint32_t k = *nstk;
        if (k >= (uint32_t)R3_MAXS) { __trap(); }
        stk[k * 6] = (uint32_t)lo;
        stk[k * 6 + 1] = (uint32_t)(lo >> 32);
        stk[k * 6 + 2] = (uint32_t)hi;
        stk[k * 6 + 3] = (uint32_t)(hi >> 32);
        stk[k * 6 + 4] = ob;
        stk[k * 6 + 5] = cnt;
        *nstk = k + 1;
    };
    if (threadIdx.x == 0) {
        *nstk = 0;
        push(kmin, kmax, 0, (uint32_t)n);
    }
    __syncthreads();
    bool first = true;
    while (true) {
        const uint32_t ns = *nstk;
        if (ns == 0) break;
        const uint32_t* top = stk + (ns - 1) * 6;
        R3Geo g;
        g.lo = (uint64_t)top[0] | ((uint64_t)top[1] << 32);
        g.hi = (uint64_t)top[2] | ((uint64_t)top[3] << 32);
        const int32_t ob = (int32_t)top[4];
        const uint32_t rcnt = top[5];
        __syncthreads();
        if (threadIdx.x == 0) *nstk = ns - 1;
        if (g.lo == g.hi) {
            r3_stream_equal(K, out, n, g.lo, ob, S.sc);
            __syncthreads();
            continue;
        }
        g = r3_geo(g.lo, g.hi);
        const bool toprange = first;   // the caller's range (not a deferred sub-range)
        const bool prebinned = toprange && pre_nfb != 0;
        first = false;
        uint32_t ftot = pre_nfb;
        if (!prebinned) {
        // ---- pass 1: coarse histogram (in starts[0..NC)) ----
        for (uint32_t b = threadIdx.x; b < (uint32_t)R3_NF + 64; b += R2_THREADS) S.starts[b] = 0;
        __syncthreads();
        for (int32_t c0 = threadIdx.x * 8; c0 < n; c0 += 8 * R2_THREADS) {
            uint32_t hv[8];
            if (c0 + 8 <= n) {
                const uint4 h0 = __ldcg(reinterpret_cast<const uint4*>(K.hi + c0));
                const uint4 h1 = __ldcg(reinterpret_cast<const uint4*>(K.hi + c0 + 4));
                hv[0] = h0.x; hv[1] = h0.y; hv[2] = h0.z; hv[3] = h0.w;
                hv[4] = h1.x; hv[5] = h1.y; hv[6] = h1.z; hv[7] = h1.w;
            } else {
#pragma unroll
                for (int u = 0; u < 8; u++) hv[u] = c0 + u < n ? __ldcg(K.hi + c0 + u) : 0xFFFFFFFFu;
            }
#pragma unroll
            for (int u = 0; u < 8; u++) {
                if (c0 + u >= n) continue;
                uint32_t cb;
                if (r3_locate_h(K, c0 + u, hv[u], g, g.cs, cb)) atomicAdd(&S.starts[cb], 1u);
            }
        }
        __syncthreads();
        K2_PHASE(2);
        // ---- sub-bins per coarse bin: 2^ceil(log2(c / T)) with T doubling until they fit ----
        constexpr int CPER = R3_NC / R2_THREADS;  // 4
        uint32_t cc[CPER];
#pragma unroll
        for (int j = 0; j < CPER; j++) cc[j] = S.starts[threadIdx.x * CPER + j];
        uint32_t T = 4;
        uint32_t lg[CPER], fex = 0;
        ftot = 0;
        if constexpr (sizeof(KT) == 4) {
            // proportional: m_c = ceil(c * (NF - nonempty) / in_range) sums to <= NF.  A geometry
            // cached for other replicas (snap) gives every coarse bin >= 1 sub-bin: their keys
            // may fall where this replica has none
            const bool all1 = toprange && snap;
            uint32_t ne = 0, tc = 0, NE = 0, TOT = 0;
#pragma unroll
            for (int j = 0; j < CPER; j++) {
                const uint32_t b = threadIdx.x * CPER + j;
                if (b < g.ncb) {
                    ne += (cc[j] > 0 || all1) ? 1u : 0u;
                    tc += cc[j];
                }
            }
            r3_scan(ne, S.sc, NE);
            r3_scan(tc, S.sc, TOT);
            const uint64_t Fn = (uint64_t)R3_NF - NE, Fd = TOT > 0 ? TOT : 1u;
            uint32_t sm = 0;
#pragma unroll
            for (int j = 0; j < CPER; j++) {
                const uint32_t b = threadIdx.x * CPER + j;
                uint32_t m = 0;
                if (b < g.ncb && (cc[j] > 0 || all1)) {
                    m = (uint32_t)min(((uint64_t)cc[j] * Fn + Fd - 1) / Fd, (uint64_t)255);
                    if (g.cs < 8) m = min(m, 1u << g.cs);
                    m = max(m, 1u);
                }
                lg[j] = m;
                sm += m;
            }
            fex = r3_scan(sm, S.sc, ftot);
        }
        while (sizeof(KT) == 8) {
            uint32_t s = 0;
#pragma unroll
            for (int j = 0; j < CPER; j++) {
                const uint32_t b = threadIdx.x * CPER + j;
                uint32_t l = 0;
                if (b < g.ncb && cc[j] > T) l = min(r3_clog2((cc[j] + T - 1) / T), g.cs);
                lg[j] = l;
                s += (b < g.ncb) ? (1u << l) : 0u;
            }
            fex = r3_scan(s, S.sc, ftot);
            if (ftot <= (uint32_t)R3_NF) break;
            T *= 2;
        }
        {
            uint32_t e = fex;
#pragma unroll
            for (int j = 0; j < CPER; j++) {
                const uint32_t b = threadIdx.x * CPER + j;
                S.coff[b] = (uint16_t)e;
                S.clog[b] = (uint8_t)lg[j];
                if (b < g.ncb) e += sizeof(KT) == 4 ? lg[j] : 1u << lg[j];
            }
        }
        __syncthreads();
        if (toprange && snap) {   // sub-bin geometry of the top range, for later pre-binned calls
            uint16_t* sc16 = reinterpret_cast<uint16_t*>(snap);
            for (uint32_t b = threadIdx.x; b < (uint32_t)R3_NC; b += R2_THREADS) {
                sc16[b] = S.coff[b];
                snap[2 * R3_NC + b] = S.clog[b];
            }
            if (threadIdx.x == 0) *reinterpret_cast<uint32_t*>(snap + 3 * R3_NC) = ftot;
        }
        // lowest key bit any fine bin depends on
        uint32_t maxl = 0;
#pragma unroll
        for (int j = 0; j < CPER; j++) maxl = max(maxl, lg[j]);
        maxl = __reduce_max_sync(0xffffffffu, maxl);
        if ((threadIdx.x & 31) == 0) S.sc[40 + (threadIdx.x >> 5)] = maxl;
        for (uint32_t b = threadIdx.x; b < (uint32_t)R3_NF + 64; b += R2_THREADS) S.starts[b] = 0;
        __syncthreads();
        uint32_t need = 0;
        for (int w = 0; w < R2_WARPS; w++) need = max(need, S.sc[40 + w]);
        need = sizeof(KT) == 4 ? 0u : g.cs - need;   // fine bins use key bits >= need
        K2_PHASE(3);
        // ---- pass 2: fine histogram ----
        for (int32_t c0 = threadIdx.x * 8; c0 < n; c0 += 8 * R2_THREADS) {
            uint32_t hv[8], fv[8];
            if (c0 + 8 <= n) {
                const uint4 h0 = __ldcg(reinterpret_cast<const uint4*>(K.hi + c0));
                const uint4 h1 = __ldcg(reinterpret_cast<const uint4*>(K.hi + c0 + 4));
                hv[0] = h0.x; hv[1] = h0.y; hv[2] = h0.z; hv[3] = h0.w;
                hv[4] = h1.x; hv[5] = h1.y; hv[6] = h1.z; hv[7] = h1.w;
            } else {
#pragma unroll
                for (int u = 0; u < 8; u++) hv[u] = c0 + u < n ? __ldcg(K.hi + c0 + u) : 0xFFFFFFFFu;
            }
#pragma unroll
            for (int u = 0; u < 8; u++) {
                fv[u] = 0xFFFFu;
                if (c0 + u >= n) continue;
                uint32_t cb;
                uint64_t key;
                if (r3_locate_hk(K, c0 + u, hv[u], g, need, cb, key)) {
                    fv[u] = r3_fine<KT>(S, g, cb, key);
                    atomicAdd(&S.starts[fv[u]], 1u);
                }
            }
            if (c0 + 8 <= n) {
                uint4 o;
                o.x = fv[0] | (fv[1] << 16); o.y = fv[2] | (fv[3] << 16);
                o.z = fv[4] | (fv[5] << 16); o.w = fv[6] | (fv[7] << 16);
                *reinterpret_cast<uint4*>(K.fb + c0) = o;
            } else {
#pragma unroll
                for (int u = 0; u < 8; u++)
                    if (c0 + u < n) K.fb[c0 + u] = (uint16_t)fv[u];
            }
        }
        __syncthreads();
        K2_PHASE(4);
        }
        const uint32_t nfb = ftot;
        // ---- prefixes over fine bins (12 per thread) + group boundaries ----
        constexpr int PER = R3_NF / R2_THREADS;  // 12
        const uint32_t H = CAPK - R3_MID;        // a multi-bin group never exceeds H + MID = CAP
        uint32_t cnts[PER], sum = 0;
#pragma unroll
        for (int j = 0; j < PER; j++) {
            cnts[j] = S.starts[threadIdx.x * PER + j];
            sum += cnts[j];
        }
        const uint32_t prev_c = threadIdx.x == 0 ? 0u : S.starts[threadIdx.x * PER - 1];
        uint32_t tot;
        const uint32_t ex = r3_scan(sum, S.sc, tot);
        uint32_t flags = 0;
        {
            uint32_t e = ex, pc = prev_c, pe = ex - prev_c;
#pragma unroll
            for (int j = 0; j < PER; j++) {
                const uint32_t b = threadIdx.x * PER + j;
                const bool big = cnts[j] > (uint32_t)R3_MID;
                const bool pbig = pc > (uint32_t)R3_MID;
                if (b < nfb && (b == 0 || big || pbig || (e / H) != (pe / H))) flags |= 1u << j;
                S.starts[b] = e;
                pe = e;
                pc = cnts[j];
                e += cnts[j];
            }
        }
        if (threadIdx.x == 0) S.starts[R3_NF] = tot;
        (void)rcnt;
        uint32_t ng;
        const uint32_t gp0 = r3_scan((uint32_t)__popc(flags), S.sc, ng);
        if (ng > (uint32_t)R3_MAXG) __trap();
        {
            uint32_t gp = gp0;
#pragma unroll
            for (int j = 0; j < PER; j++)
                if ((flags >> j) & 1u) {
                    const uint32_t b = threadIdx.x * PER + j;
                    grp[gp * 3] = b;
                    grp[gp * 3 + 1] = S.starts[b];
                    grp[gp * 3 + 2] = cnts[j] > (uint32_t)R3_MID ? 1u : 0u;
                    gp++;
                }
        }
        __syncthreads();
        K2_PHASE(5);
        for (uint32_t gi = 0; gi < ng; gi++) {
            const uint32_t b0 = grp[gi * 3], e0 = grp[gi * 3 + 1], kind = grp[gi * 3 + 2];
            const uint32_t b1 = gi + 1 < ng ? grp[(gi + 1) * 3] : nfb;
            const uint32_t e1 = gi + 1 < ng ? grp[(gi + 1) * 3 + 1] : tot;
            const uint32_t cnt = e1 - e0;
            if (cnt == 0) continue;
            if (kind == 0) {
                r3_round<KT>(K, out, n, g, b0, b1, e0, cnt, ob + (int32_t)e0, S);
            } else {
                if (threadIdx.x == 0) {
                    // key range of fine bin b0: its coarse bin c (last with coff[c] <= b0), sub-bin b0-coff[c]
                    uint32_t lo_c = 0, hi_c = g.ncb - 1;
                    while (lo_c < hi_c) {
                        const uint32_t mid = (lo_c + hi_c + 1) >> 1;
                        if ((uint32_t)S.coff[mid] <= b0) lo_c = mid;
                        else hi_c = mid - 1;
                    }
                    const uint32_t l = S.clog[lo_c];
                    uint64_t blo, bhi;
                    bool one = false;
                    if constexpr (sizeof(KT) == 4) {
                        // sub-bin s holds offsets [ceil(s W / m), ceil((s+1) W / m) - 1], W = 2^cs
                        const uint64_t cbase = (g.clb + lo_c) << g.cs, W = 1ull << g.cs, sb = b0 - S.coff[lo_c];
                        blo = cbase + (sb * W + l - 1) / l;
                        bhi = cbase + ((sb + 1) * W + l - 1) / l - 1;
                    } else {
                        const uint32_t fs = g.cs - l;
                        blo = ((g.clb + lo_c) << g.cs) + ((uint64_t)(b0 - S.coff[lo_c]) << fs);
                        bhi = blo + ((1ull << fs) - 1ull);
                        one = fs == 0;
                    }
                    if (blo < g.lo) blo = g.lo;
                    if (bhi > g.hi || bhi < blo) bhi = g.hi;
                    if (one) bhi = blo;
                    push(blo, bhi, (uint32_t)(ob + (int32_t)e0), cnt);
                }
                __syncthreads();
            }
        }
        __syncthreads();
    }
    __syncthreads();
}

// gain keys (0x3F800000 - bits(gain)) of both archs from the orderable difference D (two archs):
// D = 0: arch-1-only (gain_1 = 1), D = ~0: arch-0-only (gain_0 = 1), else d = delta_1 - delta_0.
MP_INLINE void r2_gains_from_D(uint32_t D, float hd, uint32_t& G0, uint32_t& G1) {
    if (D == 0u) {
        G0 = 0x40000000u;
        G1 = 0u;
        return;
    }
    if (D == 0xFFFFFFFFu) {
        G0 = 0u;
        G1 = 0x40000000u;
        return;
    }
    const uint32_t db = (D & 0x80000000u) ? (D & 0x7FFFFFFFu) : ~D;
    const float d = u2f(db);
    float g0, g1;
    if (hd == 0.0f) {
        g0 = g1 = 0.5f;
    } else {
        const float den = __fadd_rn(hd, hd);
        g0 = __fdiv_rn(__fadd_rn(d, hd), den);
        g1 = __fdiv_rn(__fadd_rn(__fsub_rn(0.0f, d), hd), den);   // d(t, 1) = delta_0 - delta_1 = -d
    }
    G0 = ONE_BITS - f2u(g0);
    G1 = ONE_BITS - f2u(g1);
}

// Do the sorted neighbours Da, Db have equal gain keys on arch 0 (s0) / arch 1 (s1)?
// Same as comparing r2_gains_from_D's keys, without most divisions: for two-arch
// tasks gain = RN(x / den) with x = RN(+-d + hd) in [0, den] (hd >= |d|), so
// the quotients lie in [0, 1], where every rounding interval is at most 2^-24
// wide; numerators further apart than den * 2^-24 (exact in binary64: both are
// floats) therefore give different gains, equal numerators equal gains, and
// only the remaining near-ties are divided.
MP_INLINE void r2_same_gains(uint32_t Da, uint32_t Db, float hd, bool& s0, bool& s1) {
    if (Da == Db) { s0 = s1 = true; return; }
    if (Da == 0u || Da == 0xFFFFFFFFu || Db == 0u || Db == 0xFFFFFFFFu || hd == 0.0f) {
        uint32_t A0, A1, B0, B1;
        r2_gains_from_D(Da, hd, A0, A1);
        r2_gains_from_D(Db, hd, B0, B1);
        s0 = A0 == B0;
        s1 = A1 == B1;
        return;
    }
    const float da = u2f((Da & 0x80000000u) ? (Da & 0x7FFFFFFFu) : ~Da);
    const float db = u2f((Db & 0x80000000u) ? (Db & 0x7FFFFFFFu) : ~Db);
    // screen in float: lim = den * 2^-24 is exact (den >= 2^-40 for a nonzero hd in the
    // domain), and RN is monotone, so a true |xb - xa| <= lim never rounds above lim;
    // a rounded difference above lim is a true difference above lim (different gains)
    const float den = __fadd_rn(hd, hd);
    const float lim = __fmul_rn(den, 0x1p-24f);
    const float xa = __fadd_rn(da, hd), xb = __fadd_rn(db, hd);
    s0 = xa == xb || (fabsf(__fsub_rn(xb, xa)) <= lim && __fdiv_rn(xa, den) == __fdiv_rn(xb, den));
    const float ya = __fadd_rn(__fsub_rn(0.0f, da), hd), yb = __fadd_rn(__fsub_rn(0.0f, db), hd);
    s1 = ya == yb || (fabsf(__fsub_rn(yb, ya)) <= lim && __fdiv_rn(ya, den) == __fdiv_rn(yb, den));
}


// RN(xa / den) == RN(xb / den) for numerators in [0, den] (see r2_same_gains)
MP_INLINE bool r2_same_q(float xa, float xb, float den, float lim) {
    return xa == xb || (fabsf(__fsub_rn(xb, xa)) <= lim && __fdiv_rn(xa, den) == __fdiv_rn(xb, den));
}

template <int A>
__global__ void __launch_bounds__(R2_THREADS, 1) k_rep2_sort(Rep2Args a) {
    extern __shared__ __align__(16) unsigned char r3s[];
    R3Smem S;
    S.starts = reinterpret_cast<uint32_t*>(r3s);
    S.bkraw = r3s + (size_t)(R3_NF + 64) * 4;
    S.coff = reinterpret_cast<uint16_t*>(S.bkraw + R3_RB);
    S.clog = reinterpret_cast<uint8_t*>(S.coff + R3_NC + 64);
    S.sc = reinterpret_cast<uint32_t*>(S.clog + R3_NC + 64);
    S.misc = S.sc + 96;
    __shared__ uint32_t s_tick, s_head, s_flag, s_h0, s_h1, s_mtot;
    __shared__ unsigned long long s_min[A + 1], s_max[A + 1];
    const int64_t npad = ((int64_t)a.n + 15) & ~15ll;   // 16-entry aligned scratch rows
    uint32_t* critc = a.s_cold + (int64_t)blockIdx.x * npad * (A + 1);
    uint32_t* gainc = critc + npad;   // [A][npad]
    uint32_t* dkey = a.s_key + (int64_t)blockIdx.x * npad * 2;
    uint16_t* fbuf = a.s_pi + (int64_t)blockIdx.x * npad * 2;
    uint16_t* ppos = fbuf + npad;
    uint32_t* dsorted = dkey + npad;   // (A == 2) D in sorted order (gains are recomputed from it)
    bool bad = false;
    // Two archs: a key range that holds every replica's D, from the perturbation's extremes
    // (u = 0 and u = 1 - 2^-24; every RN op on the way is monotone, so each perturbed
    // duration, and then d = delta_1 - delta_0, lies between the values at the extremes).
    // With one fixed range every replica has the same coarse bins, and the sub-bin geometry
    // built for this CTA's first replica is reused: later replicas bin their keys while
    // hashing (P0) and skip the sorter's two histogram passes.
    __shared__ uint32_t s_flo, s_fhi, s_geo_ok, s_geo_nfb, s_out, s_fast;
    unsigned char* geo = a.s_geo ? a.s_geo + (int64_t)blockIdx.x * R3_GEO_BYTES : nullptr;
    if constexpr (A == 2) {
        if (threadIdx.x == 0) {
            s_flo = ~0u; s_fhi = 0u; s_geo_ok = 0u; s_geo_nfb = 0u;
            s_fast = (a.emask == 3u && (reinterpret_cast<uintptr_t>(a.base) & 15u) == 0u) ? 1u : 0u;
        }
        __syncthreads();
        uint32_t lo = ~0u, hi = 0u;
        bool dom = true;   // every extreme a nonzero finite domain value (K1's fast-path rule)
        for (int32_t t = threadIdx.x; t < a.n; t += R2_THREADS) {
            float xl[2], xh[2];
            uint32_t enl = 0, enh = 0;
            bool dummy = false;
#pragma unroll
            for (int b = 0; b < 2; b++) {
                const float bv = __ldg(a.base + 2 * (int64_t)t + b);
                const float e0 = canon_dur(perturb_u(bv, a.sigma, 0u), dummy);
                const float e1 = canon_dur(perturb_u(bv, a.sigma, 0xFFFFFFu), dummy);
                xl[b] = e0 < e1 ? e0 : e1;
                xh[b] = e0 < e1 ? e1 : e0;
                const uint32_t ul = f2u(xl[b]), uh = f2u(xh[b]);
                if (!(ul >= 0x2B000000u && ul < 0x49800000u && uh >= 0x2B000000u && uh < 0x49800000u)) dom = false;
                if (((a.emask >> b) & 1u) && !is_inf(xl[b])) enl |= 1u << b;
                if (((a.emask >> b) & 1u) && !is_inf(xh[b])) enh |= 1u << b;
            }
            if (enl != enh || xl[0] != xl[0] || xl[1] != xl[1] || xh[0] != xh[0] || xh[1] != xh[1]) {
                lo = 0u;            // cannot bound this task: the whole key space
                hi = 0xFFFFFFFFu;
            } else if (enl == 3u) {
                const uint32_t dl = f2u(__fsub_rn(xl[1], xh[0])), dh = f2u(__fsub_rn(xh[1], xl[0]));
                lo = min(lo, (dl >> 31) ? ~dl : (dl | 0x80000000u));
                hi = max(hi, (dh >> 31) ? ~dh : (dh | 0x80000000u));
            } else if (enl != 0u) {
                const uint32_t D = enl == 1u ? 0xFFFFFFFFu : 0u;
                lo = min(lo, D);
                hi = max(hi, D);
            }
        }
        lo = __reduce_min_sync(0xffffffffu, lo);
        hi = __reduce_max_sync(0xffffffffu, hi);
        dom = __all_sync(0xffffffffu, dom);
        if ((threadIdx.x & 31) == 0) {
            atomicMin(&s_flo, lo);
            atomicMax(&s_fhi, hi);
            if (!dom) atomicAnd(&s_fast, 0u);
        }
        __syncthreads();
        if (threadIdx.x == 0 && s_flo > s_fhi) { s_flo = 0u; s_fhi = 0xFFFFFFFFu; }
        __syncthreads();
    }
    const uint64_t kfl = (uint64_t)s_flo << 32, kfh = (uint64_t)s_fhi << 32;
    const R3Geo gf = r3_geo(kfl, kfh > kfl ? kfh : kfl + (1ull << 32));
    const bool presort = A == 2 && a.mode == 1;
    const int64_t Rlim = presort ? a.pre_R : a.R;
    while (true) {
        if (threadIdx.x == 0) s_tick = atomicAdd(presort ? a.ticket_pre : a.ticket, 1u);
        if (threadIdx.x <= A) {
            s_min[threadIdx.x] = ~0ull;
            s_max[threadIdx.x] = 0ull;
        }
        __syncthreads();
        const int64_t rl = s_tick;
        __syncthreads();
        if (rl >= Rlim) break;
        K2_PHASE(0);
        // replicas sorted by the pre-sort pass: their sorted order is read back (post); the
        // pre-sort pass itself writes it per replica
        const bool post = A == 2 && a.mode == 2 && rl < a.pre_R;
        uint16_t* ppos_r = ppos;
        uint32_t* dsorted_r = dsorted;
        if (A == 2 && (presort || post)) {
            ppos_r = a.pp_pos + rl * npad;
            dsorted_r = a.pp_ds + rl * npad;
        }
        const int64_t r = a.r0 + rl;
        const float CP = a.cp[rl];
        float hdv[A];
#pragma unroll
        for (int b = 0; b < A; b++) hdv[b] = u2f(a.hd[rl * A + b]);
        // materialise critc, gainc_a (one hash per (t, a)) and, for two archs, the
        // orderable difference D(t) of the two durations; key ranges
        unsigned long long mn[A + 1], mx[A + 1];
#pragma unroll
        for (int b = 0; b <= A; b++) { mn[b] = ~0ull; mx[b] = 0ull; }
        const bool pre = A == 2 && geo && s_geo_ok && !post;
        if (pre) {   // restore the cached sub-bin geometry, zero the fine counters
            const uint16_t* g16 = reinterpret_cast<const uint16_t*>(geo);
            for (int32_t b = threadIdx.x; b < R3_NC; b += R2_THREADS) {
                S.coff[b] = __ldcg(g16 + b);
                S.clog[b] = __ldcg(geo + 2 * R3_NC + b);
            }
            for (int32_t b = threadIdx.x; b < R3_NF + 64; b += R2_THREADS) S.starts[b] = 0u;
            if (threadIdx.x == 0) s_out = 0u;
            __syncthreads();
        }
        if constexpr (A == 2) if (!post) {
            // two archs: only the orderable d is needed to sort (crit is read for equal-gain runs).
            // 4 tasks per thread and trip (t, t+1 | t+2048, t+2049): both 16-byte base loads
            // are issued before the hashing
            uint32_t dmn = ~0u, dmx = 0u;
            bool outside = false;
            auto one = [&](int32_t t, float b0v, float b1v) {
                const float bb[2] = {b0v, b1v};
                const uint64_t c0 = ((uint64_t)r * (uint64_t)a.n + (uint64_t)t) * 2u + 1u;
                uint32_t en = 0;
                float x[2];
#pragma unroll
                for (int b = 0; b < 2; b++) {
                    x[b] = canon_dur(perturb(bb[b], a.seed, a.sigma, c0 + b), bad);
                    if (((a.emask >> b) & 1u) && !is_inf(x[b])) en |= 1u << b;
                }
                if (!en) bad = true;
                uint32_t D;
                if (en == 3u) {
                    const uint32_t db = f2u(__fsub_rn(x[1], x[0]));
                    D = (db >> 31) ? ~db : (db | 0x80000000u);
                } else {
                    D = en == 1u ? 0xFFFFFFFFu : 0u;
                }
                dkey[t] = D;
                dmn = min(dmn, D);
                dmx = max(dmx, D);
                if (pre) {   // fine bin of the cached geometry (pass 2 of the sorter, fused)
                    const uint64_t key = (uint64_t)D << 32;
                    uint32_t f = 0xFFFFu;
                    if (key < gf.lo || key > gf.hi) {
                        outside = true;
                    } else {
                        f = r3_bin32(S, gf, D);
                        atomicAdd(&S.starts[f], 1u);
                    }
                    fbuf[t] = (uint16_t)f;
                }
            };
            const bool al = (reinterpret_cast<uintptr_t>(a.base) & 15u) == 0;
            const int32_t n2 = al ? (a.n & ~1) : 0;
            if (s_fast) {
                // fast path (decided per launch, as K1's): both archs enabled everywhere and no
                // perturbed duration can be 0, inf or outside the domain, so canonicalisation,
                // enabled masks and sentinels drop out; the splitmix64 state of (r, t, arch 0),
                // seed + ((r n + t) 2 + 1) golden, is walked by additions
                auto onef = [&](int32_t t, float b0v, float b1v, uint64_t X) {
                    const float x0 = perturb_x(b0v, X, a.sigma), x1 = perturb_x(b1v, X + SPLITMIX_GOLDEN, a.sigma);
                    const uint32_t db = f2u(__fsub_rn(x1, x0));
                    const uint32_t D = (db >> 31) ? ~db : (db | 0x80000000u);
                    dkey[t] = D;
                    dmn = min(dmn, D);
                    dmx = max(dmx, D);
                    if (pre) {
                        const uint64_t key = (uint64_t)D << 32;
                        uint32_t f = 0xFFFFu;
                        if (key < gf.lo || key > gf.hi) {
                            outside = true;
                        } else {
                            f = r3_bin32(S, gf, D);
                            atomicAdd(&S.starts[f], 1u);
                        }
                        fbuf[t] = (uint16_t)f;
                    }
                };
                constexpr uint64_t G2 = 2ull * SPLITMIX_GOLDEN;
                uint64_t X = a.seed + ((uint64_t)r * (uint64_t)a.n * 2u + 1u) * SPLITMIX_GOLDEN +
                             (uint64_t)(2 * threadIdx.x) * G2;
                for (int32_t t0 = 2 * threadIdx.x; t0 < n2; t0 += 4 * R2_THREADS, X += (uint64_t)(4 * R2_THREADS) * G2) {
                    const int32_t t1 = t0 + 2 * R2_THREADS;
                    const float4 v0 = __ldg(reinterpret_cast<const float4*>(a.base) + (t0 >> 1));
                    float4 v1 = make_float4(0.f, 0.f, 0.f, 0.f);
                    if (t1 < n2) v1 = __ldg(reinterpret_cast<const float4*>(a.base) + (t1 >> 1));
                    onef(t0, v0.x, v0.y, X);
                    onef(t0 + 1, v0.z, v0.w, X + G2);
                    if (t1 < n2) {
                        const uint64_t X1 = X + (uint64_t)(2 * R2_THREADS) * G2;
                        onef(t1, v1.x, v1.y, X1);
                        onef(t1 + 1, v1.z, v1.w, X1 + G2);
                    }
                }
                for (int32_t t = n2 + threadIdx.x; t < a.n; t += R2_THREADS)
                    onef(t, __ldg(a.base + 2 * (int64_t)t), __ldg(a.base + 2 * (int64_t)t + 1),
                         a.seed + (((uint64_t)r * (uint64_t)a.n + (uint64_t)t) * 2u + 1u) * SPLITMIX_GOLDEN);
            }
            for (int32_t t0 = 2 * threadIdx.x; !s_fast && t0 < n2; t0 += 4 * R2_THREADS) {
                const int32_t t1 = t0 + 2 * R2_THREADS;
                const float4 v0 = __ldg(reinterpret_cast<const float4*>(a.base) + (t0 >> 1));
                float4 v1 = make_float4(0.f, 0.f, 0.f, 0.f);
                if (t1 < n2) v1 = __ldg(reinterpret_cast<const float4*>(a.base) + (t1 >> 1));
                one(t0, v0.x, v0.y);
                one(t0 + 1, v0.z, v0.w);
                if (t1 < n2) {
                    one(t1, v1.x, v1.y);
                    one(t1 + 1, v1.z, v1.w);
                }
            }
            for (int32_t t = n2 + threadIdx.x; !s_fast && t < a.n; t += R2_THREADS)
                one(t, __ldg(a.base + 2 * (int64_t)t), __ldg(a.base + 2 * (int64_t)t + 1));
            mn[A] = (unsigned long long)dmn << 32;
            mx[A] = (unsigned long long)dmx << 32;
            if (__any_sync(0xffffffffu, outside) && (threadIdx.x & 31) == 0) s_out = 1u;
        }
        const bool vec4 = (a.n & 3) == 0;   // 16-byte loads of bl when rows stay aligned
        for (int32_t t0 = vec4 ? threadIdx.x * 4 : threadIdx.x; A != 2 && t0 < a.n; t0 += vec4 ? 4 * R2_THREADS : R2_THREADS) {
          float blq[4];
          if (vec4) {
              const float4 v4 = __ldcs(reinterpret_cast<const float4*>(a.blT + rl * a.n + t0));   // read once
              blq[0] = v4.x; blq[1] = v4.y; blq[2] = v4.z; blq[3] = v4.w;
          } else {
              blq[0] = __ldcs(a.blT + rl * a.n + t0);
          }
          const int nq = vec4 ? 4 : 1;
          for (int uq = 0; uq < nq; uq++) {
            const int32_t t = t0 + uq;
            const float blv = blq[uq];
            const float c = CP > 0.0f ? __fdiv_rn(blv, CP) : 0.0f;
            const uint32_t cc = ONE_BITS - f2u(c);
            if (A != 2) critc[t] = cc;   // two archs: crit is only needed for equal-gain runs (below)
            float x[A];
            uint32_t en;
            int k;
            float wt;
            r2_durs<A>(a, r, t, x, en, k, wt, bad);
#pragma unroll
            for (int b = 0; b < A; b++) {
                if (A == 2) break;   // two archs: gains are derived from D (general path re-materialises)
                uint32_t key = 0x40000000u;
                if ((en >> b) & 1u) {
                    float gv;
                    if (k == 1) gv = 1.0f;
                    else if (hdv[b] == 0.0f) gv = 0.5f;
                    else {
                        float ref = __uint_as_float(0x7f800000u);
#pragma unroll
                        for (int q = 0; q < A; q++)
                            if (q != b && ((en >> q) & 1u)) ref = x[q] < ref ? x[q] : ref;
                        gv = __fdiv_rn(__fadd_rn(__fsub_rn(ref, x[b]), hdv[b]), __fadd_rn(hdv[b], hdv[b]));
                    }
                    key = ONE_BITS - f2u(gv);
                }
                gainc[(int64_t)b * npad + t] = key;
                const unsigned long long full = ((unsigned long long)key << 32) | cc;
                mn[b] = full < mn[b] ? full : mn[b];
                mx[b] = full > mx[b] ? full : mx[b];
            }
            if constexpr (A == 2) {
                // d = delta_1 - delta_0 (= d(t, arch 0) = -d(t, arch 1), exact negation): gain_0 is
                // non-decreasing and gain_1 non-increasing in d (RN ops are monotone), so one order by
                // d serves both queues.  Arch-0-only tasks sort last, arch-1-only first.
                uint32_t D;
                if (en == 3u) {
                    const uint32_t db = f2u(__fsub_rn(x[1], x[0]));
                    D = (db >> 31) ? ~db : (db | 0x80000000u);
                } else {
                    D = en == 1u ? 0xFFFFFFFFu : 0u;
                }
                dkey[t] = D;
                const unsigned long long full = ((unsigned long long)D << 32) | cc;
                mn[A] = full < mn[A] ? full : mn[A];
                mx[A] = full > mx[A] ? full : mx[A];
            }
          }
        }
#pragma unroll
        for (int b = 0; b <= A; b++) {
            unsigned long long v1 = mn[b], v2 = mx[b];
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                unsigned long long y1 = __shfl_xor_sync(0xffffffffu, v1, o);
                unsigned long long y2 = __shfl_xor_sync(0xffffffffu, v2, o);
                v1 = y1 < v1 ? y1 : v1;
                v2 = y2 > v2 ? y2 : v2;
            }
            if ((threadIdx.x & 31) == 0) {
                atomicMin(&s_min[b], v1);
                atomicMax(&s_max[b], v2);
            }
        }
        __syncthreads();
        bool done = false;
        if constexpr (A == 2) {
            // one sort by (D, critc, t) -> P; then both queues in one pass (runs of equal gain fixed up)
            K2_PHASE(1);
            if (!post) {
                const uint64_t amin = s_min[A] & ~0xFFFFFFFFull, amax = s_max[A] & ~0xFFFFFFFFull;
                const R3Keys K{dkey, nullptr, fbuf};
                const R3PosOut O{ppos_r, dsorted_r};
                if (pre && !s_out) {
                    r3_sort<uint32_t>(K, O, a.n, gf.lo, gf.hi, S, s_geo_nfb);
                } else if (geo && !pre && amin >= gf.lo && amax <= gf.hi && gf.lo < gf.hi) {
                    // first replica on the fixed range: build and cache its geometry
                    if (threadIdx.x == 0) *reinterpret_cast<uint32_t*>(geo + 3 * R3_NC) = 0u;
                    __syncthreads();
                    r3_sort<uint32_t>(K, O, a.n, gf.lo, gf.hi, S, 0u, geo);
                    if (threadIdx.x == 0) {
                        s_geo_nfb = *reinterpret_cast<volatile uint32_t*>(geo + 3 * R3_NC);
                        s_geo_ok = s_geo_nfb != 0u;
                    }
                } else {
                    r3_sort<uint32_t>(K, O, a.n, amin, amax, S);
                }
            }
            K2_PHASE(7);
            if (presort) {   // the pre-sort pass stops here (its order is in pp_pos / pp_ds)
                __syncthreads();
                continue;
            }
            if (threadIdx.x == 0) { s_flag = 0; s_h0 = 0xffffffffu; s_h1 = 0xffffffffu; }
            __syncthreads();
            const int32_t cC = a.counts[rl * 2 + 0], cG = a.counts[rl * 2 + 1];
            const int32_t n1only = a.n - cC;            // arch-1-only tasks: sorted first
            int32_t* q0 = a.qtask ? a.qtask + rl * (int64_t)a.n * 2 : nullptr;
            int32_t* q1 = q0 ? q0 + cC : nullptr;
            const float h2 = hdv[0];   // hd(0) == hd(1) for two archs
            // bl of this replica in K1's [group][q][32] layout (no transpose for two archs)
            const float* blr = a.bl32 + (rl >> 5) * (int64_t)a.n * 32 + (rl & 31);
            auto critc_of = [&](uint32_t t) -> uint32_t {
                const float c = CP > 0.0f ? __fdiv_rn(__ldcg(blr + (int64_t)__ldg(a.qof + t) * 32), CP) : 0.0f;
                return ONE_BITS - f2u(c);
            };
            // sorted order into shared memory (the sort's buffers are free now) + neighbour-equality
            // bits: e0/e1 = same gain as the next position (arch 0 / arch 1)
            uint16_t* Ps = reinterpret_cast<uint16_t*>(S.bkraw);
            const int32_t nw = (a.n + 31) / 32;
            uint32_t* e0 = reinterpret_cast<uint32_t*>(Ps + ((a.n + 63) & ~63));
            uint32_t* e1 = e0 + nw;
            {   // 16-byte copies (ppos_r and Ps are 32-byte aligned)
                const int32_t n8 = a.n >> 3;
                for (int32_t i = threadIdx.x; i < n8; i += R2_THREADS)
                    reinterpret_cast<uint4*>(Ps)[i] = __ldcg(reinterpret_cast<const uint4*>(ppos_r) + i);
                for (int32_t i = (n8 << 3) + threadIdx.x; i < a.n; i += R2_THREADS) Ps[i] = ppos_r[i];
            }
            {
                K2_PHASE(8);
                // 4 consecutive positions per lane (one 16-byte load), 128 per warp and chunk,
                // two chunks in flight; nibbles of 8 lanes OR-ed into one bit word.  Near-ties
                // (different numerators less than lim apart, ~2% of the pairs) need the two
                // divisions; they are listed (position | arch << 31, in the free bin counters)
                // and divided in a compact pass, so no warp runs the division code inline
                uint32_t* nearl = S.starts + 1;
                const uint32_t ncap = (uint32_t)R3_NF + 63u;
                if (threadIdx.x == 0) S.starts[0] = 0u;
                __syncthreads();
                const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
                const bool one_arch = cC != a.n || cG != a.n;   // some D are the one-arch sentinels
                constexpr int32_t CH = 128, STEP = CH * R2_WARPS;
#ifndef MP_EQ_H
#define MP_EQ_H 2
#endif
                constexpr int EQ_H = MP_EQ_H;   // 128-position chunks per warp in flight
                for (int32_t cb0 = w * CH; cb0 < a.n; cb0 += EQ_H * STEP) {
                    uint32_t Dv[EQ_H][4], nx[EQ_H];
#pragma unroll
                    for (int h = 0; h < EQ_H; h++) {
                        const int32_t p4 = cb0 + h * STEP + lane * 4;
                        if (p4 + 4 <= a.n) {
                            const uint4 v = __ldcg(reinterpret_cast<const uint4*>(dsorted_r + p4));
                            Dv[h][0] = v.x; Dv[h][1] = v.y; Dv[h][2] = v.z; Dv[h][3] = v.w;
                        } else {
#pragma unroll
                            for (int j = 0; j < 4; j++) Dv[h][j] = p4 + j < a.n ? __ldcg(dsorted_r + p4 + j) : 0u;
                        }
                        nx[h] = (lane == 31 && p4 + 4 < a.n) ? __ldcg(dsorted_r + p4 + 4) : 0u;
                    }
#pragma unroll
                    for (int h = 0; h < EQ_H; h++) {
                        const int32_t cb = cb0 + h * STEP;
                        if (cb >= a.n) break;
                        const int32_t p4 = cb + lane * 4;
                        uint32_t nxt = __shfl_down_sync(0xffffffffu, Dv[h][0], 1);
                        if (lane == 31) nxt = nx[h];
                        // numerators x = d + hd (arch 0) and y = -d + hd (arch 1) once per position
                        uint32_t Dj[5] = {Dv[h][0], Dv[h][1], Dv[h][2], Dv[h][3], nxt};
                        float xs[5], ys[5];
                        bool gen = h2 == 0.0f;   // sentinels or hd = 0: the generic comparison
#pragma unroll
                        for (int j = 0; j < 5; j++) {
                            const uint32_t D = Dj[j];
                            if (one_arch) gen |= (D == 0u || D == 0xFFFFFFFFu) && (j < 4 ? p4 + j < a.n : p4 + 4 < a.n);
                            const float d = u2f((D & 0x80000000u) ? (D & 0x7FFFFFFFu) : ~D);
                            xs[j] = __fadd_rn(d, h2);
                            ys[j] = __fadd_rn(__fsub_rn(0.0f, d), h2);
                        }
                        const float den = __fadd_rn(h2, h2);
                        const float lim = __fmul_rn(den, 0x1p-24f);
                        uint32_t n0 = 0, n1 = 0;
#pragma unroll
                        for (int j = 0; j < 4; j++) {
                            if (p4 + j + 1 < a.n) {
                                bool s0, s1;
                                if (gen) {
                                    r2_same_gains(Dj[j], Dj[j + 1], h2, s0, s1);
                                } else {
                                    // sorted ascending: x non-decreasing, y non-increasing
                                    const float dx = __fsub_rn(xs[j + 1], xs[j]), dy = __fsub_rn(ys[j], ys[j + 1]);
                                    s0 = dx == 0.0f;
                                    s1 = dy == 0.0f;
                                    const bool c0 = !s0 && dx <= lim;
                                    const bool c1 = !s1 && dy <= lim;
                                    if (c0 || c1) {
                                        const uint32_t cnt = (c0 ? 1u : 0u) + (c1 ? 1u : 0u);
                                        const uint32_t at = atomicAdd(&S.starts[0], cnt);
                                        const uint32_t pj = (uint32_t)(p4 + j);
                                        if (at + cnt <= ncap) {
                                            if (c0) nearl[at] = pj;
                                            if (c1) nearl[at + (c0 ? 1u : 0u)] = pj | 0x80000000u;
                                        } else {   // list full (not expected): divide here
                                            if (c0) s0 = r2_same_q(xs[j], xs[j + 1], den, lim);
                                            if (c1) s1 = r2_same_q(ys[j], ys[j + 1], den, lim);
                                        }
                                    }
                                }
                                n0 |= (uint32_t)s0 << j;
                                n1 |= (uint32_t)s1 << j;
                            }
                        }
                        n0 <<= (lane & 7) * 4;
                        n1 <<= (lane & 7) * 4;
#pragma unroll
                        for (int o = 1; o < 8; o <<= 1) {
                            n0 |= __shfl_xor_sync(0xffffffffu, n0, o);
                            n1 |= __shfl_xor_sync(0xffffffffu, n1, o);
                        }
                        if ((lane & 7) == 0 && p4 < a.n) {
                            e0[(cb >> 5) + (lane >> 3)] = n0;
                            e1[(cb >> 5) + (lane >> 3)] = n1;
                        }
                    }
                }
                __syncthreads();
                const uint32_t nn = min(S.starts[0], ncap);
                const float den = __fadd_rn(h2, h2);
                for (uint32_t i = threadIdx.x; i < nn; i += R2_THREADS) {
                    const uint32_t ent = nearl[i];
                    const int32_t p = (int32_t)(ent & 0x7FFFFFFFu);
                    const uint32_t Da = __ldcg(dsorted_r + p), Db = __ldcg(dsorted_r + p + 1);   // no sentinels here
                    const float da = u2f((Da & 0x80000000u) ? (Da & 0x7FFFFFFFu) : ~Da);
                    const float db = u2f((Db & 0x80000000u) ? (Db & 0x7FFFFFFFu) : ~Db);
                    const float d0 = (ent >> 31) ? __fsub_rn(0.0f, da) : da, d1 = (ent >> 31) ? __fsub_rn(0.0f, db) : db;
                    const float xa = __fadd_rn(d0, h2), xb = __fadd_rn(d1, h2);
                    if (__fdiv_rn(xa, den) == __fdiv_rn(xb, den)) atomicOr((ent >> 31) ? &e1[p >> 5] : &e0[p >> 5], 1u << (p & 31));
                }
            }
            __syncthreads();
            // members of equal-gain runs (rare): their critc is gathered once, all loads in
            // flight together, into shared memory (the sort's bin counters are free now):
            // mw = member bits per 32 positions, mp = exclusive prefix of their popcounts,
            // crs[mp[w] + rank in word] = critc of the task at that position
            K2_PHASE(9);
            uint32_t* mw = S.starts;
            uint32_t* mp = mw + nw;
            uint32_t* crs = mp + nw;
            const uint32_t ccap = ((uint32_t)(R3_NF + 64) - 2u * (uint32_t)nw) * 4u / 6u;
            uint16_t* mpos = reinterpret_cast<uint16_t*>(crs + ccap);   // position of member #i
            auto lt = [&](int32_t wb, int32_t x) -> uint32_t {   // bits i with wb + i < x
                const int32_t c = x - wb;
                return c <= 0 ? 0u : (c >= 32 ? 0xFFFFFFFFu : ((1u << c) - 1u));
            };
            uint32_t mloc[2], pre = 0;
            {
                uint32_t cnt = 0;
#pragma unroll
                for (int h = 0; h < 2; h++) {
                    const int32_t w = 2 * (int32_t)threadIdx.x + h;
                    uint32_t m = 0;
                    if (w < nw) {
                        const int32_t wb = w * 32;
                        const uint32_t E1 = e1[w], E0 = e0[w];
                        const uint32_t P1 = (E1 << 1) | (w > 0 ? e1[w - 1] >> 31 : 0u);   // bit(e1, p-1)
                        const uint32_t P0 = (E0 << 1) | (w > 0 ? e0[w - 1] >> 31 : 0u);
                        const uint32_t m1 = (P1 | (E1 & lt(wb, cG - 1))) & lt(wb, cG);
                        const uint32_t ge0 = ~lt(wb, n1only), ge1 = ~lt(wb, n1only + 1);
                        const uint32_t m0 = (P0 & ge1) | (E0 & ge0);
                        m = (m0 | m1) & lt(wb, a.n);
                    }
                    mloc[h] = m;
                    cnt += __popc(m);
                }
                uint32_t tot;
                pre = r3_scan(cnt, S.sc, tot);
                if (threadIdx.x == 0) s_mtot = tot;
            }
#pragma unroll
            for (int h = 0; h < 2; h++) {
                const int32_t w = 2 * (int32_t)threadIdx.x + h;
                if (w < nw) {
                    mw[w] = mloc[h];
                    mp[w] = pre;
                }
                pre += __popc(mloc[h]);
            }
            __syncthreads();
            const bool mfit = s_mtot <= ccap;
#ifdef MP_PHASES
            if (threadIdx.x == 0) atomicAdd(&g_k2_phase[20], (unsigned long long)s_mtot);
#endif
            if (mfit) {
#pragma unroll
                for (int h = 0; h < 2; h++) {
                    const int32_t w = 2 * (int32_t)threadIdx.x + h;
                    if (w >= nw) continue;
                    uint32_t m = mloc[h];
                    uint32_t idx = mp[w];
                    while (m) {   // up to 4 gathers in flight per thread
                        uint32_t tq[4], ix[4];
                        int c = 0;
#pragma unroll
                        for (int u = 0; u < 4; u++) {
                            if (m) {
                                const int b = __ffs(m) - 1;
                                m &= m - 1u;
                                tq[u] = __ldg(a.qof + Ps[w * 32 + b]);
                                mpos[idx] = (uint16_t)(w * 32 + b);
                                ix[u] = idx++;
                                c = u + 1;
                            }
                        }
                        float bv[4];
#pragma unroll
                        for (int u = 0; u < 4; u++) bv[u] = u < c ? __ldcg(blr + (int64_t)tq[u] * 32) : 0.0f;
#pragma unroll
                        for (int u = 0; u < 4; u++)
                            if (u < c) crs[ix[u]] = ONE_BITS - f2u(CP > 0.0f ? __fdiv_rn(bv[u], CP) : 0.0f);
                    }
                }
            }
            __syncthreads();
            K2_PHASE(10);
            auto crit_at = [&](int32_t i) -> uint32_t {   // critc of the task at sorted position i
                if (!mfit) return critc_of(Ps[i]);
                const uint32_t m = mw[i >> 5];
                return crs[mp[i >> 5] + __popc(m & ((1u << (i & 31)) - 1u))];
            };
            auto bit = [&](const uint32_t* e, int32_t i) -> bool { return (e[i >> 5] >> (i & 31)) & 1u; };
            if (mfit) {   // positions in no equal-gain run go straight to both queues (coalesced):
                          // 4 consecutive positions per thread, 16-byte stores where aligned
                const bool v1 = q1 && ((reinterpret_cast<uintptr_t>(q1) & 15u) == 0u);
                const bool v0 = q0 && ((a.n & 3) == 0) && ((reinterpret_cast<uintptr_t>(q0) & 15u) == 0u);
                for (int32_t p4 = 4 * (int32_t)threadIdx.x; p4 < a.n; p4 += 4 * R2_THREADS) {
                    const uint32_t mb = (mw[p4 >> 5] >> (p4 & 31)) & 0xFu;
                    uint32_t tt[4];
                    if (p4 + 4 <= a.n) {
                        const uint2 v = *reinterpret_cast<const uint2*>(Ps + p4);
                        tt[0] = v.x & 0xFFFFu; tt[1] = v.x >> 16; tt[2] = v.y & 0xFFFFu; tt[3] = v.y >> 16;
                    } else {
#pragma unroll
                        for (int j = 0; j < 4; j++) tt[j] = p4 + j < a.n ? Ps[p4 + j] : 0u;
                    }
                    if (p4 == 0 && !(mb & 1u) && cG > 0) s_h1 = tt[0];
                    if (v1 && mb == 0u && p4 + 4 <= cG) {
                        __stcs(reinterpret_cast<int4*>(q1 + p4), make_int4((int)tt[0], (int)tt[1], (int)tt[2], (int)tt[3]));
                    } else if (q1) {
#pragma unroll
                        for (int j = 0; j < 4; j++)
                            if (p4 + j < cG && !((mb >> j) & 1u)) __stcs(q1 + p4 + j, (int32_t)tt[j]);
                    }
                    if (v0 && mb == 0u && p4 >= n1only && p4 + 4 <= a.n) {
                        __stcs(reinterpret_cast<int4*>(q0 + (a.n - 4 - p4)), make_int4((int)tt[3], (int)tt[2], (int)tt[1], (int)tt[0]));
                    } else if (q0) {
#pragma unroll
                        for (int j = 0; j < 4; j++) {
                            const int32_t p = p4 + j;
                            if (p < a.n && p >= n1only && !((mb >> j) & 1u)) __stcs(q0 + (a.n - 1 - p), (int32_t)tt[j]);
                        }
                    }
#pragma unroll
                    for (int j = 0; j < 4; j++)
                        if (p4 + j == a.n - 1 && !((mb >> j) & 1u)) s_h0 = tt[j];
                }
            }
            // members (all positions when they did not fit): rank inside their runs
            const int32_t nslow = mfit ? (int32_t)s_mtot : a.n;
            for (int32_t ii = threadIdx.x; ii < nslow; ii += R2_THREADS) {
                const int32_t p = mfit ? (int32_t)mpos[ii] : ii;
                const uint32_t t = Ps[p];
                // arch 1 (forward order), positions [0, cG); p and p+1 in one run iff bit(e1, p)
                if (p < cG) {
                    int32_t pos = p;
                    const bool prev = p > 0 && bit(e1, p - 1);
                    const bool next = p + 1 < cG && bit(e1, p);
                    if (prev || next) {
                        int32_t lo = p, hi = p;
                        while (lo > 0 && p - lo < 64 && bit(e1, lo - 1)) lo--;
                        while (hi + 1 < cG && hi - p < 64 && bit(e1, hi)) hi++;
                        if ((lo > 0 && bit(e1, lo - 1)) || (hi + 1 < cG && bit(e1, hi))) s_flag = 1;
                        {   // the sort ordered the run by (d, id): rank it by (critc, id)
                            const uint64_t me = ((uint64_t)crit_at(p) << 16) | t;
                            int32_t rk = 0;
                            for (int32_t i = lo; i <= hi; i++) {
                                const uint32_t ti = Ps[i];
                                rk += (((uint64_t)crit_at(i) << 16) | ti) < me ? 1 : 0;
                            }
                            pos = lo + rk;
                        }
                    }
                    if (pos == 0) s_h1 = t;
                    if (q1) __stcs(q1 + pos, (int32_t)t);
                }
                // arch 0 (reverse order), sorted positions [n1only, n)
                if (p >= n1only) {
                    int32_t pos = a.n - 1 - p;
                    const bool prev = p > n1only && bit(e0, p - 1);
                    const bool next = p + 1 < a.n && bit(e0, p);
                    if (prev || next) {
                        int32_t lo = p, hi = p;
                        while (lo > n1only && p - lo < 64 && bit(e0, lo - 1)) lo--;
                        while (hi + 1 < a.n && hi - p < 64 && bit(e0, hi)) hi++;
                        if ((lo > n1only && bit(e0, lo - 1)) || (hi + 1 < a.n && bit(e0, hi))) s_flag = 1;
                        const int32_t base = a.n - 1 - hi;   // the run's block in queue 0
                        {   // the sort ordered the run by (d, id): rank it by (critc, id)
                            const uint64_t me = ((uint64_t)crit_at(p) << 16) | t;
                            int32_t rk = 0;
                            for (int32_t i = lo; i <= hi; i++) {
                                const uint32_t ti = Ps[i];
                                rk += (((uint64_t)crit_at(i) << 16) | ti) < me ? 1 : 0;
                            }
                            pos = base + rk;
                        }
                    }
                    if (pos == 0) s_h0 = t;
                    if (q0) __stcs(q0 + pos, (int32_t)t);
                }
            }
            __syncthreads();
            K2_PHASE(11);
            if (!s_flag) {
                done = true;
                if (threadIdx.x < 2) {
                    const int b = threadIdx.x;
                    const int32_t cnt = a.counts[rl * 2 + b];
                    mp_queue_summary o;
                    o.count = cnt;
                    o.head = cnt > 0 ? (int32_t)(b == 0 ? s_h0 : s_h1) : -1;
                    const int64_t bo = (rl * 2 + b) * 2;
                    o.brw_lo = a.brw[bo];
                    o.brw_hi = (int64_t)a.brw[bo + 1];
                    o.brw = u128_to_double_scaled(a.brw[bo], a.brw[bo + 1]);
                    a.sum[rl * 2 + b] = o;
                }
            }
            __syncthreads();
        }
        K2_PHASE(12);
        if (done) continue;
        if constexpr (A == 2) {
            // fallback for this replica: materialise both archs' gain keys and ranges
            if (threadIdx.x < A) {
                s_min[threadIdx.x] = ~0ull;
                s_max[threadIdx.x] = 0ull;
            }
            if (post) {   // sorted by the pre-sort pass: this CTA has no D(t) of the replica yet
                for (int32_t t = threadIdx.x; t < a.n; t += R2_THREADS) {
                    float x[2];
                    uint32_t en = 0;
                    bool dummy = false;
                    const uint64_t c0 = ((uint64_t)r * (uint64_t)a.n + (uint64_t)t) * 2u + 1u;
#pragma unroll
                    for (int b = 0; b < 2; b++) {
                        x[b] = canon_dur(perturb(__ldg(a.base + 2 * (int64_t)t + b), a.seed, a.sigma, c0 + b), dummy);
                        if (((a.emask >> b) & 1u) && !is_inf(x[b])) en |= 1u << b;
                    }
                    uint32_t D;
                    if (en == 3u) {
                        const uint32_t db = f2u(__fsub_rn(x[1], x[0]));
                        D = (db >> 31) ? ~db : (db | 0x80000000u);
                    } else {
                        D = en == 1u ? 0xFFFFFFFFu : 0u;
                    }
                    dkey[t] = D;
                }
            }
            __syncthreads();
            unsigned long long fmn[A], fmx[A];
#pragma unroll
            for (int b = 0; b < A; b++) { fmn[b] = ~0ull; fmx[b] = 0ull; }
            for (int32_t t = threadIdx.x; t < a.n; t += R2_THREADS) {
                const float c = CP > 0.0f ? __fdiv_rn(__ldcg(a.bl32 + (rl >> 5) * (int64_t)a.n * 32 +
                                                              (int64_t)__ldg(a.qof + t) * 32 + (rl & 31)), CP)
                                          : 0.0f;
                const uint32_t cc = ONE_BITS - f2u(c);
                critc[t] = cc;
                uint32_t G[2];
                r2_gains_from_D(dkey[t], hdv[0], G[0], G[1]);
#pragma unroll
                for (int b = 0; b < A; b++) {
                    gainc[(int64_t)b * npad + t] = G[b];
                    const unsigned long long full = ((unsigned long long)G[b] << 32) | cc;
                    fmn[b] = full < fmn[b] ? full : fmn[b];
                    fmx[b] = full > fmx[b] ? full : fmx[b];
                }
            }
#pragma unroll
            for (int b = 0; b < A; b++) {
                unsigned long long v1 = fmn[b], v2 = fmx[b];
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) {
                    unsigned long long y1 = __shfl_xor_sync(0xffffffffu, v1, o);
                    unsigned long long y2 = __shfl_xor_sync(0xffffffffu, v2, o);
                    v1 = y1 < v1 ? y1 : v1;
                    v2 = y2 > v2 ? y2 : v2;
                }
                if ((threadIdx.x & 31) == 0) {
                    atomicMin(&s_min[b], v1);
                    atomicMax(&s_max[b], v2);
                }
            }
            __syncthreads();
        }
        // general path (A != 2, or an equal-gain run of > 64 entries spanning several d values)
        int64_t qoff = 0;
        for (int b = 0; b < A; b++) {
            const int32_t cnt = a.counts[rl * A + b];
            if (threadIdx.x == 0) s_head = 0xffffffffu;
            __syncthreads();
            int32_t* qdst = a.qtask ? a.qtask + rl * (int64_t)a.n * A + qoff : nullptr;
            r3_sort<uint64_t>(R3Keys{gainc + (int64_t)b * npad, critc, fbuf}, R3Out{qdst, cnt, &s_head}, a.n, s_min[b], s_max[b], S);
            __syncthreads();
            if (threadIdx.x == 0) {
                mp_queue_summary o;
                o.count = cnt;
                o.head = cnt > 0 ? (int32_t)s_head : -1;
                const int64_t bo = (rl * A + b) * 2;
                o.brw_lo = a.brw[bo];
                o.brw_hi = (int64_t)a.brw[bo + 1];
                o.brw = u128_to_double_scaled(a.brw[bo], a.brw[bo + 1]);
                a.sum[rl * A + b] = o;
            }
            qoff += cnt;
            __syncthreads();
        }
    }
    (void)bad;
}

}  // namespace mpk

namespace mph {

template <int A>
inline mp_status rep2_launch(mp_dag* dag, const float* base, uint32_t emask, uint64_t seed, float sigma, int64_t r0,
                             int32_t R, float* cp, mp_queue_summary* sum, int32_t* qtask, cudaStream_t st) {
    using namespace mpk;
    const int32_t n = dag->n;
    const int64_t groups = (R + 31) / 32;
    const int grid2 = std::max(1, std::min<int>(R, dag->num_sms));
    const int smem1 = 32 * 32 * 33 * 4;
    const int smem2 = (int)r3_smem_bytes();
    static std::atomic<uint64_t> attr{0};
    if (first_on_device(attr)) {
        MP_CUDA(cudaFuncSetAttribute(k_rep2_bl<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem1));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_bl<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem1));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_bl<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem1));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_bl<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem1));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_sort<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_sort<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_sort<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_sort<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2));
    }
    // cluster size: enough CTAs per 32-replica group to cover the SMs (strong scaling keeps K1 short)
    // (8-CTA clusters and a cross-CTA dataflow mode -- bl lines as ready flags polled from L2 --
    // measured slower: R = 512 K1 0.98 ms (4-CTA, level barriers) vs 1.58 ms (8-CTA) and
    // 1.06 ms (4-CTA dataflow); the per-group time is a latency floor of ~5 us per level)
    // the largest cluster (<= 8 CTAs) with which every group's cluster is resident at once
    // (a second wave of clusters would double K1); 1 when the groups alone fill the SMs
    // (memoised per device and group count: the occupancy queries cost host time every call)
    static std::mutex cs_mu;
    static std::map<std::pair<int, int64_t>, int> cs_memo;
    int cs = 1;
    bool memo_hit = false;
    {
        std::lock_guard<std::mutex> lk(cs_mu);
        auto it = cs_memo.find({dag->device, groups * 8 + A});
        if (it != cs_memo.end()) {
            cs = it->second;
            memo_hit = true;
        }
    }
    for (int c = 8; c >= 2 && !memo_hit; c--) {
        if (groups * c > dag->num_sms) continue;
        cudaLaunchConfig_t q = {};
        q.gridDim = dim3((unsigned)(groups * c));
        q.blockDim = dim3(R2_THREADS);
        q.dynamicSmemBytes = (size_t)smem1;
        q.stream = st;
        cudaLaunchAttribute qa[1];
        qa[0].id = cudaLaunchAttributeClusterDimension;
        qa[0].val.clusterDim.x = (unsigned)c;
        qa[0].val.clusterDim.y = 1;
        qa[0].val.clusterDim.z = 1;
        q.attrs = qa;
        q.numAttrs = 1;
        int mac = 0;
        if (cudaOccupancyMaxActiveClusters(&mac, k_rep2_bl<A>, &q) != cudaSuccess) {
            cudaGetLastError();
            continue;
        }
        if (mac >= groups) {
            cs = c;
            break;
        }
    }
    if (!memo_hit) {
        std::lock_guard<std::mutex> lk(cs_mu);
        cs_memo[{dag->device, groups * 8 + A}] = cs;
    }
    // K2 pre-sort pass (two archs, one CTA per group): K1 leaves num_sms - groups SMs idle for
    // its whole level walk; K2's hash + sort phases of the first pre_R replicas run there
    // meanwhile (about 17 replicas per idle SM fit in K1's time: K1 walks n nodes x 32 replicas
    // per SM, a pre-sort takes ~1/20 of that per replica); the main K2 pass then only finishes
    // those replicas
    const int idle = dag->num_sms - (int)(groups * cs);
    // (clusters: fewer per SM -- the pre-sort CTAs then also delay some of K1's clusters; swept
    // 4..15 per idle SM, measured net: R = 512 1.53 -> 1.44 ms, 1024 2.09 -> 1.98, 2048 3.42 ->
    // 3.33, 4096 6.01 -> 5.81 with 17 / 9: 19 leaves the pre-sort too close to K1)
#ifndef MP_PRE_FLOW
#define MP_PRE_FLOW 17
#endif
#ifndef MP_PRE_CL
#define MP_PRE_CL 9
#endif
    const int per_idle = cs == 1 ? MP_PRE_FLOW : MP_PRE_CL;
#ifndef MP_PRE_DIV
#define MP_PRE_DIV 4
#endif
    const int32_t pre_R = (A == 2 && idle > 0 && R >= 2 * 148) ? std::min<int32_t>(R / MP_PRE_DIV, idle * per_idle) : 0;
    const size_t npad_b = (size_t)((n + 15) & ~15);
    const size_t blT_elems = A == 2 ? 1 : (size_t)R * n;   // two archs: K2 reads K1's bl32 directly
    size_t bytes = align256((size_t)groups * n * 32 * 4) + align256(blT_elems * 4) + align256((size_t)R * A * 4) * 2 +
                   align256((size_t)R * A * 16) + align256((size_t)grid2 * ((n + 15) & ~15) * 4 * (A + 1)) + align256((size_t)grid2 * ((n + 15) & ~15) * 8) +
                   align256((size_t)grid2 * ((n + 15) & ~15) * 4) + align256((size_t)grid2 * R3_GEO_BYTES) +
                   align256((size_t)pre_R * npad_b * 2) + align256((size_t)pre_R * npad_b * 4);
    MP_TRY(ensure_ws(dag, bytes, st));
    Arena ar{dag->ws, dag->ws_cap};
    Rep2Args a{};
    a.n = n;
    a.A = A;
    a.L = dag->L;
    a.R = R;
    a.r0 = r0;
    a.lvlq = dag->lvlq;
    a.nodeq = dag->nodeq;
    a.rowq = dag->rowq;
    a.colq = dag->colq;
    a.qof = dag->qof;
    a.base = base;
    a.emask = emask;
    a.seed = seed;
    a.sigma = sigma;
    a.bl32 = ar.take<float>((size_t)groups * n * 32);
    a.blT = ar.take<float>(blT_elems);
    a.cp = cp;
    a.hd = ar.take<uint32_t>((size_t)R * A);
    a.counts = ar.take<int32_t>((size_t)R * A);
    a.brw = ar.take<unsigned long long>((size_t)R * A * 2);
    a.err = dag->err;
    const size_t npad = (size_t)((n + 15) & ~15);
    a.s_cold = ar.take<uint32_t>((size_t)grid2 * npad * (A + 1));
    a.s_key = ar.take<uint32_t>((size_t)grid2 * npad * 2);   // hot scratch: s_key and s_pi adjacent
    a.s_pi = ar.take<uint16_t>((size_t)grid2 * npad * 2);
    a.s_geo = A == 2 ? ar.take<unsigned char>((size_t)grid2 * R3_GEO_BYTES) : nullptr;
    a.qtask = qtask;
    a.sum = sum;
    a.ticket = dag->tickets + 56;
    a.mode = 0;
    a.pre_R = pre_R;
    a.pp_pos = pre_R > 0 ? ar.take<uint16_t>((size_t)pre_R * npad_b) : nullptr;
    a.pp_ds = pre_R > 0 ? ar.take<uint32_t>((size_t)pre_R * npad_b) : nullptr;
    a.ticket_pre = dag->tickets + 57;
    // statistics are merged with atomics: zero them (and CP) first
    MP_CUDA(cudaMemsetAsync(cp, 0, (size_t)R * 4, st));
    MP_CUDA(cudaMemsetAsync(a.hd, 0, (size_t)R * A * 4, st));
    MP_CUDA(cudaMemsetAsync(a.counts, 0, (size_t)R * A * 4, st));
    MP_CUDA(cudaMemsetAsync(a.brw, 0, (size_t)R * A * 16, st));
    if (pre_R > 0) {   // the pre-sort pass starts with K1, on a side stream
        MP_TRY(ensure_side_stream(dag));
        MP_CUDA(cudaEventRecord(dag->ev_a, st));
        MP_CUDA(cudaStreamWaitEvent(dag->side, dag->ev_a, 0));
    }
    for (;; cs = cs > 1 ? cs - 1 : 1) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3((unsigned)(groups * cs));
        cfg.blockDim = dim3(R2_THREADS);
        cfg.dynamicSmemBytes = (size_t)smem1;
        cfg.stream = st;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = (unsigned)cs;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        a.flow = cs == 1 ? 1 : 0;
        cudaError_t e;
        {
            mph::ProfScope ps("k_rep2_bl<A>", st);
            e = cudaLaunchKernelEx(&cfg, k_rep2_bl<A>, a);
        }
        if (e == cudaSuccess) break;
        cudaGetLastError();
        if (cs == 1) return fail(MP_ERR_CUDA, "k_rep2_bl launch: %s", cudaGetErrorString(e));
    }
    if (pre_R > 0) {
        MP_CUDA(cudaMemsetAsync(a.ticket_pre, 0, 4, dag->side));
        Rep2Args ap = a;
        ap.mode = 1;
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3((unsigned)idle);
        cfg.blockDim = dim3(R2_THREADS);
        cfg.dynamicSmemBytes = (size_t)smem2;
        cfg.stream = dag->side;
        {
            mph::ProfScope ps("k_rep2_pre", dag->side);
            MP_CUDA(cudaLaunchKernelEx(&cfg, k_rep2_sort<A>, ap));
        }
        MP_CUDA(cudaEventRecord(dag->ev_b, dag->side));
        MP_CUDA(cudaStreamWaitEvent(st, dag->ev_b, 0));
        a.mode = 2;
    }
    MP_CUDA(cudaMemsetAsync(a.ticket, 0, 4, st));
    {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3((unsigned)grid2);
        cfg.blockDim = dim3(R2_THREADS);
        cfg.dynamicSmemBytes = (size_t)smem2;
        cfg.stream = st;
        mph::ProfScope ps("k_rep2_sort<A>", st);
        MP_CUDA(cudaLaunchKernelEx(&cfg, k_rep2_sort<A>, a));
    }
    MP_CUDA(cudaGetLastError());
    return MP_OK;
}

// Fast replica path: n < 65536 (16-bit ids in the shared-memory sorts), A <= 4.
inline bool rep2_eligible(const mp_dag* dag, int32_t A) { return dag->n > 0 && dag->n < 65536 && A <= 4; }

inline mp_status replicas_run2(mp_dag* dag, int32_t A, const float* base, uint32_t emask, uint64_t seed, float sigma,
                               int64_t r0, int32_t R, float* cp, mp_queue_summary* sum, int32_t* qtask,
                               cudaStream_t st) {
    const int32_t chunk = 8192;
    for (int64_t b0 = 0; b0 < R; b0 += chunk) {
        const int32_t nb = (int32_t)std::min<int64_t>(chunk, R - b0);
        int32_t* q = qtask ? qtask + b0 * (int64_t)dag->n * A : nullptr;
        mp_status s;
        switch (A) {
            case 1: s = rep2_launch<1>(dag, base, emask, seed, sigma, r0 + b0, nb, cp + b0, sum + b0 * A, q, st); break;
            case 2: s = rep2_launch<2>(dag, base, emask, seed, sigma, r0 + b0, nb, cp + b0, sum + b0 * A, q, st); break;
            case 3: s = rep2_launch<3>(dag, base, emask, seed, sigma, r0 + b0, nb, cp + b0, sum + b0 * A, q, st); break;
            default: s = rep2_launch<4>(dag, base, emask, seed, sigma, r0 + b0, nb, cp + b0, sum + b0 * A, q, st); break;
        }
        if (s != MP_OK) return s;
    }
    return MP_OK;
}

}  // namespace mph
