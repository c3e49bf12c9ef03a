// path.cuh -- a3..a9 for one DAG: bottom-level (+ NOD), gain, score key, queues.
#pragma once
#include "build.cuh"

namespace mpk {

constexpr int MAX_ARCH = 8;
// Largest DAG whose bottom-levels live in one SM's shared memory.
constexpr int SMALL_CAP = 50 * 1024;

struct DurView {          // read-only duration table + enabled archs
    const float* dur;     // [n][A]
    int32_t A;
    uint32_t emask;
    int32_t wkind;        // node weight: 0 = min (c2), 1 = mean cost (N4, v1)
    int32_t W[MAX_ARCH];  // worker counts (mean cost only)
};

// w(v) = min over enabled a of delta(v,a) (reading c2), with the domain check
// (reading c20).  Sets `bad` on a domain violation or no enabled arch.
// N4 (v1): w(v) = (sum_a W_a delta(v,a)) / sum_a W_a over enabled a, in arch
// order, each op one RN binary64 op, rounded once to binary32.
MP_INLINE float task_weight(const DurView& d, int32_t v, bool& bad) {
    float w = __uint_as_float(0x7f800000u);
    bool any = false;
    double num = 0.0;
    int64_t den = 0;
    for (int a = 0; a < d.A; a++) {
        float x = canon_dur(__ldg(d.dur + (int64_t)v * d.A + a), bad);
        if (((d.emask >> a) & 1u) && !is_inf(x)) {
            any = true;
            w = x < w ? x : w;
            if (d.wkind) {
                num = __dadd_rn(num, __dmul_rn((double)d.W[a], (double)x));
                den += d.W[a];
            }
        }
    }
    if (!any) bad = true;
    if (any && d.wkind) w = __double2float_rn(__ddiv_rn(num, (double)den));
    return any ? w : 0.0f;
}

// ---- a4, small DAGs: one CTA, bottom-levels resident in shared memory ------------
// Levels are walked from the deepest (q-space is reverse level order) with one
// __syncthreads per level; bl(v) = w(v) + max bl(succ) with a single RN add.
// Nothing but the successors' bl depends on the previous level, so it is taken off
// the per-level chain: a prologue writes every w(v) into its slot sbl[q] (all loads
// in flight at once), and the next level's CSR slice -- its row offsets (rowq), node
// ids (nodeq) and successor positions (colq), contiguous ranges of q-space -- is
// copied into a shared-memory staging buffer by a TMA bulk copy (cp.async.bulk,
// mbarrier completion) while the current level computes: a staged level reads only
// shared memory, so it costs the shared-memory gathers + the barrier.  A level whose
// slice does not fit the buffer reads the CSR from L2 (prefetched there at start).
// (max is exact and order-free, so the bits are unchanged.)
MP_INLINE void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"((uint32_t)__cvta_generic_to_shared(bar)), "r"(count)
                 : "memory");
}
MP_INLINE void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(
                     (uint32_t)__cvta_generic_to_shared(bar)), "r"(bytes)
                 : "memory");
}
MP_INLINE void mbar_wait(uint64_t* bar, uint32_t phase) {
    const uint32_t a = (uint32_t)__cvta_generic_to_shared(bar);
    uint32_t done = 0;
    while (!done) {
        asm volatile(
            "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
            : "=r"(done)
            : "r"(a), "r"(phase)
            : "memory");
    }
}
// bulk copy global -> shared (16-byte aligned, size a multiple of 16), completion on bar
MP_INLINE void tma_bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     (uint32_t)__cvta_generic_to_shared(dst)),
                 "l"(src), "r"(bytes), "r"((uint32_t)__cvta_generic_to_shared(bar))
                 : "memory");
}

struct BlStage {          // one staged level: its CSR slice in the shared-memory arena
    int32_t qa, qb;       // the level's q range
    int32_t e0;           // rowq[qa]
    int32_t ok;           // staged (else read from global)
    int32_t orow, onod, ocol;   // arena offsets (int32 words) of rowq[qa], nodeq[qa], colq[e0]
    int32_t charge;       // arena words the level holds (its copies + any wrap-around gap)
};

// Producer side of a level-by-level walk that stages each level's CSR slice (rowq, nodeq,
// colq: contiguous q-space ranges) into a shared-memory ring arena with TMA bulk copies,
// up to BL_NB levels ahead (k_bl_small, k_rep2_bl's level mode).  One thread calls
// advance(r) at the start of level r (after the barrier that ended level r - 1): it
// releases level r - 1's space, then decides -- and, space permitting, stages -- the
// levels ahead; every level <= r + 1 is decided before it returns (the walk reads that
// level's record after the next barrier).  A level that does not fit is read from L2.
struct CsrStager {
    int32_t* arena;
    int32_t A;                       // arena words
    BlStage* stg;                    // [BL_NB]
    uint64_t* bars;                  // [BL_NB] mbarriers
    const int32_t* lq;               // level q starts (shared, when tab) else null
    const int32_t* le;               // level edge starts (shared, when tab) else null
    int32_t L;
    const int32_t *lvlq, *rowq, *nodeq, *colq;
    int32_t rn, head, used;          // producer state
    MP_INLINE void advance(int32_t r, int nb) {
        if (r > 0) used -= stg[(r - 1) % nb].charge;      // level r - 1 is done
        while (rn < L && rn <= r + nb - 1) {
            const int b = rn % nb;
            BlStage& S = stg[b];
            const int32_t qa = lq ? lq[rn] : __ldg(lvlq + rn), qb = lq ? lq[rn + 1] : __ldg(lvlq + rn + 1);
            const int32_t e0 = le ? le[rn] : __ldg(rowq + qa), e1 = le ? le[rn + 1] : __ldg(rowq + qb);
            // three 16-byte aligned copies: rowq[qa .. qb], nodeq[qa .. qb), colq[e0 .. e1)
            const int32_t ra = qa & ~3, rw = ((qb + 1 + 3) & ~3) - ra;
            const int32_t na = qa & ~3, nw = ((qb + 3) & ~3) - na;
            const int32_t ca = e0 & ~3, cw = ((e1 + 3) & ~3) - ca;
            const int32_t sz = rw + nw + cw;
            S.qa = qa;
            S.qb = qb;
            S.e0 = e0;
            S.ok = 0;
            S.charge = 0;
            if (sz > A) { rn++; continue; }                         // never fits: read from L2
            const int32_t start = head + sz <= A ? head : 0;
            const int32_t charge = head + sz <= A ? sz : (A - head) + sz;
            if (used + charge > A) {
                if (rn <= r + 1) { rn++; continue; }                 // due now: read from L2
                break;                                               // wait for space
            }
            head = start + sz;
            used += charge;
            S.charge = charge;
            S.orow = start + (qa - ra);
            S.onod = start + rw + (qa - na);
            S.ocol = start + rw + nw + (e0 - ca);
            int32_t* dst = arena + start;
            mbar_expect_tx(&bars[b], (uint32_t)sz * 4u);
            tma_bulk_g2s(dst, rowq + ra, (uint32_t)rw * 4u, &bars[b]);
            tma_bulk_g2s(dst + rw, nodeq + na, (uint32_t)nw * 4u, &bars[b]);
            if (cw > 0) tma_bulk_g2s(dst + rw + nw, colq + ca, (uint32_t)cw * 4u, &bars[b]);
            S.ok = 1;
            rn++;
        }
    }
};

constexpr int BL_NB = 16;       // k_bl_small: levels staged ahead of the walk, at most
constexpr int BL_LTAB = 4096;   // level-bound table in shared memory for L < BL_LTAB

// GBL = false: bl of every position in shared memory (n <= SMALL_CAP).  GBL = true
// (k_bl_one, medium DAGs with moderate edge counts): the same single-CTA walk with bl in
// a q-indexed global array `blg` (L2-resident; the block barrier orders a level's stores
// before the next level's loads), so the whole shared memory holds the staging arena.
template <bool GBL>
__global__ void __launch_bounds__(1024) k_bl_small(int32_t L, const int32_t* __restrict__ lvlq,
                                                   const int32_t* __restrict__ nodeq,
                                                   const int32_t* __restrict__ rowq,
                                                   const int32_t* __restrict__ colq, DurView d, float* bl,
                                                   float* cp, uint32_t* err, int32_t arena_words, float* blg) {
    extern __shared__ __align__(16) float sdyn[];
    float* sbl = GBL ? blg : sdyn;
    __shared__ __align__(8) uint64_t bars[BL_NB];
    __shared__ BlStage stg[BL_NB];
    bool bad = false;
    float cpm = 0.0f;
    const int32_t t = (int32_t)threadIdx.x;
    const int32_t nq = __ldg(lvlq + L);
    // after sbl: the level-bound table (q start and edge start of every level, when L is
    // small enough), then the staging arena (arena_words int32, a ring: levels are staged
    // in order and released in order; 0: no staging)
    const bool tab = L < BL_LTAB;
    int32_t* lq = reinterpret_cast<int32_t*>(GBL ? sdyn : sdyn + ((nq + 3) & ~3));   // [L + 1] q starts
    int32_t* le = lq + (tab ? ((L + 1 + 3) & ~3) : 0);                      // [L + 1] edge starts
    int32_t* arena = le + (tab ? ((L + 1 + 3) & ~3) : 0);
    const int32_t A = arena_words & ~3;
    const int32_t prod = (int32_t)blockDim.x - 1;   // producer thread: the last one
    CsrStager stager{arena, A, stg, bars, tab ? lq : nullptr, tab ? le : nullptr, L, lvlq, rowq, nodeq, colq, 0, 0, 0};
    {
        // the level walk reads every successor id and row bound once, a level at a time:
        // pull them into L2 now (one prefetch per 128-byte line) so no level waits on HBM
        const int32_t E = __ldg(rowq + nq);
        for (int32_t e = t * 32; e < E; e += blockDim.x * 32) asm volatile("prefetch.global.L2 [%0];" ::"l"(colq + e));
        for (int32_t q = t * 32; q <= nq; q += blockDim.x * 32) asm volatile("prefetch.global.L2 [%0];" ::"l"(rowq + q));
    }
    if (t == prod) {
        for (int b = 0; b < BL_NB; b++) mbar_init(&bars[b], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (tab)
        for (int32_t r = t; r <= L; r += blockDim.x) {
            const int32_t q = __ldg(lvlq + r);
            lq[r] = q;
            le[r] = __ldg(rowq + q);
        }
    {   // weights: the ids of 8 positions per thread first, then their durations (loads in flight)
        constexpr int U = 8;
        const int32_t stride = (int32_t)blockDim.x;
        for (int32_t q0 = t; q0 < nq; q0 += U * stride) {
            int32_t vv[U];
#pragma unroll
            for (int u = 0; u < U; u++) vv[u] = q0 + u * stride < nq ? __ldg(nodeq + q0 + u * stride) : -1;
#pragma unroll
            for (int u = 0; u < U; u++)
                if (vv[u] >= 0) sbl[q0 + u * stride] = task_weight(d, vv[u], bad);
        }
    }
    __syncthreads();
    if (t == prod && A > 0) stager.advance(-1, BL_NB);
    if (t == prod && A <= 0)
        for (int b = 0; b < BL_NB; b++) stg[b].ok = 0;
    __syncthreads();   // stg[] visible to every thread
    uint32_t ph = 0u;  // bit b: parity of buffer b's next phase
    for (int32_t r = 0; r < L; r++) {
        const int b = r % BL_NB;
        if (t == prod && A > 0) stager.advance(r, BL_NB);
        const BlStage S = stg[b];
        const int32_t qa = tab ? lq[r] : __ldg(lvlq + r), qb = tab ? lq[r + 1] : __ldg(lvlq + r + 1);
        if (A > 0 && S.ok) {
            mbar_wait(&bars[b], (ph >> b) & 1u);
            const int32_t* srow = arena + S.orow - qa;       // srow[q] = rowq[q]
            const int32_t* snod = arena + S.onod - qa;       // snod[q] = nodeq[q]
            const int32_t* scol = arena + S.ocol - S.e0;     // scol[e] = colq[e]
            for (int32_t q = qa + t; q < qb; q += blockDim.x) {
                int32_t e = srow[q];
                const int32_t e1 = srow[q + 1];
                const int32_t v = snod[q];
                float m = 0.0f;  // bl >= 0, and w + 0 = w: same as "bl = w without successors"
                if constexpr (GBL) {   // bl in L2: a high out-degree node keeps 16 gathers in flight
                    // (hier 0.61 -> 0.55 ms, lu64 0.35 -> 0.34; the shared-memory walk of c2 gains nothing)
                    for (; e + 16 <= e1; e += 16) {
                        float g[16];
#pragma unroll
                        for (int u = 0; u < 16; u++) g[u] = sbl[scol[e + u]];
#pragma unroll
                        for (int u = 0; u < 16; u++) m = fmaxf(m, g[u]);
                    }
                }
                for (; e + 4 <= e1; e += 4)
                    m = fmaxf(m, fmaxf(fmaxf(sbl[scol[e]], sbl[scol[e + 1]]), fmaxf(sbl[scol[e + 2]], sbl[scol[e + 3]])));
                for (; e < e1; e++) m = fmaxf(m, sbl[scol[e]]);
                const float bb = __fadd_rn(sbl[q], m);
                sbl[q] = bb;
                bl[v] = bb;
                cpm = fmaxf(cpm, bb);
            }
            ph ^= 1u << b;
        } else {
            for (int32_t q = qa + t; q < qb; q += blockDim.x) {
                int32_t e = __ldg(rowq + q);
                const int32_t e1 = __ldg(rowq + q + 1);
                const int32_t v = __ldg(nodeq + q);
                float m = 0.0f;
                for (; e + 4 <= e1; e += 4) {
                    const int32_t c0 = __ldg(colq + e), c1 = __ldg(colq + e + 1);
                    const int32_t c2 = __ldg(colq + e + 2), c3 = __ldg(colq + e + 3);
                    m = fmaxf(m, fmaxf(fmaxf(sbl[c0], sbl[c1]), fmaxf(sbl[c2], sbl[c3])));
                }
                for (; e < e1; e++) m = fmaxf(m, sbl[__ldg(colq + e)]);
                const float bb = __fadd_rn(sbl[q], m);
                sbl[q] = bb;
                bl[v] = bb;
                cpm = fmaxf(cpm, bb);
            }
        }
        __syncthreads();
    }
    cpm = warp_max(cpm);
    if ((threadIdx.x & 31) == 0) atomicMax((uint32_t*)cp, f2u(cpm));
    if (__any_sync(0xffffffffu, bad) && (threadIdx.x & 31) == 0) atomicOr(err, ERR_DOMAIN_BIT);
}

// ---- a4, wide and shallow DAGs: level-synchronous, edge-parallel -----------------------
// For DAGs with few, very wide levels (an FMM octree: 13 levels, up to 343k tasks and
// millions of edges per level) the work of a level, not its latency, is the cost, and a
// high out-degree node must not serialise on one warp.  A level's successor positions
// are one contiguous colq range; every thread of a cooperative grid takes an equal
// contiguous share of it, max-reduces the successors' bl of the runs of edges that
// belong to one node, and merges each run's maximum into the node's slot with an
// atomicMax on the float bits (bl >= 0: integer order = float order, exact).  A grid
// barrier; then one thread per node adds w(v) (the same single RN add); a grid barrier.
#ifndef MP_BL_WIDE_MIN
#define MP_BL_WIDE_MIN 16384
#endif
constexpr int32_t BL_WIDE_MIN = MP_BL_WIDE_MIN;   // mean level width (n / L) that selects k_bl_wide
constexpr int BL_WIDE_THREADS = 512;
#ifndef MP_BL_ONE_MAX_E
#define MP_BL_ONE_MAX_E (1 << 20)
#endif
constexpr int64_t BL_ONE_MAX_E = MP_BL_ONE_MAX_E;   // k_bl_one: one SM's issue budget for the edges

__global__ void __launch_bounds__(BL_WIDE_THREADS) k_bl_wide(int32_t L, const int32_t* __restrict__ lvlq,
                                                              const int32_t* __restrict__ nodeq,
                                                              const int32_t* __restrict__ rowq,
                                                              const int32_t* __restrict__ colq, DurView d,
                                                              uint32_t* blq, uint32_t* mq, float* bl, float* cp,
                                                              unsigned* bar, uint32_t* err) {
    const int64_t gtid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t T = (int64_t)gridDim.x * blockDim.x;
    bool bad = false;
    float cpm = 0.0f;
    unsigned epoch = 0;
    for (int32_t r = 0; r < L; r++) {
        const int32_t qa = __ldg(lvlq + r), qb = __ldg(lvlq + r + 1);
        const int32_t ea = __ldg(rowq + qa), eb = __ldg(rowq + qb);
        const int64_t Er = (int64_t)eb - ea;
        if (Er > 0) {
            int64_t C = (Er + T - 1) / T;
            if (C < 4) C = 4;
            const int64_t e0l = ea + gtid * C;
            if (e0l < eb) {
                const int32_t e0 = (int32_t)e0l, e1 = (int32_t)(e0l + C < eb ? e0l + C : eb);
                // owner of e0: the last position q in [qa, qb) with rowq[q] <= e0
                int32_t lo = qa, hi = qb - 1;
                while (lo < hi) {
                    const int32_t mid = (lo + hi + 1) >> 1;
                    if (__ldg(rowq + mid) <= e0) lo = mid;
                    else hi = mid - 1;
                }
                int32_t q = lo, nb = __ldg(rowq + q + 1);
                uint32_t m = 0u;
                for (int32_t eb = e0; eb < e1; eb += 8) {
                    // 8 successors' bl in flight, then the runs they close
                    uint32_t x[8];
#pragma unroll
                    for (int u = 0; u < 8; u++) x[u] = eb + u < e1 ? __ldcg(blq + __ldg(colq + eb + u)) : 0u;
#pragma unroll
                    for (int u = 0; u < 8; u++) {
                        const int32_t e = eb + u;
                        if (e >= e1) break;
                        if (e == nb) {   // the run of q ends: merge it, move to the owner of e
                            atomicMax(mq + q, m);
                            m = 0u;
                            do { q++; nb = __ldg(rowq + q + 1); } while (nb == e);
                        }
                        m = x[u] > m ? x[u] : m;
                    }
                }
                atomicMax(mq + q, m);
            }
        }
        grid_barrier(bar, epoch);
        for (int64_t q = qa + gtid; q < qb; q += T) {
            const int32_t v = __ldg(nodeq + q);
            const float b = __fadd_rn(task_weight(d, v, bad), u2f(__ldcg(mq + q)));
            blq[q] = f2u(b);
            bl[v] = b;
            cpm = fmaxf(cpm, b);
        }
        grid_barrier(bar, epoch);
    }
    cpm = warp_max(cpm);
    if ((threadIdx.x & 31) == 0) atomicMax((uint32_t*)cp, f2u(cpm));
    if (__any_sync(0xffffffffu, bad) && (threadIdx.x & 31) == 0) atomicOr(err, ERR_DOMAIN_BIT);
}

// ---- a4, large DAGs: barrier-free dataflow ------------------------------------------
// Padded q-space: every level is rounded up to a multiple of 32 positions, so a
// warp's chunk of 32 positions lies in one level and never depends on itself.
// Warps take chunks in increasing order from a ticket (deepest level first);
// a chunk's successors are in strictly deeper levels = earlier chunks, already
// taken by running warps, so spinning on them cannot deadlock.  The value is its
// own ready flag (0xFFFFFFFF = not yet; bl is never NaN).  Successor loads are
// edge-parallel across the warp (coalesced col reads) and max-reduced per node
// in shared memory.  A chunk loads ALL its successors' words as soon as it is
// taken (long before most are published), reduces the published ones and lists
// the rest per warp; the list is then polled with all its loads in flight, so a
// chunk completes about one L2 round trip after its last successor is published
// (walking the edges batch by batch instead cost one round trip per batch:
// c3 1.10 -> 0.51 ms, c4 1.43 -> 0.71 ms).
constexpr int FLOW_THREADS = 256;
constexpr uint32_t NOT_READY = 0xFFFFFFFFu;
#ifndef MP_FLOW_PF
#define MP_FLOW_PF 2
#endif
#ifndef MP_FLOW_MINB
#define MP_FLOW_MINB 8
#endif
constexpr int FLOW_PF = MP_FLOW_PF;   // edges per lane whose loads k_bl_flow issues together
constexpr int FLOW_PCAP = 1024;      // pending-successor list per warp (4 B position + 1 B owner)
constexpr int FLOW_PPL = 8;          // pending entries per lane polled together

__global__ void __launch_bounds__(FLOW_THREADS, MP_FLOW_MINB) k_bl_flow(int32_t nchunks, const int32_t* __restrict__ nodep,
                                                          const int32_t* __restrict__ rowp,
                                                          const int32_t* __restrict__ colp, DurView d,
                                                          uint32_t* blp, float* bl, float* cp, uint32_t* ticket,
                                                          uint32_t* err) {
    __shared__ uint32_t smax[FLOW_THREADS / 32][32];
    __shared__ int32_t srow[FLOW_THREADS / 32][33];
    __shared__ int32_t spend[FLOW_THREADS / 32][FLOW_PCAP];
    __shared__ uint8_t sown[FLOW_THREADS / 32][FLOW_PCAP];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    bool bad = false;
    float cpm = 0.0f;
    while (true) {
        uint32_t c = 0;
        if (lane == 0) c = atomicAdd(ticket, 1u);
        c = __shfl_sync(0xffffffffu, c, 0);
        if (c >= (uint32_t)nchunks) break;
        const int32_t p = (int32_t)c * 32 + lane;
        const int32_t v = __ldg(nodep + p);
        const int32_t e0 = __ldg(rowp + p);
        srow[w][lane] = e0;
        if (lane == 31) srow[w][32] = __ldg(rowp + p + 1);
        smax[w][lane] = 0u;
        const float wt = v >= 0 ? task_weight(d, v, bad) : 0.0f;
        __syncwarp();
        const int32_t E0 = srow[w][0], E1 = srow[w][32];
        // owner of edge e: largest i with srow[i] <= e
        auto owner = [&](int32_t e) -> int {
            int lo = 0, hi = 31;
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (srow[w][mid] <= e) lo = mid;
                else hi = mid - 1;
            }
            return lo;
        };
        // every edge of the chunk is loaded first (successor position, then its bl word, FLOW_PF
        // batches of 32 in flight per lane); published words are reduced at once and the others
        // are listed (position, owner lane) in the warp's pending list, which is then polled
        // as a whole -- so once the last successor is published the chunk finishes one round
        // trip later instead of walking its remaining batches (list full: poll in place)
        uint32_t npend = 0;
        for (int32_t eb = E0; eb < E1; eb += 32 * FLOW_PF) {
            int32_t spk[FLOW_PF];
            uint32_t xs[FLOW_PF];
#pragma unroll
            for (int k = 0; k < FLOW_PF; k++) {
                const int32_t e = eb + lane + 32 * k;
                spk[k] = e < E1 ? __ldg(colp + e) : -1;
            }
#pragma unroll
            for (int k = 0; k < FLOW_PF; k++) xs[k] = spk[k] >= 0 ? ld_relaxed(blp + spk[k]) : 0u;
#pragma unroll
            for (int k = 0; k < FLOW_PF; k++) {
                const int own = spk[k] >= 0 ? owner(eb + lane + 32 * k) : 0;
                bool nr = spk[k] >= 0 && xs[k] == NOT_READY;
                const uint32_t bal = __ballot_sync(0xffffffffu, nr);
                const uint32_t at = npend + __popc(bal & ((1u << lane) - 1u));
                if (nr && at < (uint32_t)FLOW_PCAP) {
                    spend[w][at] = spk[k];
                    sown[w][at] = (uint8_t)own;
                    nr = false;
                }
                npend += __popc(bal);
                if (nr) {   // list full: wait for this one here
                    do { xs[k] = ld_relaxed(blp + spk[k]); } while (xs[k] == NOT_READY);
                }
                if (spk[k] >= 0 && xs[k] != NOT_READY) atomicMax(&smax[w][own], xs[k]);
            }
        }
        npend = min(npend, (uint32_t)FLOW_PCAP);
        __syncwarp();
        // poll the pending list: each lane owns entries lane, lane + 32, ... (all in flight)
        for (uint32_t i0 = 0; i0 < npend; i0 += 32 * FLOW_PPL) {
            int32_t ent[FLOW_PPL];
            uint32_t xv[FLOW_PPL];
#pragma unroll
            for (int k = 0; k < FLOW_PPL; k++) {
                const uint32_t i = i0 + lane + 32 * k;
                ent[k] = i < npend ? spend[w][i] : -1;
            }
            while (true) {
                bool waiting = false;
#pragma unroll
                for (int k = 0; k < FLOW_PPL; k++)
                    if (ent[k] >= 0) {
                        xv[k] = ld_relaxed(blp + ent[k]);
                        if (xv[k] != NOT_READY) {
                            atomicMax(&smax[w][sown[w][i0 + lane + 32 * k]], xv[k]);
                            ent[k] = -1;
                        } else {
                            waiting = true;
                        }
                    }
                if (!waiting) break;
            }
        }
        __syncwarp();
        if (v >= 0) {
            const float b = __fadd_rn(wt, u2f(smax[w][lane]));
            st_relaxed(blp + p, f2u(b));
            bl[v] = b;
            cpm = fmaxf(cpm, b);
        }
        __syncwarp();
    }
    cpm = warp_max(cpm);
    if (lane == 0) atomicMax((uint32_t*)cp, f2u(cpm));
    if (__any_sync(0xffffffffu, bad) && lane == 0) atomicOr(err, ERR_DOMAIN_BIT);
}

// ---- a5: NOD (eq. 2) -----------------------------------------------------------------
// indeg_a(s) = |{p in lambda^-(s) : p enabled on a}|
// (N4, v3: with `done`, completed predecessors leave lambda^-)
__global__ void k_nod_indeg(int32_t n, const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ col,
                            DurView d, const uint8_t* __restrict__ done, int32_t* inda) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n; u += (int64_t)gridDim.x * blockDim.x) {
        if (done && done[u]) continue;
        uint32_t en = 0;
        for (int a = 0; a < d.A; a++)
            if (((d.emask >> a) & 1u) && !is_inf(__ldg(d.dur + u * d.A + a))) en |= 1u << a;
        if (!en) continue;
        for (int32_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) {
            int32_t s = col[e];
            for (int a = 0; a < d.A; a++)
                if ((en >> a) & 1u) atomicAdd(&inda[(int64_t)s * d.A + a], 1);
        }
    }
}

// NOD_a(t) = sum over enabled successors s of floor(2^32 / indeg_a(s)) (exact uint64),
// converted once (RN) and scaled by 2^-32 (exact); 0 where (t,a) is not enabled.
// (N4, v3: with `done`, completed tasks and successors score / count 0)
__global__ void k_nod_sum(int32_t n, const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ col,
                          DurView d, const uint8_t* __restrict__ done, const int32_t* __restrict__ inda, float* nod) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
        const bool tdone = done && done[t];
        for (int a = 0; a < d.A; a++) {
            float out = 0.0f;
            if (!tdone && ((d.emask >> a) & 1u) && !is_inf(__ldg(d.dur + t * d.A + a))) {
                uint64_t acc = 0;
                for (int32_t e = row_ptr[t]; e < row_ptr[t + 1]; e++) {
                    int32_t s = col[e];
                    if (((d.emask >> a) & 1u) && !is_inf(__ldg(d.dur + (int64_t)s * d.A + a)) && !(done && done[s]))
                        acc += 4294967296ull / (uint64_t)inda[(int64_t)s * d.A + a];
                }
                out = __fmul_rn(__ull2float_rn(acc), 0x1p-32f);
            }
            nod[t * d.A + a] = out;
        }
    }
}

// ---- a6: gain (eq. 1) ------------------------------------------------------------------
// pass 1: flags and hd(a) = max |d(t,a)| (non-negative floats ordered as uint32)
__global__ void k_aff_hd(int32_t n, DurView d, uint8_t* flags, uint32_t* hdbits, uint32_t* err) {
    bool bad = false;
    uint32_t hl[MAX_ARCH];
    for (int a = 0; a < MAX_ARCH; a++) hl[a] = 0;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
        float x[MAX_ARCH];
        int k = 0;
        float w = __uint_as_float(0x7f800000u);
        uint32_t en = 0;
        for (int a = 0; a < d.A; a++) {
            x[a] = canon_dur(d.dur[t * d.A + a], bad);
            if (((d.emask >> a) & 1u) && !is_inf(x[a])) {
                en |= 1u << a;
                k++;
                w = x[a] < w ? x[a] : w;
            }
        }
        if (!k) bad = true;
        for (int a = 0; a < d.A; a++) {
            uint8_t f = 0;
            if ((en >> a) & 1u) {
                f = 1 | (x[a] == w ? 2 : 0);
                if (k >= 2) {
                    float ref = __uint_as_float(0x7f800000u);
                    for (int b = 0; b < d.A; b++)
                        if (b != a && ((en >> b) & 1u)) ref = x[b] < ref ? x[b] : ref;
                    float dd = __fsub_rn(ref, x[a]);
                    uint32_t ab = f2u(fabsf(dd));
                    hl[a] = ab > hl[a] ? ab : hl[a];
                }
            }
            flags[t * d.A + a] = f;
        }
    }
    for (int a = 0; a < d.A; a++) {
        uint32_t v = warp_max(hl[a]);
        if ((threadIdx.x & 31) == 0 && v) atomicMax(&hdbits[a], v);
    }
    if (__any_sync(0xffffffffu, bad) && (threadIdx.x & 31) == 0) atomicOr(err, ERR_DOMAIN_BIT);
}

// pass 2: gain = 1 (one enabled arch) | 0.5 (hd = 0) | (d + hd) / (hd + hd)
__global__ void k_aff_gain(int32_t n, DurView d, const uint8_t* flags, const uint32_t* hdbits, float* gain,
                           float* hd_out) {
    if (blockIdx.x == 0 && threadIdx.x < d.A) hd_out[threadIdx.x] = u2f(hdbits[threadIdx.x]);
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
        float x[MAX_ARCH];
        uint32_t en = 0;
        int k = 0;
        for (int a = 0; a < d.A; a++) {
            bool dummy = false;
            x[a] = canon_dur(d.dur[t * d.A + a], dummy);
            if (flags[t * d.A + a] & 1) {
                en |= 1u << a;
                k++;
            }
        }
        for (int a = 0; a < d.A; a++) {
            float g = 0.0f;
            if ((en >> a) & 1u) {
                float h = u2f(hdbits[a]);
                if (k == 1) g = 1.0f;
                else if (h == 0.0f) g = 0.5f;
                else {
                    float ref = __uint_as_float(0x7f800000u);
                    for (int b = 0; b < d.A; b++)
                        if (b != a && ((en >> b) & 1u)) ref = x[b] < ref ? x[b] : ref;
                    float dd = __fsub_rn(ref, x[a]);
                    g = __fdiv_rn(__fadd_rn(dd, h), __fadd_rn(h, h));
                }
            }
            gain[t * d.A + a] = g;
        }
    }
}

// ---- a7: crit_n and key -------------------------------------------------------------------
__global__ void k_crit_max(int64_t cnt, int32_t A, int32_t kind, const float* crit, const uint8_t* flags,
                           uint32_t* maxbits) {
    uint32_t ml[MAX_ARCH];
    for (int a = 0; a < MAX_ARCH; a++) ml[a] = 0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cnt; i += (int64_t)gridDim.x * blockDim.x) {
        float c = crit[i];
        if (kind == 0) {
            if (c > 0.0f) ml[0] = f2u(c) > ml[0] ? f2u(c) : ml[0];
        } else {
            int a = (int)(i % A);
            if ((flags[i] & 1) && c > 0.0f) {
                for (int b = 0; b < MAX_ARCH; b++)
                    if (b == a) ml[b] = f2u(c) > ml[b] ? f2u(c) : ml[b];
            }
        }
    }
    int na = kind == 0 ? 1 : A;
    for (int a = 0; a < na; a++) {
        uint32_t v = warp_max(ml[a]);
        if ((threadIdx.x & 31) == 0 && v) atomicMax(&maxbits[a], v);
    }
}

MP_INLINE uint64_t make_key(float g, float c) {
    return ((uint64_t)(ONE_BITS - f2u(g)) << 32) | (uint64_t)(ONE_BITS - f2u(c));
}

__global__ void k_score(int32_t n, int32_t A, int32_t kind, const float* crit, const float* gain,
                        const uint8_t* flags, const uint32_t* maxbits, float* crit_norm, uint64_t* key) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
        float cn0 = 0.0f;
        if (kind == 0) {
            float mx = u2f(maxbits[0]);
            cn0 = mx > 0.0f ? __fdiv_rn(crit[t], mx) : 0.0f;
            crit_norm[t] = cn0;
        }
        for (int a = 0; a < A; a++) {
            int64_t i = t * A + a;
            bool en = flags[i] & 1;
            float c = cn0;
            if (kind == 1) {
                float mx = u2f(maxbits[a]);
                c = (en && mx > 0.0f) ? __fdiv_rn(crit[i], mx) : 0.0f;
                crit_norm[i] = c;
            }
            key[i] = en ? make_key(gain[i], c) : ~0ull;
        }
    }
}

// ---- a8/a9: queues -------------------------------------------------------------------------
__global__ void k_copy_len(const int32_t* total, int64_t* len) { *len = *total; }

__global__ void k_blocked(int32_t n, const int32_t* row_ptr, const int32_t* col, const uint8_t* done,
                          uint8_t* blocked) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n; u += (int64_t)gridDim.x * blockDim.x) {
        if (done[u]) continue;
        for (int32_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) blocked[col[e]] = 1;
    }
}

// membership flags in (arch, id) order + per-arch count and exact brw (blockIdx.y = arch)
__global__ void k_q_member(int32_t n, int32_t A, const uint8_t* flags, const uint8_t* done,
                           const uint8_t* blocked, const float* dur, int32_t* memb, int32_t* counts,
                           unsigned long long* brw) {
    const int a = blockIdx.y;
    int32_t cnt = 0;
    uint64_t lo = 0, hi = 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t nround = ((int64_t)n + stride - 1) / stride;
    for (int64_t it = 0; it < nround; it++) {
        int64_t t = it * stride + blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
        if (t < n) {
            uint8_t f = flags[t * A + a];
            bool m = (f & 1) && (!done || (!done[t] && !blocked[t]));
            memb[(int64_t)a * n + t] = m ? 1 : 0;
            if (m) {
                cnt++;
                if (f & 2) {
                    bool dummy = false;
                    uint64_t l, h;
                    fixed64(canon_dur(dur[t * A + a], dummy), l, h);
                    add128(lo, hi, l, h);
                }
            }
        }
    }
    warp_sum128(lo, hi);
    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
    if ((threadIdx.x & 31) == 0) {
        if (cnt) atomicAdd(&counts[a], cnt);
        atomic_add128(brw + 2 * a, lo, hi);
    }
}

__global__ void k_q_scatter(int32_t n, int32_t A, const uint64_t* key, const int32_t* memb, const int32_t* pos,
                            uint64_t* skey, uint32_t* sval) {
    const int a = blockIdx.y;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
        int64_t i = (int64_t)a * n + t;
        if (!memb[i]) continue;
        uint64_t k = key[t * A + a];
        uint64_t gc = k >> 32, cc = k & 0xffffffffull;  // both <= 0x3F800000 < 2^30
        int32_t p = pos[i];
        skey[p] = ((uint64_t)a << 60) | (gc << 30) | cc;
        sval[p] = (uint32_t)t;
    }
}

__global__ void k_q_out(const SortPlan* plan, const uint32_t* vb0, const uint32_t* vb1, const int32_t* total, int32_t A,
                        const int32_t* counts, const unsigned long long* brw, int64_t* qptr, int32_t* qtask,
                        mp_queue_summary* sum) {
    const int32_t Q = *total;
    const uint32_t* v = Q > 0 ? (plan->final_sel ? vb1 : vb0) : nullptr;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < Q; i += (int64_t)gridDim.x * blockDim.x)
        qtask[i] = (int32_t)v[i];
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        int64_t off = 0;
        for (int a = 0; a < A; a++) {
            qptr[a] = off;
            mp_queue_summary s;
            s.count = counts[a];
            s.head = counts[a] > 0 ? (int32_t)v[off] : -1;
            s.brw_lo = brw[2 * a];
            s.brw_hi = (int64_t)brw[2 * a + 1];
            s.brw = u128_to_double_scaled(brw[2 * a], brw[2 * a + 1]);
            sum[a] = s;
            off += counts[a];
        }
        qptr[A] = off;
    }
}

}  // namespace mpk

namespace mph {

inline mp_status check_arch(int32_t A, const int32_t* h_workers) {
    if (A < 1 || A > mpk::MAX_ARCH) return fail(MP_ERR_ARG, "n_arch %d outside [1, 8]", A);
    if (!h_workers) return fail(MP_ERR_ARG, "h_workers is NULL");
    return MP_OK;
}

inline mp_status bottom_level(mp_dag* dag, int32_t A, const float* dur, const int32_t* h_workers, float* bl,
                              float* cp, float* nod, cudaStream_t st, int32_t wkind = 0) {
    using namespace mpk;
    if (!dag) return fail(MP_ERR_ARG, "dag is NULL");
    MP_TRY(check_arch(A, h_workers));
    if (wkind != 0 && wkind != 1) return fail(MP_ERR_ARG, "unknown weight kind %d", wkind);
    if (!cp || (dag->n > 0 && (!dur || !bl))) return fail(MP_ERR_ARG, "NULL buffer");
    DurView d{dur, A, enabled_mask(A, h_workers)};
    d.wkind = wkind;
    for (int a = 0; a < A; a++) d.W[a] = h_workers[a] > 0 ? h_workers[a] : 0;
    MP_CUDA(cudaMemsetAsync(cp, 0, 4, st));
    const int32_t n = dag->n;
    if (n == 0) return MP_OK;
    if (n <= SMALL_CAP) {
        // bl in shared memory; what is left of the opt-in maximum holds two CSR staging buffers
        int optin = 0;
        MP_CUDA(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dag->device));
        const size_t sbytes = (size_t)((n + 3) & ~3) * 4;
        const size_t tbytes = dag->L < BL_LTAB ? (size_t)2 * (((dag->L + 1) + 3) & ~3) * 4 : 0;   // level table
        const int64_t avail = (int64_t)optin - (int64_t)sbytes - (int64_t)tbytes - 1024;   // static smem + slack
        const int32_t arena_words = avail >= 4096 ? (int32_t)((avail / 4) & ~3) : 0;
        const size_t smem = sbytes + tbytes + (size_t)arena_words * 4;
        static std::atomic<uint64_t> attr{0};
        if (first_on_device(attr))
            MP_CUDA(cudaFuncSetAttribute(k_bl_small<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, optin - 1024));
        MP_LAUNCH(k_bl_small<false>, 1, 1024, smem, st, dag->L, dag->lvlq, dag->nodeq, dag->rowq, dag->colq, d, bl, cp,
                  dag->err, arena_words, (float*)nullptr);
    } else if (dag->E <= BL_ONE_MAX_E && (int64_t)n < (int64_t)BL_WIDE_MIN * dag->L) {
        // medium DAG, moderate edge count: one CTA, bl in L2, CSR staged in shared memory
        int optin = 0;
        MP_CUDA(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dag->device));
        MP_TRY(ensure_ws(dag, align256((size_t)n * 4), st));
        float* blg = (float*)dag->ws;
        const size_t tbytes = dag->L < BL_LTAB ? (size_t)2 * (((dag->L + 1) + 3) & ~3) * 4 : 0;
        const int64_t avail = (int64_t)optin - (int64_t)tbytes - 1024;
        const int32_t arena_words = avail >= 4096 ? (int32_t)((avail / 4) & ~3) : 0;
        const size_t smem = tbytes + (size_t)arena_words * 4;
        static std::atomic<uint64_t> attr1{0};
        if (first_on_device(attr1))
            MP_CUDA(cudaFuncSetAttribute(k_bl_small<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, optin - 1024));
        mph::ProfScope ps("k_bl_one", st);
        k_bl_small<true><<<1, 1024, smem, st>>>(dag->L, dag->lvlq, dag->nodeq, dag->rowq, dag->colq, d, bl, cp, dag->err,
                                               arena_words, blg);
    } else if (dag->L > 0 && (int64_t)n >= (int64_t)BL_WIDE_MIN * dag->L) {
        // few, wide levels: level-synchronous edge-parallel cooperative kernel
        const int32_t nq = n;
        MP_TRY(ensure_ws(dag, 2 * align256((size_t)nq * 4), st));
        uint32_t* blq = (uint32_t*)dag->ws;
        uint32_t* mq = blq + align256((size_t)nq * 4) / 4;
        MP_CUDA(cudaMemsetAsync(mq, 0, (size_t)nq * 4, st));
        MP_CUDA(cudaMemsetAsync(dag->b_bar, 0, 64 * 4, st));
        int bps = 0;
        MP_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_bl_wide, BL_WIDE_THREADS, 0));
        // 4 CTAs of 512 per SM (measured: c4fmm 0.35 ms vs 0.39 ms with one CTA of 1024 per SM)
        const int g = std::max(1, std::min(bps, 4) * dag->num_sms);
        int32_t Lv = dag->L;
        const int32_t *lvlq = dag->lvlq, *nodeq = dag->nodeq, *rowq = dag->rowq, *colq = dag->colq;
        unsigned* bar = (unsigned*)dag->b_bar;
        uint32_t* err = dag->err;
        void* args[] = {&Lv, &lvlq, &nodeq, &rowq, &colq, &d, &blq, &mq, &bl, &cp, &bar, &err};
        mph::ProfScope ps("k_bl_wide", st);
        MP_CUDA(cudaLaunchCooperativeKernel((const void*)k_bl_wide, dim3((unsigned)g), dim3(BL_WIDE_THREADS), args, 0, st));
    } else {
        size_t need = align256((size_t)dag->P * 4);
        MP_TRY(ensure_ws(dag, need, st));
        uint32_t* blp = (uint32_t*)dag->ws;
        MP_CUDA(cudaMemsetAsync(blp, 0xff, (size_t)dag->P * 4, st));
        MP_CUDA(cudaMemsetAsync(dag->tickets + 62, 0, 4, st));
        int bps = 0;
        MP_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_bl_flow, FLOW_THREADS, 0));
        int32_t nchunks = dag->P / 32;
        // 4 blocks (32 warps) per SM: fewer spinning warps measured faster on c4 than full occupancy
#ifndef MP_FLOW_BPS
#define MP_FLOW_BPS 4
#endif
        if (bps > MP_FLOW_BPS) bps = MP_FLOW_BPS;
        int64_t g = (int64_t)bps * dag->num_sms;
        int64_t want = ((int64_t)nchunks + FLOW_THREADS / 32 - 1) / (FLOW_THREADS / 32);
        if (want < g) g = want;
        if (g < 1) g = 1;
        MP_LAUNCH(k_bl_flow, (unsigned)g, FLOW_THREADS, 0, st, nchunks, dag->nodep, dag->rowp, dag->colp, d, blp, bl, cp,
                                                        dag->tickets + 62, dag->err);
    }
    MP_CUDA(cudaGetLastError());
    if (nod) {
        size_t need = align256((size_t)n * A * 4);
        MP_TRY(ensure_ws(dag, need, st));
        int32_t* inda = (int32_t*)dag->ws;
        MP_CUDA(cudaMemsetAsync(inda, 0, (size_t)n * A * 4, st));
        MP_LAUNCH(k_nod_indeg, grid_for(n), 256, 0, st, n, dag->row_ptr, dag->col, d, nullptr, inda);
        MP_LAUNCH(k_nod_sum, grid_for(n), 256, 0, st, n, dag->row_ptr, dag->col, d, nullptr, inda, nod);
        MP_CUDA(cudaGetLastError());
    }
    return MP_OK;
}

inline mp_status affinity(mp_dag* dag, int32_t A, const float* dur, const int32_t* h_workers, float* gain,
                          float* hd, uint8_t* flags, cudaStream_t st) {
    using namespace mpk;
    if (!dag) return fail(MP_ERR_ARG, "dag is NULL");
    MP_TRY(check_arch(A, h_workers));
    if (!hd || (dag->n > 0 && (!dur || !gain || !flags))) return fail(MP_ERR_ARG, "NULL buffer");
    DurView d{dur, A, enabled_mask(A, h_workers)};
    MP_TRY(ensure_ws(dag, 256, st));
    uint32_t* hdbits = (uint32_t*)dag->ws;
    MP_CUDA(cudaMemsetAsync(hdbits, 0, 4 * MAX_ARCH, st));
    const int32_t n = dag->n;
    if (n > 0) MP_LAUNCH(k_aff_hd, grid_for(n), 256, 0, st, n, d, flags, hdbits, dag->err);
    MP_LAUNCH(k_aff_gain, grid_for(n > 0 ? n : 1), 256, 0, st, n, d, flags, hdbits, gain, hd);
    MP_CUDA(cudaGetLastError());
    return MP_OK;
}

inline mp_status score(mp_dag* dag, int32_t A, int32_t kind, const float* crit, const float* gain,
                       const uint8_t* flags, float* crit_norm, uint64_t* key, cudaStream_t st) {
    using namespace mpk;
    if (!dag) return fail(MP_ERR_ARG, "dag is NULL");
    if (A < 1 || A > MAX_ARCH) return fail(MP_ERR_ARG, "n_arch %d outside [1, 8]", A);
    if (kind != 0 && kind != 1) return fail(MP_ERR_ARG, "unknown criticality kind %d", kind);
    const int32_t n = dag->n;
    if (n == 0) return MP_OK;
    if (!crit || !gain || !flags || !crit_norm || !key) return fail(MP_ERR_ARG, "NULL buffer");
    MP_TRY(ensure_ws(dag, 256, st));
    uint32_t* mx = (uint32_t*)dag->ws;
    MP_CUDA(cudaMemsetAsync(mx, 0, 4 * MAX_ARCH, st));
    int64_t cnt = kind == 0 ? n : (int64_t)n * A;
    MP_LAUNCH(k_crit_max, grid_for(cnt), 256, 0, st, cnt, A, kind, crit, flags, mx);
    MP_LAUNCH(k_score, grid_for(n), 256, 0, st, n, A, kind, crit, gain, flags, mx, crit_norm, key);
    MP_CUDA(cudaGetLastError());
    return MP_OK;
}

inline mp_status build_queues(mp_dag* dag, int32_t A, const uint64_t* key, const uint8_t* flags, const float* dur,
                              const uint8_t* done, int64_t* qptr, int32_t* qtask, mp_queue_summary* sum,
                              cudaStream_t st) {
    using namespace mpk;
    if (!dag) return fail(MP_ERR_ARG, "dag is NULL");
    if (A < 1 || A > MAX_ARCH) return fail(MP_ERR_ARG, "n_arch %d outside [1, 8]", A);
    if (!qptr || !sum) return fail(MP_ERR_ARG, "NULL buffer");
    const int32_t n = dag->n;
    const int64_t nA = (int64_t)n * A;
    if (n > 0 && (!key || !flags || !dur || !qtask)) return fail(MP_ERR_ARG, "NULL buffer");
    const int64_t cap = nA > 0 ? nA : 1;
    size_t bytes = sort_bytes(cap, 1, 8, true) + 2 * align256(cap * 4) + align256((size_t)n + 1) + 4 * 256;
    MP_TRY(ensure_ws(dag, bytes, st));
    Arena ar{dag->ws, dag->ws_cap};
    SortArgs sa = carve_sort(ar, dag, cap, 1, 0, 8, true);
    int32_t* memb = ar.take<int32_t>(cap);
    int32_t* pos = ar.take<int32_t>(cap);
    uint8_t* blocked = ar.take<uint8_t>((size_t)n + 1);
    int32_t* counts = ar.take<int32_t>(MAX_ARCH);
    unsigned long long* brw = ar.take<unsigned long long>(2 * MAX_ARCH);
    int32_t* total = ar.take<int32_t>(2);
    int64_t* dlen = ar.take<int64_t>(1);
    MP_CUDA(cudaMemsetAsync(counts, 0, 4 * MAX_ARCH, st));
    MP_CUDA(cudaMemsetAsync(brw, 0, 16 * MAX_ARCH, st));
    MP_CUDA(cudaMemsetAsync(total, 0, 8, st));
    if (n > 0) {
        if (done) {
            MP_CUDA(cudaMemsetAsync(blocked, 0, (size_t)n, st));
            MP_LAUNCH(k_blocked, grid_for(n), 256, 0, st, n, dag->row_ptr, dag->col, done, blocked);
        }
        dim3 g(grid_for(n, 256, 148 * 8), A);
        MP_LAUNCH(k_q_member, g, 256, 0, st, n, A, flags, done, blocked, dur, memb, counts, brw);
        MP_TRY(scan(dag, memb, pos, nA, total, st));
        MP_LAUNCH(k_q_scatter, g, 256, 0, st, n, A, key, memb, pos, sa.keys[0], sa.vals[0]);
        // device-side length: the sort reads Q from `total` (int32) via an int64 mirror
        sa.seg_len = nA;
        sa.d_len = dlen;
        MP_LAUNCH(k_copy_len, 1, 1, 0, st, total, dlen);
        MP_TRY(run_sort(dag, sa, st));
    }
    MP_LAUNCH(k_q_out, grid_for(nA > 0 ? nA : 1), 256, 0, st, sa.plans, sa.vals[0], sa.vals[1], total, A, counts, brw,
              qptr, qtask, sum);
    MP_CUDA(cudaGetLastError());
    return MP_OK;
}

}  // namespace mph
