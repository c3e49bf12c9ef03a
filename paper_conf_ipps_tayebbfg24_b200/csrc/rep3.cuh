// rep3.cuh -- K3 k_rep3_sort: the two-arch replica sort (a6-a9 of one replica)
// with its whole working set in the shared memory of a 2-CTA cluster.
//
// One cluster (2 CTAs on 2 SMs, DSMEM between them) per replica, persistent
// over replicas by ticket.  CTA k owns the task ids and the sorted positions
// [k h, (k+1) h), h = ceil(n/2).  Per replica:
//   P1  hash both perturbed durations of every own task (a10), the orderable
//       difference D(t) = orderable(delta_1 - delta_0) (two-arch order theorem,
//       one order by d gives both queues), Did[t]; a coarse
//       histogram of D over the launch's fixed key range.
//   G   proportional sub-bin geometry from the cluster's coarse histogram
//       (each non-empty coarse bin gets ceil(c (NF - NE) / n) fine bins, <= NF
//       in total): fine bins hold ~3 entries.
//   P1b fine histogram, 16-bit counters packed in pairs.
//   S   exclusive scan over the cluster's fine counts -> every bin's global
//       start; CTA 0's entries of a bin first, then CTA 1's.
//   P2  counting-sort scatter: task id -> its bin's next slot (local or the
//       peer's shared memory).
//   P3  every fine bin is sorted by (D, id): <= 8 entries by one thread in
//       registers, larger bins (<= 256) by a warp (rank by comparison); the
//       "same gain as the next position" bits of both archs (e0, e1) are set
//       from each entry's successor key.
//   P5  emission: positions in no equal-gain run go straight to both queues
//       (queue 1 = ascending positions [0, cG), queue 0 = descending positions
//       [n1only, n)); members of a run (<= 64) rank themselves by (critc, id)
//       with critc = 1 - bits(bl / CP) gathered from K1's bl32.
// A replica whose bins or runs exceed those bounds (degenerate key
// distributions: sigma ~ 0, long runs of one-arch tasks) is appended to a
// fallback list that k_rep2_sort (general 64-bit key path) then processes.
// No global scratch: HBM traffic is the queue output (+ the base durations,
// K1's per-replica statistics and the bl values of run members).
#pragma once
#include "rep2.cuh"

namespace mpk {

// per-phase cycle accounting of K3 (build with -DMP_PHASES; tools/k3_phases.py): thread 0 of
// CTA 0 of every cluster adds the clock64 delta since the previous mark to g_k2_phase[16 + i]
#ifdef MP_PHASES
#define K3_PHASE(i)                                                                   \
    do {                                                                              \
        if (rank == 0 && threadIdx.x == 0) {                                          \
            const long long t__ = clock64();                                          \
            if ((i) > 0) atomicAdd(&g_k2_phase[16 + (i)], (unsigned long long)(t__ - k3_t)); \
            k3_t = t__;                                                               \
        }                                                                             \
    } while (0)
#else
#define K3_PHASE(i) ((void)0)
#endif

constexpr int R4_THREADS = 1024;
constexpr int R4_NC = 4096;     // coarse bins over the launch's fixed key range
constexpr int R4_NF = 16384;    // fine bins per replica
constexpr int R4_SMALL = 8;     // fine bins up to this size: one thread, registers
constexpr int R4_BIG = 128;     // up to this size: one warp; larger: fallback
constexpr int R4_RUN = 64;      // equal-gain runs up to this length; longer: fallback
constexpr int R4_LIST = 1024;   // big-bin list / member-crit capacity per CTA
constexpr int R4_PER = 24;      // own tasks per thread held in registers in P2 (h <= 24 Ki)
constexpr int R4_RC = 4096;     // positions per P3 round (4 per thread)
constexpr int R4_MAXR = 64;     // P3 rounds per CTA

struct R4Args {
    int32_t n, R;
    int64_t r0;
    const float* base;
    uint32_t emask;
    uint64_t seed;
    float sigma;
    const float* cp;                  // [R]      K1
    const uint32_t* hd;               // [R][2]   K1 (float bits; hd(0) == hd(1))
    const int32_t* counts;            // [R][2]   K1
    const unsigned long long* brw;    // [R][2][2] K1
    const float* bl32;                // [groups][n][32] K1 (q-space rows)
    const int32_t* qof;               // [n] q-space position of each task
    int32_t* qtask;                   // [R][2n] or null
    mp_queue_summary* sum;            // [R][2]
    uint32_t* ticket;
    int32_t* fb_list;                 // [R] replicas left to k_rep2_sort
    uint32_t* fb_count;
};

// shared-memory layout (identical in both CTAs, so peer addresses map 1:1)
struct R4Layout {
    uint32_t h, hpad, ew;
    size_t o_ds, o_ps, o_cnt, o_coff, o_clog, o_e0, o_e1, o_list, o_sc, o_um, o_uo, o_crit, o_mpos, o_rb, bytes;
};
__host__ __device__ inline R4Layout r4_layout(int32_t n) {
    R4Layout L;
    L.h = (uint32_t)(n + 1) / 2;
    L.hpad = (L.h + 63u) & ~31u;          // + slack: the last window reads up to 40 slots
    L.ew = L.hpad / 32u + 1u;
    size_t o = 0;
    L.o_ds = o;   o += (size_t)L.hpad * 4;           // D in position order
    L.o_cnt = o;  o += (size_t)R4_NF / 2 * 4;        // fine counters (coarse histogram first)
    L.o_e0 = o;   o += (size_t)L.ew * 4;
    L.o_e1 = o;   o += (size_t)L.ew * 4;
    L.o_list = o; o += (size_t)R4_LIST * 4;
    L.o_sc = o;   o += 96 * 4;
    L.o_um = o;   o += (size_t)L.ew * 4;           // P5: members (either queue) per 32 positions
    L.o_uo = o;   o += (size_t)L.ew * 4;           // P5: exclusive prefix of their counts
    L.o_crit = o; o += (size_t)R4_LIST * 4;         // P5: critc of every member, in position order
    L.o_mpos = o; o += (size_t)R4_LIST * 2;         // P5: their local positions
    L.o_rb = o;   o += (size_t)(R4_MAXR + 1) * 4;  // P3: round bounds
    L.o_ps = o;   o += (size_t)L.hpad * 2;           // task id in position order
    L.o_coff = o; o += (size_t)R4_NC * 2;
    L.o_clog = o; o += (size_t)R4_NC;
    L.bytes = (o + 15) & ~(size_t)15;
    return L;
}

// D of the two perturbed durations (orderable key; arch-1-only 0, arch-0-only ~0)
MP_INLINE uint32_t r4_D(float x0, float x1, uint32_t emask) {
    uint32_t en = 0;
    if ((emask & 1u) && !is_inf(x0)) en |= 1u;
    if ((emask & 2u) && !is_inf(x1)) en |= 2u;
    if (en == 3u) {
        const uint32_t db = f2u(__fsub_rn(x1, x0));
        return (db >> 31) ? ~db : (db | 0x80000000u);
    }
    return en == 1u ? 0xFFFFFFFFu : 0u;
}

struct R4Geo {
    uint32_t lo, hi, cs;   // coarse bin of D: (D - lo) >> cs
};

MP_INLINE uint32_t r4_coarse(const R4Geo& g, uint32_t D) {
    const uint32_t c = (D < g.lo ? 0u : D - g.lo) >> g.cs;
    return c < (uint32_t)R4_NC ? c : (uint32_t)R4_NC - 1u;
}
// fine bin: coff[c] + ((D - lo - c 2^cs) * m_c) >> cs  (monotone in D, < coff[c] + m_c)
MP_INLINE uint32_t r4_fine(const R4Geo& g, const uint16_t* coff, const uint8_t* clog, uint32_t D) {
    const uint32_t c = r4_coarse(g, D);
    const uint32_t off = (D < g.lo ? 0u : D - g.lo) - (c << g.cs);
    const uint32_t m = clog[c];
    uint32_t sub = (uint32_t)(((uint64_t)off * m) >> g.cs);
    sub = m ? min(sub, m - 1u) : 0u;   // keys outside [lo, hi] (flagged: fallback) stay in range
    return min((uint32_t)coff[c] + sub, (uint32_t)R4_NF - 1u);
}

MP_INLINE uint32_t r4_half(const uint32_t* cnt, uint32_t f) { return (cnt[f >> 1] >> ((f & 1u) * 16u)) & 0xFFFFu; }

__global__ void __launch_bounds__(R4_THREADS, 1) k_rep3_sort(R4Args a) {
    extern __shared__ __align__(16) unsigned char r4s[];
    namespace cg = cooperative_groups;
    cg::cluster_group cl = cg::this_cluster();
    const uint32_t rank = cl.block_rank(), peer = rank ^ 1u;
    const int32_t n = a.n;
    const R4Layout L = r4_layout(n);
    const int32_t h = (int32_t)L.h;
    const int32_t own0 = (int32_t)rank * h;                       // first own id / position
    const int32_t hk = min(h, n - own0);                          // own count
    const int32_t own1 = own0 + hk;
    uint32_t* Ds = reinterpret_cast<uint32_t*>(r4s + L.o_ds);
    uint16_t* Ps = reinterpret_cast<uint16_t*>(r4s + L.o_ps);
    uint32_t* cnt = reinterpret_cast<uint32_t*>(r4s + L.o_cnt);
    uint16_t* coff = reinterpret_cast<uint16_t*>(r4s + L.o_coff);
    uint8_t* clog = reinterpret_cast<uint8_t*>(r4s + L.o_clog);
    uint32_t* e0 = reinterpret_cast<uint32_t*>(r4s + L.o_e0);
    uint32_t* e1 = reinterpret_cast<uint32_t*>(r4s + L.o_e1);
    uint32_t* blist = reinterpret_cast<uint32_t*>(r4s + L.o_list);
    uint32_t* sc = reinterpret_cast<uint32_t*>(r4s + L.o_sc);
    // the peer's copies (generic pointers into its shared memory); positions [0, h) live
    // in CTA 0, [h, n) in CTA 1, at local index p - rank h
    uint32_t* const DsP = cl.map_shared_rank(Ds, peer);
    uint16_t* const PsP = cl.map_shared_rank(Ps, peer);
    uint32_t* const e0P = cl.map_shared_rank(e0, peer);
    uint32_t* const e1P = cl.map_shared_rank(e1, peer);
    const uint32_t* cntP = cl.map_shared_rank(cnt, peer);

    __shared__ uint32_t s_rl, s_flag, s_head0, s_head1, s_nbig, s_lo, s_hi, s_skip;
    uint32_t* flag0 = cl.map_shared_rank(&s_flag, 0u);            // the cluster's fallback flag (CTA 0)
    uint32_t* head0p = cl.map_shared_rank(&s_head0, 0u);
    uint32_t* head1p = cl.map_shared_rank(&s_head1, 0u);
    uint32_t* rlp1 = cl.map_shared_rank(&s_rl, 1u);
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;

    // position p (global) -> its owner's arrays
    auto own = [&](int32_t p) -> bool { return p >= own0 && p < own0 + h; };
    auto Dp = [&](int32_t p) -> uint32_t* { return own(p) ? Ds + (p - own0) : DsP + (p - (int32_t)peer * h); };
    auto Pp = [&](int32_t p) -> uint16_t* { return own(p) ? Ps + (p - own0) : PsP + (p - (int32_t)peer * h); };
    auto ebit = [&](int arch, int32_t p) -> bool {
        const bool o = own(p);
        const int32_t lp = o ? p - own0 : p - (int32_t)peer * h;
        const uint32_t* E = arch ? (o ? e1 : e1P) : (o ? e0 : e0P);
        return (E[lp >> 5] >> (lp & 31)) & 1u;
    };

    // ---- fixed key range of the launch from the perturbation's extremes (u = 0 and
    //      u = 1 - 2^-24; every RN op of the perturbation and of d is monotone) ----
    if (threadIdx.x == 0) { s_lo = ~0u; s_hi = 0u; }
    __syncthreads();
    {
        uint32_t lo = ~0u, hi = 0u;
        for (int32_t t = threadIdx.x; t < n; t += R4_THREADS) {
            float xl[2], xh[2];
            uint32_t enl = 0, enh = 0;
            bool dummy = false;
#pragma unroll
            for (int b = 0; b < 2; b++) {
                const float bv = __ldg(a.base + 2 * (int64_t)t + b);
                const float u0 = canon_dur(perturb_u(bv, a.sigma, 0u), dummy);
                const float u1 = canon_dur(perturb_u(bv, a.sigma, 0xFFFFFFu), dummy);
                xl[b] = u0 < u1 ? u0 : u1;
                xh[b] = u0 < u1 ? u1 : u0;
                if (((a.emask >> b) & 1u) && !is_inf(xl[b])) enl |= 1u << b;
                if (((a.emask >> b) & 1u) && !is_inf(xh[b])) enh |= 1u << b;
            }
            if (enl != enh || xl[0] != xl[0] || xl[1] != xl[1] || xh[0] != xh[0] || xh[1] != xh[1]) {
                lo = 0u;
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
        if (lane == 0) {
            atomicMin(&s_lo, lo);
            atomicMax(&s_hi, hi);
        }
    }
    __syncthreads();
    R4Geo g;
    g.lo = s_lo <= s_hi ? s_lo : 0u;
    g.hi = s_lo <= s_hi ? s_hi : 0xFFFFFFFFu;
    {
        const uint32_t span = g.hi - g.lo;
        uint32_t cs = 0;
        while (cs < 32 && ((uint64_t)span >> cs) >= (uint64_t)R4_NC) cs++;
        g.cs = cs;
    }
    const uint64_t golden2 = 2u * SPLITMIX_GOLDEN;
#ifdef MP_PHASES
    long long k3_t = 0;
#endif
    // D(t) of replica r (a10: both perturbed durations, hashed once per pass)
    auto D_task = [&](uint64_t cbase, int32_t t) -> uint32_t {
        const float2 bb = __ldg(reinterpret_cast<const float2*>(a.base) + t);
        const uint64_t xs = cbase + (uint64_t)(uint32_t)t * golden2;
        bool dummy = false;
        const float x0 = canon_dur(perturb_x(bb.x, xs, a.sigma), dummy);
        const float x1 = canon_dur(perturb_x(bb.y, xs + SPLITMIX_GOLDEN, a.sigma), dummy);
        return r4_D(x0, x1, a.emask);
    };
    auto cbase_of = [&](uint64_t r) -> uint64_t {
        return a.seed + ((uint64_t)r * (uint64_t)n * 2u + 1u) * SPLITMIX_GOLDEN;
    };
    // ---- the launch's fine-bin geometry, built once from a reference replica (the call's
    //      first) and shared by every replica (their D follow the same distribution):
    //      every coarse bin of the range gets >= 1 fine bin (another replica may have keys
    //      where the reference has none), the rest proportionally to the reference's
    //      coarse counts -> fine bins hold ~3 entries ----
    {
        for (int32_t i = threadIdx.x; i < R4_NC; i += R4_THREADS) cnt[i] = 0u;
        __syncthreads();
        const uint64_t cb0 = cbase_of((uint64_t)a.r0);
        for (int32_t t = own0 + threadIdx.x; t < own1; t += R4_THREADS)
            atomicAdd(&cnt[r4_coarse(g, D_task(cb0, t))], 1u);
        cl.sync();
        const uint32_t ncb = (uint32_t)(((uint64_t)(g.hi - g.lo) >> g.cs) + 1);
        constexpr int CPER = R4_NC / R4_THREADS;   // 4
        uint32_t c[CPER], tc = 0;
#pragma unroll
        for (int j = 0; j < CPER; j++) {
            const uint32_t b = threadIdx.x * CPER + j;
            c[j] = cnt[b] + cntP[b];
            tc += c[j];
        }
        uint32_t TOT;
        r3_scan(tc, sc, TOT);
        const uint64_t Fn = (uint64_t)R4_NF - ncb, Fd = TOT > 0 ? TOT : 1u;
        uint32_t m[CPER], sm = 0;
#pragma unroll
        for (int j = 0; j < CPER; j++) {
            const uint32_t b = threadIdx.x * CPER + j;
            uint32_t v = 0;
            if (b < ncb) {
                v = (uint32_t)min(((uint64_t)c[j] * Fn + Fd - 1) / Fd, (uint64_t)255);
                if (g.cs < 8) v = min(v, 1u << g.cs);
                v = max(v, 1u);
            }
            m[j] = v;
            sm += v;
        }
        uint32_t ftot;
        uint32_t e = r3_scan(sm, sc, ftot);
#pragma unroll
        for (int j = 0; j < CPER; j++) {
            const uint32_t b = threadIdx.x * CPER + j;
            coff[b] = (uint16_t)e;
            clog[b] = (uint8_t)m[j];
            e += m[j];
        }
        cl.sync();   // the peer is done reading cnt
    }

    uint32_t* um = reinterpret_cast<uint32_t*>(r4s + L.o_um);
    uint32_t* uo = reinterpret_cast<uint32_t*>(r4s + L.o_uo);
    uint32_t* mcrit = reinterpret_cast<uint32_t*>(r4s + L.o_crit);
    uint16_t* mpos = reinterpret_cast<uint16_t*>(r4s + L.o_mpos);
    int32_t* rb = reinterpret_cast<int32_t*>(r4s + L.o_rb);
    __shared__ uint32_t s_nmem, s_bpair;

    while (true) {
        if (rank == 0 && threadIdx.x == 0) {
            const uint32_t tk = atomicAdd(a.ticket, 1u);
            s_rl = tk;
            *rlp1 = tk;                  // the peer reads its own copy: no DSMEM access after S0
            s_flag = 0u;                 // when the cluster exits
            s_head0 = 0xFFFFFFFFu;
            s_head1 = 0xFFFFFFFFu;
        }
        cl.sync();                                                          // S0
        const int64_t rl = s_rl;
        if (rl >= a.R) break;
        K3_PHASE(0);
        const int64_t r = a.r0 + rl;
        // ---- P1: D(t) of the own tasks into Ds (id order for now) and the fine histogram
        //      (16-bit counters in pairs) ----
        for (int32_t i = threadIdx.x; i < R4_NF / 2; i += R4_THREADS) cnt[i] = 0u;
        if (threadIdx.x == 0) { s_nbig = 0u; s_nmem = 0u; s_bpair = 0u; }
        __syncthreads();
        {
            const uint64_t cbase = cbase_of((uint64_t)r);
            bool outside = false;
            for (int32_t t = own0 + threadIdx.x; t < own1; t += R4_THREADS) {
                const uint32_t D = D_task(cbase, t);
                Ds[t - own0] = D;
                outside |= D < g.lo || D > g.hi;
                const uint32_t f = r4_fine(g, coff, clog, D);
                atomicAdd(&cnt[f >> 1], 1u << ((f & 1u) * 16u));
            }
            if (__any_sync(0xffffffffu, outside) && lane == 0) atomicOr(flag0, 1u);
        }
        cl.sync();                                                          // S1
        K3_PHASE(1);
        // ---- S: global starts; own cursors = start + (CTA 1: CTA 0's count) ----
        uint32_t Dr[R4_PER];   // P2: the own D values leave Ds (the peer scatters into it)
        {
            constexpr int WPER = R4_NF / 2 / R4_THREADS;   // 8 words = 16 bins per thread
            uint32_t w0v[WPER], w1v[WPER], sum = 0, big = 0;
#pragma unroll
            for (int j = 0; j < WPER; j++) {
                const uint32_t wi = threadIdx.x * WPER + j;
                const uint32_t mine = cnt[wi], other = cntP[wi];
                w0v[j] = rank == 0 ? mine : other;          // CTA 0's counts
                w1v[j] = rank == 0 ? other : mine;
                const uint32_t tl = (w0v[j] & 0xFFFFu) + (w1v[j] & 0xFFFFu);
                const uint32_t th = (w0v[j] >> 16) + (w1v[j] >> 16);
                sum += tl + th;
                big = max(big, max(tl, th));
            }
            uint32_t tot;
            uint32_t e = r3_scan(sum, sc, tot);
            if (big > (uint32_t)R4_BIG) atomicOr(flag0, 1u);
            uint32_t cur[WPER];
#pragma unroll
            for (int j = 0; j < WPER; j++) {
                const uint32_t c0l = w0v[j] & 0xFFFFu, c0h = w0v[j] >> 16;
                const uint32_t tl = c0l + (w1v[j] & 0xFFFFu), th = c0h + (w1v[j] >> 16);
                const uint32_t sl = e + (rank == 1 ? c0l : 0u);
                const uint32_t sh = e + tl + (rank == 1 ? c0h : 0u);
                cur[j] = (sl & 0xFFFFu) | (sh << 16);
                e += tl + th;
            }
#pragma unroll
            for (int j = 0; j < R4_PER; j++) {
                const int32_t i = threadIdx.x + j * R4_THREADS;
                Dr[j] = i < hk ? Ds[i] : 0u;
            }
            cl.sync();                                                      // S4 (peer done reading cnt; own D in registers)
            K3_PHASE(2);
#pragma unroll
            for (int j = 0; j < WPER; j++) cnt[threadIdx.x * WPER + j] = cur[j];
        }
        __syncthreads();
        // ---- P2: counting-sort scatter of (D, id) into position order ----
#pragma unroll
        for (int j = 0; j < R4_PER; j++) {
            const int32_t i = threadIdx.x + j * R4_THREADS;
            if (i < hk) {
                const uint32_t f = r4_fine(g, coff, clog, Dr[j]);
                const uint32_t sh = (f & 1u) * 16u;
                const int32_t pos = (int32_t)((atomicAdd(&cnt[f >> 1], 1u << sh) >> sh) & 0xFFFFu);
                *Dp(pos) = Dr[j];
                *Pp(pos) = (uint16_t)(own0 + i);
            }
        }
        cl.sync();                                                          // S5
        K3_PHASE(4);
        // CTA 1's cursors are the bins' ends: CTA 0 takes a copy
        if (rank == 0)
            for (int32_t i = threadIdx.x; i < R4_NF / 2; i += R4_THREADS) cnt[i] = cntP[i];
        // the cluster's fallback flag, read once per CTA and broadcast (uniform branches)
        auto flag_now = [&]() -> bool {
            if (threadIdx.x == 0) s_skip = *reinterpret_cast<volatile uint32_t*>(flag0);
            __syncthreads();
            const bool v = s_skip != 0u;
            __syncthreads();
            return v;
        };
        const bool skip = flag_now();
        const float hdv = u2f(a.hd[rl * 2]);                               // hd(0) == hd(1)
        auto end_of = [&](uint32_t f) -> int32_t { return (int32_t)r4_half(cnt, f); };
        // ---- P3: order every bin by (D, id).  Rounds of <= 4096 own positions cut at bin
        //      starts: each entry of an own bin ranks itself in its bin (smaller keys of
        //      the bin, read from shared memory); after a barrier the round's entries move
        //      to their positions.  The one own bin that reaches into the peer's positions
        //      and bins of > 16 entries: one warp each, after the rounds. ----
        if (!skip) {
            const int32_t nr = min((hk + R4_RC - 1) / R4_RC, R4_MAXR);
            for (int32_t q = threadIdx.x; q <= nr; q += R4_THREADS) {
                int32_t b = own1;
                if (q == 0) b = own0;
                else if (q < nr) {
                    const uint32_t f = r4_fine(g, coff, clog, Ds[q * R4_RC]);
                    b = max(own0, f ? end_of(f - 1) : 0);
                }
                rb[q] = b;
            }
            __syncthreads();
            constexpr int RP = R4_RC / R4_THREADS + 1;   // a round: <= 4096 + one bin
            for (int32_t q = 0; q < nr; q++) {
                const int32_t p0 = rb[q] - own0, p1 = rb[q + 1] - own0;   // local positions
                int32_t np[RP];
                uint32_t nD[RP];
                uint16_t nt[RP];
#pragma unroll
                for (int u = 0; u < RP; u++) {
                    np[u] = -1;
                    const int32_t lp = p0 + (int32_t)threadIdx.x + u * R4_THREADS;
                    if (lp >= p1) continue;
                    const uint32_t D = Ds[lp];
                    const uint32_t f = r4_fine(g, coff, clog, D);
                    const int32_t s = (f ? end_of(f - 1) : 0) - own0, e = end_of(f) - own0, k = e - s;
                    if (s < 0 || k == 1) continue;                             // the peer's bin / in place
                    if (k > 16 || e > hk) {                                    // one warp, below
                        if (lp == s) {
                            const uint32_t at = atomicAdd(&s_nbig, 1u);
                            if (at < (uint32_t)R4_LIST) blist[at] = f;
                            else atomicOr(flag0, 1u);
                        }
                        continue;
                    }
                    const uint16_t t = Ps[lp];
                    const uint64_t key = ((uint64_t)D << 16) | t;
                    uint32_t rk = 0;
                    for (int32_t j = s; j < e; j++)
                        rk += (((uint64_t)Ds[j] << 16) | Ps[j]) < key ? 1u : 0u;
                    np[u] = s + (int32_t)rk;
                    nD[u] = D;
                    nt[u] = t;
                }
                __syncthreads();
#pragma unroll
                for (int u = 0; u < RP; u++) {
                    if (np[u] < 0) continue;
                    Ds[np[u]] = nD[u];
                    Ps[np[u]] = nt[u];
                }
                __syncthreads();
            }
            // listed bins (> 16 entries, <= R4_BIG, or reaching into the peer): one warp each
            const uint32_t nbig = min(s_nbig, (uint32_t)R4_LIST);
            for (uint32_t bi = wid; bi < nbig; bi += R4_THREADS / 32) {
                const uint32_t f = blist[bi];
                const int32_t s = f ? end_of(f - 1) : 0, e = end_of(f), k = e - s;
                if (k > R4_BIG) continue;                             // flagged in S
                constexpr int PL = R4_BIG / 32;                       // entries per lane
                uint64_t kk[PL];
#pragma unroll
                for (int j = 0; j < PL; j++) {
                    const int32_t i = lane + 32 * j;
                    kk[j] = ~0ull;
                    if (i < k) kk[j] = ((uint64_t)*Dp(s + i) << 16) | *Pp(s + i);
                }
                uint32_t rk[PL];
#pragma unroll
                for (int j = 0; j < PL; j++) rk[j] = 0u;
#pragma unroll
                for (int jj = 0; jj < PL; jj++) {
                    if (jj * 32 >= k) break;
                    const int lim = min(32, k - jj * 32);
                    for (int sl = 0; sl < lim; sl++) {
                        const uint64_t o = __shfl_sync(0xffffffffu, kk[jj], sl);
#pragma unroll
                        for (int j = 0; j < PL; j++) rk[j] += o < kk[j] ? 1u : 0u;
                    }
                }
                __syncwarp();
#pragma unroll
                for (int j = 0; j < PL; j++) {
                    const int32_t i = lane + 32 * j;
                    if (i >= k) continue;
                    *Dp(s + (int32_t)rk[j]) = (uint32_t)(kk[j] >> 16);
                    *Pp(s + (int32_t)rk[j]) = (uint16_t)(kk[j] & 0xFFFFu);
                }
            }
        }
        cl.sync();                                                          // S6a: every bin sorted
        K3_PHASE(5);
        // ---- P3b: "same gain as the next position" bits of both archs, one word per warp
        //      and 32 positions (numerators x = d + hd, y = -d + hd compared; only near-ties
        //      are divided, r2_same_gains) ----
        if (!skip) {
            const uint32_t Dnext_own = own1 < n ? *Dp(own1) : 0u;   // the peer's first key
            for (int32_t lp0 = wid * 32; lp0 < hk; lp0 += R4_THREADS) {
                const int32_t lp = lp0 + lane;
                bool s0 = false, s1 = false;
                if (lp < hk && own0 + lp + 1 < n) {
                    const uint32_t Da = Ds[lp], Db = lp + 1 < hk ? Ds[lp + 1] : Dnext_own;
                    r2_same_gains(Da, Db, hdv, s0, s1);
                }
                const uint32_t b0 = __ballot_sync(0xffffffffu, s0), b1 = __ballot_sync(0xffffffffu, s1);
                if (lane == 0) {
                    e0[lp0 >> 5] = b0;
                    e1[lp0 >> 5] = b1;
                }
            }
        }
        cl.sync();                                                          // S6
        K3_PHASE(6);
        // ---- P5: emission ----
        const bool skip2 = flag_now();
        if (!skip2) {
            const int32_t cC = a.counts[rl * 2 + 0], cG = a.counts[rl * 2 + 1];
            const int32_t n1only = n - cC;                                  // arch-1-only tasks sort first
            int32_t* q0 = a.qtask ? a.qtask + rl * (int64_t)n * 2 : nullptr;
            int32_t* q1 = q0 ? q0 + cC : nullptr;
            const float CP = a.cp[rl];
            const float* blr = a.bl32 + (rl >> 5) * (int64_t)n * 32 + (rl & 31);
            auto critc_of = [&](uint32_t t) -> uint32_t {
                const float c = CP > 0.0f ? __fdiv_rn(__ldcg(blr + (int64_t)__ldg(a.qof + t) * 32), CP) : 0.0f;
                return ONE_BITS - f2u(c);
            };
            // member masks per 32 own positions (either queue), their prefix counts, and every
            // member's critc gathered into shared memory (all loads in flight together)
            auto member1 = [&](int32_t p) -> bool {
                return p < cG && ((p > 0 && ebit(1, p - 1)) || (p + 1 < cG && ebit(1, p)));
            };
            auto member0 = [&](int32_t p) -> bool {
                return p >= n1only && ((p > n1only && ebit(0, p - 1)) || (p + 1 < n && ebit(0, p)));
            };
            const int32_t nw = (hk + 31) / 32;
            uint32_t mloc = 0, cntm = 0;
            const int32_t wq = threadIdx.x;   // one word per thread (h <= 32 Ki)
            if (wq < nw) {
                const uint32_t E0 = e0[wq], E1 = e1[wq];
                const uint32_t P0 = (E0 << 1) | (wq > 0 ? e0[wq - 1] >> 31 : (own0 > 0 && ebit(0, own0 - 1) ? 1u : 0u));
                const uint32_t P1 = (E1 << 1) | (wq > 0 ? e1[wq - 1] >> 31 : (own0 > 0 && ebit(1, own0 - 1) ? 1u : 0u));
                const int32_t pb = own0 + wq * 32;
                auto lt = [&](int32_t x) -> uint32_t {   // bits i with pb + i < x
                    const int32_t c = x - pb;
                    return c <= 0 ? 0u : (c >= 32 ? 0xFFFFFFFFu : ((1u << c) - 1u));
                };
                // bit i: position p = pb + i; e(p-1) is bit i of P, e(p) bit i of E
                const uint32_t m1 = (((P1 & ~lt(1)) | (E1 & lt(cG - 1))) & lt(cG));
                const uint32_t m0 = (((P0 & ~lt(n1only + 1)) | (E0 & lt(n - 1))) & ~lt(n1only));
                mloc = (m0 | m1) & lt(own1);
                cntm = (uint32_t)__popc(mloc);
            }
            uint32_t mtot;
            const uint32_t mpre = r3_scan(cntm, sc, mtot);
            if (wq < nw) {
                um[wq] = mloc;
                uo[wq] = mpre;
            }
            const bool mfit = mtot <= (uint32_t)R4_LIST;
            if (mfit && wq < nw) {
                uint32_t m = mloc, idx = mpre;
                while (m) {
                    const int b = __ffs(m) - 1;
                    m &= m - 1u;
                    mpos[idx] = (uint16_t)(wq * 32 + b);
                    mcrit[idx++] = critc_of(Ps[wq * 32 + b]);
                }
            }
            __syncthreads();
            // non-members: straight to both queues (coalesced, no divergence)
            for (int32_t lp = threadIdx.x; lp < hk; lp += R4_THREADS) {
                if ((um[lp >> 5] >> (lp & 31)) & 1u) continue;
                const int32_t p = own0 + lp;
                const uint32_t t = Ps[lp];
                if (p < cG) {
                    if (p == 0) *head1p = t;
                    if (q1) __stcs(q1 + p, (int32_t)t);
                }
                if (p >= n1only) {
                    if (p == n - 1) *head0p = t;
                    if (q0) __stcs(q0 + (n - 1 - p), (int32_t)t);
                }
            }
            // critc of the member at position p (own and listed; else from HBM)
            auto crit_at = [&](int32_t p) -> uint32_t {
                if (mfit && p >= own0 && p < own1) {
                    const int32_t lp = p - own0;
                    return mcrit[uo[lp >> 5] + __popc(um[lp >> 5] & ((1u << (lp & 31)) - 1u))];
                }
                return critc_of(*Pp(p));
            };
            // members: one thread each, rank inside their runs
            bool longrun = false;
            const int32_t nmem = mfit ? (int32_t)mtot : hk;
            for (int32_t mi = threadIdx.x; mi < nmem; mi += R4_THREADS) {
                const int32_t lp = mfit ? (int32_t)mpos[mi] : mi;
                if (!mfit && !((um[lp >> 5] >> (lp & 31)) & 1u)) continue;
                const int32_t p = own0 + lp;
                const uint32_t t = Ps[lp];
                int32_t pos1 = p, pos0 = n - 1 - p;
                {
                    if (member1(p)) {   // queue 1: runs of equal gain_1 by (critc, id)
                        int32_t lo = p, hi = p;
                        while (lo > 0 && p - lo <= R4_RUN && ebit(1, lo - 1)) lo--;
                        while (hi + 1 < cG && hi - p <= R4_RUN && ebit(1, hi)) hi++;
                        if (hi - lo + 1 > R4_RUN) longrun = true;
                        const uint64_t me = ((uint64_t)crit_at(p) << 16) | t;
                        int32_t rk = 0;
                        for (int32_t j = lo; j <= hi; j++)
                            if (j != p) rk += (((uint64_t)crit_at(j) << 16) | *Pp(j)) < me ? 1 : 0;
                        pos1 = lo + rk;
                    }
                    if (member0(p)) {   // queue 0: runs of equal gain_0 by (critc, id)
                        int32_t lo = p, hi = p;
                        while (lo > n1only && p - lo <= R4_RUN && ebit(0, lo - 1)) lo--;
                        while (hi + 1 < n && hi - p <= R4_RUN && ebit(0, hi)) hi++;
                        if (hi - lo + 1 > R4_RUN) longrun = true;
                        const uint64_t me = ((uint64_t)crit_at(p) << 16) | t;
                        int32_t rk = 0;
                        for (int32_t j = lo; j <= hi; j++)
                            if (j != p) rk += (((uint64_t)crit_at(j) << 16) | *Pp(j)) < me ? 1 : 0;
                        pos0 = (n - 1 - hi) + rk;
                    }
                }
                if (p < cG) {       // queue 1: ascending positions [0, cG)
                    if (pos1 == 0) *head1p = t;
                    if (q1) __stcs(q1 + pos1, (int32_t)t);
                }
                if (p >= n1only) {  // queue 0: descending positions [n1only, n)
                    if (pos0 == 0) *head0p = t;
                    if (q0) __stcs(q0 + pos0, (int32_t)t);
                }
            }
            if (__any_sync(0xffffffffu, longrun) && lane == 0) atomicOr(flag0, 1u);
        }
        cl.sync();                                                          // S7
        K3_PHASE(7);
        if (rank == 0 && threadIdx.x == 0) {
            if (s_flag) {
                a.fb_list[atomicAdd(a.fb_count, 1u)] = (int32_t)rl;
            } else {
#pragma unroll
                for (int b = 0; b < 2; b++) {
                    const int32_t c = a.counts[rl * 2 + b];
                    mp_queue_summary o;
                    o.count = c;
                    o.head = c > 0 ? (int32_t)(b == 0 ? s_head0 : s_head1) : -1;
                    const int64_t bo = (rl * 2 + b) * 2;
                    o.brw_lo = a.brw[bo];
                    o.brw_hi = (int64_t)a.brw[bo + 1];
                    o.brw = u128_to_double_scaled(a.brw[bo], a.brw[bo + 1]);
                    a.sum[rl * 2 + b] = o;
                }
            }
        }
    }
}

}  // namespace mpk

namespace mph {

// K3 takes two-arch replicas whose working set (6 B per task and CTA + 55 KB) fits a CTA
inline bool r4_fits(const mp_dag* dag) {
    if (dag->n < 2) return false;
    int optin = 0;
    if (cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dag->device) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return (int64_t)(dag->n + 1) / 2 <= (int64_t)mpk::R4_PER * mpk::R4_THREADS &&
           mpk::r4_layout(dag->n).bytes + 1024 <= (size_t)optin;
}

inline mp_status rep3_launch(mp_dag* dag, const mpk::R4Args& b, cudaStream_t st) {
    using namespace mpk;
    const size_t smem = r4_layout(dag->n).bytes;
    MP_CUDA(cudaFuncSetAttribute(k_rep3_sort, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    MP_CUDA(cudaFuncSetAttribute(k_rep3_sort, cudaFuncAttributeNonPortableClusterSizeAllowed, 0));
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(R4_THREADS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    // persistent: as many clusters as can be resident at once, at most one per replica
    cfg.gridDim = dim3(2u * (unsigned)std::max(1, std::min(b.R, dag->num_sms / 2)));
    int nclu = 0;
    if (cudaOccupancyMaxActiveClusters(&nclu, k_rep3_sort, &cfg) != cudaSuccess || nclu < 1) {
        cudaGetLastError();
        nclu = dag->num_sms / 2;
    }
    cfg.gridDim = dim3(2u * (unsigned)std::max(1, std::min(b.R, nclu)));
    mph::ProfScope ps("k_rep3_sort", st);
    MP_CUDA(cudaLaunchKernelEx(&cfg, k_rep3_sort, b));
    return MP_OK;
}

}  // namespace mph
