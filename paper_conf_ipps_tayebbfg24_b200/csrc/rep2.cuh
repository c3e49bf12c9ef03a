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
#include "replicas.cuh"

namespace mpk {

constexpr int R2_THREADS = 1024;
constexpr int R2_WARPS = 32;
constexpr int R2_CAP = 16384;
constexpr int R2_NBINS = 4096;

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
    // K2
    uint32_t* s_key;             // [grid][n]   per-CTA scratch keys
    uint16_t* s_pi;              // [grid][n]   per-CTA crit order
    int32_t* qtask;              // [R][n*A] or null
    mp_queue_summary* sum;       // [R][A]
    uint32_t* ticket;
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
template <int A>
__global__ void __launch_bounds__(R2_THREADS, 1) k_rep2_bl(Rep2Args a) {
    extern __shared__ __align__(16) unsigned char r2_smem[];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t g = blockIdx.x;
    const int64_t rl = g * 32 + lane;            // replica index within this call
    const bool live = rl < a.R;
    const int64_t r = a.r0 + rl;                 // global replica id
    float* bl32 = a.bl32 + g * (int64_t)a.n * 32;
    bool bad = false;
    uint32_t hd[A];
    int32_t cnt[A];
    uint64_t blo[A], bhi[A];
#pragma unroll
    for (int q = 0; q < A; q++) { hd[q] = 0; cnt[q] = 0; blo[q] = 0; bhi[q] = 0; }
    float cpm = 0.0f;
    for (int32_t lv = 0; lv < a.L; lv++) {
        const int32_t q1 = __ldg(a.lvlq + lv + 1);
        for (int32_t q = __ldg(a.lvlq + lv) + w; q < q1; q += R2_WARPS) {
            const int32_t v = __ldg(a.nodeq + q);
            const int32_t e0 = __ldg(a.rowq + q), e1 = __ldg(a.rowq + q + 1);
            float x[A];
            uint32_t en;
            int k;
            float wt;
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
            // successors: the warp loads 32 successor positions at once (coalesced), broadcasts
            // them with shuffles and issues 8 independent 128-byte gathers at a time
            float m = 0.0f;
            for (int32_t eb = e0; eb < e1; eb += 32) {
                const int32_t cb = min(32, e1 - eb);
                const int32_t sv = lane < cb ? __ldg(a.colq + eb + lane) : 0;
                int32_t j = 0;
                for (; j + 8 <= cb; j += 8) {
                    float t8[8];
#pragma unroll
                    for (int u = 0; u < 8; u++) {
                        const int32_t sp = __shfl_sync(0xffffffffu, sv, j + u);
                        t8[u] = bl32[(int64_t)sp * 32 + lane];
                    }
#pragma unroll
                    for (int u = 0; u < 8; u++) m = fmaxf(m, t8[u]);
                }
                for (; j < cb; j++) m = fmaxf(m, bl32[(int64_t)__shfl_sync(0xffffffffu, sv, j) * 32 + lane]);
            }
            const float bb = __fadd_rn(wt, m);
            bl32[(int64_t)q * 32 + lane] = bb;
            cpm = fmaxf(cpm, bb);
        }
        __syncthreads();
    }
    // ---- per-replica reductions across the 32 warps (column = lane = replica) ----
    uint32_t* red = reinterpret_cast<uint32_t*>(r2_smem);                 // [32][33]
    unsigned long long* red64 = reinterpret_cast<unsigned long long*>(r2_smem + 32 * 33 * 4 + 64);  // [32][33]
    auto colmax = [&](uint32_t val) -> uint32_t {
        red[w * 33 + lane] = val;
        __syncthreads();
        uint32_t m = 0;
        if (w == 0)
            for (int i = 0; i < 32; i++) m = max(m, red[i * 33 + lane]);
        __syncthreads();
        return m;
    };
    auto colsum = [&](uint32_t val) -> uint32_t {
        red[w * 33 + lane] = val;
        __syncthreads();
        uint32_t m = 0;
        if (w == 0)
            for (int i = 0; i < 32; i++) m += red[i * 33 + lane];
        __syncthreads();
        return m;
    };
    const uint32_t cpb = colmax(f2u(cpm));
    uint32_t hdb[A];
    int32_t cntb[A];
#pragma unroll
    for (int q = 0; q < A; q++) {
        hdb[q] = colmax(hd[q]);
        cntb[q] = (int32_t)colsum((uint32_t)cnt[q]);
    }
    // exact 128-bit column sums: lo words (counting carries), then hi words
#pragma unroll
    for (int q = 0; q < A; q++) {
        red64[w * 33 + lane] = blo[q];
        __syncthreads();
        uint64_t lo = 0, carry = 0;
        if (w == 0)
            for (int i = 0; i < 32; i++) {
                const uint64_t s2 = lo + red64[i * 33 + lane];
                carry += (s2 < lo) ? 1ull : 0ull;
                lo = s2;
            }
        __syncthreads();
        red64[w * 33 + lane] = bhi[q];
        __syncthreads();
        if (w == 0) {
            uint64_t hi = carry;
            for (int i = 0; i < 32; i++) hi += red64[i * 33 + lane];
            if (live) {
                const int64_t o = (rl * A + q) * 2;
                a.brw[o] = lo;
                a.brw[o + 1] = hi;
            }
        }
        __syncthreads();
    }
    if (w == 0 && live) {
        a.cp[rl] = u2f(cpb);
#pragma unroll
        for (int q = 0; q < A; q++) {
            a.hd[rl * A + q] = hdb[q];
            a.counts[rl * A + q] = cntb[q];
        }
    }
    if (__any_sync(0xffffffffu, bad) && lane == 0) atomicOr(a.err, ERR_DOMAIN_BIT);
    // ---- transpose bl32 [q][32] -> blT [r][t] ----
    float* tile = reinterpret_cast<float*>(r2_smem) + w * 32 * 33;
    const int32_t nchunks = (a.n + 31) / 32;
    for (int32_t c = w; c < nchunks; c += R2_WARPS) {
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
// K2: per-replica bucketed sorts in shared memory
// ---------------------------------------------------------------------------------------
struct R2Smem {
    uint32_t* k[2];     // [R2_CAP] keys (relative to the round's low key)
    uint16_t* v[2];     // [R2_CAP] payloads
    uint32_t* hw;       // [8192]  range histogram / per-warp digit counts
    uint32_t* scan;     // [64]    block-scan scratch
    uint32_t* misc;     // [512]   groups (4 x u32 each), stack, broadcast values
};

constexpr int R2_MAXG = 40;     // groups per range
constexpr int R2_MAXS = 16;     // deferred-range stack

// exclusive block scan of one value per thread (1024 threads); returns the prefix, total via ref
MP_INLINE uint32_t r2_scan(uint32_t x, uint32_t* sc, uint32_t& total) {
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

MP_INLINE uint32_t r2_bitlen(uint32_t x) { return x ? 32u - __clz(x) : 0u; }

// stable LSD pass in shared memory: (ks,vs) -> (kd,vd) by digit (k >> sh) & 255
MP_INLINE void r2_lsd_pass(const uint32_t* ks, const uint16_t* vs, uint32_t* kd, uint16_t* vd, uint32_t cnt, int sh,
                           uint32_t* hw, uint32_t* sc) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t* wh = hw + w * 256;
    for (int d = lane; d < 256; d += 32) wh[d] = 0;
    const uint32_t per = (cnt + R2_WARPS - 1) / R2_WARPS;
    const uint32_t ws = min(cnt, w * per), we = min(cnt, ws + per);
    __syncwarp();
    const uint32_t lt = lanemask_lt();
    for (uint32_t b = ws; b < we; b += 32) {
        const uint32_t i = b + lane;
        const uint32_t d = i < we ? (ks[i] >> sh) & 255u : 256u;
        const uint32_t peers = __match_any_sync(0xffffffffu, d);
        if (d < 256 && (peers & lt) == 0) atomicAdd(&wh[d], (uint32_t)__popc(peers));
    }
    __syncthreads();
    // exclusive offsets in (digit, warp) order: thread t owns digit t/4, warps 8*(t%4)..+8
    {
        const int d = threadIdx.x >> 2, w0 = (threadIdx.x & 3) * 8;
        uint32_t loc[8], s = 0;
#pragma unroll
        for (int j = 0; j < 8; j++) {
            loc[j] = hw[(w0 + j) * 256 + d];
            s += loc[j];
        }
        uint32_t tot;
        uint32_t run = r2_scan(s, sc, tot);
#pragma unroll
        for (int j = 0; j < 8; j++) {
            hw[(w0 + j) * 256 + d] = run;
            run += loc[j];
        }
    }
    __syncthreads();
    for (uint32_t b = ws; b < we; b += 32) {
        const uint32_t i = b + lane;
        const bool ok = i < we;
        const uint32_t k = ok ? ks[i] : 0u;
        const uint32_t d = ok ? (k >> sh) & 255u : 256u;
        const uint32_t peers = __match_any_sync(0xffffffffu, d);
        uint32_t off = 0;
        if (ok) {
            off = wh[d] + __popc(peers & lt);
            kd[off] = k;
            vd[off] = vs[i];
        }
        __syncwarp();
        if (ok && (peers & lt) == 0) wh[d] += __popc(peers);
        __syncwarp();
    }
    __syncthreads();
}

// Input sequences: key(i) and payload(i) for i in [0, n)
struct R2CritIn {
    const uint32_t* key;
    MP_INLINE uint32_t k(int32_t i) const { return key[i]; }
    MP_INLINE uint16_t p(int32_t i) const { return (uint16_t)i; }
};
struct R2GainIn {
    const uint32_t* key;
    const uint16_t* pi;
    MP_INLINE uint32_t k(int32_t i) const { return key[i]; }
    MP_INLINE uint16_t p(int32_t i) const { return pi[i]; }
};
struct R2PiOut {
    uint16_t* pi;
    MP_INLINE void put(int32_t pos, uint16_t v) const { pi[pos] = v; }
};
struct R2QOut {
    int32_t* q;          // may be null
    int32_t count;
    uint32_t* head;      // smem
    MP_INLINE void put(int32_t pos, uint16_t v) const {
        if (pos == 0) *head = v;
        if (q && pos < count) q[pos] = (int32_t)v;
    }
};

template <class In, class Out>
__device__ void r2_stream_equal(const In& in, const Out& out, int32_t n, uint32_t key, int32_t obase, uint32_t* sc) {
    uint32_t run = 0;
    for (int32_t b0 = 0; b0 < n; b0 += R2_THREADS) {
        const int32_t i = b0 + threadIdx.x;
        const bool sel = i < n && in.k(i) == key;
        uint32_t tot;
        const uint32_t pos = r2_scan(sel ? 1u : 0u, sc, tot);
        if (sel) out.put(obase + (int32_t)(run + pos), in.p(i));
        run += tot;
    }
}

template <class In, class Out>
__device__ void r2_round(const In& in, const Out& out, int32_t n, uint32_t klo, uint32_t khi, uint32_t cnt,
                         int32_t obase, R2Smem& S) {
    uint32_t run = 0;
    for (int32_t b0 = 0; b0 < n; b0 += R2_THREADS) {
        const int32_t i = b0 + threadIdx.x;
        uint32_t k = 0;
        bool sel = false;
        if (i < n) {
            k = in.k(i);
            sel = k >= klo && k <= khi;
        }
        uint32_t tot;
        const uint32_t pos = r2_scan(sel ? 1u : 0u, S.scan, tot);
        if (sel) {
            S.k[0][run + pos] = k - klo;
            S.v[0][run + pos] = in.p(i);
        }
        run += tot;
    }
    __syncthreads();
    const uint32_t nb = r2_bitlen(khi - klo);
    int cur = 0;
    for (uint32_t sh = 0; sh < nb; sh += 8) {
        r2_lsd_pass(S.k[cur], S.v[cur], S.k[cur ^ 1], S.v[cur ^ 1], cnt, (int)sh, S.hw, S.scan);
        cur ^= 1;
    }
    for (uint32_t j = threadIdx.x; j < cnt; j += R2_THREADS) out.put(obase + (int32_t)j, S.v[cur][j]);
    __syncthreads();
}

// Sort in[0..n) by key (stable: equal keys keep input order); out.put(position, payload).
template <class In, class Out>
__device__ void r2_sort(const In& in, const Out& out, int32_t n, R2Smem& S) {
    if (n <= 0) return;
    // key range
    uint32_t lo = 0xffffffffu, hi = 0u;
    for (int32_t i = threadIdx.x; i < n; i += R2_THREADS) {
        const uint32_t k = in.k(i);
        lo = min(lo, k);
        hi = max(hi, k);
    }
    lo = __reduce_min_sync(0xffffffffu, lo);
    hi = __reduce_max_sync(0xffffffffu, hi);
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    if (lane == 0) {
        S.scan[w] = lo;
        S.scan[32 + w] = hi;
    }
    __syncthreads();
    uint32_t* stk = S.misc + 4 * R2_MAXG;          // [R2_MAXS][4]: lo, hi, obase, count
    uint32_t* nstk = S.misc + 4 * R2_MAXG + 4 * R2_MAXS;
    if (threadIdx.x == 0) {
        uint32_t a = 0xffffffffu, b = 0;
        for (int j = 0; j < R2_WARPS; j++) {
            a = min(a, S.scan[j]);
            b = max(b, S.scan[32 + j]);
        }
        stk[0] = a;
        stk[1] = b;
        stk[2] = 0;
        stk[3] = (uint32_t)n;
        *nstk = 1;
    }
    __syncthreads();
    while (true) {
        const uint32_t ns = *nstk;
        if (ns == 0) break;
        const uint32_t rlo = stk[(ns - 1) * 4], rhi = stk[(ns - 1) * 4 + 1];
        const int32_t rob = (int32_t)stk[(ns - 1) * 4 + 2];
        const uint32_t rcnt = stk[(ns - 1) * 4 + 3];
        __syncthreads();
        if (threadIdx.x == 0) *nstk = ns - 1;
        if (rlo == rhi) {
            r2_stream_equal(in, out, n, rlo, rob, S.scan);
            __syncthreads();
            continue;
        }
        if (rcnt <= (uint32_t)R2_CAP) {
            r2_round(in, out, n, rlo, rhi, rcnt, rob, S);
            continue;
        }
        // histogram of the range over <= 4096 bins
        const uint32_t span = rhi - rlo;
        const uint32_t shift = r2_bitlen(span) > 12 ? r2_bitlen(span) - 12 : 0;
        const uint32_t nb = (span >> shift) + 1;
        for (uint32_t b = threadIdx.x; b < R2_NBINS; b += R2_THREADS) S.hw[b] = 0;
        __syncthreads();
        for (int32_t i = threadIdx.x; i < n; i += R2_THREADS) {
            const uint32_t k = in.k(i);
            if (k >= rlo && k <= rhi) atomicAdd(&S.hw[(k - rlo) >> shift], 1u);
        }
        __syncthreads();
        // group boundaries: a new group starts at bin 0, at a bin > CAP/2 or right after one,
        // and where the exclusive prefix crosses a multiple of CAP/2 -- so every multi-bin
        // group holds <= CAP entries; a single bin > CAP becomes a deferred (finer) range.
        const uint32_t H = R2_CAP / 2;
        uint32_t c4[4], s4 = 0;
#pragma unroll
        for (int j = 0; j < 4; j++) {
            const uint32_t b = threadIdx.x * 4 + j;
            c4[j] = b < nb ? S.hw[b] : 0u;
            s4 += c4[j];
        }
        const uint32_t up = __shfl_up_sync(0xffffffffu, c4[3], 1);
        const uint32_t prev_c = threadIdx.x == 0 ? 0u : (lane == 0 ? S.hw[threadIdx.x * 4 - 1] : up);
        uint32_t tot;
        const uint32_t ex = r2_scan(s4, S.scan, tot);   // (contains barriers: hw reads above are done)
        uint32_t flags = 0;
        {
            uint32_t e = ex, pc = prev_c, pe = ex - prev_c;
#pragma unroll
            for (int j = 0; j < 4; j++) {
                const uint32_t b = threadIdx.x * 4 + j;
                if (b < nb && (b == 0 || c4[j] > H || pc > H || (e / H) != (pe / H))) flags |= 1u << j;
                S.hw[b] = e;  // exclusive prefix of bin b (bins >= nb: the total)
                pe = e;
                pc = c4[j];
                e += c4[j];
            }
        }
        uint32_t ng;
        const uint32_t gpos = r2_scan((uint32_t)__popc(flags), S.scan, ng);
        uint32_t* grp = S.misc;  // [R2_MAXG][4]: start bin, start prefix
        if (ng > R2_MAXG) {
            // cannot happen for n < 65536 (<= 2n/(CAP/2)+1 groups); stay correct anyway:
            // split the range at the middle bin into two deferred ranges with exact counts.
            if (threadIdx.x == 0) {
                const uint32_t m = nb / 2;
                const uint32_t pm = S.hw[m];
                uint32_t k2 = *nstk;
                stk[k2 * 4] = rlo; stk[k2 * 4 + 1] = rlo + (m << shift) - 1u;
                stk[k2 * 4 + 2] = (uint32_t)rob; stk[k2 * 4 + 3] = pm;
                k2++;
                stk[k2 * 4] = rlo + (m << shift); stk[k2 * 4 + 1] = rhi;
                stk[k2 * 4 + 2] = (uint32_t)rob + pm; stk[k2 * 4 + 3] = tot - pm;
                k2++;
                *nstk = k2;
            }
            __syncthreads();
            continue;
        }
        {
            uint32_t e = ex, gp = gpos;
#pragma unroll
            for (int j = 0; j < 4; j++) {
                if ((flags >> j) & 1u) {
                    grp[gp * 4] = threadIdx.x * 4 + j;
                    grp[gp * 4 + 1] = e;
                    gp++;
                }
                e += c4[j];
            }
        }
        __syncthreads();
        for (uint32_t gi = 0; gi < ng; gi++) {
            const uint32_t b0 = grp[gi * 4], e0 = grp[gi * 4 + 1];
            const uint32_t b1 = gi + 1 < ng ? grp[(gi + 1) * 4] : nb;
            const uint32_t e1 = gi + 1 < ng ? grp[(gi + 1) * 4 + 1] : tot;
            const uint32_t cnt = e1 - e0;
            if (cnt == 0) continue;
            const uint32_t klo = rlo + (b0 << shift);
            const uint32_t khi = b1 >= nb ? rhi : rlo + (b1 << shift) - 1u;
            if (cnt <= (uint32_t)R2_CAP) {
                r2_round(in, out, n, klo, khi, cnt, rob + (int32_t)e0, S);
            } else {
                __syncthreads();
                if (threadIdx.x == 0) {
                    uint32_t k2 = *nstk;
                    stk[k2 * 4] = klo;
                    stk[k2 * 4 + 1] = khi;
                    stk[k2 * 4 + 2] = (uint32_t)(rob + (int32_t)e0);
                    stk[k2 * 4 + 3] = cnt;
                    *nstk = k2 + 1;
                }
                __syncthreads();
            }
        }
        __syncthreads();
    }
    __syncthreads();
}

template <int A>
__global__ void __launch_bounds__(R2_THREADS, 1) k_rep2_sort(Rep2Args a) {
    extern __shared__ __align__(16) unsigned char r2s[];
    R2Smem S;
    S.k[0] = reinterpret_cast<uint32_t*>(r2s);
    S.k[1] = S.k[0] + R2_CAP;
    S.v[0] = reinterpret_cast<uint16_t*>(S.k[1] + R2_CAP);
    S.v[1] = S.v[0] + R2_CAP;
    S.hw = reinterpret_cast<uint32_t*>(S.v[1] + R2_CAP);
    S.scan = S.hw + 8192;
    S.misc = S.scan + 64;
    __shared__ uint32_t s_tick, s_head;
    uint32_t* skey = a.s_key + (int64_t)blockIdx.x * a.n;
    uint16_t* spi = a.s_pi + (int64_t)blockIdx.x * a.n;
    bool bad = false;
    while (true) {
        if (threadIdx.x == 0) s_tick = atomicAdd(a.ticket, 1u);
        __syncthreads();
        const int64_t rl = s_tick;
        __syncthreads();
        if (rl >= a.R) break;
        const int64_t r = a.r0 + rl;
        const float CP = a.cp[rl];
        for (int32_t t = threadIdx.x; t < a.n; t += R2_THREADS) {
            const float blv = a.blT[rl * a.n + t];
            const float c = CP > 0.0f ? __fdiv_rn(blv, CP) : 0.0f;
            skey[t] = ONE_BITS - f2u(c);
        }
        __syncthreads();
        r2_sort(R2CritIn{skey}, R2PiOut{spi}, a.n, S);
        __syncthreads();
        int64_t qoff = 0;
        for (int b = 0; b < A; b++) {
            const float h = u2f(a.hd[rl * A + b]);
            const int32_t cnt = a.counts[rl * A + b];
            for (int32_t p = threadIdx.x; p < a.n; p += R2_THREADS) {
                const int32_t t = spi[p];
                float x[A];
                uint32_t en;
                int k;
                float wt;
                r2_durs<A>(a, r, t, x, en, k, wt, bad);
                uint32_t key = 0x40000000u;  // not enabled: after every real key (<= 0x3F800000)
                if ((en >> b) & 1u) {
                    float gv;
                    if (k == 1) gv = 1.0f;
                    else if (h == 0.0f) gv = 0.5f;
                    else {
                        float ref = __uint_as_float(0x7f800000u);
#pragma unroll
                        for (int q = 0; q < A; q++)
                            if (q != b && ((en >> q) & 1u)) ref = x[q] < ref ? x[q] : ref;
                        gv = __fdiv_rn(__fadd_rn(__fsub_rn(ref, x[b]), h), __fadd_rn(h, h));
                    }
                    key = ONE_BITS - f2u(gv);
                }
                skey[p] = key;
            }
            if (threadIdx.x == 0) s_head = 0xffffffffu;
            __syncthreads();
            int32_t* qdst = a.qtask ? a.qtask + rl * (int64_t)a.n * A + qoff : nullptr;
            r2_sort(R2GainIn{skey, spi}, R2QOut{qdst, cnt, &s_head}, a.n, S);
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
    size_t bytes = align256((size_t)groups * n * 32 * 4) + align256((size_t)R * n * 4) + align256((size_t)R * A * 4) * 2 +
                   align256((size_t)R * A * 16) + align256((size_t)grid2 * n * 4) + align256((size_t)grid2 * n * 2);
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
    a.blT = ar.take<float>((size_t)R * n);
    a.cp = cp;
    a.hd = ar.take<uint32_t>((size_t)R * A);
    a.counts = ar.take<int32_t>((size_t)R * A);
    a.brw = ar.take<unsigned long long>((size_t)R * A * 2);
    a.err = dag->err;
    a.s_key = ar.take<uint32_t>((size_t)grid2 * n);
    a.s_pi = ar.take<uint16_t>((size_t)grid2 * n);
    a.qtask = qtask;
    a.sum = sum;
    a.ticket = dag->tickets + 56;
    static bool attr = false;
    const int smem1 = 32 * 32 * 33 * 4;
    const int smem2 = (2 * R2_CAP * 4) + (2 * R2_CAP * 2) + 8192 * 4 + 64 * 4 + 512 * 4;
    if (!attr) {
        MP_CUDA(cudaFuncSetAttribute(k_rep2_bl<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem1));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_bl<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem1));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_bl<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem1));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_bl<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem1));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_sort<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_sort<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_sort<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2));
        MP_CUDA(cudaFuncSetAttribute(k_rep2_sort<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2));
        attr = true;
    }
    MP_LAUNCH(k_rep2_bl<A>, (unsigned)groups, R2_THREADS, smem1, st, a);
    MP_CUDA(cudaMemsetAsync(a.ticket, 0, 4, st));
    MP_LAUNCH(k_rep2_sort<A>, (unsigned)grid2, R2_THREADS, smem2, st, a);
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
