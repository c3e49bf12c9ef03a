// replicas.cuh -- a10: batched duration-perturbed replicas of one DAG.
//
// Small DAGs (n <= SMALL_CAP): one CTA per replica computes, in shared memory,
// the perturbed durations' statistics (hd, counts, exact best_remaining_work),
// the bottom-levels level by level, CP, then the 60-bit keys of every (arch,
// task) entry; a segmented radix sort (segment = (replica, arch)) orders the
// entries and k_rep_out emits queues and summaries.  Larger DAGs run the
// single-DAG path once per replica on perturbed durations.
#pragma once
#include "path.cuh"

namespace mpk {

struct RepArgs {
    int32_t n, A, L;
    const int32_t* lvlq;
    const int32_t* nodeq;
    const int32_t* rowq;
    const int32_t* colq;
    const int32_t* qof;
    const float* base;
    uint32_t emask;
    uint64_t seed;
    float sigma;
    int64_t r0;                 // global replica id of blockIdx.x == 0
    uint64_t* skeys;            // [RB][A][n]
    uint32_t* svals;            // [RB][A][n]
    float* cp;                  // [RB]
    int32_t* counts;            // [RB][A]
    unsigned long long* brw;    // [RB][A][2]
    uint32_t* err;
};

MP_INLINE void rep_durs(const RepArgs& a, int64_t r, int32_t t, float* x, uint32_t& en, int& k, float& w,
                        bool& bad) {
    en = 0;
    k = 0;
    w = __uint_as_float(0x7f800000u);
    for (int b = 0; b < a.A; b++) {
        uint64_t c = ((uint64_t)r * (uint64_t)a.n + (uint64_t)t) * (uint64_t)a.A + (uint64_t)b + 1u;
        float d = perturb(__ldg(a.base + (int64_t)t * a.A + b), a.seed, a.sigma, c);
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

__global__ void __launch_bounds__(1024) k_rep_main(RepArgs a) {
    extern __shared__ float sbl[];
    __shared__ uint32_t s_hd[MAX_ARCH];
    __shared__ int32_t s_cnt[MAX_ARCH];
    __shared__ unsigned long long s_brw[MAX_ARCH][2];
    __shared__ uint32_t s_cp;
    const int64_t b = blockIdx.x;
    const int64_t r = a.r0 + b;
    const int lane = threadIdx.x & 31;
    if (threadIdx.x < MAX_ARCH) {
        s_hd[threadIdx.x] = 0;
        s_cnt[threadIdx.x] = 0;
        s_brw[threadIdx.x][0] = 0;
        s_brw[threadIdx.x][1] = 0;
    }
    if (threadIdx.x == 0) s_cp = 0;
    __syncthreads();
    bool bad = false;
    // phase 1: per-task statistics of the perturbed durations
    {
        uint32_t hl[MAX_ARCH];
        int32_t cl[MAX_ARCH];
        uint64_t blo[MAX_ARCH], bhi[MAX_ARCH];
        for (int q = 0; q < MAX_ARCH; q++) { hl[q] = 0; cl[q] = 0; blo[q] = 0; bhi[q] = 0; }
        const int32_t rounds = (a.n + blockDim.x - 1) / blockDim.x;
        for (int32_t it = 0; it < rounds; it++) {
            int32_t t = it * blockDim.x + threadIdx.x;
            if (t < a.n) {
                float x[MAX_ARCH];
                uint32_t en;
                int k;
                float w;
                rep_durs(a, r, t, x, en, k, w, bad);
                for (int q = 0; q < a.A; q++) {
                    if (!((en >> q) & 1u)) continue;
                    cl[q]++;
                    if (x[q] == w) {
                        uint64_t l, h;
                        fixed64(x[q], l, h);
                        add128(blo[q], bhi[q], l, h);
                    }
                    if (k >= 2) {
                        float ref = __uint_as_float(0x7f800000u);
                        for (int p = 0; p < a.A; p++)
                            if (p != q && ((en >> p) & 1u)) ref = x[p] < ref ? x[p] : ref;
                        uint32_t ab = f2u(fabsf(__fsub_rn(ref, x[q])));
                        hl[q] = ab > hl[q] ? ab : hl[q];
                    }
                }
            }
        }
        for (int q = 0; q < a.A; q++) {
            uint32_t h = warp_max(hl[q]);
            int32_t c = cl[q];
            for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
            uint64_t lo = blo[q], hi = bhi[q];
            warp_sum128(lo, hi);
            if (lane == 0) {
                if (h) atomicMax(&s_hd[q], h);
                if (c) atomicAdd(&s_cnt[q], c);
                if (lo || hi) {
                    unsigned long long old = atomicAdd(&s_brw[q][0], (unsigned long long)lo);
                    uint64_t carry = (old + lo < old) ? 1ull : 0ull;
                    if (hi + carry) atomicAdd(&s_brw[q][1], (unsigned long long)(hi + carry));
                }
            }
        }
    }
    // phase 2: bottom-levels, deepest level first, one barrier per level
    float cpm = 0.0f;
    for (int32_t lv = 0; lv < a.L; lv++) {
        const int32_t q1 = __ldg(a.lvlq + lv + 1);
        for (int32_t q = __ldg(a.lvlq + lv) + threadIdx.x; q < q1; q += blockDim.x) {
            const int32_t v = __ldg(a.nodeq + q);
            float x[MAX_ARCH];
            uint32_t en;
            int k;
            float w;
            rep_durs(a, r, v, x, en, k, w, bad);
            if (!k) w = 0.0f;
            float m = 0.0f;
            const int32_t e1 = __ldg(a.rowq + q + 1);
            for (int32_t e = __ldg(a.rowq + q); e < e1; e++) m = fmaxf(m, sbl[__ldg(a.colq + e)]);
            const float bb = __fadd_rn(w, m);
            sbl[q] = bb;
            cpm = fmaxf(cpm, bb);
        }
        __syncthreads();
    }
    cpm = warp_max(cpm);
    if (lane == 0) atomicMax(&s_cp, f2u(cpm));
    __syncthreads();
    const float CP = u2f(s_cp);
    // phase 3: keys of every (arch, task) entry: ((1-gain bits) << 30) | (1-crit_n bits)
    for (int32_t t = threadIdx.x; t < a.n; t += blockDim.x) {
        float x[MAX_ARCH];
        uint32_t en;
        int k;
        float w;
        rep_durs(a, r, t, x, en, k, w, bad);
        const float blv = sbl[__ldg(a.qof + t)];
        const float cn = CP > 0.0f ? __fdiv_rn(blv, CP) : 0.0f;
        for (int q = 0; q < a.A; q++) {
            uint64_t key = 1ull << 60;  // not enabled: sorts after every entry
            if ((en >> q) & 1u) {
                float g;
                float h = u2f(s_hd[q]);
                if (k == 1) g = 1.0f;
                else if (h == 0.0f) g = 0.5f;
                else {
                    float ref = __uint_as_float(0x7f800000u);
                    for (int p = 0; p < a.A; p++)
                        if (p != q && ((en >> p) & 1u)) ref = x[p] < ref ? x[p] : ref;
                    g = __fdiv_rn(__fadd_rn(__fsub_rn(ref, x[q]), h), __fadd_rn(h, h));
                }
                key = ((uint64_t)(ONE_BITS - f2u(g)) << 30) | (uint64_t)(ONE_BITS - f2u(cn));
            }
            int64_t o = (b * a.A + q) * (int64_t)a.n + t;
            a.skeys[o] = key;
            a.svals[o] = (uint32_t)t;
        }
    }
    if (threadIdx.x < a.A) {
        a.counts[b * a.A + threadIdx.x] = s_cnt[threadIdx.x];
        a.brw[(b * a.A + threadIdx.x) * 2] = s_brw[threadIdx.x][0];
        a.brw[(b * a.A + threadIdx.x) * 2 + 1] = s_brw[threadIdx.x][1];
    }
    if (threadIdx.x == 0) a.cp[b] = CP;
    if (__any_sync(0xffffffffu, bad) && lane == 0) atomicOr(a.err, ERR_DOMAIN_BIT);
}

// one block per segment (replica b, arch q): queue copy + summary
__global__ void k_rep_out(int32_t n, int32_t A, const SortPlan* plans, const uint32_t* vals0,
                          const uint32_t* vals1, const int32_t* counts, const unsigned long long* brw,
                          mp_queue_summary* sum, int32_t* qtask) {
    const int64_t s = blockIdx.x;
    const int64_t b = s / A;
    const int q = (int)(s % A);
    const uint32_t* v = (plans[s].final_sel ? vals1 : vals0) + s * (int64_t)n;
    const int32_t cnt = counts[s];
    if (qtask) {
        int64_t off = b * (int64_t)n * A;
        for (int p = 0; p < q; p++) off += counts[b * A + p];
        for (int32_t i = threadIdx.x; i < cnt; i += blockDim.x) qtask[off + i] = (int32_t)v[i];
    }
    if (threadIdx.x == 0) {
        mp_queue_summary o;
        o.count = cnt;
        o.head = cnt > 0 ? (int32_t)v[0] : -1;
        o.brw_lo = brw[2 * s];
        o.brw_hi = (int64_t)brw[2 * s + 1];
        o.brw = u128_to_double_scaled(brw[2 * s], brw[2 * s + 1]);
        sum[s] = o;
    }
}

__global__ void k_perturb(int32_t n, int32_t A, const float* base, uint64_t seed, float sigma, int64_t r,
                          float* out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (int64_t)n * A;
         i += (int64_t)gridDim.x * blockDim.x) {
        uint64_t c = (uint64_t)r * (uint64_t)n * (uint64_t)A + (uint64_t)i + 1u;
        out[i] = perturb(base[i], seed, sigma, c);
    }
}

}  // namespace mpk

namespace mph {

inline bool rep2_eligible(const mp_dag* dag, int32_t A);
inline mp_status replicas_run2(mp_dag* dag, int32_t A, const float* base, uint32_t emask, uint64_t seed, float sigma,
                               int64_t r0, int32_t R, float* cp, mp_queue_summary* sum, int32_t* qtask,
                               cudaStream_t st);

inline mp_status replicas_run(mp_dag* dag, int32_t A, const float* base, const int32_t* h_workers, uint64_t seed,
                              float sigma, int64_t r0, int32_t R, float* cp, mp_queue_summary* sum,
                              int32_t* qtask, cudaStream_t st) {
    using namespace mpk;
    if (!dag) return fail(MP_ERR_ARG, "dag is NULL");
    MP_TRY(check_arch(A, h_workers));
    if (R < 0 || r0 < 0) return fail(MP_ERR_ARG, "negative replica range");
    if (R == 0) return MP_OK;
    if (!cp || !sum || (dag->n > 0 && !base)) return fail(MP_ERR_ARG, "NULL buffer");
    const int32_t n = dag->n;
    const uint32_t emask = enabled_mask(A, h_workers);
    if (n == 0) {
        // every replica of an empty DAG: CP 0, empty queues
        std::vector<mp_queue_summary> h((size_t)R * A);
        for (auto& x : h) { x.count = 0; x.head = -1; x.brw_lo = 0; x.brw_hi = 0; x.brw = 0.0; }
        MP_CUDA(cudaMemsetAsync(cp, 0, (size_t)R * 4, st));
        MP_CUDA(cudaMemcpyAsync(sum, h.data(), h.size() * sizeof(mp_queue_summary), cudaMemcpyHostToDevice, st));
        MP_CUDA(cudaStreamSynchronize(st));
        return MP_OK;
    }
    if (rep2_eligible(dag, A))
        return replicas_run2(dag, A, base, emask, seed, sigma, r0, R, cp, sum, qtask, st);
    if (n <= SMALL_CAP) {
        const int64_t per = (int64_t)A * n;
        int32_t RB = (int32_t)std::min<int64_t>(R, std::max<int64_t>(1, (int64_t)(256ll << 20) / (per * 24)));
        RB = std::max(1, std::min(RB, 1024));
        const size_t bytes = sort_bytes(n, RB * A, 8, true) + align256((size_t)RB * A * 4) +
                             align256((size_t)RB * A * 16) + align256((size_t)RB * 4);
        MP_TRY(ensure_ws(dag, bytes, st));
        Arena ar{dag->ws, dag->ws_cap};
        SortArgs sa = carve_sort(ar, dag, n, RB * A, 0, 8, true);
        int32_t* counts = ar.take<int32_t>((size_t)RB * A);
        unsigned long long* brw = ar.take<unsigned long long>((size_t)RB * A * 2);
        static std::atomic<uint64_t> attr{0};
        if (first_on_device(attr))
            MP_CUDA(cudaFuncSetAttribute(k_rep_main, cudaFuncAttributeMaxDynamicSharedMemorySize, SMALL_CAP * 4));
        for (int64_t b0 = 0; b0 < R; b0 += RB) {
            const int32_t nb = (int32_t)std::min<int64_t>(RB, R - b0);
            RepArgs ra{n, A, dag->L, dag->lvlq, dag->nodeq, dag->rowq, dag->colq, dag->qof, base, emask, seed, sigma,
                       r0 + b0, sa.keys[0], sa.vals[0], cp + b0, counts, brw, dag->err};
            MP_LAUNCH(k_rep_main, nb, 1024, (size_t)n * 4, st, ra);
            MP_CUDA(cudaGetLastError());
            SortArgs s2 = sa;
            s2.nseg = nb * A;
            MP_TRY(run_sort(dag, s2, st));
            MP_LAUNCH(k_rep_out, nb * A, 256, 0, st, n, A, s2.plans, s2.vals[0], s2.vals[1], counts, brw, sum + b0 * A,
                                              qtask ? qtask + b0 * (int64_t)n * A : nullptr);
            MP_CUDA(cudaGetLastError());
        }
        return MP_OK;
    }
    // large DAGs: the single-DAG path per replica on perturbed durations
    const int64_t nA = (int64_t)n * A;
    float *dr, *bl, *gain, *critn, *hd;
    uint8_t* flags;
    uint64_t* key;
    int64_t* qptr;
    int32_t* qscratch = nullptr;
    MP_CUDA(cudaMallocAsync(&dr, nA * 4, st));
    MP_CUDA(cudaMallocAsync(&bl, (size_t)n * 4, st));
    MP_CUDA(cudaMallocAsync(&gain, nA * 4, st));
    MP_CUDA(cudaMallocAsync(&critn, (size_t)n * 4, st));
    MP_CUDA(cudaMallocAsync(&hd, 64, st));
    MP_CUDA(cudaMallocAsync(&flags, nA, st));
    MP_CUDA(cudaMallocAsync(&key, nA * 8, st));
    MP_CUDA(cudaMallocAsync(&qptr, 8 * (MAX_ARCH + 1), st));
    if (!qtask) MP_CUDA(cudaMallocAsync(&qscratch, nA * 4, st));
    mp_status rc = MP_OK;
    for (int64_t i = 0; i < R && rc == MP_OK; i++) {
        MP_LAUNCH(k_perturb, grid_for(nA), 256, 0, st, n, A, base, seed, sigma, r0 + i, dr);
        rc = bottom_level(dag, A, dr, h_workers, bl, cp + i, nullptr, st);
        if (rc == MP_OK) rc = affinity(dag, A, dr, h_workers, gain, hd, flags, st);
        if (rc == MP_OK) rc = score(dag, A, 0, bl, gain, flags, critn, key, st);
        if (rc == MP_OK)
            rc = build_queues(dag, A, key, flags, dr, nullptr, qptr, qtask ? qtask + i * nA : qscratch, sum + i * A,
                              st);
    }
    cudaFreeAsync(dr, st);
    cudaFreeAsync(bl, st);
    cudaFreeAsync(gain, st);
    cudaFreeAsync(critn, st);
    cudaFreeAsync(hd, st);
    cudaFreeAsync(flags, st);
    cudaFreeAsync(key, st);
    cudaFreeAsync(qptr, st);
    if (qscratch) cudaFreeAsync(qscratch, st);
    return rc;
}

}  // namespace mph
