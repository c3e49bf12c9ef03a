// variants.cuh -- SURVEY §8(f) N4: ablations of readings c2 / c4 / c10.
//   mp_bottom_level_w   : bottom-level with the HEFT mean-cost node weight (v1)
//                         -- the weight lives in path.cuh's task_weight
//   mp_affinity_prefix  : hd(a) "recorded so far" (P:l.176) as a running max
//                         along a push order (v2): an inclusive max-scan
//   mp_nod_remaining    : NOD on the remaining graph (v3) -- path.cuh's NOD
//                         kernels with a `done` mask
#pragma once
#include "path.cuh"

namespace mpk {

constexpr int PFX_TILE = 1024;   // push positions per block, one per thread

// |d(t,a)| bits for a two-or-more-arch task enabled on a (c5), else 0; the
// rounded d itself, the enabled mask and w(t) for the gain pass.
MP_INLINE void pfx_absd(const DurView& d, int32_t t, uint32_t x[MAX_ARCH], float dd[MAX_ARCH], uint32_t& en,
                        float& w, int& k, bool& bad) {
    float v[MAX_ARCH];
    en = 0;
    k = 0;
    w = __uint_as_float(0x7f800000u);
#pragma unroll
    for (int a = 0; a < MAX_ARCH; a++) {
        v[a] = 0.0f;
        if (a < d.A) {
            v[a] = canon_dur(__ldg(d.dur + (int64_t)t * d.A + a), bad);
            if (((d.emask >> a) & 1u) && !is_inf(v[a])) {
                en |= 1u << a;
                k++;
                w = v[a] < w ? v[a] : w;
            }
        }
    }
    if (!k) bad = true;
#pragma unroll
    for (int a = 0; a < MAX_ARCH; a++) {
        x[a] = 0u;
        dd[a] = 0.0f;
        if (a < d.A && ((en >> a) & 1u) && k >= 2) {
            float ref = __uint_as_float(0x7f800000u);
#pragma unroll
            for (int b = 0; b < MAX_ARCH; b++)
                if (b < d.A && b != a && ((en >> b) & 1u)) ref = v[b] < ref ? v[b] : ref;
            dd[a] = __fsub_rn(ref, v[a]);
            x[a] = f2u(fabsf(dd[a]));
        }
    }
}

MP_INLINE int32_t pfx_task(const int32_t* order, int32_t i, int32_t n, bool& badarg) {
    int32_t t = order ? order[i] : i;
    if ((uint32_t)t >= (uint32_t)n) {
        badarg = true;
        return -1;
    }
    return t;
}

// pass 1: max |d| per arch over each tile of push positions
__global__ void __launch_bounds__(PFX_TILE) k_pfx_tile_max(int32_t n, DurView d, const int32_t* __restrict__ order,
                                                           uint32_t* agg, uint32_t* err) {
    __shared__ uint32_t sm[PFX_TILE / 32][MAX_ARCH];
    const int32_t i = blockIdx.x * PFX_TILE + threadIdx.x;
    uint32_t x[MAX_ARCH];
    float dd[MAX_ARCH];
    uint32_t en;
    float w;
    int k;
    bool bad = false, badarg = false;
#pragma unroll
    for (int a = 0; a < MAX_ARCH; a++) x[a] = 0u;
    if (i < n) {
        int32_t t = pfx_task(order, i, n, badarg);
        if (t >= 0) pfx_absd(d, t, x, dd, en, w, k, bad);
    }
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
    for (int a = 0; a < MAX_ARCH; a++) {
        uint32_t v = warp_max(x[a]);
        if (lane == 0) sm[wid][a] = v;
    }
    __syncthreads();
    if (wid == 0) {
#pragma unroll
        for (int a = 0; a < MAX_ARCH; a++) {
            uint32_t v = warp_max(sm[lane][a]);
            if (lane == 0) agg[(int64_t)blockIdx.x * MAX_ARCH + a] = v;
        }
    }
    if (bad) atomicOr(err, ERR_DOMAIN_BIT);
    if (badarg) atomicOr(err, ERR_ARG_BIT);
}

// pass 2 (one block): exclusive max-scan of the tile maxima per arch; the
// total is hd(a) (= mp_affinity's hd)
__global__ void __launch_bounds__(1024) k_pfx_scan_agg(int32_t nblk, int32_t A, const uint32_t* agg,
                                                       uint32_t* carry, float* hd) {
    __shared__ uint32_t wt[32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (int a = 0; a < A; a++) {
        uint32_t run = 0u;
        for (int32_t b0 = 0; b0 < nblk; b0 += 1024) {
            int32_t b = b0 + threadIdx.x;
            uint32_t v = b < nblk ? agg[(int64_t)b * MAX_ARCH + a] : 0u;
            uint32_t inc = v;                                   // inclusive warp scan (max)
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
                if (lane >= o) inc = y > inc ? y : inc;
            }
            if (lane == 31) wt[wid] = inc;
            __syncthreads();
            if (wid == 0) {
                uint32_t s = wt[lane];
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    uint32_t y = __shfl_up_sync(0xffffffffu, s, o);
                    if (lane >= o) s = y > s ? y : s;
                }
                wt[lane] = s;
            }
            __syncthreads();
            uint32_t before = wid > 0 ? wt[wid - 1] : 0u;
            uint32_t excl = __shfl_up_sync(0xffffffffu, inc, 1);
            if (lane == 0) excl = 0u;
            excl = excl > before ? excl : before;
            excl = excl > run ? excl : run;
            if (b < nblk) carry[(int64_t)b * MAX_ARCH + a] = excl;
            uint32_t tot = wt[31];
            run = tot > run ? tot : run;
            __syncthreads();
        }
        if (threadIdx.x == 0) hd[a] = u2f(run);
    }
}

// pass 3: per position, hd_prefix(a) = max(carry, inclusive scan in the tile);
// gain = 1 (one arch) | 0.5 (hd_prefix = 0) | (d + hd) / (hd + hd); flags as mp_affinity
__global__ void __launch_bounds__(PFX_TILE) k_pfx_gain(int32_t n, DurView d, const int32_t* __restrict__ order,
                                                       const uint32_t* carry, float* gain, uint8_t* flags) {
    __shared__ uint32_t wt[PFX_TILE / 32][MAX_ARCH];
    const int32_t i = blockIdx.x * PFX_TILE + threadIdx.x;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    uint32_t x[MAX_ARCH];
    float dd[MAX_ARCH];
    uint32_t en = 0;
    float w = 0.0f;
    int k = 0;
    bool bad = false, badarg = false;
    int32_t t = -1;
#pragma unroll
    for (int a = 0; a < MAX_ARCH; a++) x[a] = 0u;
    if (i < n) {
        t = pfx_task(order, i, n, badarg);
        if (t >= 0) pfx_absd(d, t, x, dd, en, w, k, bad);
    }
    uint32_t inc[MAX_ARCH];
#pragma unroll
    for (int a = 0; a < MAX_ARCH; a++) {
        inc[a] = x[a];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(0xffffffffu, inc[a], o);
            if (lane >= o) inc[a] = y > inc[a] ? y : inc[a];
        }
        if (lane == 31) wt[wid][a] = inc[a];
    }
    __syncthreads();
    if (wid == 0) {
#pragma unroll
        for (int a = 0; a < MAX_ARCH; a++) {
            uint32_t s = wt[lane][a];
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                uint32_t y = __shfl_up_sync(0xffffffffu, s, o);
                if (lane >= o) s = y > s ? y : s;
            }
            wt[lane][a] = s;
        }
    }
    __syncthreads();
    if (t < 0) return;
    for (int a = 0; a < d.A; a++) {
        uint32_t run = inc[a];
        if (wid > 0) run = wt[wid - 1][a] > run ? wt[wid - 1][a] : run;
        uint32_t c = carry[(int64_t)blockIdx.x * MAX_ARCH + a];
        run = c > run ? c : run;
        float g = 0.0f;
        uint8_t f = 0;
        if ((en >> a) & 1u) {
            float x_a = canon_dur(__ldg(d.dur + (int64_t)t * d.A + a), bad);
            f = 1 | (x_a == w ? 2 : 0);
            float h = u2f(run);
            if (k == 1) g = 1.0f;
            else if (h == 0.0f) g = 0.5f;
            else g = __fdiv_rn(__fadd_rn(dd[a], h), __fadd_rn(h, h));
        }
        gain[(int64_t)t * d.A + a] = g;
        flags[(int64_t)t * d.A + a] = f;
    }
}

}  // namespace mpk

namespace mph {

inline mp_status affinity_prefix(mp_dag* dag, int32_t A, const float* dur, const int32_t* h_workers,
                                 const int32_t* order, float* gain, float* hd, uint8_t* flags, cudaStream_t st) {
    using namespace mpk;
    if (!dag) return fail(MP_ERR_ARG, "dag is NULL");
    MP_TRY(check_arch(A, h_workers));
    if (!hd || (dag->n > 0 && (!dur || !gain || !flags))) return fail(MP_ERR_ARG, "NULL buffer");
    DurView d{dur, A, enabled_mask(A, h_workers)};
    const int32_t n = dag->n;
    int32_t nblk = std::max<int32_t>(1, (n + PFX_TILE - 1) / PFX_TILE);
    MP_TRY(ensure_ws(dag, 2 * align256((size_t)nblk * MAX_ARCH * 4), st));
    Arena ar{dag->ws, dag->ws_cap};
    uint32_t* agg = ar.take<uint32_t>((size_t)nblk * MAX_ARCH);
    uint32_t* carry = ar.take<uint32_t>((size_t)nblk * MAX_ARCH);
    if (n == 0) {
        MP_CUDA(cudaMemsetAsync(hd, 0, (size_t)A * 4, st));
        return MP_OK;
    }
    MP_LAUNCH(k_pfx_tile_max, nblk, PFX_TILE, 0, st, n, d, order, agg, dag->err);
    MP_LAUNCH(k_pfx_scan_agg, 1, 1024, 0, st, nblk, A, agg, carry, hd);
    MP_LAUNCH(k_pfx_gain, nblk, PFX_TILE, 0, st, n, d, order, carry, gain, flags);
    MP_CUDA(cudaGetLastError());
    return MP_OK;
}

inline mp_status nod_remaining(mp_dag* dag, int32_t A, const float* dur, const int32_t* h_workers,
                               const uint8_t* done, float* nod, cudaStream_t st) {
    using namespace mpk;
    if (!dag) return fail(MP_ERR_ARG, "dag is NULL");
    MP_TRY(check_arch(A, h_workers));
    const int32_t n = dag->n;
    if (n == 0) return MP_OK;
    if (!dur || !done || !nod) return fail(MP_ERR_ARG, "NULL buffer");
    DurView d{dur, A, enabled_mask(A, h_workers)};
    MP_TRY(ensure_ws(dag, align256((size_t)n * A * 4), st));
    int32_t* inda = (int32_t*)dag->ws;
    MP_CUDA(cudaMemsetAsync(inda, 0, (size_t)n * A * 4, st));
    MP_LAUNCH(k_nod_indeg, grid_for(n), 256, 0, st, n, dag->row_ptr, dag->col, d, done, inda);
    MP_LAUNCH(k_nod_sum, grid_for(n), 256, 0, st, n, dag->row_ptr, dag->col, d, done, inda, nod);
    MP_CUDA(cudaGetLastError());
    return MP_OK;
}

}  // namespace mph
