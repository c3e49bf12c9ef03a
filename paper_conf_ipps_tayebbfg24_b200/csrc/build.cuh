// build.cuh -- a1 + a2: DAG ingest (deduplicated successor CSR) and topological
// levels, plus the reverse-level "q-space" layouts the bottom-level kernels
// walk.  PAPER.md l.83-84 (Table I: lambda^-, lambda^+ as sets), l.89 (G=(V,E)),
// l.91 (a task is ready when all its predecessors are done).
#pragma once
#include <cooperative_groups.h>

#include <vector>

#include "handle.cuh"

namespace cg = cooperative_groups;

namespace mpk {

// ---- a1: counting-sort CSR ingest ------------------------------------------------------
// Edges are bucketed by source (count -> scan -> fill), then every row is sorted and
// deduplicated by one warp in registers; rows longer than CSR_WARP_MAX go through the
// radix sorter instead.  The result is the deduplicated successor CSR with each row
// ascending (the canonical order every later step relies on).
constexpr int CSR_WARP_K = 8;                    // elements per lane
constexpr int CSR_WARP_MAX = 32 * CSR_WARP_K;    // longest row a warp sorts (256)

// warp-aggregated validation + out-degree count.  Invalid edges set ERR_ARG_BIT and are
// dropped (the build then fails).
__global__ void k_csr_count(const int32_t* src, const int32_t* dst, int64_t m, int32_t n, int32_t* cnt,
                            uint32_t* err, int32_t* backward) {
    const int lane = threadIdx.x & 31;
    const int64_t wstride = (int64_t)gridDim.x * blockDim.x;
    bool bad = false, back = false;
    for (int64_t base = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) & ~31ll; base < m; base += wstride) {
        int64_t i = base + lane;
        int32_t u = -1;
        if (i < m) {
            int32_t uu = src[i], v = dst[i];
            if (uu < 0 || uu >= n || v < 0 || v >= n || uu == v) bad = true;
            else u = uu;
            back |= uu > v;
        }
        unsigned peers = __match_any_sync(0xffffffffu, u);
        int leader = __ffs(peers) - 1;
        if (u >= 0 && lane == leader) atomicAdd(&cnt[u], __popc(peers));
    }
    if (__any_sync(0xffffffffu, bad) && lane == 0) atomicOr(err, ERR_ARG_BIT);
    if (__any_sync(0xffffffffu, back) && lane == 0) *backward = 1;   // id order is not topological
}

// scatter dst into its source's bucket: rs = exclusive scan of the counts; cnt counts down
// to 0 (order inside a bucket is arbitrary, the row sort makes it canonical).
__global__ void k_csr_fill(const int32_t* src, const int32_t* dst, int64_t m, int32_t n, const int32_t* rs,
                           int32_t* cnt, int32_t* tmp) {
    const int lane = threadIdx.x & 31;
    const int64_t wstride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) & ~31ll; base < m; base += wstride) {
        int64_t i = base + lane;
        int32_t u = -1, v = 0;
        if (i < m) {
            int32_t uu = src[i];
            v = dst[i];
            if (!(uu < 0 || uu >= n || v < 0 || v >= n || uu == v)) u = uu;
        }
        unsigned peers = __match_any_sync(0xffffffffu, u);
        int leader = __ffs(peers) - 1;
        int k = __popc(peers);
        int old = 0;
        if (u >= 0 && lane == leader) old = atomicSub(&cnt[u], k);
        old = __shfl_sync(0xffffffffu, old, leader);
        if (u >= 0) tmp[rs[u] + old - k + __popc(peers & lanemask_lt())] = v;
    }
}

// one warp, one row of L <= 32*K entries: rank sort in registers (ties by slot) into a
// shared-memory run, then dedup + compaction straight to srt.  Returns the unique count.
template <int K>
__device__ __forceinline__ int csr_row_sort(const int32_t* in, int32_t L, int32_t* run, int32_t* out, int lane) {
    int32_t e[K];
    int rank[K];
#pragma unroll
    for (int k = 0; k < K; k++) {
        int j = k * 32 + lane;
        e[k] = j < L ? in[j] : 0x7fffffff;
        rank[k] = 0;
    }
#pragma unroll
    for (int kk = 0; kk < K; kk++) {
        const int lim = min(32, L - kk * 32);
        for (int l = 0; l < lim; l++) {
            const int32_t y = __shfl_sync(0xffffffffu, e[kk], l);
#pragma unroll
            for (int k = 0; k < K; k++)
                rank[k] += (y < e[k] || (y == e[k] && (kk < k || (kk == k && l < lane)))) ? 1 : 0;
        }
    }
#pragma unroll
    for (int k = 0; k < K; k++)
        if (k * 32 + lane < L) run[rank[k]] = e[k];
    __syncwarp();
    int cnt = 0;
#pragma unroll
    for (int k = 0; k < K; k++) {
        const int j = k * 32 + lane;
        int32_t x = 0;
        bool keep = false;
        if (j < L) {
            x = run[j];
            keep = (j == 0) || run[j - 1] != x;
        }
        unsigned bm = __ballot_sync(0xffffffffu, keep);
        if (keep) out[cnt + __popc(bm & lanemask_lt())] = x;
        cnt += __popc(bm);
    }
    __syncwarp();
    return cnt;
}

// one warp, one row of 32 < L <= P entries (P a power of two): bitonic sort of the
// INT_MAX-padded run in shared memory, then dedup + compaction straight to out.
template <int P>
__device__ __forceinline__ int csr_row_bitonic(const int32_t* in, int32_t L, int32_t* run, int32_t* out, int lane) {
#pragma unroll
    for (int j = lane; j < P; j += 32) run[j] = j < L ? in[j] : 0x7fffffff;
    __syncwarp();
#pragma unroll
    for (int k = 2; k <= P; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
#pragma unroll
            for (int t = lane; t < P / 2; t += 32) {
                const int i = ((t & ~(j - 1)) << 1) | (t & (j - 1));
                const int32_t x = run[i], y = run[i + j];
                const bool up = (i & k) == 0;
                if ((x > y) == up) {
                    run[i] = y;
                    run[i + j] = x;
                }
            }
            __syncwarp();
        }
    }
    int cnt = 0;
#pragma unroll
    for (int k = 0; k < P / 32; k++) {
        const int j = k * 32 + lane;
        int32_t x = 0;
        bool keep = false;
        if (j < L) {
            x = run[j];
            keep = (j == 0) || run[j - 1] != x;
        }
        unsigned bm = __ballot_sync(0xffffffffu, keep);
        if (keep) out[cnt + __popc(bm & lanemask_lt())] = x;
        cnt += __popc(bm);
    }
    __syncwarp();
    return cnt;
}

// one warp per row (rows longer than CSR_WARP_MAX are listed for the radix path).
// srt[rs[r] .. rs[r] + ucnt[r]) = sorted distinct successors of r.
// 32 rows per warp: rows of <= 8 entries are sorted by their own lane in registers
// (odd-even transposition network, then dedup), longer rows one at a time by the whole
// warp (rows longer than CSR_WARP_MAX are listed for the radix path).
// srt[rs[r] .. rs[r] + ucnt[r]) = sorted distinct successors of r.
constexpr int CSR_LANE_MAX = 8;
__device__ __forceinline__ int csr_row_warp(const int32_t* tmp, int32_t s, int32_t L, int32_t* run, int32_t* srt,
                                            int lane) {
    if (L <= 32) return csr_row_sort<1>(tmp + s, L, run, srt + s, lane);
    if (L <= 64) return csr_row_bitonic<64>(tmp + s, L, run, srt + s, lane);
    if (L <= 128) return csr_row_bitonic<128>(tmp + s, L, run, srt + s, lane);
    return csr_row_bitonic<CSR_WARP_MAX>(tmp + s, L, run, srt + s, lane);
}

// rpw rows per warp (1..32; the host picks fewer for small n so every warp has work);
// mid_list != null: rows of CSR_LANE_MAX < L <= CSR_WARP_MAX are listed for
// k_csr_rowsort_mid (one warp each) instead of being sorted one after another here.
__global__ void __launch_bounds__(256) k_csr_rowsort(int32_t n, const int32_t* rs, const int32_t* tmp, int32_t* srt,
                                                     int32_t* ucnt, int32_t* big_list,
                                                     int32_t* big_ctr /* [0]=rows, [1]=entries, [2]=mid rows */,
                                                     int32_t* big_off, int rpw, int32_t* mid_list) {
    __shared__ int32_t runs[8][CSR_WARP_MAX];
    const int lane = threadIdx.x & 31;
    int32_t* run = runs[threadIdx.x >> 5];
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r0 = ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5) * rpw; r0 < n; r0 += nw * rpw) {
        const int64_t rl = r0 + lane;
        int32_t sl = 0, Ll = 0;
        if (lane < rpw && rl < n) {
            sl = rs[rl];
            Ll = rs[rl + 1] - sl;
        }
        if (lane < rpw && rl < n && Ll <= CSR_LANE_MAX) {
            int32_t x[CSR_LANE_MAX];
#pragma unroll
            for (int q = 0; q < CSR_LANE_MAX; q++) x[q] = q < Ll ? tmp[sl + q] : 0x7fffffff;
#pragma unroll
            for (int rd = 0; rd < CSR_LANE_MAX; rd++) {
#pragma unroll
                for (int q = rd & 1; q + 1 < CSR_LANE_MAX; q += 2) {
                    const int32_t lo = min(x[q], x[q + 1]), hi = max(x[q], x[q + 1]);
                    x[q] = lo;
                    x[q + 1] = hi;
                }
            }
            int c = 0;
#pragma unroll
            for (int q = 0; q < CSR_LANE_MAX; q++) {
                if (q < Ll && (q == 0 || x[q] != x[q - 1])) {
                    srt[sl + c] = x[q];
                    c++;
                }
            }
            ucnt[rl] = c;
        }
        const bool listed = mid_list && lane < rpw && rl < n && Ll > CSR_LANE_MAX && Ll <= CSR_WARP_MAX;
        if (listed) {
            cg::coalesced_group g = cg::coalesced_threads();
            int32_t base = 0;
            if (g.thread_rank() == 0) base = atomicAdd(&big_ctr[2], (int32_t)g.size());
            mid_list[g.shfl(base, 0) + (int32_t)g.thread_rank()] = (int32_t)rl;
        }
        unsigned bigm = __ballot_sync(0xffffffffu, !listed && lane < rpw && rl < n && Ll > CSR_LANE_MAX);
        while (bigm) {
            const int l = __ffs(bigm) - 1;
            bigm &= bigm - 1;
            const int64_t r = r0 + l;
            const int32_t s = __shfl_sync(0xffffffffu, sl, l), L = __shfl_sync(0xffffffffu, Ll, l);
            if (L > CSR_WARP_MAX) {
                if (lane == 0) {
                    int idx = atomicAdd(&big_ctr[0], 1);
                    big_list[idx] = (int32_t)r;
                    big_off[idx] = atomicAdd(&big_ctr[1], L);
                }
                continue;
            }
            const int c = csr_row_warp(tmp, s, L, run, srt, lane);
            if (lane == 0) ucnt[r] = c;
        }
    }
}

// the listed medium rows, one warp each
__global__ void __launch_bounds__(256) k_csr_rowsort_mid(const int32_t* mid_list, const int32_t* mid_cnt,
                                                         const int32_t* rs, const int32_t* tmp, int32_t* srt,
                                                         int32_t* ucnt) {
    __shared__ int32_t runs[8][CSR_WARP_MAX];
    const int lane = threadIdx.x & 31;
    int32_t* run = runs[threadIdx.x >> 5];
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int32_t cnt = *mid_cnt;
    for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; i < cnt; i += nw) {
        const int32_t r = mid_list[i];
        const int32_t s = rs[r], L = rs[r + 1] - s;
        const int c = csr_row_warp(tmp, s, L, run, srt, lane);
        if (lane == 0) ucnt[r] = c;
    }
}

// long rows: gather (row << b | dst) keys of every long row for the radix sorter
__global__ void k_csr_big_gather(const int32_t* big_list, const int32_t* big_off, const int32_t* rs,
                                 const int32_t* tmp, int b, uint64_t* keys) {
    const int32_t r = big_list[blockIdx.x];
    const int32_t s = rs[r], L = rs[r + 1] - s;
    uint64_t* o = keys + big_off[blockIdx.x];
    for (int j = threadIdx.x; j < L; j += blockDim.x) o[j] = ((uint64_t)(uint32_t)r << b) | (uint32_t)tmp[s + j];
}

// long rows after the sort: one block per row finds its run (binary search), keeps the
// first of every equal run, and compacts into srt with a block-wide ballot scan.
__global__ void k_csr_big_compact(const int32_t* big_list, const SortPlan* plan, uint64_t* const* kb, int64_t tot,
                                  const int32_t* rs, int b, int32_t* srt, int32_t* ucnt) {
    __shared__ int32_t wsum[32];
    __shared__ int64_t start_s;
    const uint64_t* k = kb[plan->final_sel];
    const int32_t r = big_list[blockIdx.x];
    const int32_t s = rs[r], L = rs[r + 1] - s;
    if (threadIdx.x == 0) {
        const uint64_t want = (uint64_t)(uint32_t)r << b;
        int64_t lo = 0, hi = tot;
        while (lo < hi) {
            int64_t mid = (lo + hi) >> 1;
            if (k[mid] < want) lo = mid + 1;
            else hi = mid;
        }
        start_s = lo;
    }
    __syncthreads();
    const uint64_t* kr = k + start_s;
    const uint64_t mask = (1ull << b) - 1;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nwarp = blockDim.x >> 5;
    int32_t out = 0;
    for (int base = 0; base < L; base += blockDim.x) {
        int j = base + threadIdx.x;
        bool keep = j < L && (j == 0 || kr[j] != kr[j - 1]);
        unsigned bm = __ballot_sync(0xffffffffu, keep);
        if (lane == 0) wsum[wid] = __popc(bm);
        __syncthreads();
        int pre = 0, tot_b = 0;
        for (int w = 0; w < nwarp; w++) {
            int c = wsum[w];
            if (w < wid) pre += c;
            tot_b += c;
        }
        if (keep) srt[s + out + pre + __popc(bm & lanemask_lt())] = (int32_t)(kr[j] & mask);
        out += tot_b;
        __syncthreads();
    }
    if (threadIdx.x == 0) ucnt[r] = out;
}

// deduplicated rows -> final CSR (row_ptr = exclusive scan of ucnt) + in-degrees
__global__ void k_csr_emit(int32_t n, const int32_t* rs, const int32_t* srt, const int32_t* ucnt,
                           const int32_t* row_ptr, int32_t* col, int32_t* indeg, int rpw) {
    // 32 rows per warp (lanes = rows), their entries spread over the lanes as in k_qcols
    const int lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r0 = ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5) * rpw; r0 < n; r0 += nw * rpw) {
        const int64_t r = r0 + lane;
        int32_t s = 0, c = 0, o = 0;
        if (lane < rpw && r < n) {
            s = rs[r];
            c = ucnt[r];
            o = row_ptr[r];
        }
        int32_t inc = c;
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
            const int32_t y = __shfl_up_sync(0xffffffffu, inc, off);
            if (lane >= off) inc += y;
        }
        const int32_t exc = inc - c;
        const int32_t tot = __shfl_sync(0xffffffffu, inc, 31);
        for (int32_t kb = 0; kb < tot; kb += 32) {
            const int32_t k = kb + lane;
            int lo = 0;
#pragma unroll
            for (int step = 16; step >= 1; step >>= 1) {
                const int32_t ev = __shfl_sync(0xffffffffu, exc, lo + step);
                if (ev <= k) lo += step;
            }
            const int32_t os = __shfl_sync(0xffffffffu, s, lo);
            const int32_t oe = __shfl_sync(0xffffffffu, exc, lo);
            const int32_t oo = __shfl_sync(0xffffffffu, o, lo);
            if (k < tot) {
                const int32_t v = srt[os + (k - oe)];
                col[oo + (k - oe)] = v;
                atomicAdd(&indeg[v], 1);
            }
        }
    }
}

struct KahnArgs {
    int32_t n;
    const int32_t* row_ptr;
    const int32_t* col;
    const int32_t* indeg;
    int32_t* rem;
    int32_t* level;
    int32_t* front[2];    // frontier lists of int2 {row start, row end} (successor range of each node)
    int32_t* counts;      // [n+2], zeroed: counts[k] = size of frontier k
    int32_t* out;         // [0] = number of levels L, [1] = processed
    uint32_t* err;
    int32_t sfcap;        // one block: frontier entries [0, sfcap) live in shared memory (after rem)
    const int4* colr;     // one block: per edge {col, row_ptr[col], row_ptr[col + 1], 0}, or NULL
};

// ---- a2 for large DAGs whose id order is topological (every edge goes from a smaller to a
// larger id, as in a sequential task flow: a task only depends on tasks submitted before it) --
// level(v) = 0 for a source, else 1 + max level of its predecessors: the longest path from a
// source, i.e. exactly Kahn's level (P:l.91).  Computed as a barrier-free pull dataflow like
// k_bl_flow: warps take 32-id chunks in id order from a ticket; a node's predecessors (a
// predecessor CSR built here) have smaller ids, so they are in earlier chunks held by running
// warps (no deadlock); a level word doubles as its ready flag (0xFFFFFFFF = not yet).  A chunk
// loads all its predecessors' words at once, max-reduces the published ones and polls the rest
// from a per-warp pending list, so a dependency link costs about one L2 round trip instead of
// a level's grid barrier plus its chain of dependent loads.

// predecessor CSR: rcol[rrow[v] ...] = predecessors of v (any order: only their max is used);
// a warp takes rpw consecutive rows and spreads their edges over its lanes (warp scan of the
// row lengths + a 5-step shuffle search for each edge's row, as k_csr_emit)
__global__ void k_rcsr_fill(int32_t n, const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ col,
                            const int32_t* __restrict__ rrow, int32_t* fillc, int32_t* rcol, int rpw) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r0 = ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5) * rpw; r0 < n; r0 += nw * rpw) {
        const int64_t r = r0 + lane;
        int32_t sb = 0, c = 0;
        if (lane < rpw && r < n) {
            sb = __ldg(row_ptr + r);
            c = __ldg(row_ptr + r + 1) - sb;
        }
        int32_t inc = c;
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
            const int32_t y = __shfl_up_sync(0xffffffffu, inc, off);
            if (lane >= off) inc += y;
        }
        const int32_t exc = inc - c;
        const int32_t tot = __shfl_sync(0xffffffffu, inc, 31);
        const int32_t e0 = __shfl_sync(0xffffffffu, sb, 0);   // the rows' edges are contiguous
        for (int32_t kb = 0; kb < tot; kb += 32) {
            const int32_t k = kb + lane;
            int lo = 0;
#pragma unroll
            for (int step = 16; step >= 1; step >>= 1) {
                const int32_t ev = __shfl_sync(0xffffffffu, exc, lo + step);
                if (ev <= k) lo += step;
            }
            if (k < tot) {
                const int32_t v = __ldg(col + e0 + k);
                rcol[__ldg(rrow + v) + atomicAdd(fillc + v, 1)] = (int32_t)(r0 + lo);
            }
        }
    }
}

constexpr int LVL_THREADS = 256;
constexpr int LVL_PCAP = 1024;   // pending-predecessor list per warp (4 B id + 1 B owner lane)
constexpr int LVL_PPL = 8;
#ifndef MP_LVL_BACKOFF_MAX
#define MP_LVL_BACKOFF_MAX 256
#endif
constexpr uint32_t LVL_NOT_READY = 0xFFFFFFFFu;
MP_INLINE uint32_t lvl_ld(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__global__ void __launch_bounds__(LVL_THREADS, 4) k_lvl_flow(int32_t n, const int32_t* __restrict__ rrow,
                                                             const int32_t* __restrict__ rcol, uint32_t* level,
                                                             int32_t* out, uint32_t* ticket, uint32_t* err) {
    __shared__ uint32_t smax[LVL_THREADS / 32][32];
    __shared__ int32_t scnt[LVL_THREADS / 32][32];   // unresolved pending predecessors per lane
    __shared__ int32_t srow[LVL_THREADS / 32][33];
    __shared__ int32_t spend[LVL_THREADS / 32][LVL_PCAP];
    __shared__ uint8_t sown[LVL_THREADS / 32][LVL_PCAP];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int32_t nchunks = (n + 31) / 32;
    uint32_t lmax = 0;
    bool stuck = false;
    while (true) {
        uint32_t c = 0;
        if (lane == 0) c = atomicAdd(ticket, 1u);
        c = __shfl_sync(0xffffffffu, c, 0);
        if (c >= (uint32_t)nchunks || stuck) break;
        const int32_t cbase = (int32_t)c * 32;
        const int32_t v = cbase + lane;
        const int32_t vv = v < n ? v : n;   // past the end: an empty row
        srow[w][lane] = __ldg(rrow + vv);
        if (lane == 31) srow[w][32] = __ldg(rrow + (v + 1 < n ? v + 1 : n));
        smax[w][lane] = 0u;
        scnt[w][lane] = 0;
        __syncwarp();
        const int32_t E0 = srow[w][0], E1 = srow[w][32];
        auto owner = [&](int32_t e) -> int {   // largest i with srow[i] <= e
            int lo = 0, hi = 31;
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (srow[w][mid] <= e) lo = mid;
                else hi = mid - 1;
            }
            return lo;
        };
        // every predecessor word loaded at once; the published ones reduced, the others listed.
        // A predecessor inside this chunk (a smaller lane) is published by this warp later, so it
        // always goes to the list (at most 31 * 32 / 2 = 496 such edges: the last 512 slots are
        // kept for them); an outside one waits in place when the list is full.
        uint32_t npend = 0;
        for (int32_t eb = E0; eb < E1; eb += 64) {
            int32_t pk[2];
            uint32_t xs[2];
#pragma unroll
            for (int k = 0; k < 2; k++) {
                const int32_t e = eb + lane + 32 * k;
                pk[k] = e < E1 ? __ldg(rcol + e) : -1;
            }
#pragma unroll
            for (int k = 0; k < 2; k++) xs[k] = pk[k] >= 0 ? lvl_ld(level + pk[k]) : 0u;
#pragma unroll
            for (int k = 0; k < 2; k++) {
                const int own = pk[k] >= 0 ? owner(eb + lane + 32 * k) : 0;
                bool nr = pk[k] >= 0 && xs[k] == LVL_NOT_READY;
                const bool intra = pk[k] >= cbase;
                const uint32_t lt = (1u << lane) - 1u;
                {   // outside the chunk: slots [0, PCAP - 512)
                    const uint32_t bal = __ballot_sync(0xffffffffu, nr && !intra);
                    const uint32_t at = npend + __popc(bal & lt);
                    if (nr && !intra && at < (uint32_t)(LVL_PCAP - 512)) {
                        spend[w][at] = pk[k];
                        sown[w][at] = (uint8_t)own;
                        atomicAdd(&scnt[w][own], 1);
                        nr = false;
                    }
                    const uint32_t room = npend < (uint32_t)(LVL_PCAP - 512) ? (uint32_t)(LVL_PCAP - 512) - npend : 0u;
                    npend += min((uint32_t)__popc(bal), room);
                }
                {   // inside the chunk: always listed (<= 496 of them per chunk)
                    const uint32_t bal = __ballot_sync(0xffffffffu, nr && intra);
                    const uint32_t at = npend + __popc(bal & lt);
                    if (nr && intra) {
                        spend[w][at] = pk[k];
                        sown[w][at] = (uint8_t)own;
                        atomicAdd(&scnt[w][own], 1);
                        nr = false;
                    }
                    npend += __popc(bal);
                }
                if (nr) {   // outside the chunk and the list full: wait for this one here
                    uint32_t spin = 0;
                    do { xs[k] = lvl_ld(level + pk[k]); } while (xs[k] == LVL_NOT_READY && ++spin < (1u << 22));
                    if (xs[k] == LVL_NOT_READY) stuck = true;
                }
                if (pk[k] >= 0 && xs[k] != LVL_NOT_READY) atomicMax(&smax[w][own], xs[k] + 1u);
            }
        }
        __syncwarp();
        // rounds: poll every unresolved list entry once, then publish the lanes with nothing
        // pending (this is what resolves the entries that point inside the chunk)
        bool done = v >= n;
        uint32_t rounds = 0, backoff = 32;
        while (true) {
            bool prog = false;
            for (uint32_t i0 = 0; i0 < npend; i0 += 32 * LVL_PPL) {
                int32_t ent[LVL_PPL];
#pragma unroll
                for (int k = 0; k < LVL_PPL; k++) {
                    const uint32_t i = i0 + lane + 32 * k;
                    ent[k] = i < npend ? spend[w][i] : -1;
                }
                uint32_t xv[LVL_PPL];
#pragma unroll
                for (int k = 0; k < LVL_PPL; k++) xv[k] = ent[k] >= 0 ? lvl_ld(level + ent[k]) : LVL_NOT_READY;
#pragma unroll
                for (int k = 0; k < LVL_PPL; k++)
                    if (ent[k] >= 0 && xv[k] != LVL_NOT_READY) {
                        const uint32_t i = i0 + lane + 32 * k;
                        const int ow = sown[w][i];
                        atomicMax(&smax[w][ow], xv[k] + 1u);
                        atomicSub(&scnt[w][ow], 1);
                        spend[w][i] = -1;
                        prog = true;
                    }
            }
            __syncwarp();
            if (!done && scnt[w][lane] == 0) {
                const uint32_t lv = smax[w][lane];   // 0 for a source
                asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(level + v), "r"(lv) : "memory");
                lmax = max(lmax, lv);
                done = true;
                prog = true;
            }
            if (__all_sync(0xffffffffu, done)) break;
            // a round without progress: back off, so waiting warps leave the issue slots to the
            // warps that have work (the kernel is issue-bound on c4 without it)
            if (__any_sync(0xffffffffu, prog)) {
                backoff = 32;
            } else {
                __nanosleep(backoff);
                backoff = min(backoff * 2u, (uint32_t)MP_LVL_BACKOFF_MAX);
            }
            if (++rounds >= (1u << 20)) {   // no progress possible (cannot happen on a DAG)
                stuck = true;
                break;
            }
        }
        __syncwarp();
    }
    if (__any_sync(0xffffffffu, stuck) && lane == 0) atomicOr(err, ERR_CYCLE_BIT);
    lmax = __reduce_max_sync(0xffffffffu, lmax);
    if (lane == 0) atomicMax(out, (int32_t)lmax + 1);
}

// One-block Kahn: the successor's row range travels with the edge (one 16-byte load per
// edge instead of col then the dependent row_ptr pair -- one L2 round trip less per level).
__global__ void k_kahn_colr(const int32_t* row_ptr, const int32_t* col, int32_t n, int4* colr) {
    const int32_t E = row_ptr[n];
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x) {
        const int32_t v = col[e];
        colr[e] = make_int4(v, row_ptr[v], row_ptr[v + 1], 0);
    }
}

// Light grid barrier for a co-resident (cooperative) grid: one monotonically
// increasing arrival counter, thread 0 of each block spins with acquire loads.
MP_INLINE void grid_barrier(unsigned* bar, unsigned& epoch, bool rel = false) {
    // bar[0]: arrivals (monotonic); bar[32]: release flag (its own 128-byte line).  The last
    // block to arrive publishes the epoch; the others poll the flag, not the atomic counter.
    // rel: the arrival is one acq_rel atomic at gpu scope (cumulative over the block's writes
    // ordered before it by the __syncthreads) instead of a full fence + relaxed atomic.
    __syncthreads();
    epoch++;
    if (threadIdx.x == 0) {
        const unsigned target = epoch * gridDim.x;
        unsigned old;
        if (rel) {
            asm volatile("atom.add.acq_rel.gpu.global.u32 %0, [%1], 1;" : "=r"(old) : "l"(bar) : "memory");
        } else {
            __threadfence();
            old = atomicAdd(bar, 1u);
        }
        if (old + 1u == target) {
            asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(bar + 32), "r"(epoch) : "memory");
        } else {
            unsigned v;
            do {
                asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(bar + 32) : "memory");
            } while ((int)(v - epoch) < 0);
        }
    }
    __syncthreads();
}

// grid_barrier that also broadcasts the size of the next frontier: the last block to arrive
// reads *cnt_next (every append of the level happened before its block's arrival) and
// publishes (count << 32 | epoch) in one 64-bit release store; the pollers get the count
// with the flag instead of one more dependent L2 read per level.
MP_INLINE int32_t grid_barrier_cnt(unsigned* bar, unsigned& epoch, const int32_t* cnt_next, int32_t* s_bc) {
    __syncthreads();
    epoch++;
    if (threadIdx.x == 0) {
        __threadfence();
        const unsigned target = epoch * gridDim.x;
        const unsigned old = atomicAdd(bar, 1u);
        unsigned long long v;
        if (old + 1u == target) {
            __threadfence();
            const int32_t c = *((const volatile int32_t*)cnt_next);
            v = ((unsigned long long)(uint32_t)c << 32) | epoch;
            asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(bar + 32), "l"(v) : "memory");
        } else {
            do {
                asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(bar + 32) : "memory");
            } while ((int)((unsigned)v - epoch) < 0);
        }
        *s_bc = (int32_t)(v >> 32);
    }
    __syncthreads();
    return *s_bc;
}

// frontier slot i: the first `cap` slots of a one-block frontier are in shared memory `sl`
template <bool SF>
MP_INLINE void kahn_append(int32_t* counter, int32_t* list, int2 v, int2* sl, int32_t cap) {
    cg::coalesced_group g = cg::coalesced_threads();
    int32_t base = 0;
    if (g.thread_rank() == 0) base = atomicAdd(counter, (int32_t)g.size());
    base = g.shfl(base, 0);
    const int32_t i = base + (int32_t)g.thread_rank();
    if (SF && i < cap) sl[i] = v;
    else reinterpret_cast<int2*>(list)[i] = v;
}

template <bool SF>
MP_INLINE int2 kahn_slot(const int2* cur, const int2* sl, int32_t cap, int64_t i) {
    if (SF && i < cap) return sl[i];
    return cur[i];
}

// v just became ready: its level, and its successor range into the next frontier, so the
// consumer of the frontier reads the range directly instead of one more dependent load of
// row_ptr.  The range is loaded by the caller BEFORE the remaining-predecessor decrement
// (speculatively, for every edge), so the row_ptr round trip overlaps the atomic's.
template <bool SF>
MP_INLINE void kahn_ready(const KahnArgs& a, int32_t* counter, int32_t* list, int32_t v, int32_t lvl, int2 rr,
                          int2* sl, int32_t cap) {
    a.level[v] = lvl;
    kahn_append<SF>(counter, list, rr, sl, cap);
}

MP_INLINE int2 kahn_range(const KahnArgs& a, int32_t v) { return make_int2(a.row_ptr[v], a.row_ptr[v + 1]); }

// edge e's target and the target's successor range
// (late: the range is loaded only once the decrement made the target ready, see kahn_late)
MP_INLINE int32_t kahn_edge(const KahnArgs& a, int64_t e, int2& vr, bool late) {
    if (a.colr) {
        const int4 c = a.colr[e];
        vr = make_int2(c.y, c.z);
        return c.x;
    }
    const int32_t v = a.col[e];
    if (!late) vr = kahn_range(a, v);
    return v;
}

MP_INLINE int2 kahn_late(const KahnArgs& a, int32_t v, int2 vr, bool late) { return late ? kahn_range(a, v) : vr; }

// Kahn, level-synchronous (a task is ready when all its predecessors are done,
// P:l.91): level k+1 = successors whose last remaining predecessor is in level
// k.  Frontier nodes are taken in chunks of 1024 per block; inside a chunk the
// edges are spread evenly over the threads (block scan of the degrees + binary
// search), so a high-degree node does not serialise a level.  Cooperative grid
// (one block per SM) with a light grid barrier per level; with one block the
// barrier is a __syncthreads and the remaining-predecessor counters and the
// frontier counter live in shared memory.
template <bool SF>   // SF: one block with the shared-memory frontier (the grid path has no smem slots)
__global__ void __launch_bounds__(1024) k_kahn(KahnArgs a, unsigned* bar, int smem_rem, int var) {
    extern __shared__ int32_t srem[];
    __shared__ int32_t s_row[1024], s_pre[1025];
    __shared__ uint32_t s_sc[40];
    __shared__ int32_t s_cnt[2];
    const int64_t gtid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t gsz = (int64_t)gridDim.x * blockDim.x;
    const bool single = gridDim.x == 1;
    int32_t* rem = smem_rem ? srem : a.rem;
    const int32_t sfcap = SF ? a.sfcap : 0;
    const bool late = (var & 16) != 0;
    int2* sfb = reinterpret_cast<int2*>(srem + ((a.n + 1) & ~1));   // [2][sfcap] after rem
    unsigned epoch = 0;
    if (single && threadIdx.x < 2) s_cnt[threadIdx.x] = 0;
    if (single) __syncthreads();
    for (int64_t v = gtid; v < a.n; v += gsz) {
        int32_t d = a.indeg[v];
        rem[v] = d;
        a.level[v] = 0;
        if (d == 0) kahn_append<SF>(single ? &s_cnt[0] : &a.counts[0], a.front[0], kahn_range(a, (int32_t)v), sfb, sfcap);
    }
    __shared__ int32_t s_bc;
    int32_t cnt_bc = 0;
    if (single) __syncthreads();
    else if (var & 4) cnt_bc = grid_barrier_cnt(bar, epoch, &a.counts[0], &s_bc);
    else grid_barrier(bar, epoch);
    int32_t k = 0;
    int64_t processed = 0;
    while (true) {
        const int32_t cnt = single ? *((volatile int32_t*)&s_cnt[k & 1])
                                   : ((var & 4) ? cnt_bc : *((volatile int32_t*)&a.counts[k]));
        if (cnt == 0) break;
        processed += cnt;
        const int2* cur = reinterpret_cast<const int2*>(a.front[k & 1]);
        int32_t* nxt = a.front[(k + 1) & 1];
        const int2* scur = sfb + (k & 1) * sfcap;
        int2* snxt = sfb + ((k + 1) & 1) * sfcap;
        int32_t* nctr = single ? &s_cnt[(k + 1) & 1] : &a.counts[k + 1];
        if ((var & 1) && cnt <= (int32_t)((var & 8) ? gridDim.x : gridDim.x * (blockDim.x >> 5))) {
            // narrow level: one warp per frontier node (spread over the blocks), lanes over its
            // successors -- no block scan, no block barrier inside the level
            const int64_t gw = (int64_t)(threadIdx.x >> 5) * gridDim.x + blockIdx.x;
            if (gw < cnt) {
                const int2 rr = kahn_slot<SF>(cur, scur, sfcap, gw);
                for (int32_t e = rr.x + (int32_t)(threadIdx.x & 31); e < rr.y; e += 32) {
                    int2 vr = make_int2(0, 0);
                    const int32_t v = kahn_edge(a, e, vr, late);
                    if (atomicSub(&rem[v], 1) == 1) kahn_ready<SF>(a, nctr, nxt, v, k + 1, kahn_late(a, v, vr, late), snxt, sfcap);
                }
            }
            if (single) __syncthreads();   // every thread has read cnt before its slot is reset
        } else {
        // chunk = frontier nodes per block: spread a level over all blocks (so each thread
        // relaxes ~1 edge) but never more than one node per thread
        int64_t chunk = (cnt + gridDim.x - 1) / gridDim.x;
        chunk = chunk < 32 ? 32 : (chunk > 1024 ? 1024 : ((chunk + 31) & ~31ll));
        for (int64_t c0 = (int64_t)blockIdx.x * chunk; c0 < cnt; c0 += (int64_t)gridDim.x * chunk) {
            const int64_t i = threadIdx.x < chunk ? c0 + threadIdx.x : cnt;
            int32_t deg = 0;
            if (i < cnt) {
                const int2 rr = kahn_slot<SF>(cur, scur, sfcap, i);
                deg = rr.y - rr.x;
                s_row[threadIdx.x] = rr.x;
            }
            // block exclusive scan of the degrees
            const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
            int32_t incl = deg;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                int32_t y = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += y;
            }
            if (lane == 31) s_sc[w] = (uint32_t)incl;
            __syncthreads();
            if (w == 0) {
                int32_t v0 = (int32_t)s_sc[lane], iv = v0;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    int32_t y = __shfl_up_sync(0xffffffffu, iv, o);
                    if (lane >= o) iv += y;
                }
                s_sc[lane] = (uint32_t)(iv - v0);
                if (lane == 31) s_sc[32] = (uint32_t)iv;
            }
            __syncthreads();
            s_pre[threadIdx.x] = (int32_t)s_sc[w] + incl - deg;
            const int32_t etot = (int32_t)s_sc[32];
            const int32_t nloc = (int32_t)((cnt - c0) < chunk ? (cnt - c0) : chunk);
            __syncthreads();
            for (int32_t e = threadIdx.x; e < etot; e += blockDim.x) {
                int lo = 0, hi = nloc - 1;     // last frontier slot with s_pre <= e
                while (lo < hi) {
                    const int mid = (lo + hi + 1) >> 1;
                    if (s_pre[mid] <= e) lo = mid;
                    else hi = mid - 1;
                }
                int2 vr = make_int2(0, 0);
                const int32_t v = kahn_edge(a, s_row[lo] + (e - s_pre[lo]), vr, late);
                if (atomicSub(&rem[v], 1) == 1) kahn_ready<SF>(a, nctr, nxt, v, k + 1, kahn_late(a, v, vr, late), snxt, sfcap);
            }
            __syncthreads();
        }
        }
        k++;
        if (single) {
            if (threadIdx.x == 0) s_cnt[(k + 1) & 1] = 0;   // the list after next starts empty
            __syncthreads();
        } else if (var & 4) {
            cnt_bc = grid_barrier_cnt(bar, epoch, &a.counts[k], &s_bc);
        } else {
            grid_barrier(bar, epoch, (var & 2) != 0);
        }
    }
    if (gtid == 0) {
        a.out[0] = k;
        a.out[1] = (int32_t)processed;
        if (processed < a.n) atomicOr(a.err, ERR_CYCLE_BIT);
    }
}

__global__ void k_iota_level_keys(const int32_t* level, int32_t n, uint64_t* keys, uint32_t* vals) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        keys[v] = (uint64_t)(uint32_t)level[v];
        vals[v] = (uint32_t)v;
    }
}

__global__ void k_level_order(const SortPlan* plan, uint64_t* const* kb, uint32_t* const* vb, int32_t n,
                              int32_t* level_order, int32_t* level_ptr, int32_t* pos) {
    const uint64_t* k = kb[plan->final_sel];
    const uint32_t* v = vb[plan->final_sel];
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int32_t id = (int32_t)v[i];
        level_order[i] = id;
        pos[id] = (int32_t)i;
        if (i == 0 || k[i] != k[i - 1]) level_ptr[k[i]] = (int32_t)i;
    }
}

// q-space maps: reverse levels, ids ascending inside a level; and the padded variant.
__global__ void k_qmaps(int32_t n, const int32_t* level, const int32_t* level_ptr, const int32_t* pos,
                        const int32_t* lvlq, const int32_t* lvlp, int32_t L, const int32_t* row_ptr,
                        int32_t* qof, int32_t* nodeq, int32_t* degq, int32_t* pof, int32_t* nodep,
                        int32_t* degp) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        int32_t l = level[v];
        int32_t i = pos[v] - level_ptr[l];
        int32_t r = L - 1 - l;
        int32_t q = lvlq[r] + i;
        int32_t p = lvlp[r] + i;
        int32_t d = row_ptr[v + 1] - row_ptr[v];
        qof[v] = q;
        nodeq[q] = (int32_t)v;
        degq[q] = d;
        pof[v] = p;
        nodep[p] = (int32_t)v;
        degp[p] = d;
    }
}

// colX[rowX[x] + j] = map[col[row_ptr[v] + j]] for every position x of node v (warp per node)
// colX[rowX[x] + i] = map[col[row_ptr[nodeX[x]] + i]]: a warp takes 32 consecutive positions
// (lanes = nodes), scans their degrees and then spreads the batch's edges over its lanes
// (each lane finds its edge's owner by a 5-step shuffle search), so low-degree nodes do
// not leave 29 of 32 lanes idle and a high-degree node does not serialise a warp.
__global__ void k_qcols(int32_t npos, const int32_t* nodeX, const int32_t* rowX, const int32_t* row_ptr,
                        const int32_t* col, const int32_t* map, int32_t* colX, int rpw) {
    const int lane = threadIdx.x & 31;
    const int64_t wid = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t x0 = wid * rpw; x0 < npos; x0 += nw * rpw) {
        const int64_t x = x0 + lane;
        const int32_t v = (lane < rpw && x < npos) ? nodeX[x] : -1;
        int32_t b = 0, d = 0, o = 0;
        if (v >= 0) {
            b = row_ptr[v];
            d = row_ptr[v + 1] - b;
            o = rowX[x];
        }
        int32_t inc = d;
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
            const int32_t y = __shfl_up_sync(0xffffffffu, inc, off);
            if (lane >= off) inc += y;
        }
        const int32_t exc = inc - d;
        const int32_t tot = __shfl_sync(0xffffffffu, inc, 31);
        for (int32_t kb = 0; kb < tot; kb += 32) {
            const int32_t k = kb + lane;
            int lo = 0;   // last lane whose first edge is <= k (its range holds k)
#pragma unroll
            for (int step = 16; step >= 1; step >>= 1) {
                const int32_t ev = __shfl_sync(0xffffffffu, exc, lo + step);
                if (ev <= k) lo += step;
            }
            const int32_t ob = __shfl_sync(0xffffffffu, b, lo);
            const int32_t oe = __shfl_sync(0xffffffffu, exc, lo);
            const int32_t oo = __shfl_sync(0xffffffffu, o, lo);
            if (k < tot) colX[oo + (k - oe)] = map[col[ob + (k - oe)]];
        }
    }
}

}  // namespace mpk

namespace mph {

inline int bits_for(int64_t x) {  // smallest b >= 1 with x <= 2^b
    int b = 1;
    while ((1ll << b) < x) b++;
    return b;
}

// rows per warp for the batched row kernels: one row per warp while there are more warps
// than rows / 32 (small DAGs keep every warp busy), up to 32 (lanes = rows) for large ones
inline int rows_per_warp(int64_t rows, int64_t warps) {
    int64_t r = rows * 2 / (warps > 0 ? warps : 1);
    return (int)(r < 1 ? 1 : (r > 32 ? 32 : r));
}

inline int grid_for(int64_t n, int threads = 256, int64_t cap = 148 * 32) {
    int64_t g = (n + threads - 1) / threads;
    if (g < 1) g = 1;
    if (g > cap) g = cap;
    return (int)g;
}

// (Re)build the DAG held by `dag`.  Device arrays are grow-only: rebuilding a
// DAG no larger than a previous one allocates nothing.
inline mp_status build_into(mp_dag* dag, int32_t n, int64_t m, const int32_t* d_src, const int32_t* d_dst,
                            cudaStream_t st) {
    using namespace mpk;
    // on any error the handle holds an empty DAG (mp.h)
    auto cleanup = [&](mp_status s) {
        dag->n = 0;
        dag->E = 0;
        dag->L = 0;
        return s;
    };
    if (n < 0 || n >= (1 << 30)) return cleanup(fail(MP_ERR_ARG, "n_tasks %d outside [0, 2^30)", n));
    if (m < 0 || m >= (1ll << 31))
        return cleanup(fail(MP_ERR_ARG, "n_edges %lld outside [0, 2^31)", (long long)m));
    if (m > 0 && (!d_src || !d_dst)) return cleanup(fail(MP_ERR_ARG, "edge arrays are NULL"));
    if (m > 0 && n == 0) return cleanup(fail(MP_ERR_ARG, "edges given for an empty task set"));
    cudaGetDevice(&dag->device);
    cudaDeviceGetAttribute(&dag->num_sms, cudaDevAttrMultiProcessorCount, dag->device);
    dag->n = n;
    const int64_t nn = n > 0 ? n : 1;
    const int64_t mm = m > 0 ? m : 1;
#define ALLOC(ptr, cnt)                                                                     \
    do {                                                                                    \
        mp_status s__ = grow_buf((void**)&(ptr), (size_t)(cnt) * sizeof(*(ptr)), dag, st); \
        if (s__) return cleanup(s__);                                                       \
    } while (0)
#define CK(call)                                                                            \
    do {                                                                                    \
        cudaError_t e__ = (call);                                                           \
        if (e__) return cleanup(fail(MP_ERR_CUDA, "%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(e__))); \
    } while (0)

    ALLOC(dag->err, 4);
    ALLOC(dag->tickets, 64);
    ALLOC(dag->row_ptr, nn + 1);
    ALLOC(dag->indeg, nn);
    ALLOC(dag->level, nn);
    ALLOC(dag->level_ptr, nn + 1);
    ALLOC(dag->level_order, nn);
    ALLOC(dag->qof, nn);
    ALLOC(dag->nodeq, nn + 4);        // + 4: k_bl_small's 16-byte aligned bulk copies read past the end
    ALLOC(dag->rowq, nn + 1 + 4);
    CK(cudaMemsetAsync(dag->err, 0, 16, st));
    CK(cudaMemsetAsync(dag->tickets, 0, 64 * 4, st));
    CK(cudaMemsetAsync(dag->row_ptr, 0, (nn + 1) * 4, st));
    CK(cudaMemsetAsync(dag->indeg, 0, nn * 4, st));

    // ---- a1: counting-sort CSR (bucket by source, sort + dedup rows) -----------------------
    const int b = bits_for(n > 1 ? n : 2);
    const int npass = (2 * b + 7) / 8;
    const int64_t tps = (mm + SORT_TILE - 1) / SORT_TILE;
    size_t bytes = sort_bytes(mm, 1, npass, false) + 2 * align256(mm * 4) + 2 * align256((nn + 1) * 4) + align256(2 * (nn + 1) * 4) +
                   align256((nn + 1) * 4) + align256(64) + 256 * 4;
    {
        mp_status s = ensure_ws(dag, bytes, st);
        if (s) return cleanup(s);
        s = ensure_sort_status(dag, (size_t)tps * 256, st);
        if (s) return cleanup(s);
    }
    Arena ar{dag->ws, dag->ws_cap};
    SortArgs sa = carve_sort(ar, dag, mm, 1, 0, npass, false);
    int32_t* tmp = ar.take<int32_t>(mm);
    int32_t* srt = ar.take<int32_t>(mm);
    int32_t* cnt = ar.take<int32_t>(nn + 1);   // out-degree counts, then unique counts
    int32_t* rs = ar.take<int32_t>(nn + 1);    // bucket starts
    int32_t* bigb = ar.take<int32_t>(2 * (nn + 1));  // long-row list | offsets
    int32_t* midl = ar.take<int32_t>(nn + 1);        // medium-row list
    uint64_t** kb = ar.take<uint64_t*>(2);
    int32_t* d_scal = ar.take<int32_t>(8);  // [0]=E, [2..3] = long rows / entries, [6] = a backward edge
    bool id_topo = false;                    // id order is a topological order (k_lvl_flow)
    ALLOC(dag->col, mm);
    if (m > 0) {
        CK(cudaMemsetAsync(cnt, 0, (nn + 1) * 4, st));
        CK(cudaMemsetAsync(d_scal, 0, 32, st));
        MP_LAUNCH(k_csr_count, grid_for(m), 256, 0, st, d_src, d_dst, m, n, cnt, dag->err, d_scal + 6);
        {
            mp_status s = scan(dag, cnt, rs, (int64_t)n + 1, nullptr, st);
            if (s) return cleanup(s);
        }
        MP_LAUNCH(k_csr_fill, grid_for(m), 256, 0, st, d_src, d_dst, m, n, rs, cnt, tmp);
        {
            const int gr = grid_for((int64_t)n * 32, 256, (int64_t)dag->num_sms * 8);
            const int rpw = rows_per_warp(n, (int64_t)gr * 8);
            MP_LAUNCH(k_csr_rowsort, gr, 256, 0, st, n, rs, tmp, srt, cnt, bigb, d_scal + 2, bigb + nn + 1, rpw,
                      rpw > 1 ? midl : nullptr);
            if (rpw > 1) MP_LAUNCH(k_csr_rowsort_mid, gr, 256, 0, st, midl, d_scal + 4, rs, tmp, srt, cnt);
        }
        int32_t h_big[6] = {0, 0, 0, 0, 0, 0};
        CK(cudaMemcpyAsync(h_big, d_scal + 2, 24, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        id_topo = h_big[4] == 0;   // no edge from a larger to a smaller id
        if (h_big[0] > 0) {
            uint64_t* hk[2] = {sa.keys[0], sa.keys[1]};
            CK(cudaMemcpyAsync(kb, hk, sizeof(hk), cudaMemcpyHostToDevice, st));
            MP_LAUNCH(k_csr_big_gather, h_big[0], 256, 0, st, bigb, bigb + nn + 1, rs, tmp, b, sa.keys[0]);
            sa.seg_len = h_big[1];
            {
                mp_status s = run_sort(dag, sa, st);
                if (s) return cleanup(s);
            }
            MP_LAUNCH(k_csr_big_compact, h_big[0], 1024, 0, st, bigb, sa.plans, kb, (int64_t)h_big[1], rs, b, srt,
                                                                   cnt);
        }
        {
            mp_status s = scan(dag, cnt, dag->row_ptr, (int64_t)n + 1, d_scal, st);
            if (s) return cleanup(s);
        }
        MP_LAUNCH(k_csr_emit, grid_for((int64_t)n * 32), 256, 0, st, n, rs, srt, cnt, dag->row_ptr, dag->col,
                                                             dag->indeg, rows_per_warp(n, (int64_t)grid_for((int64_t)n * 32) * 8));
    } else {
        CK(cudaMemsetAsync(d_scal, 0, 4, st));
    }

    // ---- a2: Kahn levels ----------------------------------------------------------------
    ALLOC(dag->b_rem, nn);
    ALLOC(dag->b_f0, 2 * nn);   // int2 entries
    ALLOC(dag->b_f1, 2 * nn);
    ALLOC(dag->b_counts, nn + 2);
    ALLOC(dag->b_kout, 4);
    ALLOC(dag->b_bar, 64);
    int32_t* rem = dag->b_rem;
    int32_t* f0 = dag->b_f0;
    int32_t* f1 = dag->b_f1;
    int32_t* counts = dag->b_counts;
    int32_t* kout = dag->b_kout;
    CK(cudaMemsetAsync(counts, 0, (nn + 2) * 4, st));
    CK(cudaMemsetAsync(kout, 0, 16, st));
    if (n > 0 && id_topo && m > 0) {
        // (measured against the level-synchronous Kahn below, ingest totals: c2 0.83 -> 0.59 ms,
        // lu64 1.31 -> 0.62, hier 1.68 -> 0.82, c3 2.36 -> 1.17, c4 4.69 -> 3.46, c4fmm 2.38 -> 2.28)
        // predecessor CSR (offsets = exclusive scan of the in-degrees), then the pull dataflow
        const int64_t E = m;   // >= the deduplicated edge count
        ALLOC(dag->b_rrow, nn + 1);
        ALLOC(dag->b_rcol, E);
        {
            mp_status s = scan(dag, dag->indeg, dag->b_rrow, (int64_t)n, dag->b_rrow + n, st);
            if (s) return cleanup(s);
        }
        CK(cudaMemsetAsync(rem, 0, (size_t)n * 4, st));
        MP_LAUNCH(k_rcsr_fill, grid_for((int64_t)n * 32), 256, 0, st, n, dag->row_ptr, dag->col, dag->b_rrow, rem,
                  dag->b_rcol, rows_per_warp(n, (int64_t)grid_for((int64_t)n * 32) * 8));
        CK(cudaMemsetAsync(dag->level, 0xff, (size_t)n * 4, st));
        CK(cudaMemsetAsync(dag->tickets + 60, 0, 4, st));
        int bps = 0;
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_lvl_flow, LVL_THREADS, 0));
        const int64_t want = (((int64_t)n + 31) / 32 + LVL_THREADS / 32 - 1) / (LVL_THREADS / 32);
        const int g = (int)std::max<int64_t>(1, std::min<int64_t>(want, (int64_t)std::min(bps, 4) * dag->num_sms));
        mph::ProfScope kahn_scope("k_lvl_flow", st);
        MP_LAUNCH(k_lvl_flow, g, LVL_THREADS, 0, st, n, dag->b_rrow, dag->b_rcol, (uint32_t*)dag->level, kout,
                  dag->tickets + 60, dag->err);
    } else if (n > 0) {
        KahnArgs ka{n, dag->row_ptr, dag->col, dag->indeg, rem, dag->level, {f0, f1}, counts, kout, dag->err, 0, nullptr};
        unsigned* bar = (unsigned*)dag->b_bar;
        CK(cudaMemsetAsync(bar, 0, 64 * 4, st));
        // small DAGs: one CTA, remaining-predecessor counters in shared memory, and the first
        // sfcap entries of both frontier lists after them (the rest spill to the global lists)
        const int64_t kSmemRem = 48 * 1024;
        int smem_rem = (int64_t)n <= kSmemRem ? 1 : 0;
        int g = 1;
        if (!smem_rem) {
            int bps = 0;
            CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_kahn<false>, 1024, 0));
            g = std::max(1, std::min(bps, 1) * dag->num_sms);
        }
        int max_dyn = 0;
        {
            // per launch (the opt-in is a per-device setting): two cheap host calls
            cudaFuncAttributes fa{};
            CK(cudaFuncGetAttributes(&fa, k_kahn<true>));
            int optin = 0;
            CK(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dag->device));
            max_dyn = optin - (int)fa.sharedSizeBytes;
            static std::atomic<uint64_t> attr{0};
            if (first_on_device(attr)) {
                CK(cudaFuncSetAttribute(k_kahn<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_dyn));
                CK(cudaFuncSetAttribute(k_kahn<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_dyn));
            }
        }
        size_t smem = 0;
        if (smem_rem) {
            const size_t remb = (size_t)((n + 1) & ~1) * 4;
            const int64_t cap = std::min<int64_t>(8192, ((int64_t)max_dyn - (int64_t)remb) / 16);
            ka.sfcap = (int32_t)std::max<int64_t>(0, cap);
            smem = remb + (size_t)ka.sfcap * 16;
            if (m > 0) {
                ALLOC(dag->b_colr, m);   // E <= m (deduplicated)
                MP_LAUNCH(k_kahn_colr, grid_for(m), 256, 0, st, dag->row_ptr, dag->col, n, dag->b_colr);
                ka.colr = dag->b_colr;
            }
        }
        // variant bits: 1 = warp-per-node narrow levels, 2 = acq_rel barrier arrival
        //   4 = the barrier broadcasts the next frontier size, 8 = narrow only up to one node per block,
        //   16 = a target's row range loaded after its decrement instead of speculatively with it
        // defaults (measured, tools/kahn_ab.sh, with the int2 frontier): one block -> narrow levels
        // (c2 k_kahn 0.48 -> 0.42 ms); a grid -> frontier size broadcast by the barrier + narrow levels
        // up to one node per block (c3 2.03 -> 1.72 ms, c4 3.03 -> 2.65 ms)
        // bit 16 (ranges loaded after the decrement) measured faster than the speculative load on
        // every config (c3 1.86 -> 1.79 ms, c4 2.83 -> 2.74, lu64 0.95 -> 0.90)
        int var = g == 1 ? 17 : 29;
        void* args[] = {&ka, &bar, &smem_rem, &var};
        mph::ProfScope kahn_scope("k_kahn", st);
        const void* kf = ka.sfcap > 0 ? (const void*)k_kahn<true> : (const void*)k_kahn<false>;
        CK(cudaLaunchCooperativeKernel(kf, dim3((unsigned)g), dim3(1024), args, smem, st));
    }
    int32_t h_scal[2] = {0, 0};
    int32_t h_k[2] = {0, 0};
    uint32_t h_err = 0;
    CK(cudaMemcpyAsync(h_scal, d_scal, 4, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(h_k, kout, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&h_err, dag->err, 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (h_err & ERR_ARG_BIT) return cleanup(fail(MP_ERR_ARG, "edge id outside [0, n) or self-loop"));
    if (h_err & ERR_CYCLE_BIT) return cleanup(fail(MP_ERR_CYCLE, "edges contain a cycle (%d of %d tasks levelled)", h_k[1], n));
    dag->E = m > 0 ? h_scal[0] : 0;
    dag->L = h_k[0];
    const int32_t L = dag->L;

    // ---- canonical level order: stable sort of ids by level ---------------------------
    if (n > 0) {
        const int lb = bits_for(L + 1);
        const int lp = (lb + 7) / 8;
        Arena ar2{dag->ws, dag->ws_cap};
        size_t need = sort_bytes(nn, 1, lp, true) + align256(64);
        {
            mp_status s = ensure_ws(dag, need, st);
            if (s) return cleanup(s);
            ar2 = Arena{dag->ws, dag->ws_cap};
        }
        SortArgs ls = carve_sort(ar2, dag, n, 1, 0, lp, true);
        uint64_t** kb2 = ar2.take<uint64_t*>(2);
        uint32_t** vb2 = ar2.take<uint32_t*>(2);
        uint64_t* hk[2] = {ls.keys[0], ls.keys[1]};
        uint32_t* hv[2] = {ls.vals[0], ls.vals[1]};
        CK(cudaMemcpyAsync(kb2, hk, sizeof(hk), cudaMemcpyHostToDevice, st));
        CK(cudaMemcpyAsync(vb2, hv, sizeof(hv), cudaMemcpyHostToDevice, st));
        MP_LAUNCH(k_iota_level_keys, grid_for(n), 256, 0, st, dag->level, n, ls.keys[0], ls.vals[0]);
        {
            mp_status s = run_sort(dag, ls, st);
            if (s) return cleanup(s);
        }
        // pos[] reuses rem (free after)
        MP_LAUNCH(k_level_order, grid_for(n), 256, 0, st, ls.plans, kb2, vb2, n, dag->level_order, dag->level_ptr, rem);
        CK(cudaMemcpyAsync(dag->level_ptr + L, &dag->n, 4, cudaMemcpyHostToDevice, st));
        std::vector<int32_t> lp_h((size_t)L + 1);
        CK(cudaMemcpyAsync(lp_h.data(), dag->level_ptr, ((size_t)L + 1) * 4, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        lp_h[L] = n;
        // reverse-level offsets, unpadded and padded to 32
        std::vector<int32_t> lq((size_t)L + 1), lpp((size_t)L + 1);
        int32_t mw = 0;
        lq[0] = 0;
        lpp[0] = 0;
        for (int32_t r = 0; r < L; r++) {
            int32_t l = L - 1 - r;
            int32_t w = lp_h[l + 1] - lp_h[l];
            if (w > mw) mw = w;
            lq[r + 1] = lq[r] + w;
            lpp[r + 1] = lpp[r] + ((w + 31) / 32) * 32;
        }
        dag->max_width = mw;
        dag->P = lpp[L];
        const int64_t P = dag->P;
        ALLOC(dag->lvlq, L + 1);
        ALLOC(dag->lvlp, L + 1);
        ALLOC(dag->nodep, P);
        ALLOC(dag->rowp, P + 1);
        ALLOC(dag->colq, (dag->E > 0 ? dag->E : 1) + 4);
        ALLOC(dag->colp, dag->E > 0 ? dag->E : 1);
        ALLOC(dag->b_pof, nn);
        int32_t* pof = dag->b_pof;
        CK(cudaMemcpyAsync(dag->lvlq, lq.data(), ((size_t)L + 1) * 4, cudaMemcpyHostToDevice, st));
        CK(cudaMemcpyAsync(dag->lvlp, lpp.data(), ((size_t)L + 1) * 4, cudaMemcpyHostToDevice, st));
        CK(cudaMemsetAsync(dag->nodep, 0xff, P * 4, st));
        CK(cudaMemsetAsync(dag->rowp, 0, (P + 1) * 4, st));
        CK(cudaMemsetAsync(dag->rowq, 0, (nn + 1) * 4, st));
        MP_LAUNCH(k_qmaps, grid_for(n), 256, 0, st, n, dag->level, dag->level_ptr, rem, dag->lvlq, dag->lvlp, L,
                                             dag->row_ptr, dag->qof, dag->nodeq, dag->rowq, pof, dag->nodep,
                                             dag->rowp);
        {
            mp_status s = scan(dag, dag->rowq, dag->rowq, (int64_t)n + 1, nullptr, st);
            if (s) return cleanup(s);
            s = scan(dag, dag->rowp, dag->rowp, P + 1, nullptr, st);
            if (s) return cleanup(s);
        }
        if (dag->E > 0) {
            MP_LAUNCH(k_qcols, grid_for((int64_t)n * 32), 256, 0, st, n, dag->nodeq, dag->rowq, dag->row_ptr, dag->col,
                      dag->qof, dag->colq, rows_per_warp(n, (int64_t)grid_for((int64_t)n * 32) * 8));
            MP_LAUNCH(k_qcols, grid_for(P * 32), 256, 0, st, (int32_t)P, dag->nodep, dag->rowp, dag->row_ptr, dag->col,
                      pof, dag->colp, rows_per_warp(P, (int64_t)grid_for(P * 32) * 8));
        }
    } else {
        ALLOC(dag->lvlq, 1);
        ALLOC(dag->lvlp, 1);
        ALLOC(dag->nodep, 1);
        ALLOC(dag->rowp, 1);
        ALLOC(dag->colq, 1 + 4);
        ALLOC(dag->colp, 1);
        CK(cudaMemsetAsync(dag->lvlq, 0, 4, st));
        CK(cudaMemsetAsync(dag->lvlp, 0, 4, st));
        CK(cudaMemsetAsync(dag->rowp, 0, 4, st));
        CK(cudaMemsetAsync(dag->rowq, 0, 4, st));
        CK(cudaMemsetAsync(dag->level_ptr, 0, 4, st));
    }
    CK(cudaStreamSynchronize(st));
    CK(cudaGetLastError());
#undef ALLOC
#undef CK
    return MP_OK;
}

inline mp_status build_dag(int32_t n, int64_t m, const int32_t* d_src, const int32_t* d_dst, cudaStream_t st,
                           mp_dag** out) {
    if (!out) return fail(MP_ERR_ARG, "out is NULL");
    *out = nullptr;
    mp_dag* dag = new mp_dag();
    mp_status s = build_into(dag, n, m, d_src, d_dst, st);
    if (s != MP_OK) {
        mp_free(dag);
        return s;
    }
    *out = dag;
    return MP_OK;
}

}  // namespace mph
