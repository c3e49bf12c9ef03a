// scan.cuh -- single-pass exclusive prefix sum of int32 with decoupled
// look-back (tiles taken in ticket order).  out[i] = sum in[0..i); *total = sum.
// `in` may alias `out`.  Used by the DAG build (a1/a2), never by the oracle.
#pragma once
#include "common.cuh"

namespace mpk {

constexpr int SCAN_THREADS = 256;
constexpr int SCAN_IPT = 8;
constexpr int SCAN_TILE = SCAN_THREADS * SCAN_IPT;

struct ScanWs {
    unsigned long long* status;   // [ntiles], zeroed once
    uint32_t* ticket;             // [1]
    uint32_t* depoch;             // device scan counter (status tags; graph-replay safe)
};

// before a scan: reset the tile ticket and bump the epoch (one thread)
__global__ void k_scan_prep(ScanWs ws) {
    *ws.ticket = 0u;
    *ws.depoch = *ws.depoch + 1u;
}

__global__ void __launch_bounds__(SCAN_THREADS)
k_scan_excl(const int32_t* in, int32_t* out, int64_t n, int32_t* total, ScanWs ws) {
    const uint32_t epoch = *(volatile uint32_t*)ws.depoch & 0x3fffffffu;
    __shared__ uint32_t tile_sh;
    __shared__ int32_t wsum[SCAN_THREADS / 32];
    __shared__ int64_t excl_sh;
    if (threadIdx.x == 0) tile_sh = atomicAdd(ws.ticket, 1u);
    __syncthreads();
    const int64_t tile = tile_sh;
    const int64_t base = tile * SCAN_TILE + (int64_t)threadIdx.x * SCAN_IPT;
    int32_t v[SCAN_IPT];
    int32_t s = 0;
#pragma unroll
    for (int k = 0; k < SCAN_IPT; k++) {
        v[k] = base + k < n ? in[base + k] : 0;
        s += v[k];
    }
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int32_t x = s;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) wsum[w] = x;
    __syncthreads();
    int32_t woff = 0, tot = 0;
    for (int i = 0; i < SCAN_THREADS / 32; i++) {
        if (i < w) woff += wsum[i];
        tot += wsum[i];
    }
    if (threadIdx.x == 0) {
        uint64_t tag = (uint64_t)epoch << 34;
        int64_t excl = 0;
        if (tile == 0) {
            st_relaxed64((uint64_t*)&ws.status[0], tag | (2ull << 32) | (uint32_t)tot);
        } else {
            st_relaxed64((uint64_t*)&ws.status[tile], tag | (1ull << 32) | (uint32_t)tot);
            int64_t t = tile - 1;
            while (true) {
                uint64_t sv;
                do {
                    sv = ld_relaxed64((const uint64_t*)&ws.status[t]);
                } while ((sv >> 34) != epoch || ((sv >> 32) & 3ull) == 0);
                excl += (int64_t)(uint32_t)(sv & 0xffffffffull);
                if (((sv >> 32) & 3ull) == 2ull) break;
                t--;
            }
            st_relaxed64((uint64_t*)&ws.status[tile], tag | (2ull << 32) | (uint32_t)(excl + tot));
        }
        excl_sh = excl;
        int64_t last = (n + SCAN_TILE - 1) / SCAN_TILE - 1;
        if (tile == last && total) *total = (int32_t)(excl + tot);
    }
    __syncthreads();
    int32_t run = (int32_t)excl_sh + woff + x - s;
#pragma unroll
    for (int k = 0; k < SCAN_IPT; k++) {
        if (base + k < n) out[base + k] = run;
        run += v[k];
    }
}

inline cudaError_t scan_excl(const int32_t* in, int32_t* out, int64_t n, int32_t* d_total, ScanWs ws,
                             cudaStream_t st) {
    if (n <= 0) {
        if (d_total) return cudaMemsetAsync(d_total, 0, sizeof(int32_t), st);
        return cudaSuccess;
    }
    MP_LAUNCH(k_scan_prep, 1, 1, 0, st, ws);
    int64_t ntiles = (n + SCAN_TILE - 1) / SCAN_TILE;
    MP_LAUNCH(k_scan_excl, (unsigned)ntiles, SCAN_THREADS, 0, st, in, out, n, d_total, ws);
    return cudaGetLastError();
}

}  // namespace mpk
