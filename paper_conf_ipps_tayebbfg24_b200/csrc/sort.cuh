// sort.cuh -- stable LSD radix sort of (uint64 key, uint32 value) pairs over
// equal-length segments, one kernel per 8-bit digit pass with decoupled
// look-back (single pass over the data per digit, "onesweep"-style).
//
//  - k_sort_hist   : per-segment digit histograms of every pass in ONE read
//  - k_sort_plan   : per-segment digit bases; passes whose digit is constant
//                    over a segment are skipped ON THE DEVICE (no host sync):
//                    each segment records which ping-pong buffer every pass
//                    reads, and where its result finally lives (final_sel).
//  - k_sort_pass   : tiles of 4096 keys taken in ticket order; warp-level
//                    stable ranking with __match_any_sync; tile aggregates
//                    published per digit and resolved by look-back restricted
//                    to the tile's segment; scatter staged through shared
//                    memory so that global writes are digit-run contiguous.
// Stability: tiles in index order, warps in order, items (k-major, lane-minor)
// in index order  =>  equal keys keep their input order.
#pragma once
#include "common.cuh"

namespace mpk {

constexpr int SORT_THREADS = 256;
constexpr int SORT_WARPS = SORT_THREADS / 32;
constexpr int SORT_IPT = 16;
constexpr int SORT_TILE = SORT_THREADS * SORT_IPT;  // 4096
constexpr int SORT_MAX_PASS = 8;

struct SortPlan {                     // one per segment
    uint32_t base[SORT_MAX_PASS][256];
    int32_t src[SORT_MAX_PASS];        // buffer read by pass p, -1 = skipped
    int32_t final_sel;                 // buffer holding the result
    int32_t pad_[7];
};

struct SortArgs {
    uint64_t* keys[2];
    uint32_t* vals[2];                 // vals[0] == nullptr: keys only
    int64_t seg_len;
    int32_t nseg;
    int32_t bit_lo;
    int32_t npass;
    int32_t tiles_per_seg;
    SortPlan* plans;                   // [nseg]
    uint32_t* hist;                    // [nseg][npass][256]
    unsigned long long* status;        // [nseg*tiles_per_seg][256]
    uint32_t* tickets;                 // [npass]
    const int64_t* d_len;              // optional device-side length (<= seg_len), all segments
    uint32_t* depoch;                  // device sort counter (the status tags; graph-replay safe)
};

MP_INLINE int64_t eff_len(const SortArgs& a) {
    if (!a.d_len) return a.seg_len;
    int64_t l = *a.d_len;
    return l < a.seg_len ? (l < 0 ? 0 : l) : a.seg_len;
}

MP_INLINE uint32_t digit_of(uint64_t k, int shift) { return (uint32_t)(k >> shift) & 255u; }

// grid: (chunks, nseg); each block scans a chunk of its segment
__global__ void k_sort_hist(SortArgs a, int chunk) {
    __shared__ uint32_t h[SORT_MAX_PASS][256];
    for (int i = threadIdx.x; i < SORT_MAX_PASS * 256; i += blockDim.x) (&h[0][0])[i] = 0;
    __syncthreads();
    int64_t s = blockIdx.y;
    int64_t b = (int64_t)blockIdx.x * chunk;
    int64_t e = min(b + chunk, eff_len(a));
    const uint64_t* k = a.keys[0] + s * a.seg_len;
    for (int64_t i = b + threadIdx.x; i < e; i += blockDim.x) {
        uint64_t key = k[i];
        for (int p = 0; p < a.npass; p++) atomicAdd(&h[p][digit_of(key, a.bit_lo + 8 * p)], 1u);
    }
    __syncthreads();
    uint32_t* g = a.hist + s * a.npass * 256;
    for (int i = threadIdx.x; i < a.npass * 256; i += blockDim.x) {
        uint32_t v = (&h[0][0])[i];
        if (v) atomicAdd(&g[i], v);
    }
}

// grid: nseg blocks of 256 threads
__global__ void k_sort_plan(SortArgs a) {
    __shared__ uint32_t sc[256];
    __shared__ int trivial;
    int s = blockIdx.x;
    int d = threadIdx.x;
    if (s == 0 && d < a.npass) a.tickets[d] = 0;
    if (s == 0 && d == 0) *a.depoch = *a.depoch + 1u;   // this sort's epochs: depoch * 8 + pass
    int sel = 0;
    const int64_t len = eff_len(a);
    for (int p = 0; p < a.npass; p++) {
        uint32_t c = a.hist[((int64_t)s * a.npass + p) * 256 + d];
        if (d == 0) trivial = 0;
        __syncthreads();
        if ((int64_t)c == len) trivial = 1;
        sc[d] = c;
        __syncthreads();
        // exclusive scan (Hillis-Steele over 256)
        for (int o = 1; o < 256; o <<= 1) {
            uint32_t v = d >= o ? sc[d - o] : 0u;
            __syncthreads();
            sc[d] += v;
            __syncthreads();
        }
        a.plans[s].base[p][d] = sc[d] - c;
        int triv = trivial;
        if (d == 0) a.plans[s].src[p] = triv ? -1 : sel;
        if (!triv) sel ^= 1;
        __syncthreads();
    }
    if (d == 0) a.plans[s].final_sel = sel;
}

constexpr uint64_t ST_AGG = 1ull << 32;
constexpr uint64_t ST_PRE = 2ull << 32;

__global__ void __launch_bounds__(SORT_THREADS) k_sort_pass(SortArgs a, int pass) {
    // status tags come from a device counter bumped once per sort by k_sort_plan, so a
    // replayed CUDA graph never meets its previous replay's tags
    const uint32_t epoch = (*(volatile uint32_t*)a.depoch * (uint32_t)SORT_MAX_PASS + (uint32_t)pass) & 0x3fffffffu;
    __shared__ uint32_t whist[SORT_WARPS][256];
    __shared__ uint32_t tstart[256];       // digit start within the tile
    __shared__ int64_t gdelta[256];        // global position = gdelta[d] + tile-local index
    extern __shared__ __align__(16) unsigned char sort_dyn[];
    uint64_t* skeys = (uint64_t*)sort_dyn;                    // [SORT_TILE]
    uint32_t* svals = (uint32_t*)(sort_dyn + SORT_TILE * 8);  // [SORT_TILE]
    __shared__ uint32_t tile_sh;

    if (threadIdx.x == 0) tile_sh = atomicAdd(&a.tickets[pass], 1u);
    __syncthreads();
    const uint32_t tile = tile_sh;
    const int64_t s = tile / a.tiles_per_seg;
    const int64_t j = tile % a.tiles_per_seg;
    const SortPlan& plan = a.plans[s];
    const int src = plan.src[pass];
    if (src < 0) return;                   // digit constant over the segment
    const bool has_vals = a.vals[0] != nullptr;
    const uint64_t* kin = a.keys[src] + s * a.seg_len;
    uint64_t* kout = a.keys[src ^ 1] + s * a.seg_len;
    const uint32_t* vin = has_vals ? a.vals[src] + s * a.seg_len : nullptr;
    uint32_t* vout = has_vals ? a.vals[src ^ 1] + s * a.seg_len : nullptr;
    const int shift = a.bit_lo + 8 * pass;

    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < SORT_WARPS * 256; i += SORT_THREADS) (&whist[0][0])[i] = 0;
    __syncthreads();

    const int64_t tbase = j * SORT_TILE;
    const int64_t tlen = min((int64_t)SORT_TILE, eff_len(a) - tbase);
    if (tlen <= 0) return;                 // beyond a device-side length
    uint64_t key[SORT_IPT];
    uint32_t val[SORT_IPT];
    uint32_t rk[SORT_IPT];
#pragma unroll
    for (int k = 0; k < SORT_IPT; k++) {
        int64_t li = (int64_t)w * 32 * SORT_IPT + k * 32 + lane;
        if (li < tlen) {
            key[k] = kin[tbase + li];
            val[k] = has_vals ? vin[tbase + li] : 0u;
        } else {
            key[k] = ~0ull;
            val[k] = 0u;
        }
    }
    const uint32_t lt = lanemask_lt();
#pragma unroll
    for (int k = 0; k < SORT_IPT; k++) {
        int64_t li = (int64_t)w * 32 * SORT_IPT + k * 32 + lane;
        uint32_t d = li < tlen ? digit_of(key[k], shift) : 256u;
        uint32_t peers = __match_any_sync(0xffffffffu, d);
        uint32_t below = __popc(peers & lt);
        uint32_t cnt = d < 256 ? whist[w][d] : 0u;
        rk[k] = cnt + below;
        __syncwarp();
        if (d < 256 && (31 - __clz(peers)) == lane) whist[w][d] = cnt + __popc(peers);
        __syncwarp();
    }
    __syncthreads();
    // per digit: exclusive over warps, tile total
    uint32_t total = 0;
    {
        int d = threadIdx.x;  // SORT_THREADS == 256
        for (int ww = 0; ww < SORT_WARPS; ww++) {
            uint32_t c = whist[ww][d];
            whist[ww][d] = total;
            total += c;
        }
        // publish the tile aggregate early
        unsigned long long* st = a.status + (int64_t)tile * 256 + d;
        uint64_t tag = (uint64_t)epoch << 34;
        if (j == 0) st_relaxed64((uint64_t*)st, tag | ST_PRE | total);
        else st_relaxed64((uint64_t*)st, tag | ST_AGG | total);
        tstart[d] = total;
    }
    __syncthreads();
    // exclusive scan of tile totals over digits -> tstart
    {
        int d = threadIdx.x;
        uint32_t v = tstart[d];
        // warp scan then across warps
        uint32_t x = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= o) x += y;
        }
        __shared__ uint32_t wsum[SORT_WARPS];
        if (lane == 31) wsum[w] = x;
        __syncthreads();
        uint32_t off = 0;
        for (int ww = 0; ww < w; ww++) off += wsum[ww];
        tstart[d] = off + x - v;
    }
    // decoupled look-back for digit d within this segment
    {
        int d = threadIdx.x;
        uint64_t excl = 0;
        if (j > 0) {
            int64_t t = (int64_t)tile - 1;
            int64_t t0 = (int64_t)tile - j;   // first tile of the segment
            const uint64_t want = (uint64_t)epoch;
            while (true) {
                uint64_t sv;
                do {
                    sv = ld_relaxed64((const uint64_t*)(a.status + t * 256 + d));
                } while ((sv >> 34) != want || ((sv >> 32) & 3ull) == 0);
                excl += (sv & 0xffffffffull);
                if (((sv >> 32) & 3ull) == 2ull || t == t0) break;
                t--;
            }
            st_relaxed64((uint64_t*)(a.status + (int64_t)tile * 256 + d),
                         ((uint64_t)epoch << 34) | ST_PRE | (excl + total));
        }
        gdelta[d] = (int64_t)plan.base[pass][d] + (int64_t)excl - (int64_t)tstart[d];
    }
    __syncthreads();
    // stage in digit order
#pragma unroll
    for (int k = 0; k < SORT_IPT; k++) {
        int64_t li = (int64_t)w * 32 * SORT_IPT + k * 32 + lane;
        if (li < tlen) {
            uint32_t d = digit_of(key[k], shift);
            uint32_t pos = tstart[d] + whist[w][d] + rk[k];
            skeys[pos] = key[k];
            svals[pos] = val[k];
        }
    }
    __syncthreads();
    for (int i = threadIdx.x; i < tlen; i += SORT_THREADS) {
        uint64_t kk = skeys[i];
        int64_t g = gdelta[digit_of(kk, shift)] + i;
        kout[g] = kk;
        if (has_vals) vout[g] = svals[i];
    }
}

inline size_t sort_plan_bytes(int nseg) { return (size_t)nseg * sizeof(SortPlan); }

// Launch the whole sort. hist must be zeroed (done here); status (and the device epoch
// counter a.depoch) must be zero-initialised once at allocation.  No host state: the
// launch sequence can be captured in a CUDA graph and replayed.
inline cudaError_t sort_launch(SortArgs a, cudaStream_t st) {
    if (a.seg_len <= 0 || a.nseg <= 0 || a.npass <= 0) return cudaSuccess;
    a.tiles_per_seg = (int32_t)((a.seg_len + SORT_TILE - 1) / SORT_TILE);
    cudaError_t e = cudaMemsetAsync(a.hist, 0, (size_t)a.nseg * a.npass * 256 * sizeof(uint32_t), st);
    if (e) return e;
    int chunk = 16384;
    dim3 g((unsigned)((a.seg_len + chunk - 1) / chunk), (unsigned)a.nseg);
    MP_LAUNCH(k_sort_hist, g, 256, 0, st, a, chunk);
    MP_LAUNCH(k_sort_plan, a.nseg, 256, 0, st, a);
    int64_t ntiles = (int64_t)a.tiles_per_seg * a.nseg;
    static std::atomic<uint64_t> attr_set{0};
    const int dyn = SORT_TILE * 12;
    if (mph::first_on_device(attr_set)) {
        e = cudaFuncSetAttribute(k_sort_pass, cudaFuncAttributeMaxDynamicSharedMemorySize, dyn);
        if (e) return e;
    }
    for (int p = 0; p < a.npass; p++) MP_LAUNCH(k_sort_pass, (unsigned)ntiles, SORT_THREADS, dyn, st, a, p);
    return cudaGetLastError();
}

}  // namespace mpk
