// common.cuh -- device utilities shared by the libmp kernels (not by the oracle).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>

#include "../../include/mp.h"
#include "prof.cuh"

#define MP_INLINE __device__ __forceinline__

namespace mph {
// Function attributes (the dynamic shared-memory opt-in) are per device: true
// the first time it is asked for the current device and this flag set.
inline bool first_on_device(std::atomic<uint64_t>& mask) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return true; }
    const uint64_t b = 1ull << (dev & 63);
    return (mask.fetch_or(b) & b) == 0;
}
}  // namespace mph

namespace mpk {

constexpr uint32_t ONE_BITS = 0x3F800000u;      // bits(1.0f)
constexpr uint32_t ERR_DOMAIN_BIT = 1u;
constexpr uint32_t ERR_ARG_BIT = 2u;
constexpr uint32_t ERR_CYCLE_BIT = 4u;

MP_INLINE uint32_t f2u(float x) { return __float_as_uint(x); }
MP_INLINE float u2f(uint32_t x) { return __uint_as_float(x); }

MP_INLINE uint32_t ld_relaxed(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
MP_INLINE void st_relaxed(uint32_t* p, uint32_t v) {
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
MP_INLINE uint64_t ld_relaxed64(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
MP_INLINE void st_relaxed64(uint64_t* p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

MP_INLINE uint32_t lanemask_lt() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// Duration domain (reading c20): {+inf} U {0} U [2^-41, 2^20).  -0 -> +0.
// Returns the canonical value; sets *bad on a domain violation.
MP_INLINE float canon_dur(float d, bool& bad) {
    uint32_t u = f2u(d);
    if ((u & 0x7fffffffu) == 0u) return 0.0f;           // +-0
    if (u == 0x7f800000u) return d;                      // +inf
    // negative (incl. -inf), NaN, or outside [2^-41, 2^20)
    if ((u >> 31) || u > 0x7f800000u || u < 0x2B000000u /*2^-41*/ || u >= 0x49800000u /*2^20*/) bad = true;
    return d;
}
MP_INLINE bool is_inf(float d) { return f2u(d) == 0x7f800000u; }

// 128-bit fixed point (units 2^-64 ms) of a domain duration.
MP_INLINE void fixed64(float d, uint64_t& lo, uint64_t& hi) {
    uint32_t u = f2u(d);
    lo = hi = 0;
    if (u == 0u) return;
    uint32_t e = (u >> 23) & 0xff;                       // normal: d = (2^23|m) * 2^(e-150)
    uint64_t mant = (uint64_t)((u & 0x7fffffu) | 0x800000u);
    int sh = (int)e - 150 + 64;                          // >= 0 in domain (e >= 86)
    if (sh < 64) {
        lo = mant << sh;
        hi = sh == 0 ? 0 : (mant >> (64 - sh));
    } else {
        hi = mant << (sh - 64);
    }
}

MP_INLINE void add128(uint64_t& lo, uint64_t& hi, uint64_t blo, uint64_t bhi) {
    uint64_t r = lo + blo;
    hi = hi + bhi + (r < lo ? 1ull : 0ull);
    lo = r;
}

// warp-reduce a 128-bit unsigned sum, result valid in every lane
MP_INLINE void warp_sum128(uint64_t& lo, uint64_t& hi) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        uint64_t l2 = __shfl_xor_sync(0xffffffffu, lo, o);
        uint64_t h2 = __shfl_xor_sync(0xffffffffu, hi, o);
        add128(lo, hi, l2, h2);
    }
}

// atomically add a 128-bit value into (p[0]=lo, p[1]=hi)
MP_INLINE void atomic_add128(unsigned long long* p, uint64_t lo, uint64_t hi) {
    if (lo == 0 && hi == 0) return;
    unsigned long long old = atomicAdd(p, (unsigned long long)lo);
    uint64_t carry = (old + lo < old) ? 1ull : 0ull;
    if (hi + carry) atomicAdd(p + 1, (unsigned long long)(hi + carry));
}

// exact 128-bit integer x = hi:lo times 2^-64, rounded once to binary64 (RN-even)
MP_INLINE double u128_to_double_scaled(uint64_t lo, uint64_t hi) {
    if (hi == 0 && lo == 0) return 0.0;
    int msb = hi ? 127 - __clzll((long long)hi) : 63 - __clzll((long long)lo);
    int shift = msb - 52;
    if (shift <= 0) return ldexp((double)lo, -64);       // x < 2^53: exact
    uint64_t m, r_lo, r_hi, h_lo, h_hi;
    if (shift < 64) {
        m = (lo >> shift) | (hi << (64 - shift));
        r_lo = lo & ((1ull << shift) - 1);
        r_hi = 0;
    } else {
        m = hi >> (shift - 64);
        r_lo = lo;
        r_hi = shift == 64 ? 0ull : (hi & ((1ull << (shift - 64)) - 1));
    }
    if (shift - 1 < 64) { h_lo = 1ull << (shift - 1); h_hi = 0; }
    else { h_lo = 0; h_hi = 1ull << (shift - 65); }
    bool gt = r_hi > h_hi || (r_hi == h_hi && r_lo > h_lo);
    bool eq = r_hi == h_hi && r_lo == h_lo;
    if (gt || (eq && (m & 1))) {
        m += 1;
        if (m == (1ull << 53)) { m >>= 1; shift += 1; }
    }
    return ldexp((double)m, shift - 64);
}

template <typename T>
MP_INLINE T warp_max(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        T w = __shfl_xor_sync(0xffffffffu, v, o);
        v = v > w ? v : w;
    }
    return v;
}

// splitmix64 at a counter (north_star replica perturbation)
MP_INLINE uint64_t splitmix64(uint64_t seed, uint64_t c) {
    uint64_t x = seed + c * 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

// perturb() split at the splitmix64 state: x = seed + counter * golden (callers that walk
// counters add multiples of golden instead of multiplying); the same bits as perturb()
MP_INLINE float perturb_x(float d, uint64_t x, float sigma) {
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    x ^= x >> 31;
    float u = __fmul_rn((float)(uint32_t)(x >> 40), 0x1p-24f);
    float s = __fsub_rn(__fmul_rn(2.0f, u), 1.0f);
    float f = __fadd_rn(1.0f, __fmul_rn(sigma, s));
    return __fmul_rn(d, f);
}
constexpr uint64_t SPLITMIX_GOLDEN = 0x9E3779B97F4A7C15ull;

// the same with u = k * 2^-24 given (k < 2^24): the perturbation at a chosen draw
MP_INLINE float perturb_u(float d, float sigma, uint32_t k) {
    float u = __fmul_rn((float)k, 0x1p-24f);
    float s = __fsub_rn(__fmul_rn(2.0f, u), 1.0f);
    float f = __fadd_rn(1.0f, __fmul_rn(sigma, s));
    return __fmul_rn(d, f);
}

// delta_r(t,a) = delta * (1 + sigma*(2u-1)); explicit RN ops, no contraction
MP_INLINE float perturb(float d, uint64_t seed, float sigma, uint64_t counter) {
    float u = __fmul_rn((float)(uint32_t)(splitmix64(seed, counter) >> 40), 0x1p-24f);
    float s = __fsub_rn(__fmul_rn(2.0f, u), 1.0f);
    float f = __fadd_rn(1.0f, __fmul_rn(sigma, s));
    return __fmul_rn(d, f);
}

}  // namespace mpk
