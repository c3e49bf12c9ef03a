// micro.cuh -- per-level latency microbenchmarks (SURVEY §8(d) two-term roofline, §7 H1).
//
// A level-synchronous pass over a DAG of depth L costs at least L x t_level, where
// t_level is the cost of one level boundary plus the dependent memory round trips a
// level needs.  These kernels measure the candidates on their own, independently of
// the product kernels (which also do per-task work):
//   MP_MB_SYNC     one CTA of 1024 threads, L x __syncthreads
//   MP_MB_CLUSTER  one cluster of `arg` CTAs (2..8), L x cluster barrier
//   MP_MB_GRID     one CTA per SM, L x grid barrier (cooperative launch, cg::grid sync)
//   MP_MB_CHAIN    one thread, L dependent L2 loads (pointer chasing, ld.global.cg)
// bench.py times them with CUDA events and reports microseconds per level.
#pragma once
#include <cooperative_groups.h>

#include "common.cuh"

namespace mpk {

__global__ void __launch_bounds__(1024) k_mb_sync(int32_t L, uint32_t* sink) {
    __shared__ uint32_t x;
    if (threadIdx.x == 0) x = 0;
    for (int32_t r = 0; r < L; r++) {
        __syncthreads();
        if (threadIdx.x == (uint32_t)(r & 1023)) x += 1;
    }
    __syncthreads();
    if (threadIdx.x == 0) sink[0] = x;
}

__global__ void __launch_bounds__(1024) k_mb_cluster(int32_t L, uint32_t* sink) {
    namespace cg = cooperative_groups;
    cg::cluster_group cl = cg::this_cluster();
    __shared__ uint32_t x;
    if (threadIdx.x == 0) x = 0;
    for (int32_t r = 0; r < L; r++) {
        cl.sync();
        if (threadIdx.x == 0) x += 1;
    }
    cl.sync();
    if (threadIdx.x == 0 && cl.block_rank() == 0) sink[0] = x;
}

__global__ void __launch_bounds__(1024) k_mb_grid(int32_t L, uint32_t* sink) {
    namespace cg = cooperative_groups;
    cg::grid_group g = cg::this_grid();
    uint32_t x = 0;
    for (int32_t r = 0; r < L; r++) {
        g.sync();
        x += 1;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) sink[0] = x;
}

__global__ void k_mb_chain(int32_t L, const uint32_t* __restrict__ next, uint32_t* sink) {
    uint32_t p = 0;
    for (int32_t r = 0; r < L; r++) p = __ldcg(next + p);
    sink[0] = p;
}

}  // namespace mpk
