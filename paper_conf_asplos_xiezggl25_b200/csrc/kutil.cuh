// kutil.cuh -- small device helpers shared by the CUDA kernels (not by the oracle).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "frugal_internal.cuh"

namespace frugal {

#define FULL 0xffffffffu

__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// grid sized as a multiple of the SM count, capped by the work
static inline int grid_for(int64_t work, int per_block, int max_waves = 8) {
    int64_t b = (work + per_block - 1) / per_block;
    int64_t cap = (int64_t)kSMs * max_waves;
    if (b > cap) b = cap;
    if (b < 1) b = 1;
    return (int)b;
}

__device__ __forceinline__ void chunk_range(int n, int nblk, int b, int& lo, int& hi) {
    int per = (n + nblk - 1) / nblk;
    per = (per + kTile - 1) / kTile * kTile;
    lo = min(n, b * per);
    hi = min(n, lo + per);
}

template <int GS>
struct RowGroup {
    // lanes [grp*GS, grp*GS+GS) of the warp handle one row; returns global group id/stride
    static __device__ __forceinline__ void ids(int64_t& gid, int64_t& gstride, int& l) {
        int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
        gid = t / GS;
        gstride = ((int64_t)gridDim.x * blockDim.x) / GS;
        l = threadIdx.x & (GS - 1);
    }
};

// block-aggregated counter: every thread passes its count, one atomic per block.  The closing
// barrier keeps thread 0's reset of the next call away from this call's read (the shared word
// is one per block across calls; compute-sanitizer racecheck flagged the unordered pair)
__device__ __forceinline__ void block_count(unsigned long long* dst, unsigned v) {
    __shared__ unsigned s_cnt;
    if (threadIdx.x == 0) s_cnt = 0;
    __syncthreads();
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((threadIdx.x & 31) == 0 && v) atomicAdd(&s_cnt, v);
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned t = s_cnt;
        if (t) atomicAdd(dst, (unsigned long long)t);
    }
    __syncthreads();
}

// make this block's prior (host-memory) writes visible system-wide before anything the
// block's thread 0 -- or a later kernel in stream order -- publishes: CTA barrier, then one
// fence.sc.sys (cumulative over the writes ordered before it by the barrier).  Needed
// only when other processes read the host table (world > 1); all threads must call it.
__device__ __forceinline__ void block_fence_system() {
    __syncthreads();
    if (threadIdx.x == 0) __threadfence_system();
}

// host-table row slot of global row k (frugal_config.host_order); hs == nullptr: slot = k
__device__ __forceinline__ int64_t host_row(const int32_t* __restrict__ hs, int64_t k) {
    return hs ? (int64_t)hs[k] : k;
}

static inline int group_size(int d4) {
    int gs = 1;
    while (gs < d4 && gs < 32) gs <<= 1;
    return gs;
}

#define DISPATCH_GS(gs, ...)                  \
    switch (gs) {                             \
        case 1: { constexpr int GS = 1; __VA_ARGS__; } break;   \
        case 2: { constexpr int GS = 2; __VA_ARGS__; } break;   \
        case 4: { constexpr int GS = 4; __VA_ARGS__; } break;   \
        case 8: { constexpr int GS = 8; __VA_ARGS__; } break;   \
        case 16: { constexpr int GS = 16; __VA_ARGS__; } break; \
        default: { constexpr int GS = 32; __VA_ARGS__; } break; \
    }


}  // namespace frugal
