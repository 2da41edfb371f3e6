// device_util.cuh -- warp/block primitives and a decoupled look-back tile prefix for sm_100a.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "gp_internal.cuh"

namespace gp {

__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31u; }

__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// Proposal key of neighbour v over edge weight w (P12.s23, R3): heavier first, then the
// lower id.  key > 0 for every valid (w >= 1) arc; 0 means "no candidate".
__device__ __forceinline__ unsigned long long pack_key(int32_t w, int32_t v) {
    return ((unsigned long long)(uint32_t)w << 32) | (unsigned long long)(~(uint32_t)v);
}
__device__ __forceinline__ int32_t key_vertex(unsigned long long k) {
    return k ? (int32_t)(~(uint32_t)k) : kNone;
}

__device__ __forceinline__ unsigned long long umax64(unsigned long long a, unsigned long long b) {
    return a > b ? a : b;
}

template <int WIDTH>
__device__ __forceinline__ unsigned long long group_max64(unsigned long long k) {
#pragma unroll
    for (int off = WIDTH / 2; off > 0; off >>= 1) k = umax64(k, __shfl_xor_sync(0xffffffffu, k, off, WIDTH));
    return k;
}

__device__ __forceinline__ int32_t warp_sum(int32_t v) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
    return v;
}

__device__ __forceinline__ unsigned long long warp_sum64(unsigned long long v) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
    return v;
}

// Warp-aggregated append of the lanes with `pred` to list[*counter ...].  Must be called by
// all 32 lanes.  One atomic per warp (Guideline 12).
__device__ __forceinline__ void warp_append(int32_t *list, int32_t *counter, bool pred, int32_t value) {
    unsigned m = __ballot_sync(0xffffffffu, pred);
    if (m == 0) return;
    int leader = __ffs(m) - 1;
    int base = 0;
    if ((int)lane_id() == leader) base = atomicAdd(counter, __popc(m));
    base = __shfl_sync(0xffffffffu, base, leader);
    if (pred) list[base + __popc(m & lanemask_lt())] = value;
}

// Inclusive warp scan of int32.
__device__ __forceinline__ int32_t warp_incl_scan(int32_t v) {
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        int32_t t = __shfl_up_sync(0xffffffffu, v, off);
        if ((int)lane_id() >= off) v += t;
    }
    return v;
}

// Exclusive block scan of one int32 per thread; returns the exclusive prefix and the block
// total.  `smem` holds >= 33 ints.  All threads of the block must call.
template <int NT>
__device__ __forceinline__ int32_t block_excl_scan(int32_t v, int32_t *smem, int32_t &total) {
    constexpr int NW = NT / 32;
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    int32_t inc = warp_incl_scan(v);
    if (l == 31) smem[w] = inc;
    __syncthreads();
    if (w == 0) {
        int32_t x = (l < NW) ? smem[l] : 0;
        int32_t xi = warp_incl_scan(x);
        if (l < NW) smem[l] = xi - x;
        if (l == NW - 1) smem[32] = xi;
    }
    __syncthreads();
    total = smem[32];
    int32_t r = smem[w] + inc - v;
    __syncthreads();
    return r;
}

// ---------------------------------------------------------------------------------------
// Decoupled look-back (single-pass scan).  Status word per tile:
//   bits 63..34 epoch, 33..32 flag (1 = aggregate, 2 = inclusive prefix), 31..0 value.
// The epoch changes on every scan launch, so the status array never needs a memset.
// Called by warp 0 of the block; returns the exclusive prefix of `tile` (all lanes).
// ---------------------------------------------------------------------------------------
__device__ __forceinline__ void lb_store(unsigned long long *p, unsigned long long v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long lb_load(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ int32_t lookback_prefix(unsigned long long *status, uint32_t epoch, int tile,
                                                   int32_t aggregate) {
    const int l = lane_id();
    const unsigned long long tagA = ((unsigned long long)((epoch << 2) | 1u)) << 32;
    const unsigned long long tagP = ((unsigned long long)((epoch << 2) | 2u)) << 32;
    if (tile == 0) {
        if (l == 0) lb_store(status, tagP | (uint32_t)aggregate);
        return 0;
    }
    if (l == 0) lb_store(status + tile, tagA | (uint32_t)aggregate);
    int32_t prefix = 0;
    int pred = tile - 1;
    while (true) {
        int idx = pred - l;
        uint32_t flag = 2, val = 0;
        if (idx >= 0) {
            unsigned long long s;
            do {
                s = lb_load(status + idx);
                flag = ((uint32_t)(s >> 32) >> 2) == epoch ? ((uint32_t)(s >> 32) & 3u) : 0u;
            } while (flag == 0);
            val = (uint32_t)s;
        }
        unsigned incl = __ballot_sync(0xffffffffu, flag == 2);
        if (incl) {
            int first = __ffs(incl) - 1;  // nearest predecessor holding an inclusive prefix
            int32_t contrib = (l <= first) ? (int32_t)val : 0;
#pragma unroll
            for (int off = 16; off > 0; off >>= 1) contrib += __shfl_xor_sync(0xffffffffu, contrib, off);
            prefix += contrib;
            break;
        }
        int32_t contrib = (int32_t)val;
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) contrib += __shfl_xor_sync(0xffffffffu, contrib, off);
        prefix += contrib;
        pred -= 32;
    }
    if (l == 0) lb_store(status + tile, tagP | (uint32_t)(prefix + aggregate));
    return prefix;
}

}  // namespace gp
