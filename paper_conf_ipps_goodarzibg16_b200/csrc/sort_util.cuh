// sort_util.cuh -- key sorts and run merges shared by the contraction kernels (contract.cu,
// part.cu): keys are (coarse id << 32 | weight); equal coarse ids are merged by summing
// their weights (R8, P12.s28).
#pragma once

#include <stdint.h>

#include "device_util.cuh"

namespace gp {

__device__ __forceinline__ unsigned long long ckey(int32_t cx, int32_t w) {
    return ((unsigned long long)(uint32_t)cx << 32) | (uint32_t)w;
}

__device__ __forceinline__ void cswap(unsigned long long &a, unsigned long long &b) {
    const unsigned long long lo = a < b ? a : b, hi = a < b ? b : a;
    a = lo;
    b = hi;
}

// Sort len keys in place (any len) with the flip bitonic network; comparators whose upper
// index is >= len are skipped (virtual +inf padding never moves).
template <typename Sync>
__device__ __forceinline__ void coop_sort(unsigned long long *keys, int len, int tid, int nthr, Sync sync) {
    int S = 1;
    while (S < len) S <<= 1;
    // power-of-two strides: index arithmetic by shifts and masks (a runtime division per
    // comparator was most of the instruction count of the C1h sorts)
    for (int lh = 0; (2 << lh) <= S; ++lh) {
        const int size = 2 << lh, half = 1 << lh;
        for (int i = tid; i < S / 2; i += nthr) {
            const int base = (i >> lh) << (lh + 1), o = i & (half - 1);
            const int x = base + o, y = base + size - 1 - o;
            if (y < len) {
                const unsigned long long p = keys[x], q = keys[y];
                if (p > q) {
                    keys[x] = q;
                    keys[y] = p;
                }
            }
        }
        sync();
        for (int lj = lh - 1; lj >= 0; --lj) {
            const int j = 1 << lj;
            for (int i = tid; i < S / 2; i += nthr) {
                const int x = ((i >> lj) << (lj + 1)) + (i & (j - 1)), y = x + j;
                if (y < len) {
                    const unsigned long long p = keys[x], q = keys[y];
                    if (p > q) {
                        keys[x] = q;
                        keys[y] = p;
                    }
                }
            }
            sync();
        }
    }
}

// Run-length merge of sorted (cx<<32|w) keys, in place and without compaction: the entry
// at the head of every run of equal cx receives (cx<<32 | run sum); other entries are left
// as they are, and a head is recognised later by cx(i) != cx(i-1).  Thread `tid` owns the
// contiguous chunk [lo,hi) and only ever writes head entries inside its chunk; a run that
// crosses chunk borders is completed with the leading partial sums of the following chunks
// (`lead`/`has`, nthr entries each, filled before any write).  Returns the number of runs.
// `scan(v, total)` = exclusive prefix over the group.  Sums fit int32 (R14).
template <typename Scan, typename Sync>
__device__ __forceinline__ int32_t coop_runsum(unsigned long long *keys, int len, int tid, int nthr, int32_t *lead,
                                               int32_t *has, Scan scan, Sync sync) {
    const int per = (len + nthr - 1) / nthr;
    const int lo = min(len, tid * per), hi = min(len, lo + per);
    int32_t heads = 0, lp = 0;
    int first_head = hi;
    for (int i = lo; i < hi; ++i) {
        if (i == 0 || (keys[i] >> 32) != (keys[i - 1] >> 32)) {
            if (heads == 0) first_head = i;
            ++heads;
        } else if (heads == 0) {
            lp += (int32_t)(uint32_t)keys[i];  // continues the previous chunk's run
        }
    }
    lead[tid] = lp;
    has[tid] = heads;
    sync();
    int32_t total;
    scan(heads, total);
    int i = first_head;
    while (i < hi) {
        const uint32_t cx = (uint32_t)(keys[i] >> 32);
        int32_t sum = (int32_t)(uint32_t)keys[i];
        int k = i + 1;
        while (k < hi && (uint32_t)(keys[k] >> 32) == cx) sum += (int32_t)(uint32_t)keys[k++];
        if (k == hi)  // run reaches my chunk's end: add the following chunks' lead partials
            for (int t = tid + 1; t < nthr; ++t) {
                sum += lead[t];
                if (has[t]) break;
            }
        keys[i] = ((unsigned long long)cx << 32) | (uint32_t)sum;  // my own head entry
        i = k;
    }
    sync();
    return total;
}

// ---------------------------------------------------------------------------------------
// one-warp register merge of a row with <= 64 entries: element e = r*32 + lane lives in
// v[r]; ascending flip-bitonic network with shuffles, then a segmented scan of the weights
// and ballot compaction of the run tails (cx < 2^32-1; padding = kMaxKey).
// ---------------------------------------------------------------------------------------
__device__ __forceinline__ unsigned long long shfl_xor64(unsigned long long x, int m) {
    return __shfl_xor_sync(0xffffffffu, x, m);
}

__device__ __forceinline__ void warp_sort64(unsigned long long (&v)[2]) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int size = 2; size <= 64; size <<= 1) {
        if (size == 64) {  // mirrored step across the two registers
            const unsigned long long o0 = shfl_xor64(v[1], 31), o1 = shfl_xor64(v[0], 31);
            v[0] = v[0] < o0 ? v[0] : o0;  // element lane pairs with 63-lane (higher)
            v[1] = v[1] > o1 ? v[1] : o1;
        } else {
            const int m = size - 1;
            const bool lower = (lane & (size >> 1)) == 0;
#pragma unroll
            for (int r = 0; r < 2; ++r) {
                const unsigned long long o = shfl_xor64(v[r], m);
                v[r] = lower ? (v[r] < o ? v[r] : o) : (v[r] > o ? v[r] : o);
            }
        }
#pragma unroll
        for (int j = size / 4; j > 0; j >>= 1) {
            const bool lower = (lane & j) == 0;
#pragma unroll
            for (int r = 0; r < 2; ++r) {
                const unsigned long long o = shfl_xor64(v[r], j);
                v[r] = lower ? (v[r] < o ? v[r] : o) : (v[r] > o ? v[r] : o);
            }
        }
    }
}

// merges the sorted v into (cx<<32|sum) entries written to out[0..count); returns count
__device__ __forceinline__ int32_t warp_runmerge64(const unsigned long long (&v)[2], unsigned long long *out) {
    const int lane = threadIdx.x & 31;
    uint32_t cx[2], w[2];
    bool head[2], tail[2];
#pragma unroll
    for (int r = 0; r < 2; ++r) {
        cx[r] = (uint32_t)(v[r] >> 32);
        w[r] = (uint32_t)v[r];
    }
    // neighbours in element order
    const uint32_t prev0 = __shfl_up_sync(0xffffffffu, cx[0], 1);
    const uint32_t prev1 = __shfl_up_sync(0xffffffffu, cx[1], 1);
    const uint32_t last0 = __shfl_sync(0xffffffffu, cx[0], 31);
    const uint32_t next0 = __shfl_down_sync(0xffffffffu, cx[0], 1);
    const uint32_t next1 = __shfl_down_sync(0xffffffffu, cx[1], 1);
    const uint32_t first1 = __shfl_sync(0xffffffffu, cx[1], 0);
    head[0] = lane == 0 || prev0 != cx[0];
    head[1] = (lane == 0) ? (last0 != cx[1]) : (prev1 != cx[1]);
    tail[0] = (lane == 31) ? (first1 != cx[0]) : (next0 != cx[0]);
    tail[1] = lane == 31 || next1 != cx[1];
    // segmented inclusive scan of the weights per register
    uint32_t sum[2];
    bool seen[2];
#pragma unroll
    for (int r = 0; r < 2; ++r) {
        uint32_t val = w[r];
        bool f = head[r];
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
            const uint32_t tv = __shfl_up_sync(0xffffffffu, val, off);
            const bool tf = __shfl_up_sync(0xffffffffu, f ? 1 : 0, off);
            if (lane >= off) {
                if (!f) val += tv;
                f = f || tf;
            }
        }
        sum[r] = val;
        seen[r] = f;
    }
    // the run that crosses from register 0 into register 1 carries register 0's tail sum
    const uint32_t carry = __shfl_sync(0xffffffffu, sum[0], 31);
    if (!seen[1]) sum[1] += carry;
    // emit at run tails, skipping padding, in element order
    const bool e0 = tail[0] && cx[0] != 0xFFFFFFFFu;
    const bool e1 = tail[1] && cx[1] != 0xFFFFFFFFu;
    const unsigned b0 = __ballot_sync(0xffffffffu, e0), b1 = __ballot_sync(0xffffffffu, e1);
    const unsigned lt = lanemask_lt();
    if (e0) out[__popc(b0 & lt)] = ((unsigned long long)cx[0] << 32) | sum[0];
    if (e1) out[__popc(b0) + __popc(b1 & lt)] = ((unsigned long long)cx[1] << 32) | sum[1];
    return __popc(b0) + __popc(b1);
}

// Half-warp (16-lane segment) version for rows of 17..32 entries: two rows per warp step.
// Element e = r*16 + l of a segment lives in v[r] of segment lane l; same flip-bitonic
// network (15 stages instead of 21) and segmented run merge.  `out` is this segment's row.
__device__ __forceinline__ void seg_sort32(unsigned long long (&v)[2]) {
    const int l = threadIdx.x & 15;
#pragma unroll
    for (int size = 2; size <= 32; size <<= 1) {
        if (size == 32) {  // mirrored step across the two registers
            const unsigned long long o0 = __shfl_xor_sync(0xffffffffu, v[1], 15, 16);
            const unsigned long long o1 = __shfl_xor_sync(0xffffffffu, v[0], 15, 16);
            v[0] = v[0] < o0 ? v[0] : o0;
            v[1] = v[1] > o1 ? v[1] : o1;
        } else {
            const bool lower = (l & (size >> 1)) == 0;
#pragma unroll
            for (int r = 0; r < 2; ++r) {
                const unsigned long long o = __shfl_xor_sync(0xffffffffu, v[r], size - 1, 16);
                v[r] = lower ? (v[r] < o ? v[r] : o) : (v[r] > o ? v[r] : o);
            }
        }
#pragma unroll
        for (int j = size / 4; j > 0; j >>= 1) {
            const bool lower = (l & j) == 0;
#pragma unroll
            for (int r = 0; r < 2; ++r) {
                const unsigned long long o = __shfl_xor_sync(0xffffffffu, v[r], j, 16);
                v[r] = lower ? (v[r] < o ? v[r] : o) : (v[r] > o ? v[r] : o);
            }
        }
    }
}

__device__ __forceinline__ int32_t seg_runmerge32(const unsigned long long (&v)[2], unsigned long long *out) {
    const int lane = threadIdx.x & 31, l = lane & 15;
    const unsigned seg = (lane & 16) ? 0xFFFF0000u : 0x0000FFFFu;
    uint32_t cx[2], w[2];
    bool head[2], tail[2];
#pragma unroll
    for (int r = 0; r < 2; ++r) {
        cx[r] = (uint32_t)(v[r] >> 32);
        w[r] = (uint32_t)v[r];
    }
    const uint32_t prev0 = __shfl_up_sync(0xffffffffu, cx[0], 1, 16);
    const uint32_t prev1 = __shfl_up_sync(0xffffffffu, cx[1], 1, 16);
    const uint32_t last0 = __shfl_sync(0xffffffffu, cx[0], 15, 16);
    const uint32_t next0 = __shfl_down_sync(0xffffffffu, cx[0], 1, 16);
    const uint32_t next1 = __shfl_down_sync(0xffffffffu, cx[1], 1, 16);
    const uint32_t first1 = __shfl_sync(0xffffffffu, cx[1], 0, 16);
    head[0] = l == 0 || prev0 != cx[0];
    head[1] = (l == 0) ? (last0 != cx[1]) : (prev1 != cx[1]);
    tail[0] = (l == 15) ? (first1 != cx[0]) : (next0 != cx[0]);
    tail[1] = l == 15 || next1 != cx[1];
    uint32_t sum[2];
    bool seen[2];
#pragma unroll
    for (int r = 0; r < 2; ++r) {
        uint32_t val = w[r];
        bool f = head[r];
#pragma unroll
        for (int off = 1; off < 16; off <<= 1) {
            const uint32_t tv = __shfl_up_sync(0xffffffffu, val, off, 16);
            const bool tf = __shfl_up_sync(0xffffffffu, f ? 1 : 0, off, 16);
            if (l >= off) {
                if (!f) val += tv;
                f = f || tf;
            }
        }
        sum[r] = val;
        seen[r] = f;
    }
    const uint32_t carry = __shfl_sync(0xffffffffu, sum[0], 15, 16);
    if (!seen[1]) sum[1] += carry;
    const bool e0 = tail[0] && cx[0] != 0xFFFFFFFFu;
    const bool e1 = tail[1] && cx[1] != 0xFFFFFFFFu;
    const unsigned b0 = __ballot_sync(0xffffffffu, e0) & seg, b1 = __ballot_sync(0xffffffffu, e1) & seg;
    const unsigned lt = lanemask_lt();
    if (e0) out[__popc(b0 & lt)] = ((unsigned long long)cx[0] << 32) | sum[0];
    if (e1) out[__popc(b0) + __popc(b1 & lt)] = ((unsigned long long)cx[1] << 32) | sum[1];
    return __popc(b0) + __popc(b1);
}

}  // namespace gp
