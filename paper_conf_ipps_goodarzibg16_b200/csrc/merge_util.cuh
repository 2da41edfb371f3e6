// merge_util.cuh -- register sort network shared by the contraction kernels (contract.cu,
// small.cu): one thread sorts up to 16 (coarse id, weight) pairs by coarse id.
#pragma once

#include <stdint.h>

namespace gp {

// Batcher odd-even merge sort network for 16 inputs (63 comparators; generated and checked
// against sorted() offline).
// sort (cx, w) pairs by cx only: equal coarse ids are summed afterwards, so their order is
// irrelevant; a comparator is one 32-bit compare and four selects
__device__ __forceinline__ void cx_sort16(uint32_t (&cx)[16], int32_t (&w)[16]) {
#define GP_CE(i, j)                                                      \
    {                                                                    \
        const bool sw = cx[i] > cx[j];                                   \
        const uint32_t c0 = sw ? cx[j] : cx[i], c1 = sw ? cx[i] : cx[j]; \
        const int32_t w0 = sw ? w[j] : w[i], w1 = sw ? w[i] : w[j];      \
        cx[i] = c0;                                                      \
        cx[j] = c1;                                                      \
        w[i] = w0;                                                       \
        w[j] = w1;                                                       \
    }
    GP_CE(0, 1)
    GP_CE(2, 3)
    GP_CE(0, 2)
    GP_CE(1, 3)
    GP_CE(1, 2)
    GP_CE(4, 5)
    GP_CE(6, 7)
    GP_CE(4, 6)
    GP_CE(5, 7)
    GP_CE(5, 6)
    GP_CE(0, 4)
    GP_CE(2, 6)
    GP_CE(2, 4)
    GP_CE(1, 5)
    GP_CE(3, 7)
    GP_CE(3, 5)
    GP_CE(1, 2)
    GP_CE(3, 4)
    GP_CE(5, 6)
    GP_CE(8, 9)
    GP_CE(10, 11)
    GP_CE(8, 10)
    GP_CE(9, 11)
    GP_CE(9, 10)
    GP_CE(12, 13)
    GP_CE(14, 15)
    GP_CE(12, 14)
    GP_CE(13, 15)
    GP_CE(13, 14)
    GP_CE(8, 12)
    GP_CE(10, 14)
    GP_CE(10, 12)
    GP_CE(9, 13)
    GP_CE(11, 15)
    GP_CE(11, 13)
    GP_CE(9, 10)
    GP_CE(11, 12)
    GP_CE(13, 14)
    GP_CE(0, 8)
    GP_CE(4, 12)
    GP_CE(4, 8)
    GP_CE(2, 10)
    GP_CE(6, 14)
    GP_CE(6, 10)
    GP_CE(2, 4)
    GP_CE(6, 8)
    GP_CE(10, 12)
    GP_CE(1, 9)
    GP_CE(5, 13)
    GP_CE(5, 9)
    GP_CE(3, 11)
    GP_CE(7, 15)
    GP_CE(7, 11)
    GP_CE(3, 5)
    GP_CE(7, 9)
    GP_CE(11, 13)
    GP_CE(1, 2)
    GP_CE(3, 4)
    GP_CE(5, 6)
    GP_CE(7, 8)
    GP_CE(9, 10)
    GP_CE(11, 12)
    GP_CE(13, 14)
#undef GP_CE
}

// Batcher odd-even merge sort network for 8 inputs (19 comparators; checked exhaustively on
// 0-1 inputs), for rows of <= 8 merged entries (part.cu)
__device__ __forceinline__ void cx_sort8(uint32_t (&cx)[8], int32_t (&w)[8]) {
#define GP_CE(i, j)                                                      \
    {                                                                    \
        const bool sw = cx[i] > cx[j];                                   \
        const uint32_t c0 = sw ? cx[j] : cx[i], c1 = sw ? cx[i] : cx[j]; \
        const int32_t w0 = sw ? w[j] : w[i], w1 = sw ? w[i] : w[j];      \
        cx[i] = c0;                                                      \
        cx[j] = c1;                                                      \
        w[i] = w0;                                                       \
        w[j] = w1;                                                       \
    }
    GP_CE(0, 1)
    GP_CE(2, 3)
    GP_CE(4, 5)
    GP_CE(6, 7)
    GP_CE(0, 2)
    GP_CE(1, 3)
    GP_CE(4, 6)
    GP_CE(5, 7)
    GP_CE(1, 2)
    GP_CE(5, 6)
    GP_CE(0, 4)
    GP_CE(1, 5)
    GP_CE(2, 6)
    GP_CE(3, 7)
    GP_CE(2, 4)
    GP_CE(3, 5)
    GP_CE(1, 2)
    GP_CE(3, 4)
    GP_CE(5, 6)
#undef GP_CE
}

}  // namespace gp
