// contract.cu -- A4 leftover + A5 cmap + A6 sizing + A7 merge + A8 coarse CSR assembly.
//
// Paper: the mapping array CM is built by four kernels (flag u<=M[u], CUB inclusive scan,
// subtract one, partner copy; P18.s16-27).  Contraction sizes each thread's output by the
// pair's degree sum (P20.s5-11), merges the two neighbour lists by quicksort + duplicate
// removal or by a per-thread hash table (P20.s14-21), counts, scans again and copies the
// rows into the final arrays (P20.s22-26).
//
// B200 design:
//  * A4+A5+A6 are ONE single-pass kernel (decoupled look-back scan over the leader flags):
//    the leftover self-match, the exclusive scan (= the paper's inclusive scan minus one),
//    the leader list, the partner's CM (written by its leader, so no second pass), the
//    coarse vertex weight and the merged-row upper bound are all produced in one read of M.
//  * A7 bins coarse rows by their upper bound: <= 16 entries are merged by one thread in
//    registers (bitonic network + run-length sum); <= 256 by a warp in shared memory;
//    <= 8192 by a CTA in shared memory; longer (R-MAT hubs) by a CTA in global scratch.
//    Rows are emitted in ascending coarse id (R10) with weights of repeated coarse
//    neighbours summed (R8) and the collapsed edge dropped (R9).
//  * A8: look-back scan of the merged counts + compaction into the final arrays.
#include <cuda_runtime.h>

#include "device_util.cuh"
#include "gp_internal.cuh"

namespace gp {

constexpr int kScanItems = 8;
constexpr int kTile = kBlock * kScanItems;  // 2048 elements per look-back tile
constexpr int kNet = 16;                    // thread-bin capacity
constexpr int kWarpCap = 256;               // warp-bin capacity (entries)
constexpr int kCtaCap = 8192;               // CTA-bin capacity (entries, 64 KB smem)
constexpr unsigned long long kMaxKey = ~0ull;

struct ContractBufs {
    int32_t *leaders, *ub, *off, *cnt;
    int32_t *binW, *binC, *binG;
    int32_t *tadj, *tw;           // merged rows at off[c] (P20.s11-13 "temporary" arrays)
    unsigned long long *gkeys;    // global-bin sort space at off[c]
};

// ---------------------------------------------------------------------------------------
// A4 leftover + A5 cmap + A6 sizing: one decoupled look-back pass over u in [0, n)
// ---------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kBlock) k_cmap_scan(int32_t n, const int32_t *__restrict__ adjp,
                                                      const int32_t *__restrict__ vwgt, int32_t *__restrict__ M,
                                                      int32_t *__restrict__ CM, ContractBufs b,
                                                      int32_t *__restrict__ cvwgt, unsigned long long *status,
                                                      uint32_t epoch, LevelCtl *ctl, int apply_leftover) {
    __shared__ int32_t s_scan[33];
    __shared__ int32_t s_tile, s_prefix;
    const int ntiles = (n + kTile - 1) / kTile;
    while (true) {
        if (threadIdx.x == 0) s_tile = (int32_t)atomicAdd(&ctl->tile_ctr[0], 1u);
        __syncthreads();
        const int tile = s_tile;
        __syncthreads();
        if (tile >= ntiles) break;
        const long long base = (long long)tile * kTile + (long long)threadIdx.x * kScanItems;
        int32_t m[kScanItems];
        int32_t cnt = 0;
#pragma unroll
        for (int i = 0; i < kScanItems; ++i) {
            const long long u = base + i;
            m[i] = -2;
            if (u < n) {
                m[i] = M[u];
                if (m[i] == kFree && apply_leftover) {
                    m[i] = (int32_t)u;  // leftover: matched to itself (P18.s12-13)
                    M[u] = (int32_t)u;
                }
                cnt += (u <= m[i]) ? 1 : 0;  // leader flag (P18.s18, R7)
            }
        }
        int32_t total;
        int32_t excl = block_excl_scan<kBlock>(cnt, s_scan, total);
        if (threadIdx.x < 32) {
            int32_t pre = lookback_prefix(status, epoch, tile, total);
            if (threadIdx.x == 0) s_prefix = pre;
        }
        __syncthreads();
        int32_t c = s_prefix + excl;
        if (tile == ntiles - 1 && threadIdx.x == 0) ctl->n_coarse = s_prefix + total;
#pragma unroll
        for (int i = 0; i < kScanItems; ++i) {
            const long long u = base + i;
            if (u < n && u <= m[i]) {
                const int32_t v = m[i];
                CM[u] = c;                      // exclusive scan = inclusive - 1 (P18.s20-24)
                b.leaders[c] = (int32_t)u;
                int32_t d = adjp[u + 1] - adjp[u];
                int32_t vw = vwgt[u];
                if (v != u) {
                    CM[v] = c;                  // partner copies its leader's id (P18.s26)
                    d += adjp[v + 1] - adjp[v];  // sizing: deg(u) + deg(v) (P20.s6-8)
                    vw += vwgt[v];               // w(c) = w(u) + w(v) (P12.s27)
                }
                b.ub[c] = d;
                cvwgt[c] = vw;
                ++c;
            }
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------------------
// generic exclusive scan: out[i] = sum_{j<i} in[j] for i <= count, count read from device
// ---------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kBlock) k_scan_excl(const int32_t *__restrict__ in, int32_t *__restrict__ out,
                                                      const int32_t *count_ptr, int32_t *total_out,
                                                      unsigned long long *status, uint32_t epoch,
                                                      uint32_t *tile_ctr) {
    __shared__ int32_t s_scan[33];
    __shared__ int32_t s_tile, s_prefix;
    const int32_t count = *count_ptr;
    const int ntiles = count > 0 ? (count + kTile - 1) / kTile : 0;
    if (count == 0) {
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            out[0] = 0;
            if (total_out) *total_out = 0;
        }
        return;
    }
    while (true) {
        if (threadIdx.x == 0) s_tile = (int32_t)atomicAdd(tile_ctr, 1u);
        __syncthreads();
        const int tile = s_tile;
        __syncthreads();
        if (tile >= ntiles) break;
        const long long base = (long long)tile * kTile + (long long)threadIdx.x * kScanItems;
        int32_t x[kScanItems];
        int32_t sum = 0;
#pragma unroll
        for (int i = 0; i < kScanItems; ++i) {
            x[i] = (base + i < count) ? in[base + i] : 0;
            sum += x[i];
        }
        int32_t total;
        int32_t excl = block_excl_scan<kBlock>(sum, s_scan, total);
        if (threadIdx.x < 32) {
            int32_t pre = lookback_prefix(status, epoch, tile, total);
            if (threadIdx.x == 0) s_prefix = pre;
        }
        __syncthreads();
        int32_t run = s_prefix + excl;
#pragma unroll
        for (int i = 0; i < kScanItems; ++i) {
            if (base + i < count) out[base + i] = run;
            run += x[i];
        }
        if (tile == ntiles - 1 && threadIdx.x == 0) {
            out[count] = s_prefix + total;
            if (total_out) *total_out = s_prefix + total;
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------------------
// A7 helpers
// ---------------------------------------------------------------------------------------
// coarse key of one arc: coarse neighbour id in the high word, edge weight in the low word
__device__ __forceinline__ unsigned long long ckey(int32_t cx, int32_t w) {
    return ((unsigned long long)(uint32_t)cx << 32) | (uint32_t)w;
}

__device__ __forceinline__ void cswap(unsigned long long &a, unsigned long long &b) {
    unsigned long long lo = a < b ? a : b, hi = a < b ? b : a;
    a = lo;
    b = hi;
}

// ascending bitonic network on N registers (flip formulation: all comparators ascending)
template <int N>
__device__ __forceinline__ void reg_sort(unsigned long long (&k)[N]) {
#pragma unroll
    for (int size = 2; size <= N; size <<= 1) {
#pragma unroll
        for (int i = 0; i < N; ++i) {
            const int partner = i ^ (size - 1);
            if ((i & (size / 2)) == 0 && partner > i) cswap(k[i], k[partner]);
        }
#pragma unroll
        for (int j = size / 4; j > 0; j >>= 1) {
#pragma unroll
            for (int i = 0; i < N; ++i)
                if ((i & j) == 0) cswap(k[i], k[i ^ j]);
        }
    }
}

// Sort len keys in place (any len) with the flip bitonic network; comparators whose
// upper index is >= len are skipped (virtual +inf padding never moves).
// Cooperative over `nthr` threads with index `tid`; `sync()` separates steps.
template <typename Sync>
__device__ __forceinline__ void coop_sort(unsigned long long *keys, int len, int tid, int nthr, Sync sync) {
    int S = 1;
    while (S < len) S <<= 1;
    for (int size = 2; size <= S; size <<= 1) {
        for (int i = tid; i < S / 2; i += nthr) {
            // i-th comparator of the flip step: block of `size`, lower half index
            const int blk = i / (size / 2), off = i % (size / 2);
            const int a = blk * size + off, bb = blk * size + size - 1 - off;
            if (bb < len) {
                unsigned long long x = keys[a], y = keys[bb];
                if (x > y) {
                    keys[a] = y;
                    keys[bb] = x;
                }
            }
        }
        sync();
        for (int j = size / 4; j > 0; j >>= 1) {
            for (int i = tid; i < S / 2; i += nthr) {
                const int blk = i / j, off = i % j;
                const int a = blk * 2 * j + off, bb = a + j;
                if (bb < len) {
                    unsigned long long x = keys[a], y = keys[bb];
                    if (x > y) {
                        keys[a] = y;
                        keys[bb] = x;
                    }
                }
            }
            sync();
        }
    }
}

// run-length merge of sorted keys into (coarse id, summed weight); threads own contiguous
// chunks; `scan(v, total)` returns the exclusive prefix of v over the cooperating threads.
template <typename Scan>
__device__ __forceinline__ int32_t coop_dedup(const unsigned long long *keys, int len, int tid, int nthr,
                                              int32_t *out_adj, int32_t *out_w, Scan scan) {
    const int per = (len + nthr - 1) / nthr;
    const int lo = min(len, tid * per), hi = min(len, lo + per);
    int32_t heads = 0;
    for (int i = lo; i < hi; ++i)
        if (i == 0 || (keys[i] >> 32) != (keys[i - 1] >> 32)) ++heads;
    int32_t total;
    int32_t o = scan(heads, total);
    for (int i = lo; i < hi; ++i) {
        const uint32_t cx = (uint32_t)(keys[i] >> 32);
        if (i == 0 || (keys[i - 1] >> 32) != cx) {
            int32_t s = (int32_t)(uint32_t)keys[i];
            for (int k = i + 1; k < len && (uint32_t)(keys[k] >> 32) == cx; ++k) s += (int32_t)(uint32_t)keys[k];
            out_adj[o] = (int32_t)cx;
            out_w[o] = s;
            ++o;
        }
    }
    return total;
}

// ---------------------------------------------------------------------------------------
// A7, thread bin (ub <= 16) + routing of longer rows to the warp / CTA / global bins
// ---------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kBlock) k_merge_small(const int32_t *__restrict__ adjp,
                                                        const int32_t *__restrict__ adjncy,
                                                        const int32_t *__restrict__ adjwgt,
                                                        const int32_t *__restrict__ M,
                                                        const int32_t *__restrict__ CM, ContractBufs b,
                                                        LevelCtl *ctl) {
    const int32_t nc = ctl->n_coarse;
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long base = (long long)blockIdx.x * blockDim.x + (threadIdx.x & ~31); base < nc; base += stride) {
        const long long cc = base + (threadIdx.x & 31);
        int32_t ub = 0, s0 = 0;
        const bool valid = cc < nc;
        if (valid) {
            s0 = b.off[cc];
            ub = b.off[cc + 1] - s0;
        }
        warp_append(b.binW, &ctl->n_big_w, valid && ub > kNet && ub <= kWarpCap, (int32_t)cc);
        warp_append(b.binC, &ctl->n_big_c, valid && ub > kWarpCap && ub <= kCtaCap, (int32_t)cc);
        warp_append(b.binG, &ctl->n_big_g, valid && ub > kCtaCap, (int32_t)cc);
        if (!valid || ub > kNet) continue;
        const int32_t c = (int32_t)cc;
        const int32_t u = b.leaders[c];
        const int32_t v = M[u];
        const int32_t su = adjp[u], du = adjp[u + 1] - su;
        const int32_t sv = (v != u) ? adjp[v] : 0;
        unsigned long long k[kNet];
#pragma unroll
        for (int i = 0; i < kNet; ++i) {
            k[i] = kMaxKey;
            if (i < ub) {
                const int32_t j = (i < du) ? su + i : sv + (i - du);
                const int32_t cx = CM[__ldg(adjncy + j)];
                if (cx != c) k[i] = ckey(cx, __ldg(adjwgt + j));  // drop the collapsed edge (R9)
            }
        }
        reg_sort<kNet>(k);
        int32_t o = 0, prev = -1, acc = 0;
#pragma unroll
        for (int i = 0; i < kNet; ++i) {
            if (k[i] != kMaxKey) {
                const int32_t cx = (int32_t)(k[i] >> 32), w = (int32_t)(uint32_t)k[i];
                if (cx == prev) {
                    acc += w;  // repeated coarse neighbour: weights summed (R8, P12.s28)
                } else {
                    if (prev >= 0) {
                        b.tadj[s0 + o] = prev;
                        b.tw[s0 + o] = acc;
                        ++o;
                    }
                    prev = cx;
                    acc = w;
                }
            }
        }
        if (prev >= 0) {
            b.tadj[s0 + o] = prev;
            b.tw[s0 + o] = acc;
            ++o;
        }
        b.cnt[c] = o;
    }
}

// gather the (filtered) coarse keys of row c into dst[0..len), cooperative over a group;
// returns len.  Order of the gathered keys is irrelevant (they are sorted next).
template <typename Count>
__device__ __forceinline__ void gather_row(const int32_t *adjp, const int32_t *adjncy, const int32_t *adjwgt,
                                           const int32_t *M, const int32_t *CM, const int32_t *leaders, int32_t c,
                                           int tid, int nthr, unsigned long long *dst, Count claim) {
    const int32_t u = leaders[c];
    const int32_t v = M[u];
    for (int side = 0; side < (v != u ? 2 : 1); ++side) {
        const int32_t y = side ? v : u;
        const int32_t s = adjp[y], e = adjp[y + 1];
        for (int32_t j = s + tid; j < e; j += nthr) {
            const int32_t cx = CM[__ldg(adjncy + j)];
            if (cx != c) dst[claim()] = ckey(cx, __ldg(adjwgt + j));
        }
    }
}

// ---------------------------------------------------------------------------------------
// A7, warp bin (16 < ub <= 256): one warp per row, keys in shared memory
// ---------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kBlock) k_merge_warp(const int32_t *__restrict__ adjp,
                                                       const int32_t *__restrict__ adjncy,
                                                       const int32_t *__restrict__ adjwgt,
                                                       const int32_t *__restrict__ M,
                                                       const int32_t *__restrict__ CM, ContractBufs b,
                                                       LevelCtl *ctl) {
    __shared__ unsigned long long s_keys[kBlock / 32][kWarpCap];
    __shared__ int32_t s_len[kBlock / 32];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int nW = ctl->n_big_w;
    unsigned long long *keys = s_keys[wib];
    for (int i = blockIdx.x * (kBlock / 32) + wib; i < nW; i += gridDim.x * (kBlock / 32)) {
        const int32_t c = b.binW[i];
        if (lane == 0) s_len[wib] = 0;
        __syncwarp();
        gather_row(adjp, adjncy, adjwgt, M, CM, b.leaders, c, lane, 32, keys,
                   [&]() { return atomicAdd(&s_len[wib], 1); });
        __syncwarp();
        const int len = s_len[wib];
        coop_sort(keys, len, lane, 32, []() { __syncwarp(); });
        const int32_t s0 = b.off[c];
        int32_t o = coop_dedup(keys, len, lane, 32, b.tadj + s0, b.tw + s0, [&](int32_t v, int32_t &tot) {
            int32_t inc = warp_incl_scan(v);
            tot = __shfl_sync(0xffffffffu, inc, 31);
            return inc - v;
        });
        if (lane == 0) b.cnt[c] = o;
        __syncwarp();
    }
}

// ---------------------------------------------------------------------------------------
// A7, CTA bin (256 < ub <= 8192): one CTA per row, keys in (dynamic) shared memory
// A7, global bin (ub > 8192, hubs): one CTA per row, keys in global scratch
// ---------------------------------------------------------------------------------------
template <bool kGlobal>
__global__ void __launch_bounds__(kBlock) k_merge_cta(const int32_t *__restrict__ adjp,
                                                      const int32_t *__restrict__ adjncy,
                                                      const int32_t *__restrict__ adjwgt,
                                                      const int32_t *__restrict__ M,
                                                      const int32_t *__restrict__ CM, ContractBufs b,
                                                      LevelCtl *ctl) {
    extern __shared__ unsigned long long s_dyn[];
    __shared__ int32_t s_scan[33];
    __shared__ int32_t s_len;
    const int nB = kGlobal ? ctl->n_big_g : ctl->n_big_c;
    const int32_t *bin = kGlobal ? b.binG : b.binC;
    for (int i = blockIdx.x; i < nB; i += gridDim.x) {
        const int32_t c = bin[i];
        const int32_t s0 = b.off[c];
        unsigned long long *keys = kGlobal ? (b.gkeys + s0) : s_dyn;
        if (threadIdx.x == 0) s_len = 0;
        __syncthreads();
        gather_row(adjp, adjncy, adjwgt, M, CM, b.leaders, c, threadIdx.x, kBlock, keys,
                   [&]() { return atomicAdd(&s_len, 1); });
        __syncthreads();
        const int len = s_len;
        coop_sort(keys, len, threadIdx.x, kBlock, []() { __syncthreads(); });
        int32_t o = coop_dedup(keys, len, threadIdx.x, kBlock, b.tadj + s0, b.tw + s0,
                               [&](int32_t v, int32_t &tot) { return block_excl_scan<kBlock>(v, s_scan, tot); });
        if (threadIdx.x == 0) b.cnt[c] = o;
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------------------
// A8 compaction: merged rows from the temporary arrays into the final coarse CSR
// (P20.s22-24); G lanes per row.
// ---------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kBlock) k_compact(const int32_t *__restrict__ off, const int32_t *__restrict__ cnt,
                                                    const int32_t *__restrict__ cadjp,
                                                    const int32_t *__restrict__ tadj, const int32_t *__restrict__ tw,
                                                    int32_t *__restrict__ cadjncy, int32_t *__restrict__ cadjwgt,
                                                    LevelCtl *ctl) {
    constexpr int G = 8;
    const int32_t nc = ctl->n_coarse;
    const long long gid = ((long long)blockIdx.x * blockDim.x + threadIdx.x) / G;
    const int gl = threadIdx.x % G;
    const long long ng = ((long long)gridDim.x * blockDim.x) / G;
    for (long long c = gid; c < nc; c += ng) {
        const int32_t s = off[c], d = cadjp[c], k = cnt[c];
        for (int32_t j = gl; j < k; j += G) {
            cadjncy[d + j] = tadj[s + j];
            cadjwgt[d + j] = tw[s + j];
        }
    }
}

// ---------------------------------------------------------------------------------------
// host driver of one contraction
// ---------------------------------------------------------------------------------------
static uint32_t next_epoch(Ctx *ctx) {
    uint32_t e = ctx->epoch;
    ctx->epoch = (ctx->epoch + 1) & 0x3FFFFFFFu;
    if (ctx->epoch == 0) ctx->epoch = 1;
    return e;
}

gp_status contract_level(Ctx *ctx, const Graph *g, int32_t *M, int32_t *CM, bool apply_leftover,
                         Graph **coarse_out) {
    *coarse_out = nullptr;
    const int32_t n = g->n, nnz = g->nnz;
    const size_t nn = (size_t)n;
    const size_t ints = 7 * nn + 4 + 2 * (size_t)nnz;
    const size_t bytes = ((ints * 4 + 15) / 16) * 16 + 8 * (size_t)nnz;
    gp_status st = ensure_scratch(ctx, bytes);
    if (st != GP_OK) return st;
    st = ensure_status(ctx, nn / kTile + 2);
    if (st != GP_OK) return st;
    int32_t *p = (int32_t *)ctx->scratch;
    ContractBufs b;
    b.leaders = p; p += nn;
    b.ub = p; p += nn + 1;
    b.off = p; p += nn + 1;
    b.cnt = p; p += nn;
    b.binW = p; p += nn;
    b.binC = p; p += nn;
    b.binG = p; p += nn;
    b.tadj = p; p += nnz;
    b.tw = p; p += nnz;
    b.gkeys = (unsigned long long *)((char *)ctx->scratch + ((ints * 4 + 15) / 16) * 16);

    Graph *cg = new Graph();
    cg->ctx = ctx;
    st = dev_alloc(ctx, (void **)&cg->adjp, sizeof(int32_t) * (nn + 1));
    if (st == GP_OK) st = dev_alloc(ctx, (void **)&cg->vwgt, sizeof(int32_t) * (nn > 0 ? nn : 1));
    if (st == GP_OK) st = dev_alloc(ctx, (void **)&cg->adjncy, sizeof(int32_t) * (nnz > 0 ? nnz : 1));
    if (st == GP_OK) st = dev_alloc(ctx, (void **)&cg->adjwgt, sizeof(int32_t) * (nnz > 0 ? nnz : 1));
    if (st != GP_OK) {
        dev_free(ctx, cg->adjp);
        dev_free(ctx, cg->vwgt);
        dev_free(ctx, cg->adjncy);
        dev_free(ctx, cg->adjwgt);
        delete cg;
        return st;
    }

    LevelCtl *ctl = ctx->ctl;
    cudaStream_t s = ctx->stream;
    GP_CUDA(cudaMemsetAsync(ctl, 0, sizeof(LevelCtl), s));
    const int grid = persistent_grid(ctx, ctx->max_threads_sm / kBlock);
    if (n > 0) {
        LaunchScope ls(ctx, GP_K_CMAP);
        k_cmap_scan<<<grid, kBlock, 0, s>>>(n, g->adjp, g->vwgt, M, CM, b, cg->vwgt, ctx->status, next_epoch(ctx),
                                            ctl, apply_leftover ? 1 : 0);
        ++ctx->launches;
    }
    {
        LaunchScope ls(ctx, GP_K_ASSEMBLE);
        k_scan_excl<<<grid, kBlock, 0, s>>>(b.ub, b.off, &ctl->n_coarse, nullptr, ctx->status, next_epoch(ctx),
                                            &ctl->tile_ctr[1]);
        ++ctx->launches;
    }
    {
        LaunchScope ls(ctx, GP_K_CONTRACT);
        k_merge_small<<<grid, kBlock, 0, s>>>(g->adjp, g->adjncy, g->adjwgt, M, CM, b, ctl);
        ++ctx->launches;
    }
    {
        LaunchScope ls(ctx, GP_K_CONTRACT);
        k_merge_warp<<<grid, kBlock, 0, s>>>(g->adjp, g->adjncy, g->adjwgt, M, CM, b, ctl);
        ++ctx->launches;
    }
    {
        LaunchScope ls(ctx, GP_K_CONTRACT);
        const size_t smem = sizeof(unsigned long long) * kCtaCap;
        k_merge_cta<false><<<persistent_grid(ctx, 2), kBlock, smem, s>>>(g->adjp, g->adjncy, g->adjwgt, M, CM, b,
                                                                         ctl);
        ++ctx->launches;
    }
    {
        LaunchScope ls(ctx, GP_K_CONTRACT);
        k_merge_cta<true><<<persistent_grid(ctx, 2), kBlock, 0, s>>>(g->adjp, g->adjncy, g->adjwgt, M, CM, b, ctl);
        ++ctx->launches;
    }
    {
        LaunchScope ls(ctx, GP_K_ASSEMBLE);
        k_scan_excl<<<grid, kBlock, 0, s>>>(b.cnt, cg->adjp, &ctl->n_coarse, &ctl->cnnz, ctx->status,
                                            next_epoch(ctx), &ctl->tile_ctr[2]);
        ++ctx->launches;
    }
    {
        LaunchScope ls(ctx, GP_K_ASSEMBLE);
        k_compact<<<grid, kBlock, 0, s>>>(b.off, b.cnt, cg->adjp, b.tadj, b.tw, cg->adjncy, cg->adjwgt, ctl);
        ++ctx->launches;
    }
    GP_CUDA(cudaGetLastError());
    GP_CUDA(cudaMemcpyAsync(ctx->ctl_host, ctl, sizeof(LevelCtl), cudaMemcpyDeviceToHost, s));
    GP_CUDA(cudaStreamSynchronize(s));
    cg->n = ctx->ctl_host->n_coarse;
    cg->nnz = ctx->ctl_host->cnnz;
    *coarse_out = cg;
    return GP_OK;
}

gp_status contract_set_attributes() {
    cudaError_t e = cudaFuncSetAttribute(k_merge_cta<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)(sizeof(unsigned long long) * kCtaCap));
    if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute(k_merge_cta)");
    return GP_OK;
}

}  // namespace gp
