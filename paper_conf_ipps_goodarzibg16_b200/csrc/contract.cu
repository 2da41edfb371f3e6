// contract.cu -- A4 leftover + A5 cmap + A6 sizing + A7 merge + A8 coarse CSR assembly of
// one level in ONE persistent cooperative kernel.
//
// Paper: CM is built by four kernels (flag u<=M[u], CUB inclusive scan, subtract one,
// partner copy; P18.s16-27).  Contraction sizes each thread's output by the pair's degree
// sum (P20.s5-11), merges the two neighbour lists by quicksort + duplicate removal or a
// per-thread hash table (P20.s14-21), counts, scans again and copies the rows into the
// final arrays (P20.s22-26).
//
// B200 design:
//  C1  one decoupled look-back pass over u in [0,n): leftover self-match, leader flags,
//      exclusive scan (= the paper's inclusive scan minus one), leader list, the partner's
//      CM (written by its leader: no second pass), cvwgt, and the exclusive prefix `off`
//      of the merged-row upper bounds ub = deg(u) + deg(partner) (P20.s6-8).  Coarse rows
//      are cut into tiles of kTileArcs upper-bound entries; C1 also records each tile's
//      first row.
//  C1b (only if some ub > kTileArcs, e.g. R-MAT hubs) such rows are merged by a whole CTA
//      in global scratch.
//  C2  one pass over the tiles in order: every row of the tile is merged into the tile's
//      shared-memory slots (ub <= 16: one thread, registers + bitonic network; longer: one
//      warp, shared-memory bitonic sort), counted, the tile total gets its global prefix
//      by decoupled look-back, and the rows are written straight into the final compact
//      cadjp/cadjncy/cadjwgt (no temporary arrays, no second scan, no copy kernel).
//  Rows come out sorted by coarse id (R10) with repeated coarse neighbours summed (R8) and
//  the collapsed edge dropped (R9).
#include <cuda_runtime.h>

#include "device_util.cuh"
#include "gp_internal.cuh"

namespace gp {

constexpr int kCNT = 256;              // threads per CTA (4 co-resident CTAs per SM)
constexpr int kCItems = 8;             // vertices per thread per C1 tile
constexpr int kCTileV = kCNT * kCItems;  // 2048 vertices per C1 tile
constexpr int kTileArcs = 2048;        // C2 tile budget (upper-bound entries); rows with a
                                       // larger bound are merged by C1b
constexpr int kTileBuf = 2 * kTileArcs;  // a row starting inside the budget ends within 2x
constexpr int kNet = 16;               // one-thread merge capacity
constexpr int kWarpNet = 64;           // one-warp register merge capacity
constexpr unsigned long long kMaxKey = ~0ull;

struct ContractArgs {
    const SizeRec *in;  // device: sizes + stop flag of this level's graph
    const int32_t *adjp, *adjncy, *adjwgt, *vwgt;
    int32_t *M, *CM;
    int32_t *leaders, *off, *cnt, *tile_start, *huge, *rlen;
    int4 *seg;                  // per coarse row: {start, deg} of the leader and of the partner
    unsigned long long *gkeys;  // C1b scratch (nnz entries)
    unsigned long long *st1;    // C1 look-back status (4 words per tile)
    unsigned long long *st2;    // C2 look-back status (2 words per tile)
    uint32_t epoch;
    int32_t *cadjp, *cadjncy, *cadjwgt, *cvwgt;  // coarse graph (upper-bound sized)
    ContractCtl *ctl;
    SizeRec *out;  // device: sizes + stop decision of the coarse graph
    int32_t apply_leftover;
    int32_t threshold, stall_pct, level, max_levels;
    LevelReport *report;  // mapped host memory (may be null)
};

struct ContractSmem {
    unsigned long long buf[kTileBuf];
    int32_t scan[40];
    int32_t tile, prefix, len;
    unsigned long long prefix2;
    int32_t wlen[kCNT / 32];
    int32_t lead[kCNT], has[kCNT];
    int32_t hub_c, hub_o;
};

// ---------------------------------------------------------------------------------------
// look-back over V values per tile (V in {1,2}); words per tile: V aggregate + V inclusive;
// a word is valid when its high half equals (epoch | 2^31).
// ---------------------------------------------------------------------------------------
template <int V>
__device__ __forceinline__ void lookback(unsigned long long *st, uint32_t epoch, int tile, const int32_t (&agg)[V],
                                         int32_t (&prefix)[V]) {
    // Wide window: lane l inspects the K predecessors pred-l*K .. pred-l*K-K+1, so one step
    // covers 32*K tiles.  With hundreds of CTAs finishing a wave of tiles at once, the
    // nearest inclusive prefix is often a whole wave back; a 32-tile window would need
    // ~wave/32 dependent steps.
    constexpr int K = 8;
    const int l = threadIdx.x & 31;
    const unsigned long long tag = ((unsigned long long)(epoch | 0x80000000u)) << 32;
    unsigned long long *me = st + (size_t)tile * 2 * V;
#pragma unroll
    for (int i = 0; i < V; ++i) prefix[i] = 0;
    if (tile == 0) {
        if (l == 0)
#pragma unroll
            for (int i = 0; i < V; ++i) lb_store(me + V + i, tag | (uint32_t)agg[i]);
        return;
    }
    if (l == 0)
#pragma unroll
        for (int i = 0; i < V; ++i) lb_store(me + i, tag | (uint32_t)agg[i]);
    int pred = tile - 1;
    while (true) {
        // my K entries, nearest first; stop at the first inclusive one
        int32_t part[V];
#pragma unroll
        for (int i = 0; i < V; ++i) part[i] = 0;
        bool found = false;
        for (int k = 0; k < K && !found; ++k) {
            const int idx = pred - l * K - k;
            if (idx < 0) {
                found = true;  // before tile 0: an inclusive prefix of 0
                break;
            }
            const unsigned long long *w = st + (size_t)idx * 2 * V;
            const long long guard = spin_start();
            unsigned backoff = 0;
            while (true) {
                spin_check(guard);
                bool inc = true, ag = true;
                unsigned long long wi[V], wa[V];
#pragma unroll
                for (int i = 0; i < V; ++i) {
                    wi[i] = lb_load(w + V + i);
                    inc &= (wi[i] & 0xFFFFFFFF00000000ull) == tag;
                }
                if (inc) {
#pragma unroll
                    for (int i = 0; i < V; ++i) part[i] += (int32_t)(uint32_t)wi[i];
                    found = true;
                    break;
                }
#pragma unroll
                for (int i = 0; i < V; ++i) {
                    wa[i] = lb_load(w + i);
                    ag &= (wa[i] & 0xFFFFFFFF00000000ull) == tag;
                }
                if (ag) {
#pragma unroll
                    for (int i = 0; i < V; ++i) part[i] += (int32_t)(uint32_t)wa[i];
                    break;
                }
                if (backoff) __nanosleep(backoff);
                backoff = backoff ? min(backoff * 2, 256u) : 32u;
            }
        }
        const unsigned incl = __ballot_sync(0xffffffffu, found);
        const int first = incl ? __ffs(incl) - 1 : 32;
#pragma unroll
        for (int i = 0; i < V; ++i) prefix[i] += warp_sum(l <= first ? part[i] : 0);
        if (incl) break;
        pred -= 32 * K;
    }
    if (l == 0)
#pragma unroll
        for (int i = 0; i < V; ++i) lb_store(me + V + i, tag | (uint32_t)(prefix[i] + agg[i]));
}

// ---------------------------------------------------------------------------------------
// merge helpers
// ---------------------------------------------------------------------------------------
__device__ __forceinline__ unsigned long long ckey(int32_t cx, int32_t w) {
    return ((unsigned long long)(uint32_t)cx << 32) | (uint32_t)w;
}

__device__ __forceinline__ void cswap(unsigned long long &a, unsigned long long &b) {
    const unsigned long long lo = a < b ? a : b, hi = a < b ? b : a;
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

// Sort len keys in place (any len) with the flip bitonic network; comparators whose upper
// index is >= len are skipped (virtual +inf padding never moves).
template <typename Sync>
__device__ __forceinline__ void coop_sort(unsigned long long *keys, int len, int tid, int nthr, Sync sync) {
    int S = 1;
    while (S < len) S <<= 1;
    for (int size = 2; size <= S; size <<= 1) {
        const int half = size >> 1;
        for (int i = tid; i < S / 2; i += nthr) {
            const int blk = i / half, o = i % half;
            const int x = blk * size + o, y = blk * size + size - 1 - o;
            if (y < len) {
                const unsigned long long p = keys[x], q = keys[y];
                if (p > q) {
                    keys[x] = q;
                    keys[y] = p;
                }
            }
        }
        sync();
        for (int j = size / 4; j > 0; j >>= 1) {
            for (int i = tid; i < S / 2; i += nthr) {
                const int x = (i / j) * 2 * j + (i % j), y = x + j;
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

__device__ __forceinline__ bool is_head(const unsigned long long *keys, int i) {
    return i == 0 || (keys[i] >> 32) != (keys[i - 1] >> 32);
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

// ---------------------------------------------------------------------------------------
// C1: leftover + cmap + cvwgt + ub prefix + tile starts
// ---------------------------------------------------------------------------------------
// Tiles are assigned statically (tile = blockIdx + i*gridDim): every CTA of a cooperative
// launch is resident, and a tile only waits on lower tiles, which their CTAs reach first.
__device__ void phase_c1(const ContractArgs &a, ContractSmem &sm, int32_t n, int32_t ntiles2) {
    const int ntiles = (n + kCTileV - 1) / kCTileV;
    for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const long long base = (long long)tile * kCTileV + (long long)threadIdx.x * kCItems;
        int32_t m[kCItems];
        int32_t d[kCItems];
        int32_t cnt = 0, ubs = 0;
#pragma unroll
        for (int i = 0; i < kCItems; ++i) {
            const long long u = base + i;
            m[i] = -2;
            d[i] = 0;
            if (u < n) {
                m[i] = a.M[u];
                if (m[i] == kFree && a.apply_leftover) {
                    m[i] = (int32_t)u;  // leftover: matched to itself (P18.s12-13)
                    a.M[u] = (int32_t)u;
                }
                if (u <= m[i]) {  // leader flag (P18.s18, R7)
                    ++cnt;
                    d[i] = __ldg(a.adjp + u + 1) - __ldg(a.adjp + u);
                    if (m[i] != u) d[i] += __ldg(a.adjp + m[i] + 1) - __ldg(a.adjp + m[i]);  // P20.s6-8
                    ubs += d[i];
                }
            }
        }
        int32_t tc, tu;
        const int32_t ec = block_excl_scan<kCNT>(cnt, sm.scan, tc);
        const int32_t eu = block_excl_scan<kCNT>(ubs, sm.scan, tu);
        if (threadIdx.x < 32) {
            const int32_t agg[2] = {tc, tu};
            int32_t pre[2];
            lookback<2>(a.st1, a.epoch, tile, agg, pre);
            if (threadIdx.x == 0) {
                sm.prefix = pre[0];
                sm.prefix2 = (unsigned long long)(uint32_t)pre[1];
            }
        }
        __syncthreads();
        int32_t c = sm.prefix + ec;
        int32_t o = (int32_t)sm.prefix2 + eu;
        if (tile == 0 && threadIdx.x == 0) a.tile_start[0] = 0;
        if (tile == ntiles - 1 && threadIdx.x == 0) {
            const int32_t nc = sm.prefix + tc;
            a.ctl->n_coarse = nc;
            a.off[nc] = (int32_t)sm.prefix2 + tu;  // = nnz
            a.tile_start[ntiles2] = nc;
        }
#pragma unroll
        for (int i = 0; i < kCItems; ++i) {
            const long long u = base + i;
            if (u < n && u <= m[i]) {
                const int32_t v = m[i];
                a.CM[u] = c;                      // exclusive scan = inclusive - 1 (P18.s20-24)
                a.leaders[c] = (int32_t)u;
                int32_t vw = __ldg(a.vwgt + u);
                if (v != u) {
                    a.CM[v] = c;                  // partner copies its leader's id (P18.s26)
                    vw += __ldg(a.vwgt + v);      // w(c) = w(u) + w(v) (P12.s27)
                }
                a.cvwgt[c] = vw;
                a.off[c] = o;
                {
                    const int32_t su = __ldg(a.adjp + u);
                    const int32_t du = __ldg(a.adjp + u + 1) - su;
                    a.seg[c] = make_int4(su, du, v != u ? __ldg(a.adjp + v) : 0, d[i] - du);
                }
                // tile t starts at the first row with off >= t*kTileArcs: row c+1 for every t
                // with off[c] < t*kTileArcs <= off[c+1]
                for (int32_t t = o / kTileArcs + 1; t <= (o + d[i]) / kTileArcs && t < ntiles2; ++t)
                    a.tile_start[t] = c + 1;
                if (d[i] > kTileArcs) a.huge[atomicAdd(&a.ctl->n_huge, 1)] = c;
                ++c;
                o += d[i];
            }
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------------------
// gather the coarse keys of row c (collapsed edge dropped) into dst via claim()
// ---------------------------------------------------------------------------------------
template <typename Claim>
__device__ __forceinline__ void gather_row(const ContractArgs &a, int32_t c, int tid, int nthr,
                                           unsigned long long *dst, Claim claim) {
    const int4 sg = __ldcg(a.seg + c);
    for (int side = 0; side < 2; ++side) {
        const int32_t s = side ? sg.z : sg.x, e = s + (side ? sg.w : sg.y);
        for (int32_t j = s + tid; j < e; j += nthr) {
            const int32_t cx = __ldcg(a.CM + __ldg(a.adjncy + j));
            if (cx != c) dst[claim()] = ckey(cx, __ldg(a.adjwgt + j));  // drop the collapsed edge (R9)
        }
    }
}

// C1b: rows whose upper bound exceeds a tile: one CTA per row in global scratch
__device__ void phase_c1b(const ContractArgs &a, ContractSmem &sm, int32_t nh) {
    for (int i = blockIdx.x; i < nh; i += gridDim.x) {
        const int32_t c = a.huge[i];
        unsigned long long *keys = a.gkeys + __ldcg(a.off + c);
        if (threadIdx.x == 0) sm.len = 0;
        __syncthreads();
        gather_row(a, c, threadIdx.x, kCNT, keys, [&]() { return atomicAdd(&sm.len, 1); });
        __syncthreads();
        const int len = sm.len;
        coop_sort(keys, len, threadIdx.x, kCNT, []() { __syncthreads(); });
        const int32_t cnt = coop_runsum(
            keys, len, threadIdx.x, kCNT, sm.lead, sm.has,
            [&](int32_t v, int32_t &tot) { return block_excl_scan<kCNT>(v, sm.scan, tot); },
            []() { __syncthreads(); });
        if (threadIdx.x == 0) {
            a.cnt[c] = cnt;
            a.rlen[c] = len;
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------------------
// C2: tiled merge + assembly
// ---------------------------------------------------------------------------------------
__device__ void phase_c2(const ContractArgs &a, ContractSmem &sm, int32_t nc, int32_t nnz, int32_t ntiles2) {
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    for (int tile = blockIdx.x; tile < ntiles2; tile += gridDim.x) {
        const int32_t r0 = __ldcg(a.tile_start + tile), r1 = __ldcg(a.tile_start + tile + 1);
        const int32_t tbase = tile * kTileArcs;
        const bool single = (r1 - r0) <= kCNT;  // one row per thread: keep pass-1 state in registers
        int32_t k_cnt = 0, k_slot = 0, k_ub = 0, k_ex = 0;
        // ---- pass 1: merge every row of the tile into its shared-memory slot, count ----
        int32_t total = 0;
        for (int32_t g0 = r0; g0 < r1; g0 += kCNT) {
            const int32_t c = g0 + threadIdx.x;
            int32_t ub = 0, slot = 0, cntc = 0;
            bool warp_row = false;
            if (c < r1) {
                const int32_t o0 = __ldcg(a.off + c);
                slot = o0 - tbase;
                ub = __ldcg(a.off + c + 1) - o0;
                if (ub > kTileArcs) {
                    cntc = __ldcg(a.cnt + c);  // merged by C1b
                } else if (ub > kNet) {
                    warp_row = true;
                } else if (ub > 0) {
                    const int4 sg = __ldcg(a.seg + c);
                    const int32_t su = sg.x, du = sg.y, sv = sg.z;
                    unsigned long long k[kNet];
#pragma unroll
                    for (int i = 0; i < kNet; ++i) {
                        k[i] = kMaxKey;
                        if (i < ub) {
                            const int32_t j = (i < du) ? su + i : sv + (i - du);
                            const int32_t cx = __ldcg(a.CM + __ldg(a.adjncy + j));
                            if (cx != c) k[i] = ckey(cx, __ldg(a.adjwgt + j));
                        }
                    }
                    reg_sort<kNet>(k);
                    int32_t prev = -1, acc = 0;
#pragma unroll
                    for (int i = 0; i < kNet; ++i) {
                        if (k[i] != kMaxKey) {
                            const int32_t cx = (int32_t)(k[i] >> 32), w = (int32_t)(uint32_t)k[i];
                            if (cx == prev) {
                                acc += w;  // repeated coarse neighbour: weights summed (R8, P12.s28)
                            } else {
                                if (prev >= 0) sm.buf[slot + cntc++] = ckey(prev, acc);
                                prev = cx;
                                acc = w;
                            }
                        }
                    }
                    if (prev >= 0) sm.buf[slot + cntc++] = ckey(prev, acc);
                }
            }
            // rows of 17..64 entries: one warp each, registers + shuffles
            unsigned m64 = __ballot_sync(0xffffffffu, warp_row && ub <= kWarpNet);
            while (m64) {
                const int src = __ffs(m64) - 1;
                m64 &= m64 - 1;
                const int32_t cw = __shfl_sync(0xffffffffu, c, src);
                const int32_t sl = __shfl_sync(0xffffffffu, slot, src);
                const int4 sg = __ldcg(a.seg + cw);
                unsigned long long v[2];
#pragma unroll
                for (int r = 0; r < 2; ++r) {
                    const int32_t e = r * 32 + lane;
                    v[r] = kMaxKey;
                    if (e < sg.y + sg.w) {
                        const int32_t j = (e < sg.y) ? sg.x + e : sg.z + (e - sg.y);
                        const int32_t cx = __ldcg(a.CM + __ldg(a.adjncy + j));
                        if (cx != cw) v[r] = ckey(cx, __ldg(a.adjwgt + j));  // collapsed edge dropped (R9)
                    }
                }
                warp_sort64(v);
                const int32_t cc = warp_runmerge64(v, sm.buf + sl);  // compacted in the slot
                if (lane == src) cntc = cc;
            }
            // rows of 65..kTileArcs entries: one warp each, shared-memory sort in their slot
            unsigned mm = __ballot_sync(0xffffffffu, warp_row && ub > kWarpNet);
            while (mm) {
                const int src = __ffs(mm) - 1;
                mm &= mm - 1;
                const int32_t cw = __shfl_sync(0xffffffffu, c, src);
                const int32_t sl = __shfl_sync(0xffffffffu, slot, src);
                unsigned long long *keys = sm.buf + sl;
                if (lane == 0) sm.wlen[wib] = 0;
                __syncwarp();
                gather_row(a, cw, lane, 32, keys, [&]() { return atomicAdd(&sm.wlen[wib], 1); });
                __syncwarp();
                const int len = sm.wlen[wib];
                coop_sort(keys, len, lane, 32, []() { __syncwarp(); });
                const int32_t cc = coop_runsum(
                    keys, len, lane, 32, sm.lead + wib * 32, sm.has + wib * 32,
                    [&](int32_t v, int32_t &tot) {
                        const int32_t inc = warp_incl_scan(v);
                        tot = __shfl_sync(0xffffffffu, inc, 31);
                        return inc - v;
                    },
                    []() { __syncwarp(); });
                if (lane == src) {
                    cntc = cc;
                    a.rlen[cw] = len;
                }
            }
            int32_t part;
            const int32_t ex = block_excl_scan<kCNT>(cntc, sm.scan, part);
            if (single) {
                k_cnt = cntc;
                k_slot = slot;
                k_ub = ub;
                k_ex = ex;
            } else if (c < r1) {
                a.cnt[c] = cntc;
            }
            total += part;
        }
        // ---- tile prefix by decoupled look-back ----
        if (threadIdx.x < 32) {
            const int32_t agg[1] = {total};
            int32_t pre[1];
            lookback<1>(a.st2, a.epoch, tile, agg, pre);
            if (threadIdx.x == 0) sm.prefix = pre[0];
        }
        __syncthreads();
        int32_t pos0 = sm.prefix;
        if (tile == ntiles2 - 1 && threadIdx.x == 0) {
            a.cadjp[nc] = pos0 + total;
            a.ctl->cnnz = pos0 + total;
        }
        // ---- pass 2: cadjp and the rows, straight into the final arrays ----
        for (int32_t g0 = r0; g0 < r1; g0 += kCNT) {
            const int32_t c = g0 + threadIdx.x;
            int32_t cntc = 0, ub = 0, slot = 0, o = 0, part = 0;
            if (single) {
                cntc = k_cnt;
                slot = k_slot;
                ub = k_ub;
                o = pos0 + k_ex;
                part = total;
            } else {
                if (c < r1) {
                    cntc = __ldcg(a.cnt + c);
                    slot = __ldcg(a.off + c) - tbase;
                    ub = __ldcg(a.off + c + 1) - __ldcg(a.off + c);
                }
                const int32_t ex = block_excl_scan<kCNT>(cntc, sm.scan, part);
                o = pos0 + ex;
            }
            if (c < r1) {
                a.cadjp[c] = o;
                if (ub <= kWarpNet) {
                    for (int32_t j = 0; j < cntc; ++j) {
                        const unsigned long long k = sm.buf[slot + j];
                        a.cadjncy[o + j] = (int32_t)(k >> 32);
                        a.cadjwgt[o + j] = (int32_t)(uint32_t)k;
                    }
                }
            }
            // rows sorted in shared memory by a warp: the warp writes the run heads
            unsigned mw = __ballot_sync(0xffffffffu, c < r1 && ub > kWarpNet && ub <= kTileArcs);
            while (mw) {
                const int src = __ffs(mw) - 1;
                mw &= mw - 1;
                const int32_t cw = __shfl_sync(0xffffffffu, c, src);
                const int32_t sl = __shfl_sync(0xffffffffu, slot, src);
                const int32_t ow = __shfl_sync(0xffffffffu, o, src);
                const unsigned long long *keys = sm.buf + sl;
                const int32_t len = __ldcg(a.rlen + cw);
                int32_t run = 0;
                for (int32_t b0 = 0; b0 < len; b0 += 32) {
                    const int32_t i = b0 + lane;
                    const bool h = i < len && is_head(keys, i);
                    const unsigned hm = __ballot_sync(0xffffffffu, h);
                    if (h) {
                        const int32_t pos = ow + run + __popc(hm & lanemask_lt());
                        a.cadjncy[pos] = (int32_t)(keys[i] >> 32);
                        a.cadjwgt[pos] = (int32_t)(uint32_t)keys[i];
                    }
                    run += __popc(hm);
                }
            }
            // a row merged by C1b (at most one per tile, its last row): copied by the CTA
            const int hub_here = __syncthreads_or(c < r1 && ub > kTileArcs);
            if (hub_here) {
                if (c < r1 && ub > kTileArcs) {
                    sm.hub_c = c;
                    sm.hub_o = o;
                }
                __syncthreads();
                const int32_t hc = sm.hub_c, oc = sm.hub_o;
                const unsigned long long *src = a.gkeys + __ldcg(a.off + hc);
                const int32_t len = __ldcg(a.rlen + hc);
                int32_t run = 0;
                for (int32_t b0 = 0; b0 < len; b0 += kCNT) {
                    const int32_t i = b0 + threadIdx.x;
                    const bool h = i < len && is_head(src, i);
                    int32_t tot;
                    const int32_t ex = block_excl_scan<kCNT>(h ? 1 : 0, sm.scan, tot);
                    if (h) {
                        a.cadjncy[oc + run + ex] = (int32_t)(src[i] >> 32);
                        a.cadjwgt[oc + run + ex] = (int32_t)(uint32_t)src[i];
                    }
                    run += tot;
                }
            }
            pos0 += part;
        }
        __syncthreads();  // the slots are reused by the next tile
    }
}

__global__ void __launch_bounds__(kCNT, 4) k_contract_level(const __grid_constant__ ContractArgs a) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    ContractSmem &sm = *reinterpret_cast<ContractSmem *>(smem_raw);
    ContractCtl *ctl = a.ctl;
    const volatile SizeRec *in = a.in;
    if (in->stop) {  // an earlier level ended the coarsening: propagate and leave
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            a.out->n = in->n;
            a.out->nnz = in->nnz;
            a.out->stop = 1;
            a.out->stop_reason = in->stop_reason;
            if (a.report) {
                a.report->skipped = 1;
                __threadfence_system();
                *((volatile int32_t *)&a.report->ready) = 1;
            }
        }
        return;
    }
    const int32_t n = in->n;
    const int32_t nnz = in->nnz;
    const int32_t ntiles2 = nnz > 0 ? (nnz + kTileArcs - 1) / kTileArcs : 0;
    trace_mark(ctl->trace, 0);
    if (n > 0) {
        phase_c1(a, sm, n, ntiles2);
        trace_mark(ctl->trace, 1);
        grid_barrier(ctl->bar);
    }
    trace_mark(ctl->trace, 2);
    const int32_t nc = *(volatile int32_t *)&ctl->n_coarse;
    const int32_t nh = *(volatile int32_t *)&ctl->n_huge;
    if (nh > 0) {
        phase_c1b(a, sm, nh);
        grid_barrier(ctl->bar);
    }
    trace_mark(ctl->trace, 3);
    if (ntiles2 > 0) phase_c2(a, sm, nc, nnz, ntiles2);
    trace_mark(ctl->trace, 4);
    if (ntiles2 == 0) {  // no arcs: every coarse row is empty
        for (long long c = (long long)blockIdx.x * kCNT + threadIdx.x; c <= nc; c += (long long)gridDim.x * kCNT)
            a.cadjp[c] = 0;
        if (blockIdx.x == 0 && threadIdx.x == 0) ctl->cnnz = 0;
    }
    // the last CTA to finish publishes the coarse sizes and the stop decision
    __shared__ bool last;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) last = atomicAdd(&ctl->blocks_done, 1u) == gridDim.x - 1;
    __syncthreads();
    if (last && threadIdx.x == 0) {
        __threadfence();
        const int32_t ncv = *((volatile int32_t *)&ctl->n_coarse);
        const int32_t cnnz = *((volatile int32_t *)&ctl->cnnz);
        // stop rule (P12.s30, P20.s30; R12, R13): stall first, then threshold, then levels
        int32_t reason = GP_STOP_NONE;
        if (100LL * ncv > (long long)a.stall_pct * n) reason = GP_STOP_STALL;
        else if (ncv <= a.threshold) reason = GP_STOP_THRESHOLD;
        else if (a.level + 1 >= a.max_levels) reason = GP_STOP_MAX_LEVELS;
        a.out->n = ncv;
        a.out->nnz = cnnz;
        a.out->stop = reason != GP_STOP_NONE;
        a.out->stop_reason = reason;
        __threadfence();
        if (a.report) {
            a.report->n_coarse = ncv;
            a.report->cnnz = cnnz;
            a.report->stop = reason != GP_STOP_NONE;
            a.report->stop_reason = reason;
            a.report->skipped = 0;
            __threadfence_system();
            *((volatile int32_t *)&a.report->ready) = 1;
        }
    }
}

// ---------------------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------------------
int contract_grid(Ctx *ctx) {
    static int per_sm = -1;
    if (per_sm < 0) {
        int b = 0;
        cudaFuncSetAttribute(k_contract_level, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)sizeof(ContractSmem));
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_contract_level, kCNT, sizeof(ContractSmem));
        per_sm = b > 0 ? (b > 4 ? 4 : b) : 1;
    }
    return ctx->num_sms * per_sm;
}

size_t contract_status_words(int32_t n, int32_t nnz) {
    const size_t t1 = (size_t)(n + kCTileV - 1) / kCTileV + 1;
    const size_t t2 = (size_t)(nnz + kTileArcs - 1) / kTileArcs + 1;
    return 4 * t1 + 2 * t2;
}

size_t contract_tiles(int32_t nnz) { return (size_t)(nnz + kTileArcs - 1) / kTileArcs + 2; }

gp_status enqueue_contract(Ctx *ctx, const LevelBufs &lb, int32_t *M, int32_t *CM, Graph *cg, ContractCtl *ctl,
                           SizeRec *out_sizes, LevelReport *report, const ContractParams &prm) {
    ContractArgs a;
    a.in = lb.in;
    a.adjp = lb.adjp;
    a.adjncy = lb.adjncy;
    a.adjwgt = lb.adjwgt;
    a.vwgt = lb.vwgt;
    a.M = M;
    a.CM = CM;
    a.leaders = lb.leaders;
    a.off = lb.off;
    a.cnt = lb.cnt;
    a.tile_start = lb.tile_start;
    a.huge = lb.huge;
    a.rlen = lb.rlen;
    a.seg = lb.seg;
    a.gkeys = lb.gkeys;
    a.st1 = ctx->status;
    a.st2 = ctx->status + 4 * ((size_t)(prm.n_bound + kCTileV - 1) / kCTileV + 1);
    a.epoch = ctx->epoch;
    ctx->epoch = (ctx->epoch + 1) & 0x7FFFFFFFu;
    if (ctx->epoch == 0) ctx->epoch = 1;
    a.cadjp = cg->adjp;
    a.cadjncy = cg->adjncy;
    a.cadjwgt = cg->adjwgt;
    a.cvwgt = cg->vwgt;
    a.ctl = ctl;
    a.out = out_sizes;
    a.apply_leftover = prm.leftover ? 1 : 0;
    a.threshold = prm.threshold;
    a.stall_pct = prm.stall_pct;
    a.level = prm.level;
    a.max_levels = prm.max_levels;
    a.report = report;
    gp_status st = ensure_status(ctx, contract_status_words(prm.n_bound, prm.nnz_bound));
    if (st != GP_OK) return st;
    a.st1 = ctx->status;
    a.st2 = ctx->status + 4 * ((size_t)(prm.n_bound + kCTileV - 1) / kCTileV + 1);
    void *args[] = {&a};
    LaunchScope ls(ctx, GP_K_CONTRACT);
    GP_CUDA(cudaLaunchCooperativeKernel((const void *)k_contract_level, dim3(contract_grid(ctx)), dim3(kCNT), args,
                                        sizeof(ContractSmem), ctx->stream));
    ++ctx->launches;
    return GP_OK;
}

}  // namespace gp
