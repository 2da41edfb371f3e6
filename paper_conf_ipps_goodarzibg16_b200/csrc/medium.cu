// medium.cu -- the coarse-level tail for graphs too big for one SM's shared memory but small
// enough that a full grid mostly waits (PAPER.md P16.s6-7, P20.s28-33):
// every remaining level in ONE launch of one thread-block CLUSTER (16 CTAs on 16 SMs when the
// device allows non-portable cluster sizes, else 8), graph and state in global memory (L2-resident
// at these sizes), cluster barriers (~0.2 us) instead of grid barriers, no kernel boundary and no
// host round trip between levels.
//
// The level algorithm is small.cu's, spread over the cluster's threads:
//   * event-driven synchronous rounds: only the vertices whose target was matched rescan, only
//     the changed vertices commit; live count, rounds and maximality are the rule's (§2.1);
//   * cmap by a cluster-wide scan (block scans + the CTA totals through distributed shared
//     memory);
//   * contraction: rows of <= 16 merged entries by one thread each (the register network of
//     merge_util.cuh, counted in pass 1, re-merged and written in pass 2); wider rows by one CTA
//     each (flip-bitonic sort of (coarse id, weight) keys in shared memory, global memory beyond
//     4096 keys, run sums), staged at their upper-bound offset and copied in pass 2;
//   * coarse CSR offsets by a cluster-wide scan of the row counts; stop rule as everywhere.
// Results are bit-identical to the level kernels and to the oracle (tests/test_gpu_tail.py).
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <stdlib.h>

#include "device_util.cuh"
#include "gp_internal.cuh"
#include "merge_util.cuh"

namespace cg = cooperative_groups;

namespace gp {

constexpr int kMT = 512;        // threads per CTA (128 registers: no spills)
constexpr int kMaxCS = 16;      // cluster size (non-portable); 8 portable
constexpr int kWideSmem = 4096; // keys of a wide row sorted in shared memory

struct MediumLevelOut {  // one arena slot (same layout as small.cu's SmallLevelOut)
    int32_t *M, *CM, *cadjp, *cadjncy, *cadjwgt, *cvwgt;
};

struct MediumArgs {
    const SizeRec *in;
    const int32_t *adjp, *adjncy, *adjwgt, *vwgt;  // the first level's input graph
    MediumLevelOut *slots;
    int32_t nslots, level0, cap_n, cap_nnz;
    LevelDev *levdev;
    LevelReport *reports;
    int32_t threshold, stall_pct, max_levels, max_rounds;
    uint32_t tie_seed;
    // global scratch (sized by cap_n / cap_nnz)
    int32_t *M, *P, *R0, *R1, *cnt, *woff, *wide;
    uint8_t *stamp;
    unsigned long long *stage;
    int32_t *ctr;  // [0] next list length, [1] pairs, [2] dead, [3] wide rows, [4] wide claim, [8..] scan totals
};

enum { kCtrRn = 0, kCtrPairs = 1, kCtrDead = 2, kCtrWide = 3, kCtrClaim = 4 };  // (rounds: slots 8 and 16)

struct MediumShared {
    int32_t scan[40];
    int32_t tot[kMaxCS];  // CTA totals of a cluster scan (read through DSMEM from rank 0)
    int32_t bcast[4];
    unsigned long long keys[kWideSmem];
};

__device__ __forceinline__ int32_t ld32(const int32_t *p) { return __ldcg(p); }

// cluster-wide exclusive scan of one value per thread over (rank, thread) order
__device__ int32_t cluster_excl_scan(cg::cluster_group &cl, MediumShared &sm, int32_t v, int32_t &total) {
    int32_t btot;
    const int32_t ex = block_excl_scan<kMT>(v, sm.scan, btot);
    MediumShared *s0 = cl.map_shared_rank(&sm, 0);
    if (threadIdx.x == 0) s0->tot[cl.block_rank()] = btot;
    cl.sync();
    int32_t pre = 0, all = 0;
    const int r = (int)cl.block_rank(), cs = (int)cl.num_blocks();
    for (int q = 0; q < cs; ++q) {
        const int32_t x = s0->tot[q];
        if (q < r) pre += x;
        all += x;
    }
    cl.sync();  // the totals are rewritten by the next scan
    total = all;
    return pre + ex;
}

// warp-aggregated append to list[ctr++]
__device__ __forceinline__ void wappend(int32_t *list, int32_t *ctr, bool pred, int32_t value) {
    const unsigned m = __ballot_sync(__activemask(), pred);
    if (!pred) return;
    const int leader = __ffs(m) - 1;
    const int lane = threadIdx.x & 31;
    int32_t base = 0;
    if (lane == leader) base = atomicAdd(ctr, __popc(m));
    base = __shfl_sync(m, base, leader);
    list[base + __popc(m & lanemask_lt())] = value;
}

template <bool H>
__device__ __forceinline__ int32_t m_rescan(const MediumArgs &a, const int32_t *adjp, const int32_t *adjncy,
                                            const int32_t *adjwgt, int32_t u, unsigned long long &arcs) {
    unsigned long long best = 0;
    const int32_t s0 = ld32(adjp + u), e0 = ld32(adjp + u + 1);
    int32_t j = s0;
    for (; j + 4 <= e0; j += 4) {
        int32_t x[4], w[4], f[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            x[q] = ld32(adjncy + j + q);
            w[q] = ld32(adjwgt + j + q);
        }
#pragma unroll
        for (int q = 0; q < 4; ++q) f[q] = ld32(a.M + x[q]);
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if (f[q] == kFree) {
                const unsigned long long kk = pack_key<H>(a.tie_seed, w[q], x[q]);
                best = kk > best ? kk : best;
            }
    }
    for (; j < e0; ++j) {
        const int32_t x = ld32(adjncy + j);
        if (ld32(a.M + x) == kFree) {
            const unsigned long long kk = pack_key<H>(a.tie_seed, ld32(adjwgt + j), x);
            best = kk > best ? kk : best;
        }
    }
    arcs += (unsigned long long)(e0 - s0);
    const int32_t b = key_vertex<H>(a.tie_seed, best);
    return b == kNone ? -2 : b;
}

// flip-bitonic ascending sort of len 64-bit keys by one CTA (shared or global memory)
__device__ void m_cta_sort(unsigned long long *keys, int32_t len) {
    int32_t S = 1, lg = 0;
    while (S < len) {
        S <<= 1;
        ++lg;
    }
    for (int32_t ls = 1; ls <= lg; ++ls) {
        const int32_t lh = ls - 1;
        for (int32_t i = threadIdx.x; i < S / 2; i += kMT) {
            const int32_t blk = i >> lh, o = i & ((1 << lh) - 1);
            const int32_t x = (blk << ls) + o, y = (blk << ls) + (1 << ls) - 1 - o;
            if (y < len && keys[x] > keys[y]) {
                const unsigned long long t = keys[x];
                keys[x] = keys[y];
                keys[y] = t;
            }
        }
        __syncthreads();
        for (int32_t lj = ls - 2; lj >= 0; --lj) {
            const int32_t j = 1 << lj;
            for (int32_t i = threadIdx.x; i < S / 2; i += kMT) {
                const int32_t x = ((i >> lj) << (lj + 1)) + (i & (j - 1)), y = x + j;
                if (y < len && keys[x] > keys[y]) {
                    const unsigned long long t = keys[x];
                    keys[x] = keys[y];
                    keys[y] = t;
                }
            }
            __syncthreads();
        }
    }
}

// merge of coarse row cc (<= 16 entries) in registers; writes entries when `out` and returns
// the count
__device__ __forceinline__ int32_t m_row16(const int32_t *adjp, const int32_t *adjncy, const int32_t *adjwgt,
                                           const int32_t *CM, const int32_t *M, const int32_t *lead, int32_t cc,
                                           int32_t *oadj, int32_t *owgt) {
    const uint32_t kDrop = 0xFFFFFFFFu;
    const int32_t u = ld32(lead + cc), v = ld32(M + u);
    const int32_t su = ld32(adjp + u), du = ld32(adjp + u + 1) - su;
    const int32_t sv = v != u ? ld32(adjp + v) : 0, dv = v != u ? ld32(adjp + v + 1) - sv : 0;
    uint32_t kc[16];
    int32_t kw[16];
#pragma unroll
    for (int q = 0; q < 16; ++q) {
        kc[q] = kDrop;
        kw[q] = 0;
        if (q < du + dv) {
            const int32_t jj = q < du ? su + q : sv + (q - du);
            const uint32_t cx = (uint32_t)ld32(CM + ld32(adjncy + jj));
            if (cx != (uint32_t)cc) {  // collapsed edge dropped (R9)
                kc[q] = cx;
                kw[q] = ld32(adjwgt + jj);
            }
        }
    }
    cx_sort16(kc, kw);
    uint32_t prev = kDrop;
    int32_t acc = 0, n = 0;
#pragma unroll
    for (int q = 0; q < 16; ++q) {
        if (kc[q] == prev) {
            acc += kw[q];  // repeated coarse neighbour: weights summed (R8, P12.s28)
        } else {
            if (prev != kDrop) {
                if (oadj) {
                    oadj[n] = (int32_t)prev;
                    owgt[n] = acc;
                }
                ++n;
            }
            prev = kc[q];
            acc = kw[q];
        }
    }
    if (prev != kDrop) {
        if (oadj) {
            oadj[n] = (int32_t)prev;
            owgt[n] = acc;
        }
        ++n;
    }
    return n;
}

template <bool H>
__global__ void __launch_bounds__(kMT, 1) k_medium(const __grid_constant__ MediumArgs a) {
    extern __shared__ __align__(16) unsigned char msmem[];
    MediumShared &sm = *reinterpret_cast<MediumShared *>(msmem);
    cg::cluster_group cl = cg::this_cluster();
    const int rank = (int)cl.block_rank(), CS = (int)cl.num_blocks();
    const int t = threadIdx.x;
    const long long gt = (long long)rank * kMT + t, GT = (long long)CS * kMT;
    int32_t *M = a.M, *P = a.P, *CM = nullptr, *ctr = a.ctr;
    uint8_t *stamp = a.stamp;
    int32_t *Rl[2] = {a.R0, a.R1};

    const volatile SizeRec *in = a.in;
    int32_t n = in->n, nnz = in->nnz;
    int level = 0;
    bool stopped = in->stop != 0;
    int32_t prev_reason = in->stop_reason;
    const int32_t *gadjp = a.adjp, *gadjncy = a.adjncy, *gadjwgt = a.adjwgt, *gvwgt = a.vwgt;
    while (!stopped && level < a.nslots) {
        const int gl = a.level0 + level;
        const MediumLevelOut o = a.slots[level];
        CM = o.CM;  // written in place (the level's output)
        unsigned long long *tr = a.levdev[gl].match.trace;
        if (rank == 0) trace_mark(tr, 0);
        for (long long u = gt; u < n; u += GT) {
            M[u] = kFree;
            stamp[u] = 1;
        }
        cl.sync();
        // ---- matching rounds (event driven; small.cu) ----
        unsigned long long arcs = 0, rows = 0, visits = 0;
        int32_t rounds = 0, maximal = 0;
        int32_t mylive = 0;
        for (long long u = gt; u < n; u += GT) {
            const int32_t b = m_rescan<H>(a, gadjp, gadjncy, gadjwgt, (int32_t)u, arcs);
            P[u] = b;
            mylive += b >= 0;
        }
        int32_t live;
        cluster_excl_scan(cl, sm, mylive, live);  // (total; the cluster syncs inside)
        int32_t rn = n, cur = 0;
        for (int k = 1;; ++k) {
            if (live == 0) {
                maximal = 1;
                break;
            }
            if (a.max_rounds > 0 && rounds >= a.max_rounds) break;
            // counters by round parity (slot k & 1 reset in round k - 1 after its first barrier,
            // when every read of round k - 2's values is done)
            int32_t *cs = ctr + 8 * (k & 1);
            if (k == 1 && gt == 0) ctr[8 + kCtrRn] = ctr[8 + kCtrPairs] = ctr[8 + kCtrDead] = 0;
            cl.sync();
            if (gt == 0) {
                int32_t *cz = ctr + 8 * ((k + 1) & 1);
                cz[kCtrRn] = cz[kCtrPairs] = cz[kCtrDead] = 0;
            }
            int32_t *Rn = Rl[cur ^ 1];
            for (long long i = gt; i < rn; i += GT) {
                const int32_t x = k == 1 ? (int32_t)i : ld32(Rl[cur] + i);
                if (x < 0) continue;  // matched in the previous round (marked by the rescan pass)
                const int32_t d = ld32(P + x);
                if (d < 0) continue;
                ++visits;
                if (ld32(P + d) != x) continue;
                if (*(volatile uint8_t *)(stamp + d) && d < x) continue;  // both ends changed: the lower id handles it
                M[x] = d;
                M[d] = x;
                atomicAdd(&cs[kCtrPairs], 1);
#pragma unroll 1
                for (int e = 0; e < 2; ++e) {
                    const int32_t y0 = e ? d : x, other = e ? x : d;
                    const int32_t j1 = ld32(gadjp + y0 + 1);
                    for (int32_t j = ld32(gadjp + y0); j < j1; ++j) {
                        const int32_t y = ld32(gadjncy + j);
                        if (y != other && ld32(P + y) == y0) Rn[atomicAdd(&cs[kCtrRn], 1)] = y;
                    }
                }
            }
            cl.sync();
            for (long long i = gt; i < rn; i += GT) {
                const int32_t x = k == 1 ? (int32_t)i : ld32(Rl[cur] + i);
                if (x >= 0) stamp[x] = 0;
            }
            const int32_t pairs = ld32(cs + kCtrPairs), rnn = ld32(cs + kCtrRn);
            if (pairs > 0) ++rounds;
            live -= 2 * pairs;
            cl.sync();
            int32_t dead = 0;
            for (long long i = gt; i < rnn; i += GT) {
                const int32_t y = ld32(Rn + i);
                if (ld32(M + y) != kFree) {  // matched this round: out of the next round's list
                    Rn[i] = -1;
                    continue;
                }
                stamp[y] = 1;
                ++rows;
                const int32_t b = m_rescan<H>(a, gadjp, gadjncy, gadjwgt, y, arcs);
                P[y] = b;
                dead += b < 0;
            }
            if (dead) atomicAdd(&cs[kCtrDead], dead);
            cl.sync();
            live -= ld32(cs + kCtrDead);
            rn = rnn;
            cur ^= 1;
            if (k > n + 2) __trap();  // each round with proposals matches >= 1 pair
        }
        if (rank == 0) trace_mark(tr, 1);
        // ---- leftover + cmap (cluster scan over contiguous vertex chunks) ----
        const long long per = ((long long)n + GT - 1) / GT;
        const long long lo = min((long long)n, gt * per), hi = min((long long)n, lo + per);
        int32_t cntl = 0;
        for (long long u = lo; u < hi; ++u) {
            int32_t m = ld32(M + u);
            if (m == kFree) {
                m = (int32_t)u;
                M[u] = m;
            }
            if (u <= m) ++cntl;
        }
        int32_t nc;
        int32_t c = cluster_excl_scan(cl, sm, cntl, nc);
        int32_t *lead_of = P;  // free from here on
        for (long long u = lo; u < hi; ++u)
            if (u <= ld32(M + u)) {
                CM[u] = c;
                lead_of[c] = (int32_t)u;
                ++c;
            }
        cl.sync();
        for (long long u = gt; u < n; u += GT) {
            const int32_t m = ld32(M + u);
            if (u > m) CM[u] = ld32(CM + m);
            o.M[u] = m;
        }
        cl.sync();
        // ---- contraction: pass 1 counts (threads: rows <= 16; CTAs: wider rows) ----
        const long long pc = ((long long)nc + GT - 1) / GT;
        const long long clo = min((long long)nc, gt * pc), chi = min((long long)nc, clo + pc);
        if (gt == 0) {
            ctr[kCtrWide] = 0;
            ctr[kCtrClaim] = 0;
        }
        int32_t ubsum = 0;
        for (long long cc = clo; cc < chi; ++cc) {
            const int32_t u = ld32(lead_of + cc), v = ld32(M + u);
            const int32_t ub = (ld32(gadjp + u + 1) - ld32(gadjp + u)) + (v != u ? ld32(gadjp + v + 1) - ld32(gadjp + v) : 0);
            ubsum += ub;
            o.cvwgt[cc] = ld32(gvwgt + u) + (v != u ? ld32(gvwgt + v) : 0);  // P12.s27
        }
        int32_t ubtot;
        int32_t uoff = cluster_excl_scan(cl, sm, ubsum, ubtot);  // (also orders the counter reset)
        for (long long cc = clo; cc < chi; ++cc) {
            const int32_t u = ld32(lead_of + cc), v = ld32(M + u);
            const int32_t ub = (ld32(gadjp + u + 1) - ld32(gadjp + u)) + (v != u ? ld32(gadjp + v + 1) - ld32(gadjp + v) : 0);
            a.woff[cc] = uoff;
            uoff += ub;
            if (ub <= 16) {
                a.cnt[cc] = m_row16(gadjp, gadjncy, gadjwgt, CM, M, lead_of, (int32_t)cc, nullptr, nullptr);
            } else {
                a.wide[atomicAdd(&ctr[kCtrWide], 1)] = (int32_t)cc;
            }
        }
        cl.sync();
        // wide rows: one CTA each (claimed dynamically), merged into stage at woff
        {
            const int32_t nw = ld32(ctr + kCtrWide);
            for (;;) {
                if (t == 0) sm.bcast[0] = atomicAdd(&ctr[kCtrClaim], 1);
                __syncthreads();
                const int32_t wi = sm.bcast[0];
                __syncthreads();
                if (wi >= nw) break;
                const int32_t cc = ld32(a.wide + wi);
                const int32_t u = ld32(lead_of + cc), v = ld32(M + u);
                const int32_t su = ld32(gadjp + u), du = ld32(gadjp + u + 1) - su;
                const int32_t sv = v != u ? ld32(gadjp + v) : 0, dv = v != u ? ld32(gadjp + v + 1) - sv : 0;
                const int32_t ub = du + dv, o0 = ld32(a.woff + cc);
                // keys: shared memory, or the second half of the staging area for very long rows;
                // the merged row goes to the first half at its upper-bound offset
                unsigned long long *keys = ub <= kWideSmem ? sm.keys : a.stage + a.cap_nnz + o0;
                for (int32_t q = t; q < ub; q += kMT) {
                    const int32_t jj = q < du ? su + q : sv + (q - du);
                    const uint32_t cx = (uint32_t)ld32(CM + ld32(gadjncy + jj));
                    // the collapsed edge becomes the maximal key: it sorts last and is cut off
                    keys[q] = cx == (uint32_t)cc ? ~0ull
                                                 : (((unsigned long long)cx << 32) | (uint32_t)ld32(gadjwgt + jj));
                }
                __syncthreads();
                m_cta_sort(keys, ub);
                // heads (valid, first of their coarse id), block-scanned into compact positions
                int32_t nh = 0;
                const int32_t pe = (ub + kMT - 1) / kMT, elo = min(ub, t * pe), ehi = min(ub, elo + pe);
                for (int32_t i = elo; i < ehi; ++i)
                    if (keys[i] != ~0ull && (i == 0 || (keys[i] >> 32) != (keys[i - 1] >> 32))) ++nh;
                int32_t tot;
                int32_t pos = block_excl_scan<kMT>(nh, sm.scan, tot);
                for (int32_t i = elo; i < ehi; ++i) {
                    const unsigned long long kk = keys[i];
                    if (kk == ~0ull || (i > 0 && (kk >> 32) == (keys[i - 1] >> 32))) continue;
                    int32_t s = (int32_t)(uint32_t)kk;
                    for (int32_t q = i + 1; q < ub && (keys[q] >> 32) == (kk >> 32) && keys[q] != ~0ull; ++q)
                        s += (int32_t)(uint32_t)keys[q];  // fits int32 (R14)
                    a.stage[o0 + pos++] = (kk & 0xFFFFFFFF00000000ull) | (uint32_t)s;
                }
                if (t == 0) a.cnt[cc] = tot;
                __syncthreads();  // the key buffer is rebuilt by the next row
            }
        }
        cl.sync();
        if (rank == 0) trace_mark(tr, 2);
        // ---- coarse CSR: offsets by a cluster scan of the row counts, pass 2 writes ----
        int32_t csum = 0;
        for (long long cc = clo; cc < chi; ++cc) csum += ld32(a.cnt + cc);
        int32_t cnnz;
        int32_t pos = cluster_excl_scan(cl, sm, csum, cnnz);
        for (long long cc = clo; cc < chi; ++cc) {
            o.cadjp[cc] = pos;
            const int32_t k = ld32(a.cnt + cc);
            const int32_t u = ld32(lead_of + cc), v = ld32(M + u);
            const int32_t ub = (ld32(gadjp + u + 1) - ld32(gadjp + u)) + (v != u ? ld32(gadjp + v + 1) - ld32(gadjp + v) : 0);
            if (ub <= 16) {
                m_row16(gadjp, gadjncy, gadjwgt, CM, M, lead_of, (int32_t)cc, o.cadjncy + pos, o.cadjwgt + pos);
            } else {
                const unsigned long long *sk = a.stage + ld32(a.woff + cc);
                for (int32_t q = 0; q < k; ++q) {
                    const unsigned long long kv = sk[q];
                    o.cadjncy[pos + q] = (int32_t)(kv >> 32);
                    o.cadjwgt[pos + q] = (int32_t)(uint32_t)kv;
                }
            }
            pos += k;
        }
        if (gt == 0) o.cadjp[nc] = cnnz;
        // ---- statistics, stop rule (R12, R13), report ----
        arcs = warp_sum64(arcs);
        rows = warp_sum64(rows);
        visits = warp_sum64(visits);
        MatchCtl *mc = &a.levdev[gl].match;
        if ((t & 31) == 0 && (arcs | rows | visits)) {
            atomicAdd(&mc->arcs_scanned, arcs);
            atomicAdd(&mc->rows_scanned, rows);
            atomicAdd(&mc->live_visits, visits);
        }
        int32_t reason = GP_STOP_NONE;
        if (100LL * nc > (long long)a.stall_pct * n) reason = GP_STOP_STALL;
        else if (nc <= a.threshold) reason = GP_STOP_THRESHOLD;
        else if (gl + 1 >= a.max_levels) reason = GP_STOP_MAX_LEVELS;
        __threadfence();
        cl.sync();
        if (gt == 0) {
            mc->rounds = rounds;
            mc->maximal = maximal;
            SizeRec *so = &a.levdev[gl].out;
            so->n = nc;
            so->nnz = cnnz;
            so->stop = reason != GP_STOP_NONE;
            so->stop_reason = reason;
            LevelReport *r = &a.reports[gl];
            r->n_coarse = nc;
            r->cnnz = cnnz;
            r->stop = reason != GP_STOP_NONE;
            r->stop_reason = reason;
            r->skipped = 0;
            __threadfence_system();
            *((volatile int32_t *)&r->ready) = 1;
            trace_mark(tr, 3);
        }
        stopped = reason != GP_STOP_NONE;
        prev_reason = reason;
        n = nc;
        nnz = cnnz;
        gadjp = o.cadjp;
        gadjncy = o.cadjncy;
        gadjwgt = o.cadjwgt;
        gvwgt = o.cvwgt;
        ++level;
        cl.sync();
    }
    if (gt == 0) {
        for (int l = level; l < a.nslots; ++l) {
            const int gl = a.level0 + l;
            SizeRec *so = &a.levdev[gl].out;
            so->n = n;
            so->nnz = nnz;
            so->stop = 1;
            so->stop_reason = prev_reason;
            LevelReport *r = &a.reports[gl];
            r->skipped = 1;
            __threadfence_system();
            *((volatile int32_t *)&r->ready) = 1;
        }
    }
}

// Off by default (GP_MEDIUM=1 enables it): measured SLOWER than the grid-wide level kernels on
// the medium levels it targets -- C3 levels 8-11 took 0.5-0.8 ms of matching and up to 3.3 ms of
// contraction each on 16 SMs (the wide rows, one CTA each, serialise; the L2 round trips of the
// per-thread chains are not hidden by 8 K threads), against ~150 us per level on the full grid.
// Kept as a tested, bit-exact mode (tests/test_gpu_tail.py) and documented in DESIGN.md §4.3.
static int medium_enabled() {
    const char *e = getenv("GP_MEDIUM");  // knob read per call (results never depend on it)
    return (e && atoi(e) == 1) ? 1 : 0;
}
static int32_t medium_max_n() {
    const char *e = getenv("GP_MEDIUM_N");  // tuning knob (results never depend on it)
    return e ? atoi(e) : 131072;
}

bool medium_use(int32_t n_bound, int32_t nnz_bound) {
    return medium_enabled() && n_bound > 0 && n_bound <= medium_max_n() && nnz_bound <= 16 * medium_max_n();
}

size_t medium_scratch_bytes(int32_t n, int32_t nnz) {
    const size_t nn = (size_t)n + 64;
    return 4 * (7 * nn + 64) + nn + 16 * ((size_t)nnz + 64) + 512;
}

// cluster size: 16 when the device allows non-portable clusters for this kernel, else 8 (per
// device and instantiation: the attribute is per function)
static int medium_cluster(const void *fn, size_t smem, int which) {
    static int cs_dev[kMaxDevices][2] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    int &cs = cs_dev[dev < kMaxDevices ? dev : 0][which];
    if (cs > 0) return cs;
    cs = 8;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) == cudaSuccess) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(16);
        cfg.blockDim = dim3(kMT);
        cfg.dynamicSmemBytes = smem;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = 16;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        int ncl = 0;
        if (cudaOccupancyMaxActiveClusters(&ncl, fn, &cfg) == cudaSuccess && ncl >= 1) cs = 16;
    }
    cudaGetLastError();
    return cs;
}

gp_status enqueue_medium(Ctx *ctx, const MediumLaunch &L) {
    MediumArgs a;
    a.in = L.in;
    a.adjp = L.adjp;
    a.adjncy = L.adjncy;
    a.adjwgt = L.adjwgt;
    a.vwgt = L.vwgt;
    a.slots = reinterpret_cast<MediumLevelOut *>(L.slots);
    a.nslots = L.nslots;
    a.level0 = L.level0;
    a.cap_n = L.cap_n;
    a.cap_nnz = L.cap_nnz;
    a.levdev = L.levdev;
    a.reports = L.reports;
    a.threshold = L.threshold;
    a.stall_pct = L.stall_pct;
    a.max_levels = L.max_levels;
    a.max_rounds = L.max_rounds;
    a.tie_seed = ctx->tie_seed;
    {
        const size_t nn = (size_t)L.cap_n + 64;
        int32_t *p = static_cast<int32_t *>(L.scratch);
        a.M = p; p += nn;
        a.P = p; p += nn;
        a.R0 = p; p += nn;
        a.R1 = p; p += nn;
        a.cnt = p; p += nn;
        a.woff = p; p += nn;
        a.wide = p; p += nn;
        a.ctr = p; p += 64;
        a.stamp = reinterpret_cast<uint8_t *>(p);
        unsigned char *q = reinterpret_cast<unsigned char *>(p) + nn;
        q = reinterpret_cast<unsigned char *>(((uintptr_t)q + 255) & ~(uintptr_t)255);
        a.stage = reinterpret_cast<unsigned long long *>(q);
    }
    const size_t smem = sizeof(MediumShared);
    const void *fn = a.tie_seed ? (const void *)k_medium<true> : (const void *)k_medium<false>;
    GP_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const int cs = medium_cluster(fn, smem, a.tie_seed ? 1 : 0);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(cs);
    cfg.blockDim = dim3(kMT);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = ctx->stream;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = cs;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    void *args[] = {&a};
    LaunchScope ls(ctx, GP_K_OTHER);
    GP_CUDA(cudaLaunchKernelExC(&cfg, fn, args));
    ++ctx->launches;
    return GP_OK;
}

}  // namespace gp
