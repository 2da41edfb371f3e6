// small.cu -- the coarse-level tail for graphs that fit ONE SM: every
// remaining level -- matching rounds, cmap, contraction, coarse CSR -- in a single launch of
// one CTA whose working set lives in shared memory.
//
// Why (PAPER.md P16.s6-7, P20.s28-33): at small levels the GPU has too little parallelism and
// GP-metis hands the graph to the CPU (mt-metis).  On B200 the same latency problem shows as
// fixed costs per round and per level: a grid-wide round costs a few microseconds of barrier and
// L2 round trips however little work it holds (C1, 64x64 unit grid: 221 rounds over 6 levels).
// One CTA with the graph in its 227 KB of shared memory turns a round into two __syncthreads
// and shared-memory loads (~30-cycle latency instead of ~360), and the level loop needs no
// host round trip and no kernel boundary.
//
// Same rule and outputs as the level kernels (match.cu, contract.cu; R1-R17):
//   rounds:   every free vertex proposes its heaviest free neighbour (ties: lower id, or lower
//             h_s(v) with a tie seed); mutual proposals match; until no free vertex has a free
//             neighbour (or max_rounds); leftover self-match (P18.s12-13).  A proposal is
//             re-derived only when its target got matched (the free set only shrinks, so a
//             still-free target is still the heaviest free neighbour).
//   cmap:     leaders u <= M[u] numbered in id order, partners copy (P18.s16-27, R7).
//   contract: every arc (y, x) becomes the key (CM[y], CM[x]); the collapsed edge is dropped
//             (R9); the keys are sorted (flip-bitonic network in shared memory) and runs of
//             equal keys summed (R8) -- the off-diagonal of P^T A P in row-major order, i.e.
//             rows sorted by coarse id (R10); cvwgt = P^T vwgt (P12.s26-28).
//   stop:     stall, threshold, max_levels exactly as k_contract_level (R12, R13).
// Each level's M, CM and coarse CSR go to a per-level slot of a device arena owned by the
// hierarchy; the next level is loaded back from its slot (L2-resident).
#include <cuda_runtime.h>
#include <stdlib.h>

#include "device_util.cuh"
#include "gp_internal.cuh"
#include "merge_util.cuh"

namespace gp {

constexpr int kSNT = 512;                  // threads of the one CTA (128 registers each: no spills)
constexpr int kSVPT = 16;                  // cap: at most 16 vertices per thread (n <= 8192)
constexpr size_t kSmallSmemMax = 227 * 1024;

struct SmallLevelOut {  // one arena slot (device pointers)
    int32_t *M, *CM, *cadjp, *cadjncy, *cadjwgt, *cvwgt;
};

struct SmallArgs {
    const SizeRec *in;  // sizes + stop flag of the first level's input graph
    const int32_t *adjp, *adjncy, *adjwgt, *vwgt;  // the first level's input graph
    SmallLevelOut *slots;  // device array [nslots]
    int32_t nslots;
    int32_t level0;       // hierarchy index of the first level handled here
    int32_t cap_n, cap_nnz;  // shared-memory capacity (the first level's bounds)
    LevelDev *levdev;     // hierarchy control blocks: levdev[level0 + i]
    LevelReport *reports; // mapped host memory (reports[level0 + i])
    int32_t threshold, stall_pct, max_levels, max_rounds;
    uint32_t tie_seed;
};

// shared-memory layout (int32 words), each array 16-byte aligned
struct SmallLayout {
    int32_t adjp, adjncy, adjwgt, M, P, CM, R, stamp, scan, total;
};
__host__ __device__ inline int32_t small_round4(int32_t x) { return (x + 3) & ~3; }
__host__ __device__ inline SmallLayout small_layout(int32_t cap_n, int32_t cap_nnz) {
    SmallLayout L;
    int32_t o = 0;
    L.adjp = o;   o += small_round4(cap_n + 1);
    L.adjncy = o; o += small_round4(cap_nnz);
    L.adjwgt = o; o += small_round4(cap_nnz);
    L.M = o;      o += small_round4(cap_n);
    L.P = o;      o += small_round4(cap_n);
    L.CM = o;     o += small_round4(cap_n);   // also the rescan list of the even rounds
    L.R = o;      o += small_round4(cap_n);   // the rescan list of the odd rounds
    L.stamp = o;  o += small_round4((cap_n + 3) / 4);  // 1 byte per vertex: "changed this round"
    L.scan = o;   o += 64;
    L.total = o;
    return L;
}

size_t small_smem_bytes(int32_t n, int32_t nnz) { return (size_t)small_layout(n, nnz).total * 4; }

bool small_fits(int32_t n, int32_t nnz) {
    // keys (c * n_c + cx) must fit 32 bits below the drop marker: n_c <= n <= 65535
    return n > 0 && n <= kSNT * kSVPT && nnz >= 0 && small_smem_bytes(n, nnz) <= kSmallSmemMax;
}

// block-wide exclusive scan over the per-thread values (all threads call)
__device__ __forceinline__ int32_t sblock_scan(int32_t v, int32_t *scan, int32_t &total) {
    return block_excl_scan<kSNT>(v, scan, total);
}

__device__ __forceinline__ void small_load(int32_t *dst, const int32_t *src, int32_t len) {
    // 16-byte vector loads (global arrays are 16-byte aligned and padded by >= 16 bytes)
    const int32_t n4 = (len + 3) >> 2;
    const int4 *s4 = reinterpret_cast<const int4 *>(src);
    int4 *d4 = reinterpret_cast<int4 *>(dst);
    for (int32_t i = threadIdx.x; i < n4; i += kSNT) d4[i] = __ldcg(s4 + i);
}

// proposal key of neighbour x over weight w (heavier first, then the tie priority; 0 = none)
template <bool H>
__device__ __forceinline__ unsigned long long skey(uint32_t seed, int32_t w, int32_t x) {
    return pack_key<H>(seed, w, x);
}

// flip-bitonic sort of (key, val) pairs of any length (comparators past len are skipped);
// the index arithmetic is shifts and masks (sizes are powers of two)
__device__ void sort_pairs(uint32_t *key, int32_t *val, int32_t len) {
    int32_t S = 1, lg = 0;
    while (S < len) {
        S <<= 1;
        ++lg;
    }
    for (int32_t ls = 1; ls <= lg; ++ls) {
        const int32_t size = 1 << ls, lh = ls - 1;
        for (int32_t i = threadIdx.x; i < S / 2; i += kSNT) {
            const int32_t blk = i >> lh, o = i & ((1 << lh) - 1);
            const int32_t x = (blk << ls) + o, y = (blk << ls) + size - 1 - o;
            if (y < len && key[x] > key[y]) {
                const uint32_t k = key[x];
                key[x] = key[y];
                key[y] = k;
                const int32_t v = val[x];
                val[x] = val[y];
                val[y] = v;
            }
        }
        __syncthreads();
        for (int32_t lj = ls - 2; lj >= 0; --lj) {
            const int32_t j = 1 << lj;
            for (int32_t i = threadIdx.x; i < S / 2; i += kSNT) {
                const int32_t x = ((i >> lj) << (lj + 1)) + (i & (j - 1)), y = x + j;
                if (y < len && key[x] > key[y]) {
                    const uint32_t k = key[x];
                    key[x] = key[y];
                    key[y] = k;
                    const int32_t v = val[x];
                    val[x] = val[y];
                    val[y] = v;
                }
            }
            __syncthreads();
        }
    }
}

template <bool H>
__global__ void __launch_bounds__(kSNT, 1) k_small(const __grid_constant__ SmallArgs a) {
    extern __shared__ __align__(16) int32_t sw[];
    const SmallLayout Lo = small_layout(a.cap_n, a.cap_nnz);
    int32_t *adjp = sw + Lo.adjp, *adjncy = sw + Lo.adjncy, *adjwgt = sw + Lo.adjwgt;
    int32_t *M = sw + Lo.M, *P = sw + Lo.P, *CM = sw + Lo.CM, *scan = sw + Lo.scan;
    int32_t *Rl[2] = {CM, sw + Lo.R};
    uint8_t *stamp = reinterpret_cast<uint8_t *>(sw + Lo.stamp);
    const int t = threadIdx.x;
    __shared__ int32_t s_n, s_nnz;
    // round counters by round parity: slot k & 1 is reset in round k - 1 (after the barrier that
    // follows every read of round k - 2's values) and read in round k after its barriers
    __shared__ int32_t s_rn[2], s_pairs[2], s_dead[2];

    const volatile SizeRec *in = a.in;
    int32_t n = in->n, nnz = in->nnz;
    int level = 0;  // relative to level0
    bool stopped = in->stop != 0;
    int32_t prev_reason = in->stop_reason;
    const int32_t *gadjp = a.adjp, *gadjncy = a.adjncy, *gadjwgt = a.adjwgt, *gvwgt = a.vwgt;
    while (!stopped && level < a.nslots) {
        const int gl = a.level0 + level;
        const SmallLevelOut o = a.slots[level];
        unsigned long long *tr = a.levdev[gl].match.trace;  // GP_DEBUG phase marks
        trace_mark(tr, 0);
        // ---- load the level's graph into shared memory ----
        small_load(adjp, gadjp, n + 1);
        small_load(adjncy, gadjncy, nnz);
        small_load(adjwgt, gadjwgt, nnz);
        for (int32_t u = t; u < n; u += kSNT) {
            M[u] = kFree;
            stamp[u] = 1;  // round 1: every vertex proposes
        }
        __syncthreads();
        trace_mark(tr, 1);
        // ---- matching rounds (A2-A4), event driven ----
        // The synchronous rule simulated exactly, with work proportional to what changes:
        //  * a free vertex's proposal changes only when its target gets matched (the free set
        //    only shrinks, so a still-free target stays the heaviest free neighbour): those
        //    vertices -- the rescan list R -- rescan, nobody else;
        //  * a mutual pair appears only where one of its ends changed its proposal this round
        //    (else it was mutual a round earlier and matched then): the commit looks at the
        //    changed vertices only (stamp = 1), the pair is handled by its changed end (the
        //    lower id when both changed), which writes both M entries and lists the neighbours
        //    that proposed to either end for the next round's rescans (each such vertex proposes
        //    to one vertex, so it is listed once).
        //  live = free vertices with a proposal; a round with live > 0 matches >= 1 pair (§2.1).
        unsigned long long arcs = 0, rows = 0, visits = 0;
        int32_t rounds = 0, maximal = 0;
        auto rescan = [&](int32_t u) -> int32_t {  // heaviest free neighbour of u, or -2
            unsigned long long best = 0;
            const int32_t s0 = adjp[u], e0 = adjp[u + 1];
            int32_t j = s0;
            for (; j + 4 <= e0; j += 4) {  // four independent shared-memory chains
                int32_t x[4], w[4], f[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    x[q] = adjncy[j + q];
                    w[q] = adjwgt[j + q];
                }
#pragma unroll
                for (int q = 0; q < 4; ++q) f[q] = M[x[q]];
#pragma unroll
                for (int q = 0; q < 4; ++q)
                    if (f[q] == kFree) {
                        const unsigned long long kk = skey<H>(a.tie_seed, w[q], x[q]);
                        best = kk > best ? kk : best;
                    }
            }
            for (; j < e0; ++j) {
                const int32_t x = adjncy[j];
                if (M[x] == kFree) {
                    const unsigned long long kk = skey<H>(a.tie_seed, adjwgt[j], x);
                    best = kk > best ? kk : best;
                }
            }
            arcs += (unsigned long long)(e0 - s0);
            const int32_t b = key_vertex<H>(a.tie_seed, best);
            return b == kNone ? -2 : b;
        };
        // round 1 proposals: every vertex
        int32_t mylive = 0;
        for (int32_t u = t; u < n; u += kSNT) {
            P[u] = rescan(u);
            mylive += P[u] >= 0;
        }
        int32_t live;
        sblock_scan(mylive, scan, live);  // (block total; syncs: P complete)
        int32_t rn = n, cur = 0;           // the changed vertices of this round: all (round 1)
#ifdef GP_CHECKPOINTS
        long long ck0 = clock64();
#define GP_SCK(j) do { if (t == 0 && k < 16) a.levdev[gl].match.ck[k][j] = clock64() - ck0; } while (0)
#else
#define GP_SCK(j) do { } while (0)
#endif
        for (int k = 1;; ++k) {
#ifdef GP_CHECKPOINTS
            ck0 = clock64();
#endif
            if (live == 0) {
                maximal = 1;
                break;
            }
            if (a.max_rounds > 0 && rounds >= a.max_rounds) break;
            if (k == 1 && t == 0) s_rn[1] = s_pairs[1] = s_dead[1] = 0;
            __syncthreads();
            if (t == 0) s_rn[(k + 1) & 1] = s_pairs[(k + 1) & 1] = s_dead[(k + 1) & 1] = 0;
            const int sl = k & 1;
            GP_SCK(0);
            // commit (handshake) over the changed vertices
            int32_t *Rn = Rl[cur ^ 1];
            int32_t mypairs = 0;
            for (int32_t i = t; i < rn; i += kSNT) {
                const int32_t x = k == 1 ? i : Rl[cur][i];
                if (x < 0) continue;  // matched in the previous round (marked by the rescan pass)
                const int32_t d = P[x];
                if (d < 0) continue;
                ++visits;
                if (P[d] != x) continue;
                if (stamp[d] && d < x) continue;  // both ends changed: the lower id handles it
                M[x] = d;
                M[d] = x;
                ++mypairs;
                // neighbours that proposed to x or d rescan next round: four arcs at a time
                // (independent loads), one list reservation per four arcs
#pragma unroll 1
                for (int e = 0; e < 2; ++e) {
                    const int32_t y0 = e ? d : x, other = e ? x : d;
                    const int32_t j1 = adjp[y0 + 1];
                    for (int32_t j = adjp[y0]; j < j1; j += 4) {
                        int32_t y[4], py[4];
#pragma unroll
                        for (int q = 0; q < 4; ++q) y[q] = j + q < j1 ? adjncy[j + q] : other;
#pragma unroll
                        for (int q = 0; q < 4; ++q) py[q] = y[q] != other ? P[y[q]] : -1;
                        int32_t c = 0;
#pragma unroll
                        for (int q = 0; q < 4; ++q) c += py[q] == y0;
                        if (c) {
                            int32_t w = atomicAdd(&s_rn[sl], c);
#pragma unroll
                            for (int q = 0; q < 4; ++q)
                                if (py[q] == y0) Rn[w++] = y[q];
                        }
                    }
                }
            }
            if (mypairs) atomicAdd(&s_pairs[sl], mypairs);
            GP_SCK(1);
            __syncthreads();
            GP_SCK(2);
            // the stamps of this round's changed vertices are cleared, the next ones set
            for (int32_t i = t; i < rn; i += kSNT) {
                const int32_t x = k == 1 ? i : Rl[cur][i];
                if (x >= 0) stamp[x] = 0;
            }
            const int32_t pairs = s_pairs[sl], rnn = s_rn[sl];
            if (pairs > 0) ++rounds;
            live -= 2 * pairs;
            __syncthreads();
            GP_SCK(3);
            // round k+1 proposals: the rescans (a vertex matched this round is skipped)
            int32_t dead = 0;
            for (int32_t i = t; i < rnn; i += kSNT) {
                const int32_t y = Rn[i];
                if (M[y] != kFree) {  // matched this round: out of the next round's list
                    Rn[i] = -1;
                    continue;
                }
                stamp[y] = 1;
                ++rows;
                const int32_t b = rescan(y);
                P[y] = b;
                dead += b < 0;
            }
            if (dead) atomicAdd(&s_dead[sl], dead);
            GP_SCK(4);
            __syncthreads();
            GP_SCK(5);
            live -= s_dead[sl];
            rn = rnn;
            cur ^= 1;
            if (k > n + 2) __trap();  // each round with proposals matches >= 1 pair
            GP_SCK(6);
            if (t == 0 && k < 16) a.levdev[gl].match.ck[k][7] = rn, a.levdev[gl].match.ck[k][8] = rn + 1;
        }
#undef GP_SCK
        trace_mark(tr, 2);
        // ---- leftover (P18.s12-13) + cmap (P18.s16-27) ----
        const int32_t per = (n + kSNT - 1) / kSNT;
        const int32_t lo = min(n, t * per), hi = min(n, lo + per);
        int32_t cnt = 0;
        for (int32_t u = lo; u < hi; ++u) {
            if (M[u] == kFree) M[u] = u;
            if (u <= M[u]) ++cnt;
        }
        int32_t nc;
        int32_t c = sblock_scan(cnt, scan, nc);
        for (int32_t u = lo; u < hi; ++u)
            if (u <= M[u]) CM[u] = c++;
        __syncthreads();
        for (int32_t u = t; u < n; u += kSNT) {
            const int32_t m = M[u];
            if (u > m) CM[u] = CM[m];
            o.M[u] = m;
        }
        __syncthreads();
        for (int32_t u = t; u < n; u += kSNT) {
            const int32_t m = M[u], cu = CM[u];
            o.CM[u] = cu;
            if (u <= m) o.cvwgt[cu] = __ldcg(gvwgt + u) + (m != u ? __ldcg(gvwgt + m) : 0);  // P12.s27
        }
        // leaders by coarse id (P is free from here on) and the widest merged row
        int32_t *lead_of = P;
        bool wide = false;
        for (int32_t u = t; u < n; u += kSNT) {
            const int32_t m = M[u];
            if (u <= m) {
                lead_of[CM[u]] = u;
                const int32_t ub = (adjp[u + 1] - adjp[u]) + (m != u ? adjp[m + 1] - adjp[m] : 0);
                wide = wide || ub > 16;
            }
        }
        const uint32_t kDrop = 0xFFFFFFFFu;
        int32_t cnnz;
        if (!__syncthreads_or(wide)) {
            // ---- every merged row <= 16 entries: one thread per coarse row, register network ----
            // pass 1 counts, a block scan places the threads' rows, pass 2 re-merges and writes
            // (re-merging 16 registers is cheaper than staging the rows)
            const int32_t pc = (nc + kSNT - 1) / kSNT;
            const int32_t clo = min(nc, t * pc), chi = min(nc, clo + pc);
            int32_t mine = 0;
            for (int pass = 0; pass < 2; ++pass) {
                int32_t pos = 0;
                if (pass == 1) {
                    pos = sblock_scan(mine, scan, cnnz);
                    if (t == 0) o.cadjp[nc] = cnnz;
                }
                for (int32_t cc = clo; cc < chi; ++cc) {
                    const int32_t u = lead_of[cc], v = M[u];
                    const int32_t su = adjp[u], du = adjp[u + 1] - su;
                    const int32_t sv = v != u ? adjp[v] : 0, dv = v != u ? adjp[v + 1] - sv : 0;
                    uint32_t kc[16];
                    int32_t kw[16];
#pragma unroll
                    for (int q = 0; q < 16; ++q) {
                        kc[q] = kDrop;
                        kw[q] = 0;
                        if (q < du + dv) {
                            const int32_t jj = q < du ? su + q : sv + (q - du);
                            const uint32_t cx = (uint32_t)CM[adjncy[jj]];
                            if (cx != (uint32_t)cc) {  // collapsed edge dropped (R9)
                                kc[q] = cx;
                                kw[q] = adjwgt[jj];
                            }
                        }
                    }
                    cx_sort16(kc, kw);
                    if (pass == 1) o.cadjp[cc] = pos;
                    uint32_t prev = kDrop;
                    int32_t acc = 0;
#pragma unroll
                    for (int q = 0; q < 16; ++q) {
                        if (kc[q] == prev) {
                            acc += kw[q];  // repeated coarse neighbour: weights summed (R8, P12.s28)
                        } else {
                            if (prev != kDrop) {
                                if (pass == 1) {
                                    o.cadjncy[pos] = (int32_t)prev;
                                    o.cadjwgt[pos] = acc;
                                }
                                ++pos;
                            }
                            prev = kc[q];
                            acc = kw[q];
                        }
                    }
                    if (prev != kDrop) {
                        if (pass == 1) {
                            o.cadjncy[pos] = (int32_t)prev;
                            o.cadjwgt[pos] = acc;
                        }
                        ++pos;
                    }
                }
                if (pass == 0) mine = pos;
            }
            trace_mark(tr, 3);
            trace_mark(tr, 4);
        } else {
            // ---- general path: keys (CM[y], CM[x]) in place, block-wide sort, run sums ----
            uint32_t *key = reinterpret_cast<uint32_t *>(adjncy);
            for (int32_t y = t; y < n; y += kSNT) {
                const uint32_t cy = (uint32_t)CM[y];
                for (int32_t j = adjp[y]; j < adjp[y + 1]; ++j) {
                    const uint32_t cx = (uint32_t)CM[adjncy[j]];
                    key[j] = cx == cy ? kDrop : cy * (uint32_t)nc + cx;  // collapsed edge dropped (R9)
                }
            }
            // the per-coarse-row counts (lead_of is no longer needed)
            int32_t *ccnt = P;
            __syncthreads();
            for (int32_t x = t; x < nc; x += kSNT) ccnt[x] = 0;
            __syncthreads();
            trace_mark(tr, 3);
            sort_pairs(key, adjwgt, nnz);
            trace_mark(tr, 4);
            // ---- run sums (R8) + compaction into the coarse CSR ----
            const int32_t pe = (nnz + kSNT - 1) / kSNT;
            const int32_t elo = min(nnz, t * pe), ehi = min(nnz, elo + pe);
            int32_t heads = 0;
            for (int32_t i = elo; i < ehi; ++i)
                if (key[i] != kDrop && (i == 0 || key[i] != key[i - 1])) ++heads;
            int32_t pos = sblock_scan(heads, scan, cnnz);
            for (int32_t i = elo; i < ehi; ++i) {
                const uint32_t kk = key[i];
                if (kk == kDrop || (i > 0 && kk == key[i - 1])) continue;
                int32_t sum = adjwgt[i];
                for (int32_t q = i + 1; q < nnz && key[q] == kk; ++q) sum += adjwgt[q];  // fits int32 (R14)
                const int32_t cr = (int32_t)(kk / (uint32_t)nc);
                o.cadjncy[pos] = (int32_t)(kk - (uint32_t)cr * (uint32_t)nc);
                o.cadjwgt[pos] = sum;
                atomicAdd(&ccnt[cr], 1);
                ++pos;
            }
            __syncthreads();
            {
                const int32_t pc = (nc + kSNT - 1) / kSNT;
                const int32_t clo = min(nc, t * pc), chi = min(nc, clo + pc);
                int32_t sm = 0;
                for (int32_t x = clo; x < chi; ++x) sm += ccnt[x];
                int32_t tot;
                int32_t off = sblock_scan(sm, scan, tot);
                for (int32_t x = clo; x < chi; ++x) {
                    o.cadjp[x] = off;
                    off += ccnt[x];
                }
                if (t == 0) o.cadjp[nc] = cnnz;
            }
        }
        trace_mark(tr, 5);
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
        __syncthreads();
        if (t == 0) {
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
            s_n = nc;
            s_nnz = cnnz;
        }
        __syncthreads();
        stopped = reason != GP_STOP_NONE;
        prev_reason = reason;
        n = s_n;
        nnz = s_nnz;
        gadjp = o.cadjp;
        gadjncy = o.cadjncy;
        gadjwgt = o.cadjwgt;
        gvwgt = o.cvwgt;
        ++level;
    }
    // the levels the host enqueued beyond the stop: skipped reports
    if (t == 0) {
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

static int small_enabled() {
    const char *e = getenv("GP_SMALL");  // knob read per call (results never depend on it)
    return (e && atoi(e) == 0) ? 0 : 1;
}

bool small_use(int32_t n_bound, int32_t nnz_bound) { return small_enabled() && small_fits(n_bound, nnz_bound); }

gp_status enqueue_small(Ctx *ctx, const SmallLaunch &L) {
    SmallArgs a;
    a.in = L.in;
    a.adjp = L.adjp;
    a.adjncy = L.adjncy;
    a.adjwgt = L.adjwgt;
    a.vwgt = L.vwgt;
    a.slots = reinterpret_cast<SmallLevelOut *>(L.slots);
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
    const size_t smem = small_smem_bytes(L.cap_n, L.cap_nnz);
    const void *fn = a.tie_seed ? (const void *)k_small<true> : (const void *)k_small<false>;
    GP_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    void *args[] = {&a};
    LaunchScope ls(ctx, GP_K_OTHER);
    GP_CUDA(cudaLaunchKernel(fn, dim3(1), dim3(kSNT), args, smem, ctx->stream));
    ++ctx->launches;
    return GP_OK;
}

size_t small_slot_ints(int32_t n, int32_t nnz) {
    // M, CM, cadjp, cadjncy, cadjwgt, cvwgt, each padded to 64 ints (256 B)
    auto pad = [](size_t x) { return (x + 4 + 63) / 64 * 64; };
    return 2 * pad((size_t)n) + pad((size_t)n + 1) + 2 * pad((size_t)nnz) + pad((size_t)n);
}

void small_slot_carve(int32_t *base, int32_t n, int32_t nnz, void *out_slot) {
    auto pad = [](size_t x) { return (x + 4 + 63) / 64 * 64; };
    SmallLevelOut s;
    int32_t *p = base;
    s.M = p; p += pad((size_t)n);
    s.CM = p; p += pad((size_t)n);
    s.cadjp = p; p += pad((size_t)n + 1);
    s.cadjncy = p; p += pad((size_t)nnz);
    s.cadjwgt = p; p += pad((size_t)nnz);
    s.cvwgt = p;
    *reinterpret_cast<SmallLevelOut *>(out_slot) = s;
}

size_t small_slot_desc_bytes() { return sizeof(SmallLevelOut); }

}  // namespace gp
