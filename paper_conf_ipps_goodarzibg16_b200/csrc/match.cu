// match.cu -- A1-A4 of one level in ONE persistent cooperative kernel: degree-binned
// proposals, handshake commits, the round loop and the leftover pass.
//
// Rule (PAPER.md P18.s6-13 re-pinned by north_star, R1-R4): in every round each
// free vertex proposes its heaviest free neighbour (ties -> lower id; HEM, P12.s23,
// P18.s7); two vertices that propose each other match (handshake; replaces the paper's
// conflict kernel "M[u]=v and M[v]!=u => M[u]=u", P18.s10-12).  Rounds repeat until no
// free vertex has a free neighbour; the leftover pass self-matches the rest (P18.s12-13).
//
// B200 design:
//  * One launch per level, grid = SMs x co-resident CTAs; phases are separated by a grid
//    barrier (~1-2 us) instead of kernel boundaries and host round trips.
//  * Phase 0 (round-1 proposals, every vertex free, no M reads): chunks of consecutive
//    vertices whose adjacency fits a stage are staged into shared memory with TMA bulk
//    copies (cp.async.bulk, mbarrier completion, 2 stages), then reduced by groups of G
//    threads per vertex (G from the level's average degree) -> coalesced 100%-useful HBM
//    streams.  Chunks with long rows fall back to direct group / warp scans; rows longer
//    than kHubDeg go to a hub list scanned by whole CTAs.
//  * Phase k (k >= 1) fuses the commit of round k with the proposals of round k+1:
//      p = P_k[u], q = P_k[p]:   q == u           -> M[u] = p (matched; owner writes only)
//                                p kept its pair  -> p is still u's heaviest free neighbour
//                                p matched q      -> rescan u's row (lazy rescan)
//    The rescan tests a neighbour x with "M[x] free and not (P_k[P_k[x]] == x)", so the
//    round-k matches being written concurrently are seen through the read-only P_k.
//    P is double buffered by round parity; matched and dead vertices hold the same value
//    (partner / NONE) in both buffers.  Result-identical to the literal rule (oracle).
//  * Worklists are appended with one atomic per CTA (block-aggregated), round counters
//    live in a 4-slot ring so no counter is reset while another CTA may still read it.
#include <cuda_runtime.h>
#include <stdlib.h>

#include "device_util.cuh"
#include "gp_internal.cuh"

namespace gp {

constexpr int kNT = 512;            // threads per CTA of the persistent kernels
constexpr int kStageArcs = 4096;    // arcs per TMA stage (adjncy + adjwgt = 32 KB)
constexpr int kStages = 3;          // TMA pipeline depth of phase 0
constexpr int kMaxVch = 1024;       // vertices per phase-0 chunk (adjp slice staged too)
constexpr int kHubDeg = 1024;       // rows longer than this: hub phase (chunks over all CTAs)

// CTAs taking part in this launch: min(grid, ceil(n / vpc)).  The host launches the full
// persistent grid before the level's size is known; the level's kernel retires the CTAs a
// small level cannot use, which makes its grid barriers and claim counters cheaper.
__shared__ int g_nact;

struct MatchArgs {
    const SizeRec *in;  // device: sizes + stop flag of this level's graph
    const int32_t *adjp, *adjncy, *adjwgt;
    int32_t *M;
    int32_t *P[2];
    int32_t *L[2];
    int32_t *H;  // hub list of the pending hub phase
    int32_t *S;  // second-heaviest neighbour of the last full scan (NONE = none cached)
    unsigned long long *hk;  // multi-CTA hub phase: best key per listed hub (the contraction's idle gkeys)
    // parking (single-GPU whole-level launches; null: off).  parked[u] = 1 while u, whose
    // target is still free, is off the live list; pcnt[v] counts vertices that parked on v;
    // W: wake tasks (matched vertices with parked neighbours), R: woken vertices.  All live in
    // the contraction's scratch, idle while a level matches (cnt, lofs, huge, seg).
    int32_t *parked, *pcnt, *W, *R;
    MatchCtl *ctl;
    int32_t max_rounds;
    int32_t leftover;
    int32_t G;    // lanes per vertex in phase 0 (1, 2, 4, 8 or 16)
    int32_t vch;  // vertices per phase-0 chunk (about 80 % of a stage at the average degree)
    int32_t vpc;  // vertices per active CTA (small levels run on fewer CTAs)
    // sharded levels (dist.cu): the rows are the vertices [vbase, vbase + n) of a graph of
    // n_global vertices; P, S and M are indexed by global vertex id (ghost entries are
    // filled by the exchange between launches).  Single GPU: vbase = 0.
    int32_t vbase;
    int32_t lanes_mode;  // 1: short live lists use G lanes per vertex (phase_k_lanes)
    int32_t tail_live;   // live lists this short are finished by CTA 0 alone
    int32_t interleave;  // phase-k groups dealt to CTAs round-robin (1) or in contiguous ranges (0)
    int32_t static_mode; // 1: small levels walk all vertices each round (no live list; GP_MATCH_STATIC=1)
    int32_t prof;        // GP_PROF=1: per-round slowest-warp times and rescan counts (MatchCtl)
    int32_t mode;  // kMatchWhole, or one launch per phase for the sharded path
    int32_t k;     // round of a kMatchRound launch
    uint32_t tie_seed;  // 0: lower id wins ties (north_star); else RM tie priority (R17, P18.s8)
    int32_t hub_deg_small, hub_small_n;  // levels of <= hub_small_n vertices send rescans of rows
                                         // longer than hub_deg_small to the hub phase (knobs)
};
__shared__ int32_t g_hubdeg;  // this launch's hub threshold (kHubDeg or hub_deg_small)


struct MatchSmem {
    int32_t adj[kStages][kStageArcs];
    int32_t wgt[kStages][kStageArcs];
    int32_t ap[kStages][kMaxVch + 8];  // adjp[v0 .. v0+vch] of the staged chunk
    uint64_t bar[kStages];
    int32_t a0[kStages];    // aligned first arc of the staged chunk
    int32_t fits[kStages];  // 1 staged, 0 fallback
    long long cid[kStages]; // chunk staged in the stage (claimed dynamically; >= nchunks: none)
    int32_t scratch[40];
    int32_t claim;  // phase-k group claims of this CTA
    int32_t trows;  // GP_PROF: rows rescanned by this CTA's threads in the round
    unsigned long long tmax;  // GP_PROF: slowest warp of this CTA in the round (ns)
    unsigned long long red[kNT / 32];
    unsigned long long cnt3[3][kNT / 32];
};

__device__ __forceinline__ int32_t ldcg(const int32_t *p) { return __ldcg(p); }
// Loads of the current round's proposals P_k, its live list and S.  L2 (ld.global.cg) by
// default; GP_P_CA=1 at build time reads them through L1 (safe: they were written in an earlier
// phase and every phase starts after a grid barrier whose acquire invalidates the SM's L1; the
// only writes within a phase mark dead vertices NONE, which a stale read cannot turn into a
// handshake).  Measured equal on C3 / C2 / C5 (3.31 vs 3.30, 2.80 vs 2.82, 29.5 vs 29.0 ms):
// the mesh locality of these gathers is already captured by coalescing within a warp.
#if defined(GP_P_CA)
__device__ __forceinline__ int32_t ldP(const int32_t *p) { return __ldca(p); }
#elif GP_L2HINT >= 2
// GP_L2HINT=2: the gathered proposal arrays carry an L2 evict_last policy (C3 level 0:
// P[2] + S + M = 64 MB of the 126 MB L2)
__device__ __forceinline__ int32_t ldP(const int32_t *p) {
    int32_t v;
    asm("{\n\t.reg .b64 pol;\n\tcreatepolicy.fractional.L2::evict_last.b64 pol, 1.0;\n\t"
        "ld.global.cg.L2::cache_hint.s32 %0, [%1], pol;\n\t}" : "=r"(v) : "l"(p));
    return v;
}
#else
__device__ __forceinline__ int32_t ldP(const int32_t *p) { return __ldcg(p); }
#endif
// GP_L2HINT >= 1 (default): the streamed arcs (rescans, phase-0 TMA stages) carry an L2
// evict_first policy so that they do not push the gathered proposal arrays out of L2.
// Measured (scripts/r2_l2hint.sh): C3 3.17 -> 3.11 ms (level-0 match 441 -> 420 us), C5
// unchanged; adding evict_last on the P / S gathers (=2) was slower than arcs alone (3.14 ms),
// and an L2 set-aside for it (cudaLimitPersistingL2CacheSize 64 MB) slower still (3.36 ms,
// C5 34 ms).  GP_L2HINT=0 at build time removes the hints.
#if GP_L2HINT >= 1
__device__ __forceinline__ int32_t ldArc(const int32_t *p) {
    int32_t v;
    asm("{\n\t.reg .b64 pol;\n\tcreatepolicy.fractional.L2::evict_first.b64 pol, 1.0;\n\t"
        "ld.global.nc.L2::cache_hint.s32 %0, [%1], pol;\n\t}" : "=r"(v) : "l"(p));
    return v;
}
#else
__device__ __forceinline__ int32_t ldArc(const int32_t *p) { return __ldg(p); }
#endif
__device__ __forceinline__ int4 ld_volatile_v4(const int4 *p) {
    int4 v;
    asm volatile("ld.volatile.global.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p)
                 : "memory");
    return v;
}

// Warp-buffered list append (no CTA-wide synchronisation): the lanes with `pred` put `value`
// into the warp's shared queue; a full queue is flushed with ONE global atomic and a
// coalesced copy.  `qn` is the warp-uniform queue length.  All 32 lanes must call.
constexpr int kWQ = 256;
__device__ __forceinline__ void wq_flush(int32_t *q, int32_t &qn, int32_t *list, int32_t *counter) {
    const int lane = threadIdx.x & 31;
    if (qn == 0) return;
    int32_t base = 0;
    if (lane == 0) base = atomicAdd(counter, qn);
    base = __shfl_sync(0xffffffffu, base, 0);
    __syncwarp();
    for (int i = lane; i < qn; i += 32) list[base + i] = q[i];
    __syncwarp();
    qn = 0;
}
__device__ __forceinline__ void wq_push(int32_t *q, int32_t &qn, int32_t *list, int32_t *counter, bool pred,
                                        int32_t value) {
    const unsigned m = __ballot_sync(0xffffffffu, pred);
    if (pred) q[qn + __popc(m & lanemask_lt())] = value;
    qn += __popc(m);
    if (qn > kWQ - 32) wq_flush(q, qn, list, counter);
}

// x is free after round k's commits.  M is not read: a vertex matched in any
// round <= k has P_k[P_k[x]] == x (matched vertices keep their partner in both proposal
// buffers), and a dead vertex (P = NONE) never neighbours a vertex that still rescans.
__device__ __forceinline__ bool free_after(int32_t x, const int32_t *Pk) {
    const int32_t px = ldP(Pk + x);
    return !(px >= 0 && ldP(Pk + px) == x);
}

// top-2 of packed keys (k1 > k2, both 0 = none)
__device__ __forceinline__ void top2_add(unsigned long long &k1, unsigned long long &k2, unsigned long long k) {
    if (k > k1) {
        k2 = k1;
        k1 = k;
    } else if (k > k2) {
        k2 = k;
    }
}
template <int WIDTH>
__device__ __forceinline__ void group_top2(unsigned long long &k1, unsigned long long &k2) {
#pragma unroll
    for (int off = WIDTH / 2; off > 0; off >>= 1) {
        const unsigned long long o1 = __shfl_xor_sync(0xffffffffu, k1, off, WIDTH);
        const unsigned long long o2 = __shfl_xor_sync(0xffffffffu, k2, off, WIDTH);
        const unsigned long long lo = k1 < o1 ? k1 : o1;
        k1 = k1 > o1 ? k1 : o1;
        const unsigned long long m2 = k2 > o2 ? k2 : o2;
        k2 = lo > m2 ? lo : m2;
    }
}
__device__ __forceinline__ void group_top2_rt(unsigned long long &k1, unsigned long long &k2, int G) {
    switch (G) {
        case 1: return;
        case 2: group_top2<2>(k1, k2); return;
        case 4: group_top2<4>(k1, k2); return;
        case 8: group_top2<8>(k1, k2); return;
        default: group_top2<16>(k1, k2); return;
    }
}

__device__ __forceinline__ unsigned long long group_max_rt(unsigned long long k, int G) {
    switch (G) {
        case 1: return k;
        case 2: return group_max64<2>(k);
        case 4: return group_max64<4>(k);
        case 8: return group_max64<8>(k);
        default: return group_max64<16>(k);
    }
}

// ---------------------------------------------------------------------------------------
// phase 0: round-1 proposals of every vertex
// ---------------------------------------------------------------------------------------
// thread 0: stage chunk c (bounds A0/A1 already loaded) into stage st with TMA bulk copies
// of its adjp slice and arc range, or mark it as fallback (too many arcs) / empty
__device__ __forceinline__ void stage_chunk(const MatchArgs &a, MatchSmem &sm, int32_t n, long long c, int32_t s,
                                            int32_t e, int st) {
    const int32_t A0 = s & ~3, A1 = (e + 3) & ~3;
    sm.a0[st] = A0;
    const bool fits = (A1 - A0) <= kStageArcs;
    const long long nv = min((long long)a.vch, (long long)n - c * a.vch);   // vertices in the chunk
    const unsigned apb = (unsigned)((nv + 1 + 3) & ~3ll) * 4u;  // adjp slice (<= adjp[n+3]), 16-byte multiple
    if (fits) {
        sm.fits[st] = 1;
        mbar_arrive_expect_tx(&sm.bar[st], apb + (unsigned)(A1 - A0) * 8u);
        tma_load_1d(sm.ap[st], a.adjp + c * a.vch, apb, &sm.bar[st]);
        if (A1 > A0) {
            tma_load_1d(sm.adj[st], a.adjncy + A0, (unsigned)(A1 - A0) * 4u, &sm.bar[st]);
            tma_load_1d(sm.wgt[st], a.adjwgt + A0, (unsigned)(A1 - A0) * 4u, &sm.bar[st]);
        }
    } else {
        sm.fits[st] = 0;
    }
}

__device__ __forceinline__ void load_bounds(const MatchArgs &a, int32_t n, long long nchunks, long long c, int32_t &s,
                                            int32_t &e) {
    s = e = 0;
    if (c < nchunks) {
        s = __ldg(a.adjp + c * a.vch);
        e = __ldg(a.adjp + min((long long)n, (c + 1) * a.vch));
    }
}

template <bool H>
__device__ void phase0(const MatchArgs &a, MatchSmem &sm, int32_t n, unsigned long long &scanned) {
    const int G = a.G;
    const int ngroups = kNT / G;
    const long long nchunks = ((long long)n + a.vch - 1) / a.vch;
    const int t = threadIdx.x, gl = t % G, grp = t / G;
    int32_t *P1 = a.P[1], *P0 = a.P[0];
    // thread 0 claims chunks dynamically (balances the tail) and keeps kStages in flight
    long long nxt = -1;          // next claimed chunk, bounds prefetched
    int32_t nb_s = 0, nb_e = 0;
    if (t == 0) {
        for (int q = 0; q < kStages; ++q) mbar_init(&sm.bar[q], 1);
        fence_mbar_init();
        // the first kStages chunks of a CTA are static (b, b + nact, b + 2 nact): their bounds
        // load in parallel and no claim atomic precedes the first TMA (a chain of 3 claims +
        // bounds held the first copies back by ~8 us, the whole phase on small levels);
        // later chunks are claimed dynamically beyond 3 nact -- per CTA still in increasing order
        int32_t cs[kStages], ce[kStages];
#pragma unroll
        for (int q = 0; q < kStages; ++q)
            load_bounds(a, n, nchunks, (long long)blockIdx.x + (long long)q * g_nact, cs[q], ce[q]);
#pragma unroll
        for (int q = 0; q < kStages; ++q) {
            const long long c = (long long)blockIdx.x + (long long)q * g_nact;
            sm.cid[q] = c;
            if (c < nchunks) stage_chunk(a, sm, n, c, cs[q], ce[q], q);
        }
        nxt = (long long)kStages * g_nact + atomicAdd(&a.ctl->chunk_ctr, 1u);
        load_bounds(a, n, nchunks, nxt, nb_s, nb_e);
    }
    __syncthreads();
    unsigned uses[kStages] = {};
    for (long long i = 0;; ++i) {
        const int st = (int)(i % kStages);
        const long long c = sm.cid[st];
        if (c >= nchunks) break;  // chunks are claimed in order: later stages are empty too
        const bool fits = sm.fits[st] != 0;
        const int32_t A0 = sm.a0[st];
        if (fits) {
            mbar_wait(&sm.bar[st], uses[st] & 1u);
            ++uses[st];
        }
        const long long vbeg = c * a.vch, vend = min((long long)n, vbeg + a.vch);
        const int32_t *sp = sm.ap[st];
        // a uniform trip count per warp keeps the group shuffles converged
        for (long long vb = vbeg; vb < vend; vb += ngroups) {
            const long long v = vb + grp;
            const bool valid = v < vend;
            int32_t s = 0, e = 0;
            if (valid) {
                if (fits) {
                    s = sp[v - vbeg];
                    e = sp[v - vbeg + 1];
                } else {
                    s = __ldg(a.adjp + v);
                    e = __ldg(a.adjp + v + 1);
                }
            }
            unsigned long long key = 0, key2 = 0;
            bool hub = false;
            if (fits) {
                const int32_t *sa = sm.adj[st], *sw = sm.wgt[st];
                for (int32_t j = s - A0 + gl; j < e - A0; j += G) top2_add(key, key2, pack_key<H>(a.tie_seed, sw[j], sa[j]));
            } else if (valid) {
                if (e - s > kHubDeg) {
                    hub = true;
                } else {  // 8 arcs per lane per batch, all loads in flight together
                    for (int32_t j0 = s + gl; j0 < e; j0 += 8 * G) {
                        int32_t xv[8], wv[8];
#pragma unroll
                        for (int q = 0; q < 8; ++q) {
                            const int32_t j = j0 + q * G;
                            xv[q] = j < e ? ldArc(a.adjncy + j) : -1;
                            wv[q] = j < e ? ldArc(a.adjwgt + j) : 0;
                        }
#pragma unroll
                        for (int q = 0; q < 8; ++q)
                            if (xv[q] >= 0) top2_add(key, key2, pack_key<H>(a.tie_seed, wv[q], xv[q]));
                    }
                }
            }
            group_top2_rt(key, key2, G);
            if (valid && gl == 0) {
                const int32_t x = a.vbase + (int32_t)v;  // row v is vertex vbase + v
                a.M[x] = kFree;
                if (a.parked) {
                    a.parked[x] = 0;
                    a.pcnt[x] = 0;
                }
                if (hub) {
                    const int32_t h = atomicAdd(&a.ctl->slot[1].nhub, 1);
                    a.H[h] = x;
                    if (a.hk) a.hk[h] = 0ull;  // (sharded launches: per-CTA hub_phase, no hk)
                    a.S[x] = kNone;
                } else {
                    const int32_t p = key_vertex<H>(a.tie_seed, key);
                    P1[x] = p;
                    a.S[x] = key_vertex<H>(a.tie_seed, key2);  // cached second-heaviest neighbour
                    if (p == kNone) P0[x] = kNone;  // dead vertices: NONE in both buffers
                    scanned += (unsigned long long)(e - s);
                }
            }
        }
        __syncthreads();  // stage `st` is free again
        if (t == 0) {
            sm.cid[st] = nxt;
            if (nxt < nchunks) {
                stage_chunk(a, sm, n, nxt, nb_s, nb_e, st);
                nxt = (long long)kStages * g_nact + atomicAdd(&a.ctl->chunk_ctr, 1u);
                load_bounds(a, n, nchunks, nxt, nb_s, nb_e);  // in flight during the next chunk
            }
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------------------
// hub phase: every listed row (deg > kHubDeg) is scanned by a whole CTA
// kCheck = false in round 1 (every vertex free), true for rescans after round k.
// ---------------------------------------------------------------------------------------
template <bool H>
__device__ __noinline__ void hub_phase(const MatchArgs &a, MatchSmem &sm, int32_t nhub, bool check, const int32_t *Pk,
                          int32_t *Pn, int32_t *Lnext, int32_t *live_next, unsigned long long &scanned) {
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    for (int i = blockIdx.x; i < nhub; i += g_nact) {
        const int32_t u = a.H[i];
        const int32_t s = __ldg(a.adjp + (u - a.vbase)), e = __ldg(a.adjp + (u - a.vbase) + 1);
        unsigned long long key = 0;
        for (int32_t j = s + threadIdx.x; j < e; j += kNT) {
            const int32_t x = ldArc(a.adjncy + j);
            if (!check || free_after(x, Pk)) key = umax64(key, pack_key<H>(a.tie_seed, ldArc(a.adjwgt + j), x));
        }
        key = group_max64<32>(key);
        if (lane == 0) sm.red[wib] = key;
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned long long k = 0;
            for (int q = 0; q < kNT / 32; ++q) k = umax64(k, sm.red[q]);
            const int32_t p = key_vertex<H>(a.tie_seed, k);
            Pn[u] = p;
            a.S[u] = kNone;
            if (p == kNone) {
                a.P[0][u] = kNone;
                a.P[1][u] = kNone;
            } else if (Lnext) {
                Lnext[atomicAdd(live_next, 1)] = u;
            }
            scanned += (unsigned long long)(e - s);
        }
        __syncthreads();
    }
}

// Multi-CTA hub phase (kMatchWhole): the listed rows are cut into chunks of kHC arcs and the
// chunks are dealt round-robin to all CTAs, so a 400 K-arc R-MAT hub is scanned by ~100 CTAs
// at once instead of one (each thread: 8 arcs, all loads of a level in flight).  Each chunk's
// best key goes to hk[hub] by a 64-bit global atomicMax; after a grid barrier the hubs'
// proposals are written (top-1 only: S = NONE for hubs, as in hub_phase).  Every CTA walks the
// hub list in segments of kNT hubs with a block scan of the chunk counts.
constexpr int kHC = kNT * 8;  // arcs per hub chunk
template <bool H>
__device__ __noinline__ void hub_phase_mc(const MatchArgs &a, MatchSmem &sm, int32_t nhub, bool check, const int32_t *Pk,
                             int32_t *Pn, int32_t *Lnext, int32_t *live_next, unsigned long long &scanned,
                             unsigned *bar, unsigned &bar_epoch, int nact) {
    const int t = threadIdx.x, lane = t & 31, wib = t >> 5;
    int32_t *hs = reinterpret_cast<int32_t *>(&sm.adj[0][0]);  // per segment: row start, end, chunk base
    int32_t *he = hs + kNT, *hb = he + kNT;
    long long carry = 0;  // chunks of earlier segments
    for (int32_t seg = 0; seg < nhub; seg += kNT) {
        const int32_t i = seg + t;
        int32_t rs = 0, re = 0, ch = 0;
        if (i < nhub) {
            const int32_t u = a.H[i];
            rs = __ldg(a.adjp + (u - a.vbase));
            re = __ldg(a.adjp + (u - a.vbase) + 1);
            ch = (re - rs + kHC - 1) / kHC;
            if (blockIdx.x == 0) scanned += (unsigned long long)(re - rs);
        }
        int32_t tot;
        const int32_t ex = block_excl_scan<kNT>(ch, sm.scratch, tot);
        hs[t] = rs;
        he[t] = re;
        hb[t] = ex;
        __syncthreads();
        const int32_t nseg = min(kNT, nhub - seg);
        // global chunk g = carry + local; this CTA takes g = b (mod nact)
        long long g0 = carry + (((long long)blockIdx.x - carry) % nact + nact) % nact;
        for (long long g = g0; g < carry + tot; g += nact) {
            const int32_t loc = (int32_t)(g - carry);
            int32_t r = 0;  // hub of chunk loc: the last with hb <= loc
            for (int step = kNT / 2; step > 0; step >>= 1)
                if (r + step < nseg && hb[r + step] <= loc) r += step;
            const int32_t c0 = hs[r] + (loc - hb[r]) * kHC, c1 = min(he[r], c0 + kHC);
            int32_t x[8], w[8], px[8];
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const int32_t j = c0 + q * kNT + t;
                x[q] = j < c1 ? ldArc(a.adjncy + j) : -1;
                w[q] = j < c1 ? ldArc(a.adjwgt + j) : 0;
            }
            unsigned long long key = 0;
            if (check) {
#pragma unroll
                for (int q = 0; q < 8; ++q) px[q] = x[q] >= 0 ? ldP(Pk + x[q]) : -1;
#pragma unroll
                for (int q = 0; q < 8; ++q) {
                    const int32_t pp = px[q] >= 0 ? ldP(Pk + px[q]) : -1;
                    if (x[q] >= 0 && pp != x[q]) key = umax64(key, pack_key<H>(a.tie_seed, w[q], x[q]));  // x free after round k
                }
            } else {
#pragma unroll
                for (int q = 0; q < 8; ++q)
                    if (x[q] >= 0) key = umax64(key, pack_key<H>(a.tie_seed, w[q], x[q]));
            }
            key = group_max64<32>(key);
            if (lane == 0) sm.red[wib] = key;
            __syncthreads();
            if (t == 0) {
                unsigned long long k = 0;
                for (int q = 0; q < kNT / 32; ++q) k = umax64(k, sm.red[q]);
                if (k) atomicMax(&a.hk[seg + r], k);
            }
            __syncthreads();
        }
        carry += tot;
        __syncthreads();  // hs/he/hb are rewritten by the next segment
    }
    grid_barrier(bar, bar_epoch, nact);
    // finalize: one thread per hub
    for (long long i = (long long)blockIdx.x * kNT + t; i < nhub; i += (long long)nact * kNT) {
        const int32_t u = a.H[i];
        const unsigned long long k = __ldcg(a.hk + i);
        const int32_t p = key_vertex<H>(a.tie_seed, k);
        Pn[u] = p;
        a.S[u] = kNone;
        if (p == kNone) {
            a.P[0][u] = kNone;
            a.P[1][u] = kNone;
        } else if (Lnext) {
            Lnext[atomicAdd(live_next, 1)] = u;
        }
    }
}

// ---------------------------------------------------------------------------------------
// phase k >= 1: commit of round k + proposals of round k+1 (lazy rescans)
// ---------------------------------------------------------------------------------------
// CTA-aggregated final flush of the warps' list queues: one global atomic per CTA.  All
// threads of the CTA call.
__device__ __forceinline__ void cta_flush(MatchSmem &sm, const int32_t *q, int32_t qn, int32_t *list,
                                          int32_t *counter) {
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    if (lane == 0) sm.scratch[wib] = qn;
    __syncthreads();
    if (wib == 0) {  // warp 0 scans the 16 queue lengths; one atomic for the CTA
        const int32_t c = lane < kNT / 32 ? sm.scratch[lane] : 0;
        int32_t inc = c;
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
            const int32_t t = __shfl_up_sync(0xffffffffu, inc, off);
            if (lane >= off) inc += t;
        }
        const int32_t tot = __shfl_sync(0xffffffffu, inc, 31);
        int32_t base = 0;
        if (lane == 0 && tot) base = atomicAdd(counter, tot);
        base = __shfl_sync(0xffffffffu, base, 0);
        if (lane < kNT / 32) sm.scratch[lane] = inc - c;
        if (lane == 0) sm.scratch[kNT / 32] = base;
    }
    __syncthreads();
    const int32_t base = sm.scratch[kNT / 32] + sm.scratch[wib];
    for (int i = lane; i < qn; i += 32) list[base + i] = q[i];
}

// Parking.  Under the rule a free vertex u keeps proposing its target p while
// p is free, so a "keep p" vertex leaves the live list (parked) until p matches; a handshake
// with p is then detected from p's side (a vertex whose proposal changed is always live in the
// next round).  When v matches in round k it becomes a wake task; after the round barrier the
// wake phase finds the vertices parked on v (P_k[x] == v and parked) and the resolve pass
// gives them their round-(k+1) proposals exactly as the live-list protocol would have (their
// target matched in round k: cached second choice or rescan), all within round k -- so the
// proposals, handshakes and round counts are the rule's.  Each x is parked on one vertex and
// each matched vertex is listed once (by itself, or by its live partner if it was parked).
__device__ __forceinline__ void park_match(const MatchArgs &a, int32_t *Pn, RoundSlot *, int k, int32_t u,
                                           int32_t p) {
    int32_t *nw = &a.ctl->nwake[k & 3];
    if (ldcg(a.parked + p)) {  // p is off the list: u also writes p's side (P_k[p] == u already)
        a.M[p] = u;
        Pn[p] = u;
        a.parked[p] = 0;
        if (ldcg(a.pcnt + p)) a.W[atomicAdd(nw, 1)] = p;
    }
    if (ldcg(a.pcnt + u)) a.W[atomicAdd(nw, 1)] = u;
}
__device__ __forceinline__ void park_keep(const MatchArgs &a, int32_t u, int32_t p) {
    a.parked[u] = 1;
    atomicAdd(&a.pcnt[p], 1);
}

// wake phase: the rows of the wake tasks in chunks of kHC arcs over all CTAs (as the hub phase)
constexpr int kWC = kNT * 8;
__device__ __noinline__ void wake_phase(const MatchArgs &a, MatchSmem &sm, int32_t nw, const int32_t *Pk,
                                        int32_t *nres, int nact) {
    const int t = threadIdx.x;
    int32_t *hs = reinterpret_cast<int32_t *>(&sm.adj[0][0]);
    int32_t *he = hs + kNT, *hb = he + kNT, *hv = hb + kNT;
    long long carry = 0;
    for (int32_t seg = 0; seg < nw; seg += kNT) {
        const int32_t i = seg + t;
        int32_t rs = 0, re = 0, ch = 0, v = -1;
        if (i < nw) {
            v = a.W[i];
            rs = __ldg(a.adjp + (v - a.vbase));
            re = __ldg(a.adjp + (v - a.vbase) + 1);
            ch = (re - rs + kWC - 1) / kWC;
        }
        int32_t tot;
        const int32_t ex = block_excl_scan<kNT>(ch, sm.scratch, tot);
        hs[t] = rs;
        he[t] = re;
        hb[t] = ex;
        hv[t] = v;
        __syncthreads();
        const int32_t nseg = min(kNT, nw - seg);
        const long long g0 = carry + (((long long)blockIdx.x - carry) % nact + nact) % nact;
        for (long long g = g0; g < carry + tot; g += nact) {
            const int32_t loc = (int32_t)(g - carry);
            int32_t r = 0;
            for (int step = kNT / 2; step > 0; step >>= 1)
                if (r + step < nseg && hb[r + step] <= loc) r += step;
            const int32_t c0 = hs[r] + (loc - hb[r]) * kWC, c1 = min(he[r], c0 + kWC), vv = hv[r];
            int32_t x[8], px[8];
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const int32_t j = c0 + q * kNT + t;
                x[q] = j < c1 ? ldArc(a.adjncy + j) : -1;
            }
#pragma unroll
            for (int q = 0; q < 8; ++q) px[q] = x[q] >= 0 ? ldP(Pk + x[q]) : -1;
#pragma unroll
            for (int q = 0; q < 8; ++q)
                if (px[q] == vv && ldcg(a.parked + x[q])) {  // parked on the matched vv: resolve it
                    a.parked[x[q]] = 0;
                    a.R[atomicAdd(nres, 1)] = x[q];
                }
        }
        carry += tot;
        __syncthreads();
    }
}

// Short live lists (small levels, late rounds): G lanes per live vertex, so a warp covers
// 32/G vertices and a rescan reads G*4 arcs per dependent step instead of 8 per thread.
// The round's critical path is then ~8 dependent loads whatever the row length (<= kHubDeg).
// Same decisions as phase_k_impl (commit / keep p / cached second choice / rescan).
template <int G, bool H>
__device__ void phase_k_lanes(const MatchArgs &a, MatchSmem &sm, int k, int32_t len, bool park, const int32_t *Lover,
                              unsigned long long &scanned, unsigned long long &rows, unsigned long long &visits,
                              int32_t &made) {
    constexpr int VPW = 32 / G;  // live vertices per warp step
    const int32_t *Pk = a.P[k & 1];
    int32_t *Pn = a.P[(k + 1) & 1];
    int32_t *Pkw = a.P[k & 1];
    const int32_t *Lk = Lover ? Lover : a.L[k & 1];
    int32_t *Ln = a.L[(k + 1) & 1];
    RoundSlot *next = &a.ctl->slot[(k + 1) & 3];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5, gl = lane % G;
    int32_t *q = reinterpret_cast<int32_t *>(&sm.adj[0][0]) + wib * kWQ;
    int32_t qn = 0;
    const long long ngroups = ((long long)len + VPW - 1) / VPW;
    const long long g_lo = ngroups * blockIdx.x / g_nact, g_hi = ngroups * (blockIdx.x + 1) / g_nact;
    if (threadIdx.x == 0) sm.claim = 0;
    __syncthreads();
    auto claim_next = [&]() -> long long {
        int c = 0;
        if (lane == 0) c = atomicAdd(&sm.claim, 1);
        c = __shfl_sync(0xffffffffu, c, 0);
        // interleaved (group c of CTA b = b + c * nact): a spatial cluster of rescans is
        // spread over all CTAs instead of landing on one; contiguous with GP_MATCH_CONTIG=1
        return a.interleave ? (long long)blockIdx.x + (long long)c * g_nact : g_lo + c;
    };
    for (long long g = claim_next(); g < (a.interleave ? ngroups : g_hi); g = claim_next()) {
        const long long idx = g * VPW + lane / G;
        int32_t u = idx < len ? ((k == 1 && !Lover) ? a.vbase + (int32_t)idx : ldP(Lk + idx)) : -1;
        const int32_t p = u >= 0 ? ldP(Pk + u) : kNone;
        const int32_t s2r = u >= 0 ? ldP(a.S + u) : kNone;  // not predicated on p: same load level
        const int32_t rs0 = u >= 0 ? __ldg(a.adjp + (u - a.vbase)) : 0;  // speculative row bounds
        const int32_t re0 = u >= 0 ? __ldg(a.adjp + (u - a.vbase) + 1) : 0;
        const int32_t s2 = p != kNone ? s2r : kNone;
        const int32_t qq = p != kNone ? ldP(Pk + p) : kNone;
        const int32_t ps = s2 != kNone ? ldP(Pk + s2) : -1;
        const int32_t rr = (p != kNone && qq != u && qq >= 0) ? ldP(Pk + qq) : -1;
        const int32_t pps = ps >= 0 ? ldP(Pk + ps) : -1;
        bool need = false, live = false;
        if (p != kNone) {
            if (gl == 0) ++visits;
            if (qq == u) {
                if (gl == 0) {
                    a.M[u] = p;  // handshake
                    Pn[u] = p;
                    if (park) park_match(a, Pn, next, k, u, p);
                    ++made;
                }
            } else if (rr != p) {
                if (gl == 0) {
                    Pn[u] = p;  // p still free: still the heaviest free neighbour
                    if (park) park_keep(a, u, p);
                }
                live = !park;
            } else if (s2 != kNone && pps != s2) {
                if (gl == 0) {
                    Pn[u] = s2;  // cached second choice still free
                    a.S[u] = kNone;
                }
                live = true;
            } else {
                need = true;
            }
        }
        int32_t s = 0, e = 0;
        if (need) {
            s = rs0;
            e = re0;
            if (e - s > g_hubdeg) {
                if (gl == 0) {
                    const int32_t h = atomicAdd(&next->nhub, 1);
                    a.H[h] = u;
                    if (a.hk) a.hk[h] = 0ull;  // (sharded launches: per-CTA hub_phase, no hk)
                }
                need = false;
                e = s;
            } else if (gl == 0) {
                ++rows;
                scanned += (unsigned long long)(e - s);
            }
        }
        // warp-uniform trip count keeps the width-G shuffles converged
        int32_t trips = need ? (e - s + 4 * G - 1) / (4 * G) : 0;
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) trips = max(trips, __shfl_xor_sync(0xffffffffu, trips, off));
        unsigned long long key = 0, key2 = 0;
        for (int t = 0; t < trips; ++t) {
            int32_t x[4], w[4], px[4], pp[4];
#pragma unroll
            for (int b = 0; b < 4; ++b) {
                const int32_t j = s + (t * 4 + b) * G + gl;
                x[b] = (need && j < e) ? ldArc(a.adjncy + j) : -1;
                w[b] = (need && j < e) ? ldArc(a.adjwgt + j) : 0;
            }
#pragma unroll
            for (int b = 0; b < 4; ++b) px[b] = x[b] >= 0 ? ldP(Pk + x[b]) : -1;
#pragma unroll
            for (int b = 0; b < 4; ++b) pp[b] = px[b] >= 0 ? ldP(Pk + px[b]) : -1;
#pragma unroll
            for (int b = 0; b < 4; ++b)
                if (x[b] >= 0 && pp[b] != x[b]) top2_add(key, key2, pack_key<H>(a.tie_seed, w[b], x[b]));  // x free after round k
        }
        if (trips > 0) group_top2<G>(key, key2);
        if (need && gl == 0) {
            const int32_t b = key_vertex<H>(a.tie_seed, key);
            Pn[u] = b;
            a.S[u] = key_vertex<H>(a.tie_seed, key2);
            if (b == kNone) Pkw[u] = kNone;  // dead: NONE in both buffers
            live = b != kNone;
        }
        wq_push(q, qn, Ln, &next->live, live && gl == 0, u);
    }
    cta_flush(sm, q, qn, Ln, &next->live);
}

// Warp-cooperative rescan of every row of a phase-k group that needs one (lazy rescan,
// DESIGN.md §4.2): the rows' arcs are flattened into one item space (warp scan of the
// degrees) and each lane takes kFB items per batch, so the dependent loads of ALL rows
// (arc -> P_k[x] -> P_k[P_k[x]]) are in flight together instead of one row after another.
// Top-2 per row of a batch with native 32-bit shared atomics, field by field (heaviest weight,
// then the best tie word at that weight; the same among the row's other keys; a 64-bit shared
// atomicMax would be a CAS loop).  Rows longer than one batch keep a running top-2 that the
// row's owner lane merges after every batch: every item is loaded ONCE (an earlier two-pass
// version re-ran the three dependent loads per batch for the second choice, which made the
// slowest warp of a round ~15 us on coarse levels).  Rows longer than kHubDeg go to the hub
// list.  All 32 lanes call; fq lives in the phase-0 staging buffers (idle in phase k).
constexpr int kFQ = 128;  // queue entries per warp (32 lanes x kVL <= 4)
constexpr int kFB = 8;    // flat items per lane per batch (256 per warp batch)
#ifndef GP_KFB1
#define GP_KFB1 8         // items per lane per batch of the kVL = 1 groups (build-time A/B)
#endif
struct FlatQ {
    unsigned long long a1[kFQ], a2[kFQ];          // running top-2 of rows spanning batches
    uint32_t w1[kFQ], n1[kFQ], w2[kFQ], n2[kFQ];  // the batch's top-2 per row: (weight, tie word)
    int32_t s[kFQ];                               // row start (arc index)
    int32_t off[kFQ + 2];                         // row offset in the flat item space
    uint8_t own[32 * (kFB > GP_KFB1 ? kFB : GP_KFB1)];  // queue entry of every item of the batch
};
// the queues live in adj[1..2], wgt[0..2] and ap[0..2] (contiguous in MatchSmem)
static_assert(sizeof(FlatQ) * (kNT / 32) <=
                  sizeof(int32_t) * ((kStages - 1) * kStageArcs + kStages * kStageArcs + kStages * (kMaxVch + 8)),
              "flat rescan queues must fit the idle phase-0 buffers");

__device__ __forceinline__ unsigned long long wn_key(uint32_t w, uint32_t n) {
    return w ? (((unsigned long long)w << 32) | n) : 0ull;
}

template <int kVL, bool H, int KFB = (kVL == 1 ? GP_KFB1 : 4)>
__device__ __forceinline__ void flat_rescan(const MatchArgs &a, MatchSmem &sm, const int32_t *Pk, int32_t *Pn,
                                            int32_t *Pkw, RoundSlot *next, const int32_t (&u)[kVL],
                                            bool (&need)[kVL], bool (&live)[kVL], unsigned long long &scanned,
                                            unsigned long long &rows, const int32_t (&rs)[kVL],
                                            const int32_t (&re)[kVL], int i0 = 0, int i1 = kVL) {
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    FlatQ &fq = *(reinterpret_cast<FlatQ *>(&sm.adj[1][0]) + wib);
    int32_t rpos[kVL];
    int32_t qn = 0, T = 0;
#pragma unroll
    for (int i = 0; i < kVL; ++i) {
        if (i < i0 || i >= i1) continue;  // (warp-uniform)
        int32_t d = need[i] ? re[i] - rs[i] : 0;
        if (need[i]) ++rows;
        if (need[i] && d > g_hubdeg) {
            const int32_t h = atomicAdd(&next->nhub, 1);
            a.H[h] = u[i];
            if (a.hk) a.hk[h] = 0ull;  // (sharded launches: per-CTA hub_phase, no hk)
            need[i] = false;
            d = 0;
        }
        const unsigned b = __ballot_sync(0xffffffffu, need[i]);
        const int32_t inc = warp_incl_scan(d);
        const int32_t tot = __shfl_sync(0xffffffffu, inc, 31);
        rpos[i] = qn + __popc(b & lanemask_lt());
        if (need[i]) {
            fq.s[rpos[i]] = rs[i];
            fq.off[rpos[i]] = T + inc - d;
            scanned += (unsigned long long)d;
        }
        qn += __popc(b);
        T += tot;
    }
    if (qn == 0) return;  // warp-uniform
    const bool multi = T > 32 * KFB;  // some row spans batches: running top-2 per row
    for (int r = lane; r < qn; r += 32) {
        fq.w1[r] = fq.n1[r] = fq.w2[r] = fq.n2[r] = 0u;
        if (multi) fq.a1[r] = fq.a2[r] = 0ull;
    }
    for (int32_t b0 = 0; b0 < T; b0 += 32 * KFB) {
        const int32_t bn = min(T - b0, 32 * KFB);
        // every queued row marks its items inside this batch with its entry
#pragma unroll
        for (int i = 0; i < kVL; ++i)
            if (i >= i0 && i < i1 && need[i]) {
                const int32_t o = fq.off[rpos[i]];
                const int32_t lo = max(o, b0), hi = min(o + (re[i] - rs[i]), b0 + bn);
                for (int32_t q = lo; q < hi; ++q) fq.own[q - b0] = (uint8_t)rpos[i];
            }
        __syncwarp();
        // three dependent load levels for KFB items per lane: arc, P_k[x], P_k[P_k[x]]
        int32_t x[KFB], w[KFB], px[KFB];
#pragma unroll
        for (int b = 0; b < KFB; ++b) {
            const int32_t f = b * 32 + lane;
            x[b] = -1;
            w[b] = 0;
            if (f < bn) {
                const int32_t r = fq.own[f];
                const int32_t j = fq.s[r] + (b0 + f - fq.off[r]);
                x[b] = ldArc(a.adjncy + j);
                w[b] = ldArc(a.adjwgt + j);
            }
        }
#pragma unroll
        for (int b = 0; b < KFB; ++b) px[b] = x[b] >= 0 ? ldP(Pk + x[b]) : -1;
        uint32_t t[KFB];  // tie word of a candidate (x free after round k), w = 0 otherwise
#pragma unroll
        for (int b = 0; b < KFB; ++b) {
            const int32_t pp = px[b] >= 0 ? ldP(Pk + px[b]) : -1;
            const bool cand = x[b] >= 0 && pp != x[b];
            t[b] = cand ? (uint32_t)pack_key<H>(a.tie_seed, w[b], x[b]) : 0u;
            if (!cand) w[b] = 0;
        }
#pragma unroll
        for (int b = 0; b < KFB; ++b)
            if (w[b]) atomicMax(&fq.w1[fq.own[b * 32 + lane]], (uint32_t)w[b]);
        __syncwarp();
#pragma unroll
        for (int b = 0; b < KFB; ++b) {
            const int r = w[b] ? fq.own[b * 32 + lane] : 0;
            if (w[b] && (uint32_t)w[b] == fq.w1[r]) atomicMax(&fq.n1[r], t[b]);
        }
        __syncwarp();
#pragma unroll
        for (int b = 0; b < KFB; ++b) {
            const int r = w[b] ? fq.own[b * 32 + lane] : 0;
            if (w[b] && (uint32_t)w[b] == fq.w1[r] && t[b] == fq.n1[r]) w[b] = 0;  // the batch's top: not a second
            else if (w[b]) atomicMax(&fq.w2[r], (uint32_t)w[b]);
        }
        __syncwarp();
#pragma unroll
        for (int b = 0; b < KFB; ++b) {
            const int r = w[b] ? fq.own[b * 32 + lane] : 0;
            if (w[b] && (uint32_t)w[b] == fq.w2[r]) atomicMax(&fq.n2[r], t[b]);
        }
        __syncwarp();
        if (multi) {  // the rows of this batch: owner lanes merge its top-2 into the running one
            const int r0 = fq.own[0], r1 = fq.own[bn - 1];
            for (int r = r0 + lane; r <= r1; r += 32) {
                const unsigned long long t1 = wn_key(fq.w1[r], fq.n1[r]), t2 = wn_key(fq.w2[r], fq.n2[r]);
                const unsigned long long A1 = fq.a1[r], A2 = fq.a2[r];
                const unsigned long long lo = A1 < t1 ? A1 : t1, m2 = A2 > t2 ? A2 : t2;
                fq.a1[r] = A1 > t1 ? A1 : t1;
                fq.a2[r] = lo > m2 ? lo : m2;
                fq.w1[r] = fq.n1[r] = fq.w2[r] = fq.n2[r] = 0u;
            }
            __syncwarp();
        }
    }
#pragma unroll
    for (int i = 0; i < kVL; ++i) {
        if (i >= i0 && i < i1 && need[i]) {
            const int32_t r = rpos[i];
            const unsigned long long k1 = multi ? fq.a1[r] : wn_key(fq.w1[r], fq.n1[r]);
            const unsigned long long k2 = multi ? fq.a2[r] : wn_key(fq.w2[r], fq.n2[r]);
            const int32_t bv = key_vertex<H>(a.tie_seed, k1);
            Pn[u[i]] = bv;
            a.S[u[i]] = key_vertex<H>(a.tie_seed, k2);
            if (bv == kNone) Pkw[u[i]] = kNone;  // dead: NONE in both buffers
            live[i] = bv != kNone;
        }
    }
    __syncwarp();  // fq is rebuilt by the warp's next group
}

// kVL live vertices per lane per step: their dependent loads overlap.  4 on long lists, 1 on
// short ones (a wide step would leave most warps idle).
// kStatic (small levels, <= 2 vertices per thread): the round walks ALL vertices of the level
// in place of the compacted live list; u is live iff M[u] is FREE and P_k[u] != NONE (matched
// vertices keep their partner in P, dead ones NONE), read at the same level as P_k[u].  No list
// load, no list append and no atomic with a return value on the round's critical path; the
// next round's live count is a fire-and-forget reduction.
// GP_PROF=2: cycle checkpoints of warp 0 of block 0 (first group of round k < 16)
// (compiled in only with -DGP_CHECKPOINTS: GP_NVCC_DEFS=-DGP_CHECKPOINTS for _build)
#ifdef GP_CHECKPOINTS
#define GP_CK(j)                                                                                   \
    do {                                                                                           \
        if (ck_on && threadIdx.x == 0) a.ctl->ck[k][j] = clock64() - ck0;                          \
    } while (0)
#define GP_CK_ON(expr) ck_on = (expr)
#define GP_CK_SINK(expr)                                                                           \
    do {                                                                                           \
        if (ck_on) {                                                                               \
            int32_t z_ = 0;                                                                        \
            for (int i_ = 0; i_ < kVL; ++i_) z_ += expr;                                          \
            if (z_ == -7777777) a.ctl->ck[15][11] = z_;                                            \
        }                                                                                          \
    } while (0)
#else
#define GP_CK(j) do { } while (0)
#define GP_CK_ON(expr) do { } while (0)
#define GP_CK_SINK(expr) do { } while (0)
#endif

template <bool H, int kVL, bool kStatic = false>
__device__ void phase_k_impl(const MatchArgs &a, MatchSmem &sm, int k, int32_t len, bool park, const int32_t *Lover,
                             unsigned long long &scanned, unsigned long long &rows, unsigned long long &visits,
                             int32_t &made, int vpg = 32) {
    // vpg (kVL = 1 only): live vertices per warp group.  Short live lists take 4..16 vertices
    // per warp so that more warps share the round, and the flat rescan still spreads a
    // group's arcs over all 32 lanes (the old per-vertex G-lane groups walked a long row
    // 4G arcs per dependent step).
    const int32_t *Pk = a.P[k & 1];
    int32_t *Pn = a.P[(k + 1) & 1];
    int32_t *Pkw = a.P[k & 1];
    const int32_t *Lk = Lover ? Lover : a.L[k & 1];
    int32_t *Ln = a.L[(k + 1) & 1];
    RoundSlot *next = &a.ctl->slot[(k + 1) & 3];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    int32_t *q = reinterpret_cast<int32_t *>(&sm.adj[0][0]) + wib * kWQ;  // phase 0 is over
    int32_t qn = 0;
    // CTA b owns the contiguous groups [g_lo, g_hi) of 32*kVL live entries; its warps claim
    // them from a shared-memory counter.  No global atomics on a shared address: thousands
    // of warps hitting one L2 atomic unit serialise (~0.5 ns each), which dominated the
    // rounds of small levels.
    const int gsz = kVL == 1 ? vpg : 32 * kVL;  // live entries per group
#ifdef GP_CHECKPOINTS
    bool ck_on = a.prof == 2 && blockIdx.x == 0 && threadIdx.x < 32 && k < 16;
    const long long ck0 = clock64();
#endif
    const long long ngroups = ((long long)len + gsz - 1) / gsz;
    const long long g_lo = ngroups * blockIdx.x / g_nact, g_hi = ngroups * (blockIdx.x + 1) / g_nact;
    if (threadIdx.x == 0) sm.claim = 0;
    __syncthreads();
    auto claim_next = [&]() -> long long {  // warp-uniform
        int c = 0;
        if (lane == 0) c = atomicAdd(&sm.claim, 1);
        c = __shfl_sync(0xffffffffu, c, 0);
        // interleaved (group c of CTA b = b + c * nact): a spatial cluster of rescans is
        // spread over all CTAs instead of landing on one; contiguous with GP_MATCH_CONTIG=1
        return a.interleave ? (long long)blockIdx.x + (long long)c * g_nact : g_lo + c;
    };
    for (long long g = claim_next(); g < (a.interleave ? ngroups : g_hi); g = claim_next()) {
        GP_CK(0);
        const long long base = g * gsz;
        int32_t u[kVL], p[kVL], s2[kVL], qq[kVL], rr[kVL], ps[kVL], pps[kVL];
        // level 1: the vertices; level 2: P_k[u] and the cached second candidate S[u]
#pragma unroll
        for (int i = 0; i < kVL; ++i) {
            const long long idx = base + i * 32 + lane;
            u[i] = (idx < len && (kVL > 1 || lane < gsz)) ? ((kStatic || (k == 1 && !Lover)) ? a.vbase + (int32_t)idx : ldP(Lk + idx)) : -1;
        }
        GP_CK_SINK(u[i_]);
        GP_CK(1);
        int32_t rs[kVL], re[kVL];  // row bounds, loaded speculatively with P_k[u]: a rescan
                                   // then starts one dependent level earlier
#pragma unroll
        for (int i = 0; i < kVL; ++i) {
            p[i] = u[i] >= 0 ? ldP(Pk + u[i]) : kNone;
            s2[i] = u[i] >= 0 ? ldP(a.S + u[i]) : kNone;  // not predicated on p: same load level
            rs[i] = u[i] >= 0 ? __ldg(a.adjp + (u[i] - a.vbase)) : 0;
            re[i] = u[i] >= 0 ? __ldg(a.adjp + (u[i] - a.vbase) + 1) : 0;
            if (kStatic && u[i] >= 0 && k > 1 && ldcg(a.M + u[i]) != kFree) p[i] = kNone;  // matched: not live
        }
#pragma unroll
        for (int i = 0; i < kVL; ++i)
            if (p[i] == kNone) s2[i] = kNone;
        GP_CK(2);
        // The freedom test of the cached candidate (P_k[s2], P_k[P_k[s2]]) is issued with the
        // test of p (same dependent levels) on latency-bound short lists; on long lists (kVL = 4:
        // the big levels, bound by the LSU's random-gather rate) only for the vertices whose
        // target p was matched by someone else, which saves two gathers for every vertex that
        // matches or keeps p (most of them).
        constexpr bool kSpecS = kVL < 4;
        // level 3: P_k[p] and P_k[s2] (freedom test of the cached candidate, P only)
#pragma unroll
        for (int i = 0; i < kVL; ++i) {
            qq[i] = p[i] != kNone ? ldP(Pk + p[i]) : kNone;
            ps[i] = (kSpecS && s2[i] != kNone) ? ldP(Pk + s2[i]) : -1;
        }
        // level 4: P_k[q] (did p match q?) and P_k[P_k[s2]]
#pragma unroll
        for (int i = 0; i < kVL; ++i) {
            rr[i] = (p[i] != kNone && qq[i] != u[i] && qq[i] >= 0) ? ldP(Pk + qq[i]) : -1;
            pps[i] = ps[i] >= 0 ? ldP(Pk + ps[i]) : -1;
        }
        if (!kSpecS) {  // deferred: only where p matched q != u this round
#pragma unroll
            for (int i = 0; i < kVL; ++i)
                ps[i] = (p[i] != kNone && qq[i] != u[i] && rr[i] == p[i] && s2[i] != kNone) ? ldP(Pk + s2[i]) : -1;
#pragma unroll
            for (int i = 0; i < kVL; ++i) pps[i] = ps[i] >= 0 ? ldP(Pk + ps[i]) : -1;
        }
        GP_CK_SINK(rr[i_] + pps[i_]);
        GP_CK(3);
        bool need[kVL], parked_now[kVL];
#pragma unroll
        for (int i = 0; i < kVL; ++i) {
            need[i] = false;
            parked_now[i] = false;
            if (p[i] == kNone) continue;
            ++visits;
            if (qq[i] == u[i]) {
                a.M[u[i]] = p[i];  // handshake: u and p propose each other
                Pn[u[i]] = p[i];
                if (park) park_match(a, Pn, next, k, u[i], p[i]);
                ++made;
                u[i] = -1;  // done
            } else if (rr[i] != p[i]) {
                Pn[u[i]] = p[i];  // p is still free: still the heaviest free neighbour
                if (park) {
                    park_keep(a, u[i], p[i]);
                    parked_now[i] = true;
                }
            } else if (s2[i] != kNone && pps[i] != s2[i]) {
                // the cached second-heaviest neighbour of u's last scan is still free: it is
                // now u's heaviest free neighbour (the free set only shrinks)
                Pn[u[i]] = s2[i];
                a.S[u[i]] = kNone;
            } else {
                need[i] = true;  // full rescan
            }
        }
        bool live[kVL];
#pragma unroll
        for (int i = 0; i < kVL; ++i) live[i] = u[i] >= 0 && p[i] != kNone && !need[i] && !parked_now[i];
        GP_CK(4);
        flat_rescan<kVL, H>(a, sm, Pk, Pn, Pkw, next, u, need, live, scanned, rows, rs, re);
        GP_CK(5);
        if (kStatic) {
#pragma unroll
            for (int i = 0; i < kVL; ++i) qn += live[i] ? 1 : 0;  // live count only
        } else {
#pragma unroll
            for (int i = 0; i < kVL; ++i) wq_push(q, qn, Ln, &next->live, live[i], u[i]);
        }
        GP_CK(6);
        GP_CK_ON(false);  // first group only
    }
    GP_CK_ON(a.prof == 2 && blockIdx.x == 0 && threadIdx.x < 32 && k < 16);
    GP_CK(7);
    if (kStatic) {
        const int32_t c = warp_sum(qn);
        if (lane == 0 && c) atomicAdd(&next->live, c);  // result unused: a RED, no round trip
    } else {
        cta_flush(sm, q, qn, Ln, &next->live);
    }
    GP_CK(8);
}
#undef GP_CK
#undef GP_CK_ON
#undef GP_CK_SINK

template <bool H>
__device__ void phase_k(const MatchArgs &a, MatchSmem &sm, int32_t n, int k, int32_t len, bool stat, bool park,
                        const int32_t *Lover, unsigned long long &scanned, unsigned long long &rows,
                        unsigned long long &visits, int32_t &made) {
    (void)n;
    unsigned long long t0 = 0, rows0 = rows;
    if (a.prof == 1) {
        if (threadIdx.x == 0) sm.tmax = 0;
        __syncthreads();
        t0 = globaltimer();
    }
    const long long threads = (long long)g_nact * kNT;
    if (stat) {
        if ((long long)len > threads) phase_k_impl<H, 2, true>(a, sm, k, len, false, nullptr, scanned, rows, visits, made);
        else phase_k_impl<H, 1, true>(a, sm, k, len, false, nullptr, scanned, rows, visits, made);
    } else if ((long long)len >= 4LL * threads) phase_k_impl<H, 4>(a, sm, k, len, park, Lover, scanned, rows, visits, made);
    else if (a.lanes_mode == 0 || (long long)len * 2 > threads) phase_k_impl<H, 1>(a, sm, k, len, park, Lover, scanned, rows, visits, made);
    else if (a.lanes_mode == 2) {  // short lists: 4..16 vertices per warp, flat rescans over all 32 lanes
        const int vpg = (long long)len * 8 <= threads ? 4 : (long long)len * 4 <= threads ? 8 : 16;
        phase_k_impl<H, 1>(a, sm, k, len, park, Lover, scanned, rows, visits, made, vpg);
    }
    else if ((long long)len * 8 <= threads) phase_k_lanes<8, H>(a, sm, k, len, park, Lover, scanned, rows, visits, made);
    else if ((long long)len * 4 <= threads) phase_k_lanes<4, H>(a, sm, k, len, park, Lover, scanned, rows, visits, made);
    else phase_k_lanes<2, H>(a, sm, k, len, park, Lover, scanned, rows, visits, made);
    if (a.prof == 1 && k < 16) {  // one shared atomic per warp, one global atomic per CTA
        const unsigned long long dt = globaltimer() - t0;
        const int32_t dr = warp_sum((int32_t)(rows - rows0));
        if ((threadIdx.x & 31) == 0) {
            atomicMax(&sm.tmax, dt);
            if (dr) atomicAdd(&sm.trows, dr);
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            atomicMax(&a.ctl->wmax[k], sm.tmax);
            if (sm.trows) atomicAdd(&a.ctl->trows[k], sm.trows);
            sm.trows = 0;
            if (blockIdx.x == 0) a.ctl->lens[k] = len;
        }
    }
}

template <bool H>
__global__ void __launch_bounds__(kNT, 2) k_match_level(const __grid_constant__ MatchArgs a) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    // 128-byte alignment by POINTER arithmetic on the __shared__ symbol: the compiler keeps the
    // shared address space (LDS/STS/ATOMS); an integer round trip made every access generic
    MatchSmem &sm = *reinterpret_cast<MatchSmem *>(smem_raw + ((128u - (unsigned)__cvta_generic_to_shared(smem_raw)) & 127u));
    MatchCtl *ctl = a.ctl;
    const volatile SizeRec *in = a.in;
    if (in->stop) return;  // an earlier level ended the coarsening: nothing to do
    const int32_t n = in->n;
    if (n <= 0) return;
    {
        const long long want = ((long long)n + a.vpc - 1) / a.vpc;
        const int nact = (int)(want < 1 ? 1 : (want < (long long)gridDim.x ? want : (long long)gridDim.x));
        if ((int)blockIdx.x >= nact) return;  // retired: this level is too small for it
        if (threadIdx.x == 0) {
            g_nact = nact;
            g_hubdeg = (n <= a.hub_small_n && a.hub_deg_small > 0 && a.hub_deg_small < kHubDeg) ? a.hub_deg_small : kHubDeg;
        }
        __syncthreads();
    }
    unsigned long long scanned = 0, rows = 0, visits = 0;
    if (threadIdx.x == 0) sm.trows = 0;  // GP_PROF counter (published after the first barrier)
    unsigned bar_epoch = 0;  // grid barriers passed (thread 0)
    int tr = 0;
    if (a.mode == kMatchWhole || a.mode == kMatchPhase0) {
        trace_mark(ctl->trace, tr++);
        phase0<H>(a, sm, n, scanned);
        trace_mark(ctl->trace, tr++);
        grid_barrier(ctl->bar, bar_epoch, g_nact);
        trace_mark(ctl->trace, tr++);
        const int32_t nh = *(volatile int32_t *)&ctl->slot[1].nhub;
        if (nh > 0) {
            if (a.mode == kMatchWhole) {
                hub_phase_mc<H>(a, sm, nh, false, a.P[0], a.P[1], nullptr, nullptr, scanned, ctl->bar, bar_epoch, g_nact);
                grid_barrier(ctl->bar, bar_epoch, g_nact);
            } else {
                hub_phase<H>(a, sm, nh, false, a.P[0], a.P[1], nullptr, nullptr, scanned);
            }
        }
    }
    int32_t rounds = 0, maximal = 0;
    const int nact_all = g_nact;  // CTAs of this launch (g_nact drops to 1 in the tail)
    bool tail = false;            // CTA 0 alone runs the remaining (short) rounds
    int32_t known_len = -1;       // next round's live-list length, read at the end of a round
    // small level: every round walks all vertices (kStatic), at most 2 per thread
    const bool stat = a.mode == kMatchWhole && a.static_mode && (long long)n <= 2LL * nact_all * kNT;
    const bool park = a.mode == kMatchWhole && !stat && a.parked != nullptr;
    if (a.mode == kMatchWhole || a.mode == kMatchRound) {
        // kMatchWhole: the device-side round loop; kMatchRound: round a.k only (the sharded
        // driver exchanges the boundary proposals between launches and decides termination)
        for (int k = (a.mode == kMatchRound) ? a.k : 1;; ++k) {
            if (k > n + 2 && a.mode == kMatchWhole) __trap();  // each round matches >= 1 pair
            if (blockIdx.x == 0 && threadIdx.x == 0) {
                RoundSlot *z = &ctl->slot[(k + 2) & 3];  // last read two phases ago
                z->live = 0;
                z->nhub = 0;
                z->matches = 0;
                z->claim = 0;
                ctl->nwake[(k + 2) & 3] = 0;
                ctl->nres[(k + 2) & 3] = 0;
            }
            const int32_t len = (k == 1 || stat) ? n : known_len >= 0 ? known_len : *(volatile int32_t *)&ctl->slot[k & 3].live;
            int32_t made = 0;
            phase_k<H>(a, sm, n, k, len, stat, park, nullptr, scanned, rows, visits, made);
            // any match this round: one flag store per CTA (only "> 0" is used)
            if (__syncthreads_or(made > 0) && threadIdx.x == 0) *(volatile int32_t *)&ctl->slot[k & 3].matches = 1;
            trace_mark(ctl->trace, tr++);
            const bool bprof = a.prof == 1 && k < 16 && !tail;
            if (bprof) {
                __syncthreads();
                if (threadIdx.x == 0) {
                    const unsigned long long t = globaltimer();
                    atomicMax(&ctl->barr[k][0], ~t);
                    atomicMax(&ctl->barr[k][1], t);
                }
            }
            if (tail) __syncthreads();  // one CTA: the block barrier orders the round
            else grid_barrier(ctl->bar, bar_epoch, nact_all);
            if (bprof && threadIdx.x == 0) atomicMax(&ctl->barr[k][2], globaltimer());
            trace_mark(ctl->trace, tr++);
            // the next slot {live, nhub} and this round's match flag: two independent loads
            // in flight together (one L2 round trip instead of three)
            int4 nxt = ld_volatile_v4(reinterpret_cast<const int4 *>(&ctl->slot[(k + 1) & 3]));
            const int32_t made_any = *(volatile int32_t *)&ctl->slot[k & 3].matches;
            if (park) {
                const int32_t nw = *(volatile int32_t *)&ctl->nwake[k & 3];
                if (nw > 0) {  // wake phase + resolve pass, still round k (see park_match)
                    wake_phase(a, sm, nw, a.P[k & 1], &ctl->nres[k & 3], g_nact);
                    if (tail) __syncthreads();
                    else grid_barrier(ctl->bar, bar_epoch, nact_all);
                    const int32_t nr = *(volatile int32_t *)&ctl->nres[k & 3];
                    if (nr > 0) {
                        int32_t made2 = 0;
                        phase_k<H>(a, sm, n, k, nr, false, true, a.R, scanned, rows, visits, made2);
                        if (tail) __syncthreads();
                        else grid_barrier(ctl->bar, bar_epoch, nact_all);
                    }
                    nxt = ld_volatile_v4(reinterpret_cast<const int4 *>(&ctl->slot[(k + 1) & 3]));
                }
            }
            int32_t live = nxt.x;
            if (nxt.y > 0) {
                if (a.mode == kMatchWhole && !tail)
                    hub_phase_mc<H>(a, sm, nxt.y, true, a.P[k & 1], a.P[(k + 1) & 1], a.L[(k + 1) & 1],
                                 &ctl->slot[(k + 1) & 3].live, scanned, ctl->bar, bar_epoch, nact_all);
                else
                    hub_phase<H>(a, sm, nxt.y, true, a.P[k & 1], a.P[(k + 1) & 1], a.L[(k + 1) & 1],
                              &ctl->slot[(k + 1) & 3].live, scanned);
                if (tail) __syncthreads();
                else grid_barrier(ctl->bar, bar_epoch, nact_all);
                live = *(volatile int32_t *)&ctl->slot[(k + 1) & 3].live;  // hub rows may stay live
            }
            if (a.mode == kMatchRound) break;
            if (made_any > 0) ++rounds;
            known_len = live;
            if (live == 0) {
                maximal = 1;
                break;
            }
            if (a.max_rounds > 0 && rounds >= a.max_rounds) break;
            // short live list: the grid barriers (not the work) would dominate the remaining
            // rounds, so CTA 0 finishes them alone; the others wait at the barrier below
            // (not with parking: the list then holds only the changed vertices while many may
            // still be parked, and their wake/resolve passes need the whole grid)
            if (!stat && !park && !tail && nact_all > 1 && live <= a.tail_live) {
                tail = true;
                if (blockIdx.x != 0) break;
                __syncthreads();
                if (threadIdx.x == 0) g_nact = 1;
                __syncthreads();
            }
        }
        if (tail) {
            __syncthreads();
            if (threadIdx.x == 0) g_nact = nact_all;
            grid_barrier(ctl->bar, bar_epoch, nact_all);  // CTA 0's rounds are done
        }
    }
    trace_mark(ctl->trace, tr++);
    if (a.leftover && (a.mode == kMatchWhole || a.mode == kMatchFinish)) {
        for (long long u = (long long)blockIdx.x * kNT + threadIdx.x; u < n; u += (long long)g_nact * kNT)
            if (a.M[a.vbase + u] == kFree) a.M[a.vbase + u] = a.vbase + (int32_t)u;
    }
    scanned = warp_sum64(scanned);
    rows = warp_sum64(rows);
    visits = warp_sum64(visits);
    if ((threadIdx.x & 31) == 0) {
        sm.cnt3[0][threadIdx.x >> 5] = scanned;
        sm.cnt3[1][threadIdx.x >> 5] = rows;
        sm.cnt3[2][threadIdx.x >> 5] = visits;
    }
    __syncthreads();
    if (threadIdx.x < 3) {  // one atomic per CTA and counter
        unsigned long long t = 0;
        for (int w = 0; w < kNT / 32; ++w) t += sm.cnt3[threadIdx.x][w];
        if (t) atomicAdd(threadIdx.x == 0 ? &ctl->arcs_scanned : threadIdx.x == 1 ? &ctl->rows_scanned : &ctl->live_visits, t);
    }
    if (blockIdx.x == 0 && threadIdx.x == 0 && a.mode == kMatchWhole) {
        ctl->rounds = rounds;
        ctl->maximal = maximal;
    }
}

// ---------------------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------------------
static int choose_group(double avg_deg) {
    // lanes per vertex in phase 0.  The rows come from shared memory, so a thread per row is
    // cheapest in instructions (no 64-bit top-2 shuffles) up to ~12 arcs per row.
    if (avg_deg <= 12.0) return 1;
    if (avg_deg <= 24.0) return 2;
    if (avg_deg <= 48.0) return 4;
    return 8;
}

static int32_t match_vpc() {
    static int32_t v = -1;
    if (v < 0) {
        const char *e = getenv("GP_MATCH_VPC");  // tuning knob (results never depend on it)
        v = e ? atoi(e) : 512;  // r2 sweep (C3: 3.31 ms at 128, 3.30 at 256, 3.24 at 512, 3.26 at 768)
        if (v < 1) v = 1;
    }
    return v;
}

int match_grid(Ctx *ctx) {
    // per device: cudaFuncSetAttribute applies to the current device (the ctx's, DeviceGuard)
    static int per_sm_dev[kMaxDevices] = {0};
    int dummy = -1;
    int &per_sm = (ctx->device >= 0 && ctx->device < kMaxDevices) ? per_sm_dev[ctx->device] : dummy;
    if (per_sm <= 0) {
        int b = 0;
        cudaFuncSetAttribute(k_match_level<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(MatchSmem) + 128);
        cudaFuncSetAttribute(k_match_level<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(MatchSmem) + 128);
        int b1 = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_match_level<false>, kNT, sizeof(MatchSmem) + 128);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b1, k_match_level<true>, kNT, sizeof(MatchSmem) + 128);
        if (b1 < b) b = b1;  // one persistent grid size for both instantiations
        per_sm = b > 0 ? (b > 2 ? 2 : b) : 1;
    }
    return ctx->num_sms * per_sm;
}

gp_status enqueue_match(Ctx *ctx, const LevelBufs &lb, int32_t *M, MatchCtl *ctl, int32_t max_rounds,
                        bool leftover, double avg_deg_hint, int32_t vbase, int mode, int k) {
    MatchArgs a;
    a.vbase = vbase;
    a.mode = mode;
    a.k = k;
    a.in = lb.in;
    a.adjp = lb.adjp;
    a.adjncy = lb.adjncy;
    a.adjwgt = lb.adjwgt;
    a.M = M;
    a.P[0] = lb.P[0];
    a.P[1] = lb.P[1];
    a.L[0] = lb.L[0];
    a.L[1] = lb.L[1];
    a.H = lb.H;
    a.S = lb.S;
    a.hk = lb.gkeys;  // idle while a level matches (the contraction's hub-row scratch, >= nnz keys)
    {
        static int pk = -1;
        if (pk < 0) {
            const char *e = getenv("GP_MATCH_PARK");  // tuning knob (results never depend on it)
            pk = (e && atoi(e) == 1) ? 1 : 0;
        }
        const bool on = pk && mode == kMatchWhole && lb.cnt && lb.lofs && lb.huge && lb.seg;
        a.parked = on ? lb.cnt : nullptr;  // contraction scratch, idle while matching
        a.pcnt = on ? lb.lofs : nullptr;
        a.W = on ? lb.huge : nullptr;
        a.R = on ? reinterpret_cast<int32_t *>(lb.seg) : nullptr;
    }
    a.ctl = ctl;
    a.max_rounds = max_rounds;
    a.tie_seed = ctx->tie_seed;
    a.leftover = leftover ? 1 : 0;
    a.G = choose_group(avg_deg_hint);
    {
        const char *e1 = getenv("GP_HUB_DEG_SMALL"), *e2 = getenv("GP_HUB_SMALL_N");  // tuning knobs
        a.hub_deg_small = e1 ? atoi(e1) : kHubDeg;
        a.hub_small_n = e2 ? atoi(e2) : 0;
    }
    a.vpc = match_vpc();
    {
        static int lm = -1;
        if (lm < 0) {
            const char *e = getenv("GP_MATCH_LANES");  // tuning knob (results never depend on it)
            lm = e ? atoi(e) : 1;
        }
        a.lanes_mode = lm;
        static int tl = -1;
        if (tl < 0) {
            const char *e = getenv("GP_TAIL_LIVE");  // tuning knob (results never depend on it)
            tl = e ? atoi(e) : 2048;
        }
        a.tail_live = tl;
        static int il = -1;
        if (il < 0) {
            const char *e = getenv("GP_MATCH_CONTIG");  // tuning knob (results never depend on it)
            il = (e && atoi(e) == 1) ? 0 : 1;
        }
        a.interleave = il;
        static int pf = -1;
        if (pf < 0) {
            const char *e = getenv("GP_PROF");
            pf = e ? atoi(e) : 0;
        }
        a.prof = pf;
        static int sm = -1;
        if (sm < 0) {
            const char *e = getenv("GP_MATCH_STATIC");  // tuning knob (results never depend on it)
            sm = (e && atoi(e) == 1) ? 1 : 0;  // measured neutral on C3 (3.41 ms both): off
        }
        a.static_mode = sm;
    }
    {
        // vertices per chunk: ~80 % of a stage at the average degree, a multiple of the
        // number of vertex groups (kNT / G) so that no group pass runs mostly idle
        const double d = avg_deg_hint > 0.5 ? avg_deg_hint : 0.5;
        const int ng = kNT / a.G;
        int v = (int)(0.8 * kStageArcs / d);
        v = v >= ng ? (v / ng) * ng : (v / 32) * 32;
        a.vch = v < 32 ? 32 : (v > kMaxVch ? kMaxVch : v);
    }
    void *args[] = {&a};
    LaunchScope ls(ctx, GP_K_PROPOSE);
    GP_CUDA(cudaLaunchCooperativeKernel(a.tie_seed ? (const void *)k_match_level<true> : (const void *)k_match_level<false>, dim3(match_grid(ctx)), dim3(kNT), args,
                                        sizeof(MatchSmem) + 128, ctx->stream));
    ++ctx->launches;
    return GP_OK;
}

}  // namespace gp
