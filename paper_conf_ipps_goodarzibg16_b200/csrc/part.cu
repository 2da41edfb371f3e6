// part.cu -- the partitioned grid tail: every remaining level -- matching
// rounds, cmap, contraction, coarse CSR -- in ONE persistent cooperative launch over all SMs,
// once the level fits the SMs' combined shared memory.
//
// Why (PAPER.md P16.s6-7, P20.s28-33): the paper hands the small levels to the CPU because the
// GPU's per-round fixed costs dominate there.  On B200 the medium levels (C3 levels 4-11:
// 430 K .. 65 K vertices) cost ~12 us per round in the level kernels, ~10 dependent L2 round
// trips of the slowest warp plus the grid barrier, and ~55 us per contraction, for a few MB of
// data.  Here every CTA (one per SM) owns a contiguous vertex range [lo, hi) balanced on
// 2*arcs + 5*vertices, keeps its rows in shared memory and refreshes a WINDOW of the proposal
// array P (its own range plus the halo its arcs reach, two hops wide) from global memory once
// per round: every gather of a round is a shared-memory load, and a round is one grid barrier,
// one coalesced window load and shared-memory work.  Ids outside the window (graphs without id
// locality) are read from global memory: results never depend on it.
//
// Same rule and outputs as the level kernels (match.cu, contract.cu; R1-R17):
//   rounds:   every free vertex proposes its heaviest free neighbour (ties: lower id, or lower
//             h_s(v) with a tie seed); mutual proposals match (P18.s7-12 with the handshake);
//             until no free vertex has a free neighbour, or max_rounds; leftover self-match
//             (P18.s12-13).  Round k+1's proposals are fused with round k's commit: P_k is
//             read-only during the phase, "x free after round k" = not (P_k[x] >= 0 and
//             P_k[P_k[x]] == x) (a matched vertex holds its partner in both parity buffers);
//             a free vertex keeps its target while the target stays free (the free set only
//             shrinks), else it rescans its row.
//   cmap:     leaders u <= M[u] numbered in id order (per-CTA counts, prefix over CTAs), the
//             leader writes its partner's CM (P18.s16-27, R7); cvwgt = vwgt[u] + vwgt[M[u]].
//   contract: coarse row c = rows of u and M[u] through CM, the collapsed edge dropped (R9),
//             repeated coarse neighbours summed (R8), sorted by coarse id (R10).  Two passes
//             (count, then re-merge and write at the row's final offset): rows <= 16 entries
//             by one thread (register network), <= 64 by one warp (register bitonic), longer
//             <= 256 by one warp (bitonic in shared memory), longer by the whole CTA (in shared memory, or in the global staging beyond 4096).
//   stop:     stall, threshold, max_levels exactly as k_contract_level (R12, R13).
// The next level's partition bounds are found by the threads that write the coarse row
// offsets, so a level starts without a search.
#include <cuda_runtime.h>
#include <stdlib.h>

#include "device_util.cuh"
#include "gp_internal.cuh"
#include "merge_util.cuh"
#include "sort_util.cuh"

namespace gp {

constexpr int kPT = 512;             // threads per CTA (128 registers: no spills)
constexpr int kPW = kPT / 32;        // warps per CTA
constexpr int kMaxParts = 256;       // grid cap (one CTA per SM)
#ifndef GP_PART_PB
#define GP_PART_PB 4
#endif
constexpr int kPB = GP_PART_PB;      // arcs per rescan step (loads issued together)
constexpr int kPKeys = 4096;         // keys of a CTA-merged row staged in shared memory (256 per warp)
constexpr size_t kPartDyn = 216 * 1024;  // dynamic shared memory per CTA
constexpr int32_t kPartBudget = (int32_t)((kPartDyn - kPKeys * 8) / 4);  // words for the level arrays
constexpr unsigned long long kPPad = ~0ull;  // sort padding / dropped collapsed edge

struct PartLevelOut {  // one arena slot (same layout as small.cu's SmallLevelOut)
    int32_t *M, *CM, *cadjp, *cadjncy, *cadjwgt, *cvwgt;
};

struct PartCtl {  // zeroed before the launch
    unsigned bar;                  // grid barrier arrivals (cumulative over the launch)
    unsigned pad[3];
    int32_t ring[4][4];            // by global phase g & 3: {live of round g, pairs of round g}
    int32_t bnd[kMaxParts + 1];    // partition bounds of the next level
    int32_t nL[kMaxParts];         // leaders per CTA
    int32_t nA[kMaxParts];         // merged entries per CTA
};

struct PartArgs {
    const SizeRec *in;  // sizes + stop flag of the first level's input graph
    const int32_t *adjp, *adjncy, *adjwgt, *vwgt;  // the first level's input graph
    PartLevelOut *slots;
    int32_t nslots, level0;
    LevelDev *levdev;
    LevelReport *reports;
    int32_t threshold, stall_pct, max_levels, max_rounds;
    uint32_t tie_seed;
    int32_t *P0, *P1;                // proposals by round parity (cap_n each)
    unsigned long long *wkeys;       // staging of CTA-merged rows longer than kPKeys (cap_nnz)
    PartCtl *ctl;
    int32_t wmin;                    // words of work per active CTA (fewer CTAs on small levels)
    int32_t force_garcs;             // test knob: arcs always read from global memory
    int32_t wcap_max;                // test knob: window capacity cap (words; 0 = none)
    int32_t force_gstage;            // test knob: contraction staging in global memory
    int32_t cap_n, cap_nnz;          // slot / staging capacities (the first level's bounds)
    int32_t prof;                    // GP_PROF=1: slowest CTA per round / contraction step
    int32_t trace;                   // GP_DEBUG: phase timestamps of block 0 (globaltimer reads cost)
};

__device__ __forceinline__ int32_t pld(const int32_t *p) { return __ldcg(p); }
// GP_PART_CHECK builds: every shared / staging / output index is range-checked (a violation
// prints and traps) -- the memory-safety check of this kernel where compute-sanitizer is not
// available (tests run under it: scripts/part_checked.sh)
#ifdef GP_PART_CHECK
#define PCHK(cond, what, v)                                                                        \
    do {                                                                                           \
        if (!(cond)) {                                                                             \
            printf("k_part check failed: %s (%lld) block %d thread %d\n", what, (long long)(v),    \
                   (int)blockIdx.x, (int)threadIdx.x);                                             \
            __trap();                                                                              \
        }                                                                                          \
    } while (0)
#else
#define PCHK(cond, what, v) do { } while (0)
#endif
// v, or *gp (ld.global.cg) when useg: a predicated load instead of a branch
__device__ __forceinline__ int32_t ld_or(int32_t v, const int32_t *gp, bool useg) {
    asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.global.cg.s32 %0, [%1];\n\t}"
        : "+r"(v)
        : "l"(gp), "r"((unsigned)useg));
    return v;
}

// grid barrier over the nact CTAs still running (the count only grows: a barrier completes at
// the running sum of the participants of all barriers so far)
__device__ __forceinline__ void pbar(unsigned *bar, unsigned &target, int nact) {
    __syncthreads();
    if (threadIdx.x == 0) {
        target += (unsigned)nact;
        red_release_add_u32(bar, 1u);
        const long long g = spin_start();
        while ((int)(ld_acquire_u32(bar) - target) < 0) spin_check(g);
    }
    __syncthreads();
}

// The end of a round phase: the CTA's live / pair counts (warp sums, then thread 0) go into the
// round ring (live of the next round, pairs of this one; slot g + 2 is reset for reuse), then
// the grid barrier -- one CTA barrier for both.
__device__ __forceinline__ void round_bar(PartCtl *ctl, unsigned &target, int nact, int32_t g, int32_t live,
                                          int32_t pairs, int32_t *s) {
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    live = warp_sum(live);
    pairs = warp_sum(pairs);
    if (l == 0) {
        s[w] = live;
        s[kPW + w] = pairs;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        int32_t lt = 0, pt = 0;
        for (int q = 0; q < kPW; ++q) {
            lt += s[q];
            pt += s[kPW + q];
        }
        if (lt) atomicAdd(&ctl->ring[(g + 1) & 3][0], lt);
        if (pt) atomicAdd(&ctl->ring[g & 3][1], pt);
        if (blockIdx.x == 0) {
            ctl->ring[(g + 2) & 3][0] = 0;
            ctl->ring[(g + 2) & 3][1] = 0;
        }
        target += (unsigned)nact;
        red_release_add_u32(&ctl->bar, 1u);
        const long long g0 = spin_start();
        while ((int)(ld_acquire_u32(&ctl->bar) - target) < 0) spin_check(g0);
    }
    __syncthreads();
}

// CTAs for a level of W = 2*nnz + 5*n words: at least wmin words each, at most the grid
__device__ __forceinline__ int part_nact(int32_t n, int32_t nnz, int32_t wmin) {
    const long long W = 2LL * nnz + 5LL * n;
    long long k = (W + wmin - 1) / wmin;
    if (k < 1) k = 1;
    return (int)(k < (long long)gridDim.x ? k : (long long)gridDim.x);
}

// max{c in [0, n] : 2*adjp[c] + 5*c <= T}: a 512-ary search (3 dependent probes up to 2^27)
__device__ int32_t part_search(const int32_t *adjp, int32_t n, long long T) {
    int32_t lo = 0, hi = n + 1;  // invariant: W(lo) <= T < W(hi) (W(n + 1) = +inf)
    while (hi - lo > 1) {
        const int32_t step = (hi - lo + kPT - 1) / kPT;
        const int32_t c = lo + threadIdx.x * step;
        const bool ok = c < hi && c <= n && 2LL * pld(adjp + c) + 5LL * c <= T;
        const int cnt = __syncthreads_count(ok);  // W increasing: the true probes are a prefix
        const int32_t nlo = lo + (cnt - 1) * step;
        const int32_t nhi = lo + cnt * step;
        lo = nlo;
        hi = nhi < hi ? nhi : hi;
    }
    return lo;
}

// block reduction of three counters (all threads call; s holds >= 3 * kPW entries)
__device__ __forceinline__ void block_sum3(unsigned long long &x, unsigned long long &y, unsigned long long &z,
                                           unsigned long long *s) {
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    x = warp_sum64(x);
    y = warp_sum64(y);
    z = warp_sum64(z);
    if (l == 0) {
        s[w] = x;
        s[kPW + w] = y;
        s[2 * kPW + w] = z;
    }
    __syncthreads();
    x = y = z = 0;
    for (int q = 0; q < kPW; ++q) {
        x += s[q];
        y += s[kPW + q];
        z += s[2 * kPW + q];
    }
    __syncthreads();
}

// one CTA's view of its level
struct PartView {
    int32_t n, lo, hi, nv, a0, na;
    bool garcs;                          // arcs read from global memory (did not fit)
    const int32_t *gadjp, *gadjncy, *gadjwgt;
    // shared memory: sap = adjp[lo & ~3 ..] (16-byte aligned TMA copy, loff = lo & 3), sadj /
    // swgt = adjncy / adjwgt[a0 & ~3 ..] (aoff = a0 & 3), M / cnt per own vertex, the window
    int32_t *sap, *M, *cnt, *sadj, *swgt, *win;
    int32_t loff, aoff;
    int32_t wlo, wlen;
    // contraction staging in shared memory (after the window) when it fits: row i's merged
    // entries at sst[cnt[i]] (cnt holds the rows' upper-bound offsets while merging)
    unsigned long long *sst;
    bool sstage;
    int32_t sstot;   // staging entries (upper bounds) in shared memory (checks)
    int32_t capnnz;  // global staging / output capacity (checks)
    // row start of own vertex i relative to a0 (i in [0, nv])
    __device__ __forceinline__ int32_t rs(int32_t i) const {
        PCHK(i >= 0 && i <= nv, "row index", i);
        return sap[i + loff] - a0;
    }
    __device__ __forceinline__ int32_t arc(int32_t j) const {
        PCHK(j >= 0 && j < na, "arc index", j);
        return garcs ? pld(gadjncy + a0 + j) : sadj[j + aoff];
    }
    __device__ __forceinline__ int32_t wgt(int32_t j) const {
        PCHK(j >= 0 && j < na, "arc index", j);
        return garcs ? pld(gadjwgt + a0 + j) : swgt[j + aoff];
    }
    // window lookup of a global array g (P_k or CM) at x
    // branch-free: the shared load always issues (at index 0 when outside), the global load is
    // predicated -- a branch per lookup serialised the unrolled lookups of a row (no ILP)
    __device__ __forceinline__ int32_t wget(const int32_t *g, int32_t x) const {
        const unsigned d = (unsigned)(x - wlo);
        const bool out = d >= (unsigned)wlen;
        return ld_or(win[out ? 0u : d], g + x, out);
    }
};

// heaviest neighbour of own vertex i that is free after round k (k = 0: every neighbour):
// kPB arcs per step with all their loads issued together
template <bool H>
__device__ __forceinline__ int32_t part_best(const PartView &V, const int32_t *Pk, uint32_t seed, int32_t i,
                                             bool test_free) {
    unsigned long long best = 0;
    const int32_t s0 = V.rs(i), e0 = V.rs(i + 1);
    for (int32_t j0 = s0; j0 < e0; j0 += kPB) {
        int32_t x[kPB], w[kPB];
        bool f[kPB];
#pragma unroll
        for (int q = 0; q < kPB; ++q) {
            const bool ok = j0 + q < e0;
            x[q] = ok ? V.arc(j0 + q) : -1;
            w[q] = ok ? V.wgt(j0 + q) : 0;
        }
        if (test_free) {
            int32_t c[kPB];
#pragma unroll
            for (int q = 0; q < kPB; ++q) c[q] = x[q] >= 0 ? V.wget(Pk, x[q]) : -1;
#pragma unroll
            for (int q = 0; q < kPB; ++q) f[q] = x[q] >= 0 && !(c[q] >= 0 && V.wget(Pk, c[q]) == x[q]);
        } else {
#pragma unroll
            for (int q = 0; q < kPB; ++q) f[q] = x[q] >= 0;
        }
#pragma unroll
        for (int q = 0; q < kPB; ++q)
            if (f[q]) best = umax64(best, pack_key<H>(seed, w[q], x[q]));
    }
    return key_vertex<H>(seed, best);
}

// Heaviest (free, when TEST) neighbour for every lane of the warp with `need`, the rows of the
// needing lanes flattened over the lanes 32 arcs at a time: a lane finds its arc's row by a
// shuffle search over the rows' exclusive degree prefix, and per-row maxima are a segmented
// shuffle max whose segment tails update the row's slot.  Coarse levels have a heavy degree
// tail (C3 level 8: mean 3.6, p99 19): a row per lane made every warp as slow as its longest
// row.  All 32 lanes call (warp-uniform); `slot` = 32 entries of this warp.
template <bool H, bool TEST>
__device__ __forceinline__ int32_t warp_flat_best(const PartView &V, const int32_t *Pk, uint32_t seed, bool need,
                                                  int32_t i, unsigned long long *slot) {
    const int lane = threadIdx.x & 31;
    const int32_t s = need ? V.rs(i) : 0;
    const int32_t deg = need ? V.rs(i + 1) - s : 0;
    const int32_t incl = warp_incl_scan(deg), excl = incl - deg;
    const int32_t T = __shfl_sync(0xffffffffu, incl, 31);
    slot[lane] = 0;
    __syncwarp();
    for (int32_t base = 0; base < T; base += 32) {
        const int32_t e = base + lane;
        const bool valid = e < T;
        int o = 0;  // the last lane whose exclusive prefix is <= e (a lane with a positive degree)
#pragma unroll
        for (int step = 16; step > 0; step >>= 1) {
            const int32_t ex = __shfl_sync(0xffffffffu, excl, o + step);
            if (ex <= e) o += step;
        }
        const int32_t so = __shfl_sync(0xffffffffu, s, o), eo = __shfl_sync(0xffffffffu, excl, o);
        unsigned long long key = 0;
        if (valid) {
            const int32_t j = so + (e - eo);
            const int32_t x = V.arc(j), w = V.wgt(j);
            bool f = true;
            if (TEST) {
                const int32_t c = V.wget(Pk, x);
                f = !(c >= 0 && V.wget(Pk, c) == x);
            }
            if (f) key = pack_key<H>(seed, w, x);
        }
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {  // segmented inclusive max over equal owners
            const unsigned long long ok = __shfl_up_sync(0xffffffffu, key, d);
            const int oo = __shfl_up_sync(0xffffffffu, o, d);
            if (lane >= d && oo == o) key = umax64(key, ok);
        }
        const int no = __shfl_down_sync(0xffffffffu, o, 1);
        const bool nvalid = __shfl_down_sync(0xffffffffu, valid ? 1 : 0, 1) != 0;
        if (valid && (lane == 31 || no != o || !nvalid)) slot[o] = umax64(slot[o], key);
        __syncwarp();
    }
    const unsigned long long bk = slot[lane];
    __syncwarp();
    return need ? key_vertex<H>(seed, bk) : kNone;
}

// the two fine rows of coarse row c (leader u = lo + i, partner v): arc e of the merged row
struct RowSrc {
    int32_t su, du, sv, dv;  // starts (own rows: local arc index; foreign v: global) and degrees
    bool vglob;              // v's row is read from global memory
};
__device__ __forceinline__ RowSrc row_src(const PartView &V, int32_t i, int32_t m) {
    RowSrc r;
    r.su = V.rs(i);
    r.du = V.rs(i + 1) - r.su;
    r.vglob = false;
    r.sv = 0;
    r.dv = 0;
    const int32_t u = V.lo + i;
    if (m != u) {
        if (m >= V.lo && m < V.hi) {
            r.sv = V.rs(m - V.lo);
            r.dv = V.rs(m - V.lo + 1) - r.sv;
        } else {
            r.vglob = true;
            r.sv = pld(V.gadjp + m);
            r.dv = pld(V.gadjp + m + 1) - r.sv;
        }
    }
    return r;
}
// key of merged element e (cx << 32 | w), kPPad for the collapsed edge
__device__ __forceinline__ unsigned long long row_key(const PartView &V, const int32_t *CMg, const RowSrc &r,
                                                      int32_t e, int32_t c) {
    // element e: u's row, then v's (own row: shared memory; foreign partner: global)
    const bool inu = e < r.du;
    const int32_t j = inu ? r.su + e : r.sv + e - r.du;
    const bool g = !inu && r.vglob;
    int32_t x, w;
    if (V.garcs) {
        x = pld((g ? V.gadjncy : V.gadjncy + V.a0) + j);
        w = pld((g ? V.gadjwgt : V.gadjwgt + V.a0) + j);
    } else {
        const int32_t jl = g ? 0 : j + V.aoff;  // a valid shared index either way
        PCHK(g || (j >= 0 && j < V.na), "own row arc", j);
        PCHK(!g || (j >= 0 && j < V.capnnz), "foreign row arc", j);
        x = ld_or(V.sadj[jl], V.gadjncy + j, g);
        w = ld_or(V.swgt[jl], V.gadjwgt + j, g);
    }
    const int32_t cx = V.wget(CMg, x);
    return cx == c ? kPPad : ckey(cx, w);  // collapsed edge dropped (R9)
}

// The merged row of leader u and partner v is staged (as cx << 32 | w) in the global staging
// array at the two fine rows' own arc ranges: [adjp[u], adjp[u+1]) then [adjp[v], adjp[v+1]).
// Every vertex is in exactly one pair, so the ranges of different coarse rows are disjoint, and
// a merged row never has more entries than its two fine rows.
struct KeyAcc {
    unsigned long long *base0, *base1;
    int32_t d0;
    __device__ __forceinline__ unsigned long long &operator()(int32_t e) const {
        PCHK(e >= 0, "staging entry", e);
        return e < d0 ? base0[e] : base1[e - d0];
    }
};
__device__ __forceinline__ KeyAcc stage_of(const PartView &V, const RowSrc &r, unsigned long long *gkeys) {
    KeyAcc s;
    s.base0 = gkeys + V.a0 + r.su;
    s.base1 = gkeys + (r.vglob ? r.sv : V.a0 + r.sv);
    s.d0 = r.du;
    return s;
}

// where own row i (leader, sources r) stages its merged entries
__device__ __forceinline__ KeyAcc stage_at(const PartView &V, const RowSrc &r, unsigned long long *gkeys, int32_t i) {
    if (!V.sstage) return stage_of(V, r, gkeys);
    KeyAcc s;
    PCHK(V.cnt[i] >= 0 && V.cnt[i] + r.du + r.dv <= V.sstot, "shared staging slot", V.cnt[i]);
    s.base0 = V.sst + V.cnt[i];
    s.base1 = s.base0 + r.du;
    s.d0 = r.du;
    return s;
}

// ---- merged rows of <= N (8 or 16) entries: one thread, register network ----
template <int N>
__device__ __forceinline__ int32_t merge_thread(const PartView &V, const int32_t *CMg, const RowSrc &r, int32_t c,
                                                const KeyAcc &st) {
    const uint32_t kDrop = 0xFFFFFFFFu;
    uint32_t kc[N];
    int32_t kw[N];
    const int32_t ub = r.du + r.dv;
#pragma unroll
    for (int q = 0; q < N; ++q) {
        kc[q] = kDrop;
        kw[q] = 0;
        if (q < ub) {
            const unsigned long long k = row_key(V, CMg, r, q, c);
            if (k != kPPad) {
                kc[q] = (uint32_t)(k >> 32);
                kw[q] = (int32_t)(uint32_t)k;
            }
        }
    }
    if constexpr (N == 8) cx_sort8(kc, kw);
    else cx_sort16(kc, kw);
    int32_t cnt = 0;
    uint32_t prev = kDrop;
    int32_t acc = 0;
#pragma unroll
    for (int q = 0; q < N; ++q) {
        if (kc[q] == prev) {
            acc += kw[q];  // repeated coarse neighbour: weights summed (R8, P12.s28)
        } else {
            if (prev != kDrop) st(cnt++) = ckey((int32_t)prev, acc);
            prev = kc[q];
            acc = kw[q];
        }
    }
    if (prev != kDrop) st(cnt++) = ckey((int32_t)prev, acc);
    return cnt;
}

// ---- merged rows of 17..32 entries: a half warp (16-lane segment), two rows per warp step;
// `r` / `c` / `st` are this segment's row (an idle segment passes ub = 0) ----
__device__ __forceinline__ int32_t merge_seg(const PartView &V, const int32_t *CMg, const RowSrc &r, int32_t c,
                                             const KeyAcc &st, unsigned long long *sout) {
    const int l = threadIdx.x & 15;
    const int32_t ub = r.du + r.dv;
    unsigned long long v[2];
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        const int32_t e = q * 16 + l;
        v[q] = e < ub ? row_key(V, CMg, r, e, c) : kPPad;
    }
    seg_sort32(v);
    const int32_t cnt = seg_runmerge32(v, sout);
    __syncwarp();
    for (int32_t q = l; q < cnt; q += 16) st(q) = sout[q];
    __syncwarp();
    return cnt;
}

// ---- merged rows of 33..64 entries: one warp, register bitonic + segmented run merge ----
__device__ __forceinline__ int32_t merge_warp(const PartView &V, const int32_t *CMg, const RowSrc &r, int32_t c,
                                              const KeyAcc &st, unsigned long long *wout) {
    const int lane = threadIdx.x & 31;
    const int32_t ub = r.du + r.dv;
    unsigned long long v[2];
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        const int32_t e = q * 32 + lane;
        v[q] = e < ub ? row_key(V, CMg, r, e, c) : kPPad;
    }
    warp_sort64(v);
    const int32_t cnt = warp_runmerge64(v, wout);  // padding (cx = 2^32-1) is never emitted
    __syncwarp();
    for (int32_t q = lane; q < cnt; q += 32) st(q) = wout[q];
    __syncwarp();
    return cnt;
}

// ---- merged rows of 65..256 entries: one warp, flip-bitonic in its shared-memory area ----
__device__ __forceinline__ int32_t merge_warp_smem(const PartView &V, const int32_t *CMg, const RowSrc &r, int32_t c,
                                                   const KeyAcc &st, unsigned long long *wk) {
    const int lane = threadIdx.x & 31;
    const int32_t ub = r.du + r.dv;
    for (int32_t e = lane; e < ub; e += 32) wk[e] = row_key(V, CMg, r, e, c);
    __syncwarp();
    coop_sort(wk, ub, lane, 32, []() { __syncwarp(); });
    int32_t total = 0;
    for (int32_t b0 = 0; b0 < ub; b0 += 32) {
        const int32_t e = b0 + lane;
        bool h = false;
        unsigned long long k = 0;
        int32_t sum = 0;
        if (e < ub) {
            k = wk[e];
            h = k != kPPad && (e == 0 || (wk[e - 1] >> 32) != (k >> 32));
            if (h) {
                sum = (int32_t)(uint32_t)k;  // the run's weights summed (R8)
                for (int32_t q = e + 1; q < ub && (wk[q] >> 32) == (k >> 32); ++q) sum += (int32_t)(uint32_t)wk[q];
            }
        }
        const unsigned hm = __ballot_sync(0xffffffffu, h);
        if (h) st(total + __popc(hm & lanemask_lt())) = ckey((int32_t)(k >> 32), sum);
        total += __popc(hm);
    }
    __syncwarp();
    return total;
}

// ---- longer merged rows: the whole CTA.  Keys sorted in shared memory (<= kPKeys) or in the
// row's staging ranges; run heads (with their run sums) compacted to the front of the staging.
__device__ int32_t merge_cta(const PartView &V, const int32_t *CMg, const RowSrc &r, int32_t c, const KeyAcc &st,
                             unsigned long long *skeys, int32_t *s) {
    const int32_t ub = r.du + r.dv;
    KeyAcc acc = st;
    if (ub <= kPKeys) {
        acc.base0 = skeys;
        acc.base1 = skeys + r.du;
    }
    for (int32_t e = threadIdx.x; e < ub; e += kPT) acc(e) = row_key(V, CMg, r, e, c);
    __syncthreads();
    int32_t S = 1;
    while (S < ub) S <<= 1;
    for (int lh = 0; (2 << lh) <= S; ++lh) {  // flip-bitonic network (padding past ub)
        const int size = 2 << lh, half = 1 << lh;
        for (int i = threadIdx.x; i < S / 2; i += kPT) {
            const int base = (i >> lh) << (lh + 1), o = i & (half - 1);
            const int x = base + o, y = base + size - 1 - o;
            if (y < ub) {
                const unsigned long long p = acc(x), q = acc(y);
                if (p > q) {
                    acc(x) = q;
                    acc(y) = p;
                }
            }
        }
        __syncthreads();
        for (int lj = lh - 1; lj >= 0; --lj) {
            const int j = 1 << lj;
            for (int i = threadIdx.x; i < S / 2; i += kPT) {
                const int x = ((i >> lj) << (lj + 1)) + (i & (j - 1)), y = x + j;
                if (y < ub) {
                    const unsigned long long p = acc(x), q = acc(y);
                    if (p > q) {
                        acc(x) = q;
                        acc(y) = p;
                    }
                }
            }
            __syncthreads();
        }
    }
    // run heads in chunks of kPT: sums read first, the scan's barriers, then the compacted
    // writes (in place when sorted in the staging: a write lands at or before its head and
    // after every run walk of the chunk has finished)
    int32_t total = 0;
    for (int32_t b0 = 0; b0 < ub; b0 += kPT) {
        const int32_t e = b0 + threadIdx.x;
        unsigned long long k = 0;
        bool h = false;
        int32_t sum = 0;
        if (e < ub) {
            k = acc(e);
            h = k != kPPad && (e == 0 || (acc(e - 1) >> 32) != (k >> 32));
            if (h) {
                sum = (int32_t)(uint32_t)k;  // the run's weights summed (R8); fits int32 (R14)
                for (int32_t q = e + 1; q < ub; ++q) {
                    const unsigned long long kq = acc(q);
                    if ((kq >> 32) != (k >> 32)) break;
                    sum += (int32_t)(uint32_t)kq;
                }
            }
        }
        int32_t tot;
        const int32_t ex = block_excl_scan<kPT>(h ? 1 : 0, s, tot);
        if (h) st(total + ex) = ckey((int32_t)(k >> 32), sum);
        total += tot;
        __syncthreads();
    }
    return total;
}

// 1D bulk copy global -> shared (no cache-policy hint: the gathered arrays should stay in L2)
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_addr(dst)),
                 "l"(src), "r"(bytes), "r"(smem_addr(bar))
                 : "memory");
}
// Up to three copies of `words[q]` int32 (multiples of 4, 16-byte aligned) completed on one
// mbarrier phase.  All threads call after a __syncthreads (the destinations are free); thread
// 0 orders the CTA's earlier generic shared accesses and the grid's earlier global writes
// (seen through the barrier's acquire) before the async-proxy copies.
__device__ __forceinline__ void part_fetch(uint64_t *bar, unsigned &phase, int32_t *d0, const int32_t *s0, int32_t w0,
                                           int32_t *d1 = nullptr, const int32_t *s1 = nullptr, int32_t w1 = 0,
                                           int32_t *d2 = nullptr, const int32_t *s2 = nullptr, int32_t w2 = 0) {
    if (threadIdx.x == 0) {
        asm volatile("fence.proxy.async;" ::: "memory");
        mbar_arrive_expect_tx(bar, (unsigned)(w0 + w1 + w2) * 4u);
        if (w0 > 0) bulk_g2s(d0, s0, (unsigned)w0 * 4u, bar);
        if (w1 > 0) bulk_g2s(d1, s1, (unsigned)w1 * 4u, bar);
        if (w2 > 0) bulk_g2s(d2, s2, (unsigned)w2 * 4u, bar);
    }
    mbar_wait(bar, phase);
    phase ^= 1u;
}

// GP_PROF=1: the slowest CTA's time since `t0` into *slot (ns)
__device__ __forceinline__ void prof_max(const PartArgs &a, unsigned long long *slot, unsigned long long t0) {
    if (a.prof && threadIdx.x == 0) atomicMax(slot, globaltimer() - t0);
}
__device__ __forceinline__ unsigned long long prof_now(const PartArgs &a) { return a.prof ? globaltimer() : 0ull; }

template <bool H>
__global__ void __launch_bounds__(kPT, 1) k_part(const __grid_constant__ PartArgs a) {
    extern __shared__ __align__(16) unsigned char praw[];
    unsigned long long *skeys = reinterpret_cast<unsigned long long *>(praw);  // kPKeys
    int32_t *sw = reinterpret_cast<int32_t *>(praw + (size_t)kPKeys * 8);    // kPartBudget words
    __shared__ int32_t s_scan[64];
    __shared__ unsigned long long s_red[3 * kPW];
    __shared__ int32_t s_b[8];
    __shared__ int32_t s_lists[4][kPT];  // rows of 17..32 / 33..64 / 65..256 / > 256 entries of a sweep
    __shared__ int32_t s_cnt3[4];
    __shared__ int32_t s_hist[33];
    __shared__ __align__(8) uint64_t s_mbar;
    unsigned mph = 0;  // mbarrier phase of the next fetch

    const int t = threadIdx.x, b = blockIdx.x, lane = t & 31, wid = t >> 5;
    if (t == 0) {
        mbar_init(&s_mbar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    PartCtl *ctl = a.ctl;
    unsigned btarget = 0;  // barrier target (thread 0)
    int32_t g = 0;         // global phase counter (identical on every CTA)
    const volatile SizeRec *in = a.in;
    int32_t n = in->n, nnz = in->nnz;
    bool stopped = in->stop != 0;
    int32_t prev_reason = in->stop_reason;
    const int32_t *gadjp = a.adjp, *gadjncy = a.adjncy, *gadjwgt = a.adjwgt, *gvwgt = a.vwgt;
    int level = 0;
    while (!stopped && level < a.nslots) {
        const int nact = part_nact(n, nnz, a.wmin);
        if (b >= nact) return;  // retired (levels only shrink: it is never needed again)
        const int gl = a.level0 + level;
        const PartLevelOut o = a.slots[level];
        unsigned long long *tr = a.levdev[gl].match.trace;
        int tm = 0;  // GP_DEBUG phase marks of this level (block 0)
#define PT_MARK() do { if (a.trace) trace_mark(tr, tm++); } while (0)
        PT_MARK();
        // ---- partition [lo, hi) and this level's shared-memory layout ----
        PartView V;
        V.n = n;
        V.gadjp = gadjp;
        V.gadjncy = gadjncy;
        V.gadjwgt = gadjwgt;
        V.capnnz = a.cap_nnz;
        V.sstage = false;
        V.sstot = 0;
        PCHK(n <= a.cap_n && nnz <= a.cap_nnz, "level size within the slot bounds", nnz);
        if (level == 0) {
            const long long W = 2LL * nnz + 5LL * n;
            V.lo = b == 0 ? 0 : part_search(gadjp, n, (long long)b * W / nact);
            V.hi = b == nact - 1 ? n : part_search(gadjp, n, (long long)(b + 1) * W / nact);
        } else {
            V.lo = pld(ctl->bnd + b);
            V.hi = pld(ctl->bnd + b + 1);
        }
        V.nv = V.hi - V.lo;
        V.a0 = pld(gadjp + V.lo);
        V.na = pld(gadjp + V.hi) - V.a0;
        {
            V.loff = V.lo & 3;
            V.aoff = V.a0 & 3;
            const int32_t np4 = (V.nv + 1 + V.loff + 3) & ~3;  // adjp slice words (aligned copy)
            const int32_t nv4 = (V.nv + 3) & ~3, na4 = (V.na + V.aoff + 3) & ~3;
            V.sap = sw;
            V.M = V.sap + np4;
            V.cnt = V.M + nv4;
            int32_t *rest = V.cnt + nv4;
            const int32_t used = np4 + 2 * nv4;
            if (used + nv4 + 8 > kPartBudget) __trap();  // the host's bound guarantees it (part_fits)
            V.garcs = a.force_garcs || used + 2 * na4 + nv4 + 8 > kPartBudget;
            if (!V.garcs) {
                V.sadj = rest;
                V.swgt = rest + na4;
                V.win = rest + 2 * na4;
            } else {
                V.sadj = V.swgt = nullptr;
                V.win = rest;
            }
            __syncthreads();  // the previous level's shared arrays are no longer read
            if (V.garcs)
                part_fetch(&s_mbar, mph, V.sap, gadjp + (V.lo - V.loff), np4);
            else
                part_fetch(&s_mbar, mph, V.sap, gadjp + (V.lo - V.loff), np4, V.sadj, gadjncy + (V.a0 - V.aoff), na4,
                           V.swgt, gadjwgt + (V.a0 - V.aoff), na4);
        }
        int32_t wcap = (kPartBudget - (int32_t)(V.win - sw)) & ~3;
        if (a.wcap_max > 0 && wcap > a.wcap_max) wcap = a.wcap_max;
        for (int32_t i = t; i < V.nv; i += kPT) V.M[i] = kFree;
        __syncthreads();
        // window: own range + a halo of 2 * D on each side, D = the distance (outside [lo, hi))
        // that all but ~1/256 of the arcs stay within, rounded up to a power of two: the
        // neighbours x and the neighbours' proposals P[x] (two hops) of a graph with id
        // locality; the rare longer arcs read global memory
        {
            if (t < 33) s_hist[t] = 0;
            __syncthreads();
            for (int32_t i = t; i < V.nv; i += kPT) {
                const int32_t u = V.lo + i;
                (void)u;
                for (int32_t j = V.rs(i), je = V.rs(i + 1); j < je; ++j) {
                    const int32_t x = V.arc(j);
                    const uint32_t d = x < V.lo ? (uint32_t)(V.lo - x) : x >= V.hi ? (uint32_t)(x - V.hi + 1) : 0u;
                    atomicAdd(&s_hist[32 - __clz(d)], 1);  // bucket q: d < 2^q
                }
            }
            __syncthreads();
            int32_t q = 0, acc = 0;
            const int32_t keep = V.na - (V.na >> 8);
            while (q < 32 && acc + s_hist[q] < keep) acc += s_hist[q++];
            const long long D = q >= 31 ? (long long)n : (1LL << q);
            long long wl = (long long)V.lo - 2 * D, wh = (long long)V.hi + 2 * D;
            if (wl < 0) wl = 0;
            if (wh > n) wh = n;
            if (wh - wl > wcap) {  // keep the own range, as much halo as fits
                const long long extra = wcap > V.nv ? (wcap - V.nv) / 2 : 0;
                wl = (long long)V.lo - extra;
                if (wl < 0) wl = 0;
                wh = wl + wcap;
                if (wh > n) wh = n;
            }
            wl &= ~3LL;  // 16-byte aligned copies (arrays are padded past n)
            wh = (wh + 3) & ~3LL;
            if (wh - wl > wcap) wh = wl + wcap;
            V.wlo = (int32_t)wl;
            V.wlen = (int32_t)(wh - wl) > 0 ? (int32_t)(wh - wl) : 0;
            PCHK((int32_t)(V.win - sw) + V.wlen <= kPartBudget, "window in shared memory", V.wlen);
            __syncthreads();
        }
        PT_MARK();
        // ---- matching rounds (A2-A4) ----
        unsigned long long arcs = 0, rows = 0, visits = 0;
        int32_t rounds = 0, maximal = 0;
        MatchCtl *mc = &a.levdev[gl].match;
        unsigned long long t0 = prof_now(a);
        {  // round-1 proposals: every vertex is free (phase g)
            int32_t mylive = 0;
            // one row per thread: no freedom test in round 1, so a row is a short chain of
            // shared loads (the flattened scan of the later rounds measured slower here)
            for (int32_t i = t; i < V.nv; i += kPT) {
                const int32_t u = V.lo + i;
                const int32_t p = part_best<H>(V, a.P1, a.tie_seed, i, false);
                a.P1[u] = p;  // round 1 -> parity 1
                if (p < 0) a.P0[u] = kNone;  // no neighbour: dead in both parity buffers
                mylive += p >= 0;
                arcs += (unsigned long long)(V.rs(i + 1) - V.rs(i));
            }
            PT_MARK();
            prof_max(a, &mc->wmax[0], t0);
            round_bar(ctl, btarget, nact, g, mylive, 0, s_scan);
            PT_MARK();
            ++g;
        }
        for (int k = 1;; ++k) {  // phase g: commit of round k + proposals of round k + 1
            if (t == 0) {
                s_b[0] = *(volatile int32_t *)&ctl->ring[g & 3][0];
                s_b[1] = k > 1 ? *(volatile int32_t *)&ctl->ring[(g - 1) & 3][1] : 0;
            }
            __syncthreads();
            const int32_t live = s_b[0];
            if (s_b[1] > 0) ++rounds;  // round k - 1 matched (always, when it ran: §2.1)
            __syncthreads();
            if (live == 0) {
                maximal = 1;
                break;
            }
            if (a.max_rounds > 0 && rounds >= a.max_rounds) break;
            if (k > n + 2) __trap();  // each round with proposals matches >= 1 pair
            t0 = prof_now(a);
            if (a.prof && b == 0 && t == 0 && k < 16) mc->lens[k] = live;
            int32_t *Pk = (k & 1) ? a.P1 : a.P0;
            int32_t *Pn = (k & 1) ? a.P0 : a.P1;
            part_fetch(&s_mbar, mph, V.win, Pk + V.wlo, V.wlen);
            PT_MARK();
            int32_t mylive = 0, mypairs = 0;
            unsigned long long *slot = skeys + wid * 32;
            for (int32_t ib = t - lane; ib < V.nv; ib += kPT) {  // warp-uniform
                const int32_t i = ib + lane;
                const int32_t u = V.lo + i;
                int32_t p = -1, q = -1;
                bool live = false, need = false;
                if (i < V.nv && V.M[i] == kFree) {
                    p = V.wget(Pk, u);
                    live = p >= 0;  // else dead: no free neighbour (stays free: leftover)
                }
                if (live) {
                    ++visits;
                    q = V.wget(Pk, p);
                    // q == u: handshake (P18.s10-12); else p keeps being the heaviest free
                    // neighbour while it is free after round k, and u rescans if p matched q
                    need = q != u && q >= 0 && V.wget(Pk, q) == p;
                }
                const int32_t b2 = warp_flat_best<H, true>(V, Pk, a.tie_seed, need, i, slot);
                if (!live) continue;
                if (q == u) {  // matched in round k
                    V.M[i] = p;
                    Pn[u] = p;  // both parity buffers now hold the partner
                    mypairs += u < p;
                    continue;
                }
                int32_t np = p;
                if (need) {
                    np = b2;
                    ++rows;
                    arcs += (unsigned long long)(V.rs(i + 1) - V.rs(i));
                }
                Pn[u] = np;
                // a vertex without free neighbours is dead in both buffers; readers of P_k see
                // p or NONE and decide alike (u is not matched this round, so P_k[u] never
                // completes a handshake or a "matched" test)
                if (np < 0) Pk[u] = kNone;
                mylive += np >= 0;
            }
            PT_MARK();
            if (k < 16) prof_max(a, &mc->wmax[k], t0);
            round_bar(ctl, btarget, nact, g, mylive, mypairs, s_scan);
            PT_MARK();
            ++g;
        }
        PT_MARK();
        // ---- leftover (P18.s12-13) + cmap (P18.s16-27): per-thread contiguous vertex blocks ----
        const int32_t per = (V.nv + kPT - 1) / kPT;
        const int32_t i0 = min(V.nv, t * per), i1 = min(V.nv, i0 + per);
        int32_t cl = 0;
        for (int32_t i = i0; i < i1; ++i) {
            if (V.M[i] == kFree) V.M[i] = V.lo + i;
            if (V.lo + i <= V.M[i]) ++cl;
        }
        int32_t nlead;
        int32_t c = block_excl_scan<kPT>(cl, s_scan, nlead);
        if (t == 0) ctl->nL[b] = nlead;
        for (int32_t i = t; i < V.nv; i += kPT) o.M[V.lo + i] = V.M[i];
        pbar(&ctl->bar, btarget, nact);
        PT_MARK();
        if (wid == 0) {  // coarse ids: leaders in id order, CTAs in range order
            int32_t pre = 0, all = 0;
            for (int q = lane; q < nact; q += 32) {
                const int32_t x = pld(ctl->nL + q);
                all += x;
                pre += q < b ? x : 0;
            }
            pre = warp_sum(pre);
            all = warp_sum(all);
            if (lane == 0) {
                s_b[2] = pre;
                s_b[3] = all;
            }
        }
        __syncthreads();
        const int32_t cbase = s_b[2], nc = s_b[3];
        c += cbase;
        for (int32_t i = i0; i < i1; ++i) {
            const int32_t u = V.lo + i, m = V.M[i];
            if (u <= m) {
                o.CM[u] = c;
                if (m != u) o.CM[m] = c;  // the leader writes its partner's coarse id (P18.s26)
                o.cvwgt[c] = pld(gvwgt + u) + (m != u ? pld(gvwgt + m) : 0);  // P12.s27
                ++c;
            }
        }
        pbar(&ctl->bar, btarget, nact);
        PT_MARK();
        // ---- contraction (A6-A8): every coarse row merged once into the staging, counted,
        // then copied to its final offset ----
        t0 = prof_now(a);
        part_fetch(&s_mbar, mph, V.win, o.CM + V.wlo, V.wlen);
        {  // staging: shared memory after the window when the rows' upper bounds fit, else global
            int32_t myub = 0;
            for (int32_t i = i0; i < i1; ++i) {
                const int32_t m = V.M[i];
                if (V.lo + i <= m) {
                    const RowSrc r = row_src(V, i, m);
                    myub += r.du + r.dv;
                }
            }
            int32_t ubtot;
            int32_t ro = block_excl_scan<kPT>(myub, s_scan, ubtot);
            int32_t *sb = V.win + ((V.wlen + 3) & ~3);
            V.sst = reinterpret_cast<unsigned long long *>(sb);
            V.sstage = !a.force_gstage && 2LL * ubtot + 4 <= (long long)(kPartBudget - (int32_t)(sb - sw));
            V.sstot = ubtot;
            if (V.sstage)
                for (int32_t i = i0; i < i1; ++i) {
                    const int32_t m = V.M[i];
                    if (V.lo + i <= m) {
                        const RowSrc r = row_src(V, i, m);
                        V.cnt[i] = ro;  // this row's upper-bound offset in the staging
                        ro += r.du + r.dv;
                    }
                }
            __syncthreads();
        }
        PT_MARK();
        // rows of > 16 merged entries, in sweeps over windows of kPT vertices: 17..32 by half
        // warps, 33..64 by warps, longer by the whole CTA
        for (int32_t r0 = 0; r0 < V.nv; r0 += kPT) {
            if (t == 0) s_cnt3[0] = s_cnt3[1] = s_cnt3[2] = s_cnt3[3] = 0;
            __syncthreads();
            {
                const int32_t i = r0 + t;
                int which = -1;
                if (i < V.nv) {
                    const int32_t m = V.M[i];
                    if (V.lo + i <= m) {
                        const RowSrc r = row_src(V, i, m);
                        const int32_t ub = r.du + r.dv;
                        if (ub > 16) which = ub <= 32 ? 0 : ub <= 64 ? 1 : ub <= 256 ? 2 : 3;
                    }
                }
#pragma unroll
                for (int q = 0; q < 4; ++q) {  // warp-aggregated appends (one shared atomic per warp and list)
                    const unsigned bq = __ballot_sync(0xffffffffu, which == q);
                    if (bq) {
                        int32_t base = 0;
                        if (lane == __ffs(bq) - 1) base = atomicAdd(&s_cnt3[q], __popc(bq));
                        base = __shfl_sync(0xffffffffu, base, __ffs(bq) - 1);
                        if (which == q) s_lists[q][base + __popc(bq & lanemask_lt())] = i;
                    }
                }
            }
            __syncthreads();
            const int32_t nA = s_cnt3[0], nB = s_cnt3[1], nW = s_cnt3[2], nC = s_cnt3[3];
            if (nA + nB + nW + nC == 0) continue;
            unsigned long long *wbuf = skeys + wid * 256;  // this warp's shared-memory keys
            for (int32_t q = 2 * wid; q < nA; q += 2 * kPW) {  // two 17..32-entry rows per warp
                const int half = lane >> 4;
                const int32_t qi = q + half;
                RowSrc r;
                int32_t cc = 0, ii = -1;
                KeyAcc st;
                if (qi < nA) {
                    ii = s_lists[0][qi];
                    r = row_src(V, ii, V.M[ii]);
                    cc = V.wget(o.CM, V.lo + ii);
                    st = stage_at(V, r, a.wkeys, ii);
                } else {
                    r.du = r.dv = 0;  // idle segment: all padding
                    r.su = r.sv = 0;
                    r.vglob = false;
                    st = stage_of(V, r, a.wkeys);  // (unused: no entries)
                }
                const int32_t k2 = merge_seg(V, o.CM, r, cc, st, wbuf + half * 32);
                if (ii >= 0 && (lane & 15) == 0) V.cnt[ii] = k2;
            }
            for (int32_t q = wid; q < nB; q += kPW) {
                const int32_t ii = s_lists[1][q];
                const RowSrc r = row_src(V, ii, V.M[ii]);
                const int32_t k2 = merge_warp(V, o.CM, r, V.wget(o.CM, V.lo + ii), stage_at(V, r, a.wkeys, ii), wbuf);
                if (lane == 0) V.cnt[ii] = k2;
            }
            for (int32_t q = wid; q < nW; q += kPW) {
                const int32_t ii = s_lists[2][q];
                const RowSrc r = row_src(V, ii, V.M[ii]);
                const int32_t k2 =
                    merge_warp_smem(V, o.CM, r, V.wget(o.CM, V.lo + ii), stage_at(V, r, a.wkeys, ii), wbuf);
                if (lane == 0) V.cnt[ii] = k2;
            }
            __syncthreads();
            for (int32_t q = 0; q < nC; ++q) {
                const int32_t ii = s_lists[3][q];
                const RowSrc r = row_src(V, ii, V.M[ii]);
                const int32_t k2 =
                    merge_cta(V, o.CM, r, V.wget(o.CM, V.lo + ii), stage_at(V, r, a.wkeys, ii), skeys, s_scan);
                if (t == 0) V.cnt[ii] = k2;
                __syncthreads();
            }
        }
        PT_MARK();
        // rows of <= 16 entries by their thread (contiguous blocks = coarse id order)
        // (warp-uniform steps: the 8-entry network runs when every merging lane's row fits it,
        // else all merging lanes run the 16-entry one -- divergent networks would run both)
        int32_t mine = 0;
        for (int32_t r0 = 0; r0 < per; ++r0) {
            const int32_t i = i0 + r0;
            int32_t ub = 0, m = 0;
            RowSrc r;
            r.du = r.dv = r.su = r.sv = 0;
            r.vglob = false;
            bool lead = false;
            if (i < i1) {
                m = V.M[i];
                lead = V.lo + i <= m;
                if (lead) {
                    r = row_src(V, i, m);
                    ub = r.du + r.dv;
                }
            }
            const bool narrow = lead && ub <= 16;
            const bool all8 = __all_sync(0xffffffffu, !narrow || ub <= 8);
            if (narrow) {
                const KeyAcc st = stage_at(V, r, a.wkeys, i);
                const int32_t cu = V.wget(o.CM, V.lo + i);
                V.cnt[i] = all8 ? merge_thread<8>(V, o.CM, r, cu, st) : merge_thread<16>(V, o.CM, r, cu, st);
            }
            if (lead) mine += V.cnt[i];
        }
        int32_t ctot;
        const int32_t cex = block_excl_scan<kPT>(mine, s_scan, ctot);
        if (t == 0) ctl->nA[b] = ctot;
        prof_max(a, &mc->barr[0][0], t0);
        PT_MARK();
        pbar(&ctl->bar, btarget, nact);
        PT_MARK();
        if (wid == 0) {  // merged entries of the lower CTAs: this CTA's first coarse arc
            int32_t pre = 0, all = 0;
            for (int q = lane; q < nact; q += 32) {
                const int32_t x = pld(ctl->nA + q);
                all += x;
                pre += q < b ? x : 0;
            }
            pre = warp_sum(pre);
            all = warp_sum(all);
            if (lane == 0) {
                s_b[4] = pre;
                s_b[5] = all;
            }
        }
        __syncthreads();
        t0 = prof_now(a);
        const int32_t cnnz = s_b[5];
        // copy: cadjp, the staged rows at their offsets, and the next level's partition bounds
        // (row cc holds the targets T_j = j * Wt / nnext with W(cc) <= T_j < W(cc + 1),
        // W(c) = 2 * cadjp[c] + 5 * c, the same measure as part_search)
        const int nnext = part_nact(nc, cnnz, a.wmin);
        const long long Wt = 2LL * cnnz + 5LL * nc;
        if (b == 0 && t == 0) {
            ctl->bnd[0] = 0;
            ctl->bnd[nnext] = nc;
        }
        if (V.sstage) {
            // cadjp, bounds, and per vertex: M := the row's staging offset, cnt := its output
            // offset in the CTA's range (running, so non-leaders keep offsets monotone); then the
            // CTA's output copied in one coalesced sweep (an element's row: the last vertex
            // whose output offset is <= the element's, by binary search)
            int32_t ru = 0, ro = cex;
            {
                int32_t myub = 0;  // this thread's staging base = the exclusive scan of upper bounds
                for (int32_t i = i0; i < i1; ++i) {
                    const int32_t m = V.M[i];
                    if (V.lo + i <= m) {
                        const RowSrc r = row_src(V, i, m);
                        myub += r.du + r.dv;
                    }
                }
                int32_t ubtot;
                ru = block_excl_scan<kPT>(myub, s_scan, ubtot);
            }
            for (int32_t i = i0; i < i1; ++i) {
                const int32_t u = V.lo + i, m = V.M[i];
                if (u > m) {
                    V.cnt[i] = ro;
                    continue;
                }
                const RowSrc r = row_src(V, i, m);
                const int32_t cc = V.wget(o.CM, u), k2 = V.cnt[i];
                const int32_t pos = s_b[4] + ro;
                o.cadjp[cc] = pos;
                if (nnext > 1) {
                    const long long W0 = 2LL * pos + 5LL * cc, W1 = W0 + 2LL * k2 + 5;
                    long long j = (W0 * nnext + Wt - 1) / Wt;
                    if (j < 1) j = 1;
                    for (; j < nnext && (j * Wt) / nnext < W1; ++j) ctl->bnd[j] = cc;
                }
                V.M[i] = ru;
                V.cnt[i] = ro;
                ru += r.du + r.dv;
                ro += k2;
            }
            __syncthreads();
            const int32_t gbase = s_b[4];
            for (int32_t e = t; e < ctot; e += kPT) {
                int32_t lo2 = 0, hi2 = V.nv;  // last i with cnt[i] <= e
                while (hi2 - lo2 > 1) {
                    const int32_t mid = (lo2 + hi2) >> 1;
                    if (V.cnt[mid] <= e) lo2 = mid;
                    else hi2 = mid;
                }
                const unsigned long long kv = V.sst[V.M[lo2] + (e - V.cnt[lo2])];
                PCHK(V.M[lo2] >= 0 && V.M[lo2] + (e - V.cnt[lo2]) < V.sstot, "staged entry", e);
                PCHK(gbase + e < V.capnnz, "coarse arc", gbase + e);
                __stcg(o.cadjncy + gbase + e, (int32_t)(kv >> 32));
                __stcg(o.cadjwgt + gbase + e, (int32_t)(uint32_t)kv);
            }
        } else {
            int32_t pos = s_b[4] + cex;
            for (int32_t i = i0; i < i1; ++i) {
                const int32_t u = V.lo + i, m = V.M[i];
                if (u > m) continue;
                const RowSrc r = row_src(V, i, m);
                const KeyAcc st = stage_of(V, r, a.wkeys);
                const int32_t cc = V.wget(o.CM, u), k2 = V.cnt[i];
                o.cadjp[cc] = pos;
                for (int32_t q0 = 0; q0 < k2; q0 += 16) {  // 16 staged loads in flight, then the stores
                    unsigned long long kv[16];
#pragma unroll
                    for (int q = 0; q < 16; ++q) kv[q] = q0 + q < k2 ? __ldcg(&st(q0 + q)) : 0ull;
#pragma unroll
                    for (int q = 0; q < 16; ++q)
                        if (q0 + q < k2) {
                            PCHK(pos + q0 + q < V.capnnz, "coarse arc", pos + q0 + q);
                            o.cadjncy[pos + q0 + q] = (int32_t)(kv[q] >> 32);
                            o.cadjwgt[pos + q0 + q] = (int32_t)(uint32_t)kv[q];
                        }
                }
                if (nnext > 1) {
                    const long long W0 = 2LL * pos + 5LL * cc, W1 = W0 + 2LL * k2 + 5;
                    long long j = (W0 * nnext + Wt - 1) / Wt;
                    if (j < 1) j = 1;
                    for (; j < nnext && (j * Wt) / nnext < W1; ++j) ctl->bnd[j] = cc;
                }
                pos += k2;
            }
        }
        if (b == nact - 1 && t == 0) o.cadjp[nc] = cnnz;
        prof_max(a, &mc->barr[0][1], t0);
        PT_MARK();
        pbar(&ctl->bar, btarget, nact);
        // ---- statistics, stop rule (R12, R13), report ----
        block_sum3(arcs, rows, visits, s_red);
        if (t == 0 && (arcs | rows | visits)) {
            atomicAdd(&mc->arcs_scanned, arcs);
            atomicAdd(&mc->rows_scanned, rows);
            atomicAdd(&mc->live_visits, visits);
        }
        int32_t reason = GP_STOP_NONE;
        if (100LL * nc > (long long)a.stall_pct * n) reason = GP_STOP_STALL;
        else if (nc <= a.threshold) reason = GP_STOP_THRESHOLD;
        else if (gl + 1 >= a.max_levels) reason = GP_STOP_MAX_LEVELS;
        if (b == 0 && t == 0) {
            mc->rounds = rounds;
            mc->maximal = maximal;
            SizeRec *so = &a.levdev[gl].out;
            so->n = nc;
            so->nnz = cnnz;
            so->stop = reason != GP_STOP_NONE;
            so->stop_reason = reason;
        }
        PT_MARK();
        pbar(&ctl->bar, btarget, nact);  // every CTA's outputs and statistics are complete
        if (b == 0 && t == 0) {
            LevelReport *r = &a.reports[gl];
            r->n_coarse = nc;
            r->cnnz = cnnz;
            r->stop = reason != GP_STOP_NONE;
            r->stop_reason = reason;
            r->skipped = 0;
            __threadfence_system();
            *((volatile int32_t *)&r->ready) = 1;
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
#undef PT_MARK
    }
    // the levels the host enqueued beyond the stop: skipped reports
    if (b == 0 && t == 0) {
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

// ---------------------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------------------
static int part_enabled() {
    const char *e = getenv("GP_PART");  // knob read per call (results never depend on it)
    return (e && atoi(e) == 0) ? 0 : 1;
}
static int32_t part_wmin() {
    const char *e = getenv("GP_PART_W");  // tuning knob: words of work per active CTA
    const int v = e ? atoi(e) : 4096;
    return v < 64 ? 64 : v;
}
static int32_t part_knob(const char *name) {
    const char *e = getenv(name);  // test knobs (results never depend on them)
    return e ? atoi(e) : 0;
}
static int part_grid(Ctx *ctx) { return ctx->num_sms < kMaxParts ? ctx->num_sms : kMaxParts; }

// every CTA's vertex arrays (3 words + at least its own window) fit its shared memory: a CTA
// range has 5 * nv <= W / nact + 5 (W-balanced bounds), so W <= grid * 5/4 * (budget - 32)
bool part_fits(Ctx *ctx, int32_t n, int32_t nnz) {
    const long long W = 2LL * nnz + 5LL * n;
    return n > 0 && W <= (long long)part_grid(ctx) * (kPartBudget - 32) * 5 / 4 * 98 / 100;
}
bool part_use(Ctx *ctx, int32_t n_bound, int32_t nnz_bound) {
    return part_enabled() && part_fits(ctx, n_bound, nnz_bound);
}

size_t part_scratch_bytes(int32_t n, int32_t nnz) {
    return 4096 + sizeof(PartCtl) + 2 * 4 * ((size_t)n + 128) + 8 * ((size_t)nnz + 64);
}

gp_status enqueue_part(Ctx *ctx, const PartLaunch &L) {
    PartArgs a;
    a.in = L.in;
    a.adjp = L.adjp;
    a.adjncy = L.adjncy;
    a.adjwgt = L.adjwgt;
    a.vwgt = L.vwgt;
    a.slots = reinterpret_cast<PartLevelOut *>(L.slots);
    a.nslots = L.nslots;
    a.level0 = L.level0;
    a.levdev = L.levdev;
    a.reports = L.reports;
    a.threshold = L.threshold;
    a.stall_pct = L.stall_pct;
    a.max_levels = L.max_levels;
    a.max_rounds = L.max_rounds;
    a.tie_seed = ctx->tie_seed;
    a.wmin = part_wmin();
    a.force_garcs = part_knob("GP_PART_GARCS");
    a.wcap_max = part_knob("GP_PART_WCAP");
    a.force_gstage = part_knob("GP_PART_GSTAGE");
    a.cap_n = L.cap_n;
    a.cap_nnz = L.cap_nnz;
    a.prof = part_knob("GP_PROF") == 1 ? 1 : 0;
    a.trace = getenv("GP_DEBUG") ? 1 : 0;
    {
        unsigned char *p = static_cast<unsigned char *>(L.scratch);
        p = reinterpret_cast<unsigned char *>(((uintptr_t)p + 255) & ~(uintptr_t)255);
        a.ctl = reinterpret_cast<PartCtl *>(p);
        p += (sizeof(PartCtl) + 255) & ~(size_t)255;
        const size_t nn = ((size_t)L.cap_n + 64 + 63) & ~(size_t)63;  // 256-byte aligned parity buffers (TMA)
        a.P0 = reinterpret_cast<int32_t *>(p);
        a.P1 = a.P0 + nn;
        a.wkeys = reinterpret_cast<unsigned long long *>(a.P1 + nn);
    }
    GP_CUDA(cudaMemsetAsync(a.ctl, 0, sizeof(PartCtl), ctx->stream));
    const size_t smem = kPartDyn;
    const void *fn = a.tie_seed ? (const void *)k_part<true> : (const void *)k_part<false>;
    GP_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    GP_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kPT, smem));
    if (per_sm < 1) {
        set_error("k_part: one CTA per SM does not fit");
        return GP_ERR_CUDA;
    }
    void *args[] = {&a};
    LaunchScope ls(ctx, GP_K_OTHER);
    GP_CUDA(cudaLaunchCooperativeKernel(fn, dim3(part_grid(ctx)), dim3(kPT), args, smem, ctx->stream));
    ++ctx->launches;
    return GP_OK;
}

}  // namespace gp
