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
//  * Work units are WARP tiles: a warp never waits for its CTA, so an SM keeps 32
//    independent dependent-load chains in flight (a CTA-tile design kept ~4 and was
//    latency-bound; measured).  No CTA ever waits on another one except at grid barriers.
//  * Prefixes are "chunked reduce-then-scan": phase A accumulates each tile's aggregate
//    into the sum of the contiguous chunk of tiles one CTA owns in phase B (integer
//    atomics: order-free, deterministic); phase B block-scans its chunk once.
//  C1a warp tiles of 256 vertices: leftover self-match (P18.s12-13), leader flags u<=M[u]
//      (P18.s18), #leaders and the sum of merged-row upper bounds ub = deg(u)+deg(v)
//      (P20.s5-8).                                                               | barrier
//  C1b CM (= the paper's inclusive scan minus one, P18.s20-24; the leader also writes its
//      partner's CM, P18.s26), cvwgt (P12.s27), the ub prefix `off`, each coarse row's two
//      fine segments, and C2's warp-tile starts (256 upper-bound entries each). | barrier
//  C1h (only if some ub > 256): one CTA per such row merges it in shared memory (ub <=
//      4096) or global scratch and leaves it compacted.                          | barrier
//  C2a warp tiles: every row is merged (ub <= 16: one thread, registers + bitonic network;
//      <= 64: the warp, registers + shuffles; <= 256: the warp, shared-memory bitonic sort)
//      and the tile is written compacted to scratch at its own ub offset, with each row's
//      tile-local offset and the tile total.                                     | barrier
//  C2b cadjp and a coalesced copy of every tile into the final compact CSR.
//  Rows come out sorted by coarse id (R10) with repeated coarse neighbours summed (R8) and
//  the collapsed edge dropped (R9).
#include <cuda_runtime.h>

#include <algorithm>
#include <stdlib.h>

#include "device_util.cuh"
#include "gp_internal.cuh"
#include "merge_util.cuh"
#include "sort_util.cuh"

namespace gp {

constexpr int kCNT = 256;        // threads per CTA (4 co-resident CTAs per SM)
constexpr int kCW = kCNT / 32;   // warps per CTA
constexpr int kCItems = 8;       // vertices per lane of a C1 warp tile
constexpr int kVW = 32 * kCItems;  // 256 vertices per C1 warp tile
constexpr int kWB = kContractTileBudget;  // C2: rows up to this bound merged by a warp (slot area 2*kWB)
constexpr int kRT = 32;          // C2 warp tile: coarse rows (single GPU; 8..32, see k_contract_level)
constexpr int kCtaRow = 4096;    // C1h: rows up to this bound are merged in shared memory
constexpr int kNet = 16;         // one-thread merge capacity
constexpr int kWarpNet = 64;     // one-warp register merge capacity
constexpr int kBuf = 4096;       // shared u64 buffer (warp regions of 2*kWB / C1h rows / C2b)
constexpr unsigned long long kMaxKey = ~0ull;

// CTAs taking part in this launch: min(grid, ceil(max(n, nnz/4) / vpc)) (see match.cu)
__shared__ int g_cact;

struct ContractArgs {
    const SizeRec *in;  // device: sizes + stop flag of this level's graph
    const int32_t *adjp, *adjncy, *adjwgt, *vwgt;
    int32_t *M, *CM;
    int32_t *off, *cnt, *tile_start, *huge, *lofs;
    int32_t *tagg1;             // C1 warp-tile aggregates {#leaders, sum ub}
    int32_t *ttot;              // C2 warp-tile totals
    int4 *seg;                  // per coarse row: {start, deg} of the leader and of the partner
    unsigned long long *gkeys;  // C1h scratch at off[c] (nnz entries)
    unsigned long long *tout;   // C2a output scratch at each tile's ub offset (nnz entries)
    int32_t *cadjp, *cadjncy, *cadjwgt, *cvwgt;  // coarse graph (upper-bound sized)
    ContractCtl *ctl;
    SizeRec *out;  // device: sizes + stop decision of the coarse graph
    int32_t apply_leftover;
    int32_t threshold, stall_pct, level, max_levels;
    LevelReport *report;  // mapped host memory (may be null)
    int32_t vpc;          // vertices (or 4 arcs) per active CTA
    // sharded levels (dist.cu): C1 ran as separate kernels (seg, off, cvwgt, CM, tile starts,
    // huge rows and ctl->n_coarse / n_huge are given); coarse row c has the global id
    // cbase + c; adjncy/adjwgt hold the local rows followed by the shipped partner rows; the
    // host takes the stop decision.  Single GPU: dist = 0, cbase = 0.
    int32_t dist, cbase, tb_fixed, nnz_ub;
    int32_t prof;    // GP_PROF=1: slowest C2a warp tile (ctl->dbg)
    // single-pass coarse CSR assembly (single GPU): decoupled look-back over the C2 warp tiles
    unsigned long long *status;  // one status word per tile (ctx->status; epoch-tagged, never reset)
    uint32_t epoch;
    int32_t warp_max;  // single GPU: rows up to this bound merged by a warp in C2a (kWB..2*kWB)
    int32_t giant_ub;  // single GPU: C1h rows longer than this merged by the whole grid (0: off)
    int32_t knobs;  // bit 0: route 65..kWB rows of small levels to C1h (GP_C1H_SMALL=1); bit 1: two-pass only (GP_C2_SP=0)
};
__device__ __forceinline__ bool small_hub_on(const ContractArgs &a) { return a.knobs & 1; }

struct ContractSmem {
    unsigned long long buf[kBuf];
    int32_t scan[40];
    int32_t red[2][kCW];
    int32_t wlen[kCW];
    int32_t lead[kCNT], has[kCNT];
    int32_t len, last;
};

// ---------------------------------------------------------------------------------------
// merge helpers
// ---------------------------------------------------------------------------------------
// CM gathers: L2 (ld.global.cg) by default; GP_CM_CA=1 at build time reads them through L1
// (safe: CM is written by C1b, a phase that ends with a grid barrier whose acquire invalidates
// every SM's L1).
#ifdef GP_CM_CA
__device__ __forceinline__ int32_t ldCM(const int32_t *p) { return __ldca(p); }
#else
__device__ __forceinline__ int32_t ldCM(const int32_t *p) { return __ldcg(p); }
#endif

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

__device__ __forceinline__ bool is_head(const unsigned long long *keys, int i) {
    return i == 0 || (keys[i] >> 32) != (keys[i - 1] >> 32);
}

// ---------------------------------------------------------------------------------------
// block-wide helpers (all threads call)
// ---------------------------------------------------------------------------------------
__device__ __forceinline__ void block_sum2(ContractSmem &sm, int32_t &x, int32_t &y) {
    const int l = threadIdx.x & 31, w = threadIdx.x >> 5;
    int32_t a = warp_sum(x), b = warp_sum(y);
    if (l == 0) {
        sm.red[0][w] = a;
        sm.red[1][w] = b;
    }
    __syncthreads();
    a = 0;
    b = 0;
#pragma unroll
    for (int q = 0; q < kCW; ++q) {
        a += sm.red[0][q];
        b += sm.red[1][q];
    }
    __syncthreads();
    x = a;
    y = b;
}

// exclusive scan of vals[k*stride + comp] for k in [0, cnt) into out[k] (shared), plus base;
// returns the sum of the list
__device__ __forceinline__ int32_t block_scan_list(ContractSmem &sm, const int32_t *vals, int stride, int comp,
                                                   int cnt, int32_t base, int32_t *out) {
    const int per = (cnt + kCNT - 1) / kCNT;
    const int lo = min(cnt, (int)threadIdx.x * per), hi = min(cnt, lo + per);
    int32_t s = 0;
    for (int k = lo; k < hi; ++k) s += __ldcg(vals + (size_t)k * stride + comp);
    int32_t tot;
    int32_t run = base + block_excl_scan<kCNT>(s, sm.scan, tot);
    for (int k = lo; k < hi; ++k) {
        out[k] = run;
        run += __ldcg(vals + (size_t)k * stride + comp);
    }
    __syncthreads();
    return tot;
}

__device__ __forceinline__ int32_t warp_excl(int32_t v, int32_t &total) {
    const int32_t inc = warp_incl_scan(v);
    total = __shfl_sync(0xffffffffu, inc, 31);
    return inc - v;
}

// ---------------------------------------------------------------------------------------
// C1a: leftover + leader flags + warp-tile aggregates (+ chunk sums of C1b's owners)
// ---------------------------------------------------------------------------------------
__device__ void phase_c1a(const ContractArgs &a, int32_t n, int nt1, int T1) {
    const int lane = threadIdx.x & 31;
    const int gw = blockIdx.x * kCW + (threadIdx.x >> 5), nw = g_cact * kCW;
    for (int wt = gw; wt < nt1; wt += nw) {
        const long long base = (long long)wt * kVW;
        int32_t cnt = 0, ubs = 0;
#pragma unroll
        for (int i = 0; i < kCItems; ++i) {
            const long long u = base + i * 32 + lane;  // coalesced
            if (u < n) {
                int32_t m = a.M[u];
                if (m == kFree && a.apply_leftover) {
                    m = (int32_t)u;  // leftover: matched to itself (P18.s12-13)
                    a.M[u] = m;
                }
                if (u <= m) {  // leader flag (P18.s18, R7)
                    ++cnt;
                    ubs += __ldg(a.adjp + u + 1) - __ldg(a.adjp + u);
                    if (m != u) ubs += __ldg(a.adjp + m + 1) - __ldg(a.adjp + m);  // P20.s6-8
                }
            }
        }
        cnt = warp_sum(cnt);
        ubs = warp_sum(ubs);
        if (lane == 0) {
            a.tagg1[2 * wt] = cnt;
            a.tagg1[2 * wt + 1] = ubs;
            atomicAdd(&a.ctl->chunk1[2 * (wt / T1)], cnt);
            atomicAdd(&a.ctl->chunk1[2 * (wt / T1) + 1], ubs);
        }
    }
}

// ---------------------------------------------------------------------------------------
// C1b: CM, cvwgt, off, seg, C2 warp-tile starts, huge rows
// ---------------------------------------------------------------------------------------
__device__ void phase_c1b(const ContractArgs &a, ContractSmem &sm, int32_t n, int nt1, int T1, int32_t hub_ub) {
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int t_lo = blockIdx.x * T1, t_hi = min(nt1, t_lo + T1);
    if (t_lo >= t_hi) return;
    int32_t pc = 0, pu = 0;
    for (int b = threadIdx.x; b < (int)blockIdx.x; b += kCNT) {
        pc += __ldcg(a.ctl->chunk1 + 2 * b);
        pu += __ldcg(a.ctl->chunk1 + 2 * b + 1);
    }
    block_sum2(sm, pc, pu);
    int32_t *tpc = reinterpret_cast<int32_t *>(sm.buf);  // segments of <= kBuf tiles per value
    int32_t *tpu = tpc + kBuf;
    for (int s_lo = t_lo; s_lo < t_hi; s_lo += kBuf) {
    const int s_hi = min(t_hi, s_lo + kBuf);
    pc += block_scan_list(sm, a.tagg1 + 2 * s_lo, 2, 0, s_hi - s_lo, pc, tpc);
    pu += block_scan_list(sm, a.tagg1 + 2 * s_lo, 2, 1, s_hi - s_lo, pu, tpu);
    for (int t = s_lo + wib; t < s_hi; t += kCW) {
        // step i of the tile covers the vertices tbase + i*32 + lane: every load and the CM
        // store are coalesced; the scan runs step by step (ballot for the leader ranks, a
        // warp scan for the upper bounds) with running totals
        const long long tbase = (long long)t * kVW;
        int32_t m[kCItems];
#pragma unroll
        for (int i = 0; i < kCItems; ++i) {
            const long long u = tbase + i * 32 + lane;
            m[i] = u < n ? a.M[u] : -2;  // L1-cached: the grid barrier's acquire invalidated L1
        }
        int32_t su[kCItems], du[kCItems], sv[kCItems], dv[kCItems], vw[kCItems];
#pragma unroll
        for (int i = 0; i < kCItems; ++i) {
            const long long u = tbase + i * 32 + lane;
            const bool lead = u < n && u <= m[i];
            const bool pair = u < n && u < m[i];
            su[i] = lead ? __ldg(a.adjp + u) : 0;
            du[i] = lead ? __ldg(a.adjp + u + 1) : 0;
            sv[i] = pair ? __ldg(a.adjp + m[i]) : 0;
            dv[i] = pair ? __ldg(a.adjp + m[i] + 1) : 0;
            vw[i] = (lead ? __ldg(a.vwgt + u) : 0) + (pair ? __ldg(a.vwgt + m[i]) : 0);  // P12.s27
        }
        int32_t c = tpc[t - s_lo], o = tpu[t - s_lo];
        const unsigned lt = lanemask_lt();
#pragma unroll
        for (int i = 0; i < kCItems; ++i) {
            const long long u = tbase + i * 32 + lane;
            const bool lead = u < n && u <= m[i];
            const int32_t dl = du[i] - su[i];
            const int32_t d = lead ? dl + (dv[i] - sv[i]) : 0;  // P20.s6-8
            const unsigned bl = __ballot_sync(0xffffffffu, lead);
            int32_t dtot;
            const int32_t dex = warp_excl(d, dtot);
            if (lead) {
                const int32_t cc = c + __popc(bl & lt);  // exclusive scan = inclusive - 1 (P18.s20-24)
                const int32_t oo = o + dex;
                const int32_t v = m[i];
                a.CM[u] = cc;
                if (v != u) a.CM[v] = cc;  // partner copies its leader's id (P18.s26)
                a.cvwgt[cc] = vw[i];
                a.off[cc] = oo;
                a.seg[cc] = make_int4(su[i], dl, sv[i], d - dl);
                if (d > hub_ub) a.huge[atomicAdd(&a.ctl->n_huge, 1)] = cc;
                if (a.giant_ub > 0 && d > a.giant_ub) {  // merged by the whole grid (phase_c1h_giant)
                    const int32_t gi = atomicAdd(&a.ctl->n_giant, 1);
                    if (gi < kMaxGiant) a.ctl->giant[gi] = cc;
                }
            }
            c += __popc(bl);
            o += dtot;
        }
        if (t == nt1 - 1 && lane == 0) {
            a.ctl->n_coarse = c;
            a.off[c] = o;  // = nnz
        }
    }
    __syncthreads();  // the prefix arrays are rewritten by the next segment
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
            const int32_t cx = ldCM(a.CM + __ldcs(a.adjncy + j));
            if (cx != c + a.cbase) dst[claim()] = ckey(cx, __ldcs(a.adjwgt + j));  // drop the collapsed edge (R9)
        }
    }
}

// ---------------------------------------------------------------------------------------
// Long rows (> kCtaRow keys, R-MAT hubs): runs of kCtaRow keys are sorted in shared memory,
// then merged pairwise through global memory (merge path, windows of kMW outputs staged in
// shared memory; the window split points of a batch are searched by all threads at once).
// A bitonic network over global memory (the earlier design) paid ~log^2 dependent passes.
// ---------------------------------------------------------------------------------------
constexpr int kBigTile = 4096;  // C2b: tiles with more merged keys are copied by the whole CTA
constexpr int kMW = kBuf / 2;  // outputs per merge window (A and B pieces staged side by side)

// number of A elements among the first d outputs of merge(A, B) (A first on ties)
__device__ __forceinline__ int32_t merge_path(const unsigned long long *A, int32_t la, const unsigned long long *B,
                                              int32_t lb, int32_t d) {
    int32_t lo = max(0, d - lb), hi = min(d, la);
    while (lo < hi) {
        const int32_t mid = (lo + hi) >> 1;
        if (A[mid] <= B[d - mid - 1]) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

// CTA merge of sorted A[0, la) and B[0, lb) into O (all global); all threads call
__device__ void cta_merge(ContractSmem &sm, const unsigned long long *A, int32_t la, const unsigned long long *B,
                          int32_t lb, unsigned long long *O) {
    const int tid = threadIdx.x;
    const int32_t m = la + lb;
    int32_t *split = sm.lead;  // lead[] and has[] are adjacent: kCNT + 1 split points fit
    const int32_t nwin = (m + kMW - 1) / kMW;
    for (int32_t wb0 = 0; wb0 < nwin; wb0 += kCNT) {
        const int32_t nbw = min(kCNT, nwin - wb0);
        for (int t = tid; t <= nbw; t += kCNT) split[t] = merge_path(A, la, B, lb, min(m, (wb0 + t) * kMW));
        __syncthreads();
        for (int32_t w = 0; w < nbw; ++w) {
            const int32_t d0 = (wb0 + w) * kMW, d1 = min(m, d0 + kMW);
            const int32_t i0 = split[w], i1 = split[w + 1], j0 = d0 - i0, j1 = d1 - i1;
            const int32_t na = i1 - i0, nb = j1 - j0;
            for (int32_t t = tid; t < na; t += kCNT) sm.buf[t] = A[i0 + t];
            for (int32_t t = tid; t < nb; t += kCNT) sm.buf[kMW + t] = B[j0 + t];
            __syncthreads();
            constexpr int kPer = kMW / kCNT;
            const int32_t dl = tid * kPer;
            if (dl < na + nb) {
                const unsigned long long *sa = sm.buf, *sb = sm.buf + kMW;
                int32_t i = merge_path(sa, na, sb, nb, dl), j = dl - i;
#pragma unroll
                for (int k = 0; k < kPer; ++k) {
                    if (dl + k < na + nb) {
                        const bool ta = j >= nb || (i < na && sa[i] <= sb[j]);
                        O[d0 + dl + k] = ta ? sa[i] : sb[j];
                        i += ta ? 1 : 0;
                        j += ta ? 0 : 1;
                    }
                }
            }
            __syncthreads();
        }
    }
}

// sort keys[0, len) (global) in place; tmp: len entries of global scratch
__device__ __noinline__ void cta_sort_long(ContractSmem &sm, unsigned long long *keys, unsigned long long *tmp, int32_t len) {
    const int tid = threadIdx.x;
    for (int32_t r0 = 0; r0 < len; r0 += kCtaRow) {  // sorted runs of kCtaRow keys
        const int32_t rl = min(kCtaRow, len - r0);
        for (int32_t t = tid; t < rl; t += kCNT) sm.buf[t] = keys[r0 + t];
        __syncthreads();
        coop_sort(sm.buf, rl, tid, kCNT, []() { __syncthreads(); });
        for (int32_t t = tid; t < rl; t += kCNT) keys[r0 + t] = sm.buf[t];
        __syncthreads();
    }
    unsigned long long *src = keys, *dst = tmp;
    for (int32_t run = kCtaRow; run < len; run *= 2) {
        for (int32_t a0 = 0; a0 < len; a0 += 2 * run) {
            const int32_t la = min(run, len - a0), lb = max(0, min(run, len - a0 - la));
            cta_merge(sm, src + a0, la, src + a0 + la, lb, dst + a0);
        }
        unsigned long long *x = src;
        src = dst;
        dst = x;
    }
    if (src != keys) {
        for (int32_t t = tid; t < len; t += kCNT) keys[t] = src[t];
    }
    __syncthreads();
}

// Run-sum + compaction of a sorted long row keys[0, len) (global) in place, window by window
// through shared memory: each window's runs are summed and compacted in smem, the window's
// last run is held back (it may continue into the next window) and the rest is written at
// the row's compacted position (always <= the window start: no unread key is overwritten).
__device__ int32_t long_runsum_compact(ContractSmem &sm, unsigned long long *keys, int32_t len) {
    const int tid = threadIdx.x;
    int32_t wr = 0;
    unsigned long long pend = 0;
    bool has_pend = false;  // uniform
    for (int32_t w0 = 0; w0 < len; w0 += kBuf) {
        const int32_t wl = min(kBuf, len - w0);
        for (int32_t t = tid; t < wl; t += kCNT) sm.buf[t] = keys[w0 + t];
        __syncthreads();
        const int32_t cntw = coop_runsum(
            sm.buf, wl, tid, kCNT, sm.lead, sm.has,
            [&](int32_t v, int32_t &tot) { return block_excl_scan<kCNT>(v, sm.scan, tot); },
            []() { __syncthreads(); });
        int32_t hw = 0;  // compact the window's heads to sm.buf[0, cntw) (in place, as in C1h)
        for (int32_t b0 = 0; b0 < wl; b0 += kCNT) {
            const int32_t j = b0 + tid;
            const unsigned long long kv = j < wl ? sm.buf[j] : 0ull;
            const bool h = j < wl && is_head(sm.buf, j);
            int32_t tot;
            const int32_t ex = block_excl_scan<kCNT>(h ? 1 : 0, sm.scan, tot);
            if (h) sm.buf[hw + ex] = kv;
            hw += tot;
            __syncthreads();
        }
        // the pending run of the previous window: continued by this window's first run, or done
        const bool cont = has_pend && (uint32_t)(sm.buf[0] >> 32) == (uint32_t)(pend >> 32);
        __syncthreads();
        if (tid == 0) {
            if (cont) sm.buf[0] = (pend & 0xFFFFFFFF00000000ull) | (uint32_t)((uint32_t)pend + (uint32_t)sm.buf[0]);
            else if (has_pend) keys[wr] = pend;
        }
        if (has_pend && !cont) ++wr;
        __syncthreads();
        for (int32_t t = tid; t < cntw - 1; t += kCNT) keys[wr + t] = sm.buf[t];
        wr += cntw - 1;
        pend = sm.buf[cntw - 1];
        has_pend = true;
        __syncthreads();
    }
    if (has_pend) {
        if (tid == 0) keys[wr] = pend;
        ++wr;
    }
    __syncthreads();
    return wr;
}

// ---------------------------------------------------------------------------------------
// C1h giant rows (single GPU, ub > giant_ub: R-MAT hubs of 10^4-10^5 arcs): merged by GROUPS
// of CTAs, one row per group at a time, through a dense accumulator over the coarse ids and a
// presence bitmap (both in the idle `tout`): every CTA adds its share of the row's arcs into
// acc[CM[x]] (weights summed, R8; collapsed edge dropped, R9), the first add of an id sets its
// bit; each CTA then counts the bits of its slice of the bitmap, and after a prefix over the
// CTAs writes its ids in increasing order (rows come out sorted by coarse id, R10), resetting
// both as it goes.  ~3 group barriers and nc / 32 words per row, whatever the row length.
// One CTA sorting a 400 K-key hub row took 25-29 ms and was the whole C1h phase on C4.
// ---------------------------------------------------------------------------------------
// barrier of the CTAs of one group (a running count: completes at the sum of the group's
// arrivals so far)
__device__ __forceinline__ void group_barrier(unsigned *bar, unsigned &target, unsigned gs) {
    __syncthreads();
    if (threadIdx.x == 0) {
        target += gs;
        red_release_add_u32(bar, 1u);
        const long long guard = spin_start();
        while ((int)(ld_acquire_u32(bar) - target) < 0) spin_check(guard);
    }
    __syncthreads();
}

__device__ __noinline__ void phase_c1h_giant(const ContractArgs &a, ContractSmem &sm, int32_t ng, int32_t nc,
                                             int32_t G) {
    // G independent groups of CTAs (b % G), each with its own accumulator + bitmap region of
    // the idle tout and its own barrier; group gb takes giant rows gb, gb + G, ...
    ContractCtl *ctl = a.ctl;
    const int32_t nw = (nc + 31) >> 5;
    const int gb = (int)blockIdx.x % G, r = (int)blockIdx.x / G;
    const unsigned gs = (unsigned)((g_cact - gb + G - 1) / G);  // CTAs in this group
    const size_t stride = ((size_t)nc + (size_t)nw + 64) & ~(size_t)31;
    int32_t *acc = reinterpret_cast<int32_t *>(a.tout) + stride * gb;  // weights by coarse id
    uint32_t *bm = reinterpret_cast<uint32_t *>(acc + nc + 32);        // presence bits
    unsigned *gbar = ctl->gbar + gb;
    unsigned gtarget = 0;  // (thread 0)
    const long long gthreads = (long long)gs * kCNT, gtid = (long long)r * kCNT + threadIdx.x;
    for (long long i = gtid; i < nc; i += gthreads) acc[i] = 0;
    for (long long i = gtid; i < nw; i += gthreads) bm[i] = 0u;
    group_barrier(gbar, gtarget, gs);
    // this CTA's bitmap words [w0, w1) = coarse ids [32 w0, 32 w1), per thread contiguous
    const int32_t w0 = (int32_t)((long long)nw * r / gs), w1 = (int32_t)((long long)nw * (r + 1) / gs);
    const int32_t per = (w1 - w0 + kCNT - 1) / kCNT;
    const int32_t t0w = min(w1, w0 + (int32_t)threadIdx.x * per), t1w = min(w1, t0w + per);
    for (int32_t gi = gb; gi < ng; gi += G) {
        const int32_t c = ctl->giant[gi];
        const int32_t o0 = __ldcg(a.off + c);
        const int32_t ub = __ldcg(a.off + c + 1) - o0;
        const int4 sg = __ldcg(a.seg + c);
        for (long long p = gtid; p < ub; p += gthreads) {
            const int32_t pi = (int32_t)p;
            const int32_t j = pi < sg.y ? sg.x + pi : sg.z + (pi - sg.y);
            const int32_t cx = ldCM(a.CM + __ldcs(a.adjncy + j));
            if (cx != c + a.cbase) {
                if (atomicAdd(acc + cx, __ldcs(a.adjwgt + j)) == 0) atomicOr(bm + (cx >> 5), 1u << (cx & 31));
            }
        }
        group_barrier(gbar, gtarget, gs);
        int32_t mine = 0;
        for (int32_t w = t0w; w < t1w; ++w) mine += __popc(__ldcg(bm + w));
        int32_t tot;
        const int32_t ex = block_excl_scan<kCNT>(mine, sm.scan, tot);
        if (threadIdx.x == 0) ctl->chunk2[blockIdx.x] = tot;  // (C2's chunk sums: idle until C2)
        group_barrier(gbar, gtarget, gs);
        if (threadIdx.x < 32) {  // prefix over the group's lower ranks
            int32_t pre = 0, all = 0;
            for (int q = threadIdx.x; q < (int)gs; q += 32) {
                const int32_t x = __ldcg(ctl->chunk2 + gb + q * G);
                all += x;
                pre += q < r ? x : 0;
            }
            pre = warp_sum(pre);
            all = warp_sum(all);
            if (threadIdx.x == 0) {
                sm.last = pre;
                if (r == 0) a.cnt[c] = all;
            }
        }
        __syncthreads();
        unsigned long long *dst = a.gkeys + o0;
        int32_t wr = sm.last + ex;
        for (int32_t w = t0w; w < t1w; ++w) {  // ids in increasing order: rows sorted by coarse id (R10)
            uint32_t bits = __ldcg(bm + w);
            if (!bits) continue;
            bm[w] = 0u;
            while (bits) {
                const int b = __ffs(bits) - 1;
                bits &= bits - 1;
                const int32_t cx = (w << 5) + b;
                dst[wr++] = ckey(cx, __ldcg(acc + cx));  // summed weight (R8); fits int32 (R14)
                acc[cx] = 0;
            }
        }
        group_barrier(gbar, gtarget, gs);  // the accumulator is clean for the group's next row
    }
    // chunk2 accumulates C2's per-CTA sums by atomics from zero: clear this CTA's entry (made
    // visible by the grid barrier that follows C1h)
    if (threadIdx.x == 0) ctl->chunk2[blockIdx.x] = 0;
}

// ---------------------------------------------------------------------------------------
// C1h: rows with ub > kWB, one CTA each; result compacted at gkeys[off[c]], count cnt[c]
// ---------------------------------------------------------------------------------------
__device__ __noinline__ void phase_c1h(const ContractArgs &a, ContractSmem &sm, int32_t nh, bool giant_done) {
    // rows are claimed dynamically (first one static): a CTA busy with a 400 K-key hub row
    // takes no further rows, instead of a fixed 1/nact share of them
    for (int i = blockIdx.x; i < nh;) {
        const int32_t c = a.huge[i];
        const int32_t o0 = __ldcg(a.off + c);
        const int32_t ub = __ldcg(a.off + c + 1) - o0;
        if (giant_done && ub > a.giant_ub) {  // merged by the whole grid already
            if (threadIdx.x == 0) sm.last = g_cact + (int)atomicAdd(&a.ctl->hub_ctr, 1u);
            __syncthreads();
            i = sm.last;
            __syncthreads();
            continue;
        }
        const unsigned long long tc0 = a.prof ? globaltimer() : 0ull;
        unsigned long long *dst = a.gkeys + o0;
        unsigned long long *keys = (ub <= kCtaRow) ? sm.buf : dst;
        // gather at fixed positions (leader's arcs, then the partner's; 4 per thread in flight);
        // the collapsed edge becomes kMaxKey, sorts last and is cut off (no claim atomics)
        const int4 sg = __ldcg(a.seg + c);
        int32_t nself = 0, dummy = 0;
        for (int32_t p0 = threadIdx.x; p0 < ub; p0 += 4 * kCNT) {
            int32_t x[4], w[4], cx[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int32_t p = p0 + q * kCNT;
                const int32_t j = p < sg.y ? sg.x + p : sg.z + (p - sg.y);
                x[q] = p < ub ? __ldcs(a.adjncy + j) : -1;
                w[q] = p < ub ? __ldcs(a.adjwgt + j) : 0;
            }
#pragma unroll
            for (int q = 0; q < 4; ++q) cx[q] = x[q] >= 0 ? ldCM(a.CM + x[q]) : 0;
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int32_t p = p0 + q * kCNT;
                if (p < ub) {
                    const bool self = cx[q] == c + a.cbase;  // collapsed edge dropped (R9)
                    keys[p] = self ? kMaxKey : ckey(cx[q], w[q]);
                    nself += self ? 1 : 0;
                }
            }
        }
        block_sum2(sm, nself, dummy);  // (syncs: the keys are complete)
        const int len = ub - nself;
        if (ub <= kCtaRow) coop_sort(keys, ub, threadIdx.x, kCNT, []() { __syncthreads(); });
        else cta_sort_long(sm, keys, a.tout + o0, ub);  // tout is idle until C2a
        int32_t cnt;
        if (ub > kCtaRow) {
            cnt = long_runsum_compact(sm, dst, len);
        } else {
            cnt = coop_runsum(
                keys, len, threadIdx.x, kCNT, sm.lead, sm.has,
                [&](int32_t v, int32_t &tot) { return block_excl_scan<kCNT>(v, sm.scan, tot); },
                []() { __syncthreads(); });
            // compact the run heads into dst
            int32_t wr = 0;
            for (int32_t b0 = 0; b0 < len; b0 += kCNT) {
                const int32_t j = b0 + threadIdx.x;
                const unsigned long long kv = j < len ? keys[j] : 0ull;
                const bool h = j < len && is_head(keys, j);
                int32_t tot;
                const int32_t ex = block_excl_scan<kCNT>(h ? 1 : 0, sm.scan, tot);
                if (h) dst[wr + ex] = kv;
                wr += tot;
                __syncthreads();
            }
        }
        if (threadIdx.x == 0) {
            a.cnt[c] = cnt;
            sm.last = g_cact + (int)atomicAdd(&a.ctl->hub_ctr, 1u);
            if (a.prof) {  // GP_PROF=1: C1h rows: sum of upper bounds; slowest row (ns << 32 | ub)
                atomicAdd(&a.ctl->dbg[6], (unsigned long long)ub);
                atomicMax(&a.ctl->dbg[7], ((globaltimer() - tc0) << 24) | (unsigned long long)min(ub, (1 << 24) - 1));
            }
        }
        __syncthreads();
        i = sm.last;
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------------------
// C2a: warp tiles: merge every row, write the tile compacted to tout at its ub offset
// ---------------------------------------------------------------------------------------
__device__ void phase_c2a(const ContractArgs &a, ContractSmem &sm, int32_t ntiles2, int T2, int32_t nc, int32_t rt,
                          bool single_pass, int32_t hub_ub) {
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int gw = blockIdx.x * kCW + wib, nw = g_cact * kCW;
    unsigned long long *wb = sm.buf + wib * 2 * kWB;  // this warp's slots (2*kWB entries)
    // warp tiles are claimed dynamically from one global counter: the merge cost of a tile
    // varies (row mix, C1h copies), and a static split per CTA leaves barrier tails
    // (measured: +30 % on the phase at small levels)
    // (the first tile of a warp is static -- tile gw -- so no claim round trip precedes it)
    for (int wt = gw;;) {
        wt = __shfl_sync(0xffffffffu, wt, 0);
        if (wt >= ntiles2) break;
        const unsigned long long tt0 = a.prof ? globaltimer() : 0ull;
        int32_t nw64 = 0;
        int32_t r0 = 0, r1 = 0;
        if (a.dist) {  // sharded levels: tiles of <= tb upper-bound entries (dist.cu k_dc_tiles)
            if (lane < 2) r0 = __ldcg(a.tile_start + wt + lane);
            r1 = __shfl_sync(0xffffffffu, r0, 1);
            r0 = __shfl_sync(0xffffffffu, r0, 0);
        } else {  // rt (<= 32) consecutive coarse rows
            r0 = wt * rt;
            r1 = min(nc, r0 + rt);
        }
        unsigned long long *out = a.tout + (r0 < r1 ? __ldcg(a.off + r0) : 0);
        int32_t run = 0;
        // single-pass assembly (single GPU): a tile whose rows merge in ONE pass keeps them in
        // its slot area (C1h rows stay in gkeys) until its look-back prefix is known, then
        // writes them straight into cadjncy / cadjwgt; a multi-pass tile stages its passes in
        // tout (the slot area is reused) and copies them out after the look-back.
        const bool sp1 = single_pass;
        bool spilled = false;                      // an earlier pass of this tile went to tout
        int32_t myoff = INT32_MAX, myslot = 0;     // this lane's row: offset in the tile, slot
        bool myhub = false;                        // ... merged by C1h (keys in gkeys)
        for (int32_t g0 = r0; g0 < r1; g0 += 32) {
            const int32_t c = g0 + lane;
            int32_t ub = 0, hcnt = 0;
            int4 sg = make_int4(0, 0, 0, 0);
            if (c < r1) {
                const int32_t o0 = __ldcg(a.off + c);
                ub = __ldcg(a.off + c + 1) - o0;
                if (ub <= kWarpNet) sg = __ldcg(a.seg + c);
                if (ub > hub_ub) hcnt = __ldcg(a.cnt + c);  // merged by C1h
            }
            // Passes over the 32 rows: a pass takes the next lanes whose slots (ub of rows
            // <= kWB; C1h rows take none) fit the warp's 2kWB slot area -- one pass unless the
            // rows are long.  The first lane of a pass always fits (ub <= kWB).
            for (int32_t first = 0;;) {
            const bool inr = c < r1 && lane >= first;
            const int32_t used = warp_incl_scan((inr && ub <= hub_ub) ? ub : 0);  // all lanes: a shuffle scan
            const bool act = inr && used <= 2 * kWB;
            const unsigned pm = __ballot_sync(0xffffffffu, act);
            int32_t cntc = (act && ub > hub_ub) ? hcnt : 0;
            // Positions in the slot area: rows with ub <= 64 (staged) packed first, rows of
            // 65..kWB entries after them.
            const bool srow = act && ub <= kWarpNet;
            const bool mrow = act && ub > kWarpNet && ub <= hub_ub;
            int32_t S, Mt;
            const int32_t sp = warp_excl(srow ? ub : 0, S);
            const int32_t sq = S + warp_excl(mrow ? ub : 0, Mt);
            const int32_t slot = srow ? sp : sq;
            // ---- staging, coalesced: each staged row writes its arc indices into its slots
            // (the map), then lane e of a step owns flat slot idx: arc -> (adjncy, adjwgt)
            // -> CM, and overwrites the slot with the key (cx << 32 | w) ----
            if (srow) {
                for (int32_t q = 0; q < sg.y; ++q) wb[sp + q] = (unsigned long long)(sg.x + q);
                for (int32_t q = 0; q < sg.w; ++q) wb[sp + sg.y + q] = (unsigned long long)(sg.z + q);
            }
            __syncwarp();
            {
                // two sweeps of up to 16 steps (512 slots: a whole pass) so that every load of
                // a level is in flight together: (adjncy, adjwgt) -> slot as (x << 32 | w), then
                // CM[x] replaces the slot's high word -> key (cx << 32 | w)
                constexpr int kB = 16;
                uint32_t *wb32 = reinterpret_cast<uint32_t *>(wb);
                for (int32_t b0 = 0; b0 < S; b0 += 32 * kB) {
                    int32_t x[kB], w[kB];
#pragma unroll
                    for (int k = 0; k < kB; ++k) {
                        const int32_t idx = b0 + k * 32 + lane;
                        const int32_t jj = idx < S ? (int32_t)wb32[2 * idx] : -1;
                        x[k] = jj >= 0 ? __ldcs(a.adjncy + jj) : -1;
                        w[k] = jj >= 0 ? __ldcs(a.adjwgt + jj) : 0;
                    }
#pragma unroll
                    for (int k = 0; k < kB; ++k) {
                        const int32_t idx = b0 + k * 32 + lane;
                        if (idx < S) {
                            wb32[2 * idx] = (uint32_t)w[k];
                            wb32[2 * idx + 1] = (uint32_t)x[k];
                        }
                    }
                }
                __syncwarp();
                for (int32_t b0 = 0; b0 < S; b0 += 32 * kB) {
                    int32_t cx[kB];
#pragma unroll
                    for (int k = 0; k < kB; ++k) {
                        const int32_t idx = b0 + k * 32 + lane;
                        const int32_t x = idx < S ? (int32_t)wb32[2 * idx + 1] : -1;
                        cx[k] = x >= 0 ? ldCM(a.CM + x) : 0;
                    }
#pragma unroll
                    for (int k = 0; k < kB; ++k) {
                        const int32_t idx = b0 + k * 32 + lane;
                        if (idx < S) wb32[2 * idx + 1] = (uint32_t)cx[k];
                    }
                }
                __syncwarp();
            }
            const uint32_t self = (uint32_t)(c + a.cbase);  // the collapsed edge's coarse id (R9)
            // rows of 17..32 entries: two at a time, one per half-warp, merged in place
            unsigned m32 = __ballot_sync(0xffffffffu, srow && ub > kNet && ub <= 2 * kNet);
            nw64 += __popc(m32);
            while (m32) {
                const int sa = __ffs(m32) - 1;
                m32 &= m32 - 1;
                const int sb = m32 ? __ffs(m32) - 1 : -1;
                if (sb >= 0) m32 &= m32 - 1;
                const int src = (lane & 16) ? sb : sa;  // this half-warp's row (-1: idle)
                const int s0 = src < 0 ? sa : src;
                const int32_t sl = __shfl_sync(0xffffffffu, sp, s0);
                const int32_t rub0 = __shfl_sync(0xffffffffu, ub, s0);  // all lanes shuffle
                const int32_t rub = src < 0 ? 0 : rub0;
                const uint32_t rself = __shfl_sync(0xffffffffu, self, s0);
                unsigned long long v[2];
#pragma unroll
                for (int r = 0; r < 2; ++r) {
                    const int32_t e = r * 16 + (lane & 15);
                    v[r] = (e < rub) ? wb[sl + e] : kMaxKey;
                    if ((uint32_t)(v[r] >> 32) == rself) v[r] = kMaxKey;  // collapsed edge dropped
                }
                __syncwarp();
                seg_sort32(v);
                unsigned long long dummy[1];
                const int32_t cc = seg_runmerge32(v, src < 0 ? dummy : wb + sl);  // idle half: all padding
                __syncwarp();
                const int32_t cca = __shfl_sync(0xffffffffu, cc, 0), ccb = __shfl_sync(0xffffffffu, cc, 16);
                if (lane == sa) cntc = cca;  // the owners may sit in either half
                if (lane == sb) cntc = ccb;
            }
            // rows of 33..64 entries: the warp, registers + shuffles, merged in place
            unsigned m64 = __ballot_sync(0xffffffffu, srow && ub > 2 * kNet);
            nw64 += __popc(m64);
            while (m64) {
                const int src = __ffs(m64) - 1;
                m64 &= m64 - 1;
                const int32_t sl = __shfl_sync(0xffffffffu, sp, src);
                const int32_t rub = __shfl_sync(0xffffffffu, ub, src);
                const uint32_t rself = __shfl_sync(0xffffffffu, self, src);
                unsigned long long v[2];
#pragma unroll
                for (int r = 0; r < 2; ++r) {
                    const int32_t e = r * 32 + lane;
                    v[r] = (e < rub) ? wb[sl + e] : kMaxKey;
                    if ((uint32_t)(v[r] >> 32) == rself) v[r] = kMaxKey;  // collapsed edge dropped
                }
                __syncwarp();
                warp_sort64(v);
                const int32_t cc = warp_runmerge64(v, wb + sl);  // compacted in the slot
                __syncwarp();
                if (lane == src) cntc = cc;
            }
            // rows of 65..kWB entries: the warp, shared-memory sort in the slot, compacted
            unsigned mm = __ballot_sync(0xffffffffu, mrow);
            while (mm) {
                const int src = __ffs(mm) - 1;
                mm &= mm - 1;
                const int32_t cw = __shfl_sync(0xffffffffu, c, src);
                const int32_t sl = __shfl_sync(0xffffffffu, sq, src);
                unsigned long long *keys = wb + sl;
                if (lane == 0) sm.wlen[wib] = 0;
                __syncwarp();
                gather_row(a, cw, lane, 32, keys, [&]() { return atomicAdd(&sm.wlen[wib], 1); });
                __syncwarp();
                const int len = sm.wlen[wib];
                coop_sort(keys, len, lane, 32, []() { __syncwarp(); });
                const int32_t cc = coop_runsum(
                    keys, len, lane, 32, sm.lead + wib * 32, sm.has + wib * 32,
                    [&](int32_t v, int32_t &tot) { return warp_excl(v, tot); }, []() { __syncwarp(); });
                int32_t wr = 0;
                for (int32_t b0 = 0; b0 < len; b0 += 32) {
                    const int32_t i = b0 + lane;
                    const unsigned long long kv = i < len ? keys[i] : 0ull;
                    const bool h = i < len && is_head(keys, i);
                    const unsigned hm = __ballot_sync(0xffffffffu, h);
                    __syncwarp();
                    if (h) keys[wr + __popc(hm & lanemask_lt())] = kv;
                    wr += __popc(hm);
                    __syncwarp();
                }
                if (lane == src) cntc = cc;
            }
            // rows of <= 16 entries: one thread, registers + odd-even merge network, written
            // back compacted into the row's slots
            if (srow && ub > 0 && ub <= kNet) {
                uint32_t kc[kNet];
                int32_t kw[kNet];
#pragma unroll
                for (int i = 0; i < kNet; ++i) {
                    const unsigned long long kv = (i < ub) ? wb[sp + i] : kMaxKey;
                    kc[i] = (uint32_t)(kv >> 32);
                    kw[i] = (int32_t)(uint32_t)kv;
                    if (kc[i] == self) kc[i] = 0xFFFFFFFFu;  // collapsed edge dropped (R9)
                }
                cx_sort16(kc, kw);
                uint32_t prev = 0xFFFFFFFFu;
                int32_t acc = 0;
#pragma unroll
                for (int i = 0; i < kNet; ++i) {
                    if (kc[i] == prev) {
                        acc += kw[i];  // repeated coarse neighbour: weights summed (R8, P12.s28)
                    } else {
                        if (prev != 0xFFFFFFFFu) wb[sp + cntc++] = ckey((int32_t)prev, acc);
                        prev = kc[i];
                        acc = kw[i];
                    }
                }
                if (prev != 0xFFFFFFFFu) wb[sp + cntc++] = ckey((int32_t)prev, acc);
            }
            int32_t part;
            const int32_t ex = warp_excl(cntc, part);
            const bool last_pass = first + __popc(pm) >= 32 || g0 + first + __popc(pm) >= r1;
            const bool keep = sp1 && last_pass && !spilled && g0 + 32 >= r1;  // whole tile in one pass
            if (act) {
                if (sp1) {
                    myoff = run + ex;
                    myslot = slot;
                    myhub = ub > hub_ub;
                } else {
                    a.lofs[c] = run + ex;
                }
                if (ub <= hub_ub && !keep)
                    for (int32_t j = 0; j < cntc; ++j) __stcs(out + run + ex + j, wb[slot + j]);
            }
            if (!keep) spilled = true;
            // rows merged by C1h: the warp copies them in
            unsigned mh = keep ? 0u : __ballot_sync(0xffffffffu, act && ub > hub_ub);
            while (mh) {
                const int src = __ffs(mh) - 1;
                mh &= mh - 1;
                const int32_t cw = __shfl_sync(0xffffffffu, c, src);
                const int32_t k = __shfl_sync(0xffffffffu, cntc, src);
                const int32_t pos = run + __shfl_sync(0xffffffffu, ex, src);
                const unsigned long long *src_keys = a.gkeys + __ldcg(a.off + cw);
                for (int32_t j0 = 0; j0 < k; j0 += 32 * 8) {  // 8 keys per lane in flight
                    unsigned long long kk[8];
#pragma unroll
                    for (int q = 0; q < 8; ++q) {
                        const int32_t j = j0 + q * 32 + lane;
                        kk[q] = j < k ? __ldcg(src_keys + j) : 0ull;
                    }
#pragma unroll
                    for (int q = 0; q < 8; ++q) {
                        const int32_t j = j0 + q * 32 + lane;
                        if (j < k) out[pos + j] = kk[q];
                    }
                }
            }
            __syncwarp();
            run += part;
            first += __popc(pm);
            if (first >= 32 || g0 + first >= r1) break;
            }
        }
        if (a.prof && lane == 0) {
            const unsigned long long dt = globaltimer() - tt0;
            atomicMax(&a.ctl->dbg[0], (dt << 32) | (unsigned)wt);
            atomicMax(&a.ctl->dbg[1], ((unsigned long long)nw64 << 32) | (unsigned)wt);
            atomicMax(&a.ctl->dbg[2], ((unsigned long long)(r1 - r0) << 32) | (unsigned)wt);
            atomicAdd(&a.ctl->dbg[3], dt);
            atomicAdd(&a.ctl->dbg[4], 1ull);
            atomicAdd(&a.ctl->dbg[5], (unsigned long long)nw64);
        }
        if (sp1) {
            // decoupled look-back over the tiles in claim order (every earlier tile is already
            // claimed by a running warp, so the chain always completes)
            const int32_t prefix = lookback_prefix(a.status, a.epoch, wt, run);
            const int32_t c = r0 + lane;
            if (c < r1) a.cadjp[c] = prefix + myoff;  // (R11)
            if (wt == ntiles2 - 1 && lane == 0) {
                a.cadjp[nc] = prefix + run;
                a.ctl->cnnz = prefix + run;
            }
            if (!spilled) {
                // the tile's rows from the slot area / gkeys, coalesced: entry e belongs to the
                // last row whose offset is <= e (binary search over the lanes' offsets)
                const int32_t hbase = (c < r1 && myhub) ? __ldcg(a.off + c) : 0;
                for (int32_t e = lane; e - lane < run; e += 32) {
                    int r = 0;
#pragma unroll
                    for (int step = 16; step > 0; step >>= 1) {
                        const int32_t o = __shfl_sync(0xffffffffu, myoff, r + step);
                        if (o <= e) r += step;
                    }
                    const int32_t j = e - __shfl_sync(0xffffffffu, myoff, r);
                    const int32_t sl = __shfl_sync(0xffffffffu, myslot, r);
                    const bool hub = __shfl_sync(0xffffffffu, myhub ? 1 : 0, r) != 0;
                    const int32_t hb = __shfl_sync(0xffffffffu, hbase, r);
                    if (e < run) {
                        const unsigned long long kv = hub ? __ldcg(a.gkeys + hb + j) : wb[sl + j];
                        a.cadjncy[prefix + e] = (int32_t)(kv >> 32);
                        a.cadjwgt[prefix + e] = (int32_t)(uint32_t)kv;
                    }
                }
            } else {
                __syncwarp();
                for (int32_t j0 = 0; j0 < run; j0 += 32 * 8) {  // staged passes: tout -> final
                    unsigned long long kk[8];
#pragma unroll
                    for (int q = 0; q < 8; ++q) {
                        const int32_t j = j0 + q * 32 + lane;
                        kk[q] = j < run ? __ldcg(out + j) : 0ull;
                    }
#pragma unroll
                    for (int q = 0; q < 8; ++q) {
                        const int32_t j = j0 + q * 32 + lane;
                        if (j < run) {
                            a.cadjncy[prefix + j] = (int32_t)(kk[q] >> 32);
                            a.cadjwgt[prefix + j] = (int32_t)(uint32_t)kk[q];
                        }
                    }
                }
            }
            __syncwarp();  // the slot area is rebuilt by the next tile
        }
        if (lane == 0) {
            if (!sp1) {
                a.ttot[wt] = run;
                atomicAdd(&a.ctl->chunk2[wt / T2], run);
                if (run > kBigTile) a.ctl->big_flag = 1;  // read by every CTA after the grid barrier
            }
            wt = nw + (int)atomicAdd(&a.ctl->tile_ctr, 1u);
        }
    }
}

// ---------------------------------------------------------------------------------------
// C2b: cadjp + coalesced copy of the tiles of this CTA's chunk into the final CSR
// ---------------------------------------------------------------------------------------
__device__ void phase_c2b(const ContractArgs &a, ContractSmem &sm, int32_t nc, int32_t ntiles2, int T2, int32_t rt,
                          bool balanced) {
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int t_lo = blockIdx.x * T2, t_hi = min(ntiles2, t_lo + T2);
    if (t_lo >= t_hi) return;
    int32_t pre = 0, dummy = 0;
    for (int b = threadIdx.x; b < (int)blockIdx.x; b += kCNT) pre += __ldcg(a.ctl->chunk2 + b);
    block_sum2(sm, pre, dummy);
    int32_t *tp = reinterpret_cast<int32_t *>(sm.buf);
    constexpr int kCap = 2 * kBuf;
    for (int s_lo = t_lo; s_lo < t_hi; s_lo += kCap) {
    const int s_hi = min(t_hi, s_lo + kCap);
    pre += block_scan_list(sm, a.ttot + s_lo, 1, 0, s_hi - s_lo, pre, tp);
    if (threadIdx.x == 0) sm.len = 0;  // tiles too big for one warp (R-MAT hub rows): CTA copies
    __syncthreads();
    for (int t = s_lo + wib; t < s_hi; t += kCW) {
        const int32_t p = tp[t - s_lo];
        int32_t r0 = 0, r1 = 0;
        if (a.dist) {
            if (lane < 2) r0 = __ldcg(a.tile_start + t + lane);
            r1 = __shfl_sync(0xffffffffu, r0, 1);
            r0 = __shfl_sync(0xffffffffu, r0, 0);
        } else {
            r0 = t * rt;
            r1 = min(nc, r0 + rt);
        }
        const int32_t total = __ldcg(a.ttot + t);
        for (int32_t c = r0 + lane; c < r1; c += 32) a.cadjp[c] = p + __ldcg(a.lofs + c);
        bool big = false;
        if (balanced && r0 < r1 && total > kBigTile) {
            // listed for phase_c2b_big: its entries are copied by all CTAs in equal shares
            if (lane == 0) {
                const unsigned i = atomicAdd(&a.ctl->big_ctr, 1u);
                a.seg[i] = make_int4(p, total, __ldcg(a.off + r0), 0);  // seg is idle after C2a
            }
            big = true;
        } else if (r0 < r1 && total > kBigTile) {
            int slot = 0;
            if (lane == 0) slot = atomicAdd(&sm.len, 1);
            slot = __shfl_sync(0xffffffffu, slot, 0);
            if (slot < kCNT) {
                big = true;
                if (lane == 0) sm.lead[slot] = t;
            }
        }
        if (r0 < r1 && !big) {
            const unsigned long long *src = a.tout + __ldcg(a.off + r0);
            constexpr int kB = 8;
            for (int32_t j0 = 0; j0 < total; j0 += 32 * kB) {
                unsigned long long k[kB];
#pragma unroll
                for (int q = 0; q < kB; ++q) {
                    const int32_t j = j0 + q * 32 + lane;
                    k[q] = j < total ? __ldcs(src + j) : 0ull;
                }
#pragma unroll
                for (int q = 0; q < kB; ++q) {
                    const int32_t j = j0 + q * 32 + lane;
                    if (j < total) {
                        a.cadjncy[p + j] = (int32_t)(k[q] >> 32);
                        a.cadjwgt[p + j] = (int32_t)(uint32_t)k[q];
                    }
                }
            }
        }
        if (t == ntiles2 - 1 && lane == 0) {
            a.cadjp[nc] = p + total;
            a.ctl->cnnz = p + total;
        }
    }
    __syncthreads();
    const int nbig = balanced ? 0 : min(sm.len, kCNT);
    for (int b = 0; b < nbig; ++b) {  // whole-CTA copies, 8 keys per thread in flight
        const int t = sm.lead[b];
        const int32_t p = tp[t - s_lo];
        const int32_t r0 = a.dist ? __ldcg(a.tile_start + t) : t * rt;
        const int32_t total = __ldcg(a.ttot + t);
        const unsigned long long *src = a.tout + __ldcg(a.off + r0);
        constexpr int kB = 8;
        for (int32_t j0 = 0; j0 < total; j0 += kCNT * kB) {
            unsigned long long k[kB];
#pragma unroll
            for (int q = 0; q < kB; ++q) {
                const int32_t j = j0 + q * kCNT + threadIdx.x;
                k[q] = j < total ? __ldcs(src + j) : 0ull;
            }
#pragma unroll
            for (int q = 0; q < kB; ++q) {
                const int32_t j = j0 + q * kCNT + threadIdx.x;
                if (j < total) {
                    a.cadjncy[p + j] = (int32_t)(k[q] >> 32);
                    a.cadjwgt[p + j] = (int32_t)(uint32_t)k[q];
                }
            }
        }
    }
    __syncthreads();
    }
}

// ---------------------------------------------------------------------------------------
// C2b, big tiles (R-MAT: tiles holding hub rows, clustered at the low coarse ids, so the
// static tile chunks of C2b left one CTA copying ~10^8 entries -- 18-33 ms per C4 level): the
// listed tiles' entries are concatenated and every CTA copies an equal share
// ---------------------------------------------------------------------------------------
__device__ void phase_c2b_big(const ContractArgs &a, ContractSmem &sm) {
    const int32_t nb = (int32_t)*(volatile unsigned *)&a.ctl->big_ctr;
    int32_t *pre = reinterpret_cast<int32_t *>(sm.buf);  // exclusive prefix of the chunk's totals
    constexpr int kCap = 2 * kBuf - 1;
    for (int32_t c0 = 0; c0 < nb; c0 += kCap) {
        const int cnt = min(kCap, nb - c0);
        const int32_t T = block_scan_list(sm, reinterpret_cast<const int32_t *>(a.seg + c0), 4, 1, cnt, 0, pre);
        if (threadIdx.x == 0) pre[cnt] = T;
        __syncthreads();
        const long long e0 = (long long)T * blockIdx.x / g_cact, e1 = (long long)T * (blockIdx.x + 1) / g_cact;
        // first listed tile holding entry e0: the last i with pre[i] <= e0
        int lo = 0, hi = cnt - 1;
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (pre[mid] <= e0) lo = mid;
            else hi = mid - 1;
        }
        for (int i = lo; i < cnt && pre[i] < e1; ++i) {
            const int4 b = __ldcg(a.seg + c0 + i);  // {p, total, tout offset}
            const int32_t j0 = (int32_t)max((long long)pre[i], e0) - pre[i];
            const int32_t j1 = (int32_t)(min((long long)pre[i] + b.y, e1) - pre[i]);
            const unsigned long long *src = a.tout + b.z;
            constexpr int kB = 8;
            for (int32_t jb = j0; jb < j1; jb += kCNT * kB) {
                unsigned long long k[kB];
#pragma unroll
                for (int q = 0; q < kB; ++q) {
                    const int32_t j = jb + q * kCNT + threadIdx.x;
                    k[q] = j < j1 ? __ldcs(src + j) : 0ull;
                }
#pragma unroll
                for (int q = 0; q < kB; ++q) {
                    const int32_t j = jb + q * kCNT + threadIdx.x;
                    if (j < j1) {
                        a.cadjncy[b.x + j] = (int32_t)(k[q] >> 32);
                        a.cadjwgt[b.x + j] = (int32_t)(uint32_t)k[q];
                    }
                }
            }
        }
        __syncthreads();  // pre[] is rebuilt for the next chunk
    }
}

// Two instantiations that differ only in __launch_bounds__ (co-resident CTAs per SM):
// 3 (80 registers, 72 B of spills) and 4 (64 registers, 280 B of spills).  Measured
// (scripts/r2_minb.sh, r2_fold.sh): 3 is faster on C3 (3.17 vs 3.26 ms) and C2 (2.68 vs
// 2.81 ms), 4 on the n >= 2^24 graphs, C5 (29.0 vs 29.4 ms) and C4 (495 vs 521 ms: more CTAs in
// flight for the hub merges); enqueue_contract picks by the level's size bound (kBigLevel).
constexpr int32_t kBigLevel = 1 << 24;
template <int kMinB>
__global__ void __launch_bounds__(kCNT, kMinB) k_contract_level(const __grid_constant__ ContractArgs a) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    // 128-byte alignment by POINTER arithmetic on the __shared__ symbol: the compiler keeps the
    // shared address space (LDS/STS/ATOMS); an integer round trip made every access generic
    ContractSmem &sm = *reinterpret_cast<ContractSmem *>(smem_raw + ((128u - (unsigned)__cvta_generic_to_shared(smem_raw)) & 127u));
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
    // load the volatile size first: a conditional "a.dist ? a.nnz_ub : in->nnz" compiles to
    // ONE load from a selected address, and a generic load of a __grid_constant__ parameter's
    // address faults (observed with nvcc 12.9 / sm_100a)
    const int32_t nnz_in = in->nnz;
    const int32_t nnz = a.dist ? a.nnz_ub : nnz_in;
    {
        const long long work = (long long)n > (long long)nnz / 4 ? (long long)n : (long long)nnz / 4;
        const long long want = (work + a.vpc - 1) / a.vpc;
        const int nact = (int)(want < 1 ? 1 : (want < (long long)gridDim.x ? want : (long long)gridDim.x));
        if ((int)blockIdx.x >= nact) return;  // retired: this level is too small for it
        if (threadIdx.x == 0) g_cact = nact;
        __syncthreads();
    }
    unsigned bar_epoch = 0;  // grid barriers passed (thread 0)
    const int nt1 = (n + kVW - 1) / kVW;
    // Rows merged by one CTA each (C1h): ub > kWB.  GP_C1H_SMALL=1 also routes the 65..kWB rows
    // of small levels (about one C2 tile per warp) to C1h -- measured slower on C3 (C1h took
    // ~20 us at L10/L11 for a few rows per CTA), so off by default.  Sharded levels keep kWB
    // (dist.cu builds their C1h list).
    // Single-GPU levels route rows of up to 2*kWB entries (one row then fills a warp's slot
    // area) to the warp merges: on R-MAT (C4) the C1h rows of 257..512 entries, one CTA each
    // with a block-wide sort, were most of the contraction (31-38 ms of ~42 ms per level).
    const int32_t hub_ub = a.dist ? kWB
                           : ((long long)n > 32LL * 2 * g_cact * kCW || !small_hub_on(a)) ? a.warp_max : kWarpNet;
    const int T1 = (nt1 + g_cact - 1) / g_cact;            // C1b tiles per CTA
    trace_mark(ctl->trace, 0);
    if (n > 0 && !a.dist) {
        phase_c1a(a, n, nt1, T1);
        trace_mark(ctl->trace, 1);
        grid_barrier(ctl->bar, bar_epoch, g_cact);
        trace_mark(ctl->trace, 2);
        phase_c1b(a, sm, n, nt1, T1, hub_ub);
        trace_mark(ctl->trace, 3);
        grid_barrier(ctl->bar, bar_epoch, g_cact);
    }
    trace_mark(ctl->trace, 4);
    const int32_t nc = *(volatile int32_t *)&ctl->n_coarse;
    const int32_t nh = *(volatile int32_t *)&ctl->n_huge;
    if (nh > 0) {
        const int32_t ng = a.dist ? 0 : *(volatile int32_t *)&ctl->n_giant;
        // groups of >= 16 CTAs, as many as the idle tout holds accumulators + bitmaps for (none:
        // an overflowing list or no room -- every row per CTA)
        const long long per_group = (long long)nc + ((long long)nc + 31) / 32 + 96;
        int32_t G = g_cact / 16 < 32 ? g_cact / 16 : 32;
        const long long room = 2LL * nnz_in / per_group;
        if (G > room) G = (int32_t)room;
        if (G > ng) G = ng;
        const bool giant = ng > 0 && ng <= kMaxGiant && G >= 1;
        if (giant) phase_c1h_giant(a, sm, ng, nc, G);
        phase_c1h(a, sm, nh, giant);
        grid_barrier(ctl->bar, bar_epoch, g_cact);
    }
    trace_mark(ctl->trace, 5);
    // C2 warp tiles: 32 consecutive coarse rows each (single GPU); sharded levels get tiles of
    // <= tb_fixed upper-bound entries from dist.cu
    // rows per single-GPU tile: 32 (full lanes in the row merges).  Halving it on small levels
    // (more, shorter tiles) measured slower: the per-tile latency chain dominates there.
    const int32_t rt = kRT;
    const int32_t ntiles2 = nnz <= 0 ? 0 : a.dist ? (nnz + a.tb_fixed - 1) / a.tb_fixed : (nc + rt - 1) / rt;
    const int T2 = (ntiles2 + g_cact - 1) / g_cact;  // C2b tiles (and chunk sums) per CTA
    if (ntiles2 > 0) {
        // Single-pass assembly (decoupled look-back) while the tiles are few: every warp then
        // has ~1-2 tiles and the look-back chains stay short.  With many more tiles than warps
        // (C3 levels 0-3) the inclusive prefixes advance ~32 tiles per L2 round trip behind
        // ~4700 concurrent tiles, which measured slower (L0 C2: 351 us vs 242 us) than the
        // two-pass assembly (tile totals, one grid barrier, C2b copy).  Sharded levels: two-pass.
        const bool single_pass = !a.dist && !(a.knobs & 2) && ntiles2 <= 2 * g_cact * kCW;
        phase_c2a(a, sm, ntiles2, T2, nc, rt, single_pass, hub_ub);
        trace_mark(ctl->trace, 6);
        if (!single_pass) {
            grid_barrier(ctl->bar, bar_epoch, g_cact);
            trace_mark(ctl->trace, 7);
            const bool balanced = *(volatile int32_t *)&ctl->big_flag != 0;  // uniform after the barrier
            phase_c2b(a, sm, nc, ntiles2, T2, rt, balanced);
            if (balanced) {
                grid_barrier(ctl->bar, bar_epoch, g_cact);
                phase_c2b_big(a, sm);
            }
        }
    } else {  // no arcs: every coarse row is empty
        for (long long c = (long long)blockIdx.x * kCNT + threadIdx.x; c <= nc; c += (long long)g_cact * kCNT)
            a.cadjp[c] = 0;
        if (blockIdx.x == 0 && threadIdx.x == 0) ctl->cnnz = 0;
    }
    trace_mark(ctl->trace, 8);
    // the last CTA to finish publishes the coarse sizes and the stop decision
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) sm.last = atomicAdd(&ctl->blocks_done, 1u) == (unsigned)g_cact - 1;
    __syncthreads();
    if (sm.last && threadIdx.x == 0) {
        __threadfence();
        const int32_t ncv = *((volatile int32_t *)&ctl->n_coarse);
        const int32_t cnnz = *((volatile int32_t *)&ctl->cnnz);
        // stop rule (P12.s30, P20.s30; R12, R13): stall first, then threshold, then levels
        int32_t reason = GP_STOP_NONE;
        if (a.dist) reason = GP_STOP_NONE;  // global decision on the host (dist.cu)
        else if (100LL * ncv > (long long)a.stall_pct * n) reason = GP_STOP_STALL;
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
static int32_t contract_vpc() {
    static int32_t v = -1;
    if (v < 0) {
        const char *e = getenv("GP_CONTRACT_VPC");  // tuning knob (results never depend on it)
        v = e ? atoi(e) : 256;  // r2 sweep: 64 / 128 / 256 within 0.5 % (256 best by a hair)
        if (v < 1) v = 1;
    }
    return v;
}

template <int kMinB>
static int contract_grid_of(Ctx *ctx) {
    // per device: cudaFuncSetAttribute applies to the current device (the ctx's, DeviceGuard)
    static int per_sm_dev[kMaxDevices] = {0};
    int dummy = -1;
    int &per_sm = (ctx->device >= 0 && ctx->device < kMaxDevices) ? per_sm_dev[ctx->device] : dummy;
    if (per_sm <= 0) {
        int b = 0;
        cudaFuncSetAttribute(k_contract_level<kMinB>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)sizeof(ContractSmem) + 128);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_contract_level<kMinB>, kCNT, sizeof(ContractSmem) + 128);
        per_sm = b > 0 ? (b > kMinB ? kMinB : b) : 1;
    }
    const int g = ctx->num_sms * per_sm;
    return g < kMaxContractCtas ? g : kMaxContractCtas;
}

static bool contract_big(int32_t n_bound) {
    static int mb = -1;  // GP_CONTRACT_MINB=3|4 forces one instantiation (tuning knob)
    if (mb < 0) {
        const char *e = getenv("GP_CONTRACT_MINB");
        mb = e ? atoi(e) : 0;
    }
    return mb == 4 || (mb != 3 && n_bound >= kBigLevel);
}

int contract_grid(Ctx *ctx, int32_t n_bound) {
    return contract_big(n_bound) ? contract_grid_of<4>(ctx) : contract_grid_of<3>(ctx);
}

size_t contract_tiles(int32_t n, int32_t nnz) {
    // sharded tiles of >= 32 upper-bound entries, single-GPU tiles of kRT rows, C1 warp tiles
    return (size_t)(nnz + 31) / 32 + (size_t)(n + 7) / 8 + 2 * ((size_t)(n + kVW - 1) / kVW) + 8;
}

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
    a.off = lb.off;
    a.cnt = lb.cnt;
    a.tile_start = lb.tile_start;
    a.huge = lb.huge;
    a.lofs = lb.lofs;
    a.tagg1 = lb.tagg1;
    a.ttot = lb.ttot;
    a.seg = lb.seg;
    a.gkeys = lb.gkeys;
    a.tout = lb.tout;
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
    a.vpc = contract_vpc();
    a.dist = prm.dist;
    a.cbase = prm.cbase;
    a.tb_fixed = prm.tb;
    a.nnz_ub = prm.nnz_ub;
    a.status = nullptr;
    a.epoch = 0;
    {
        const char *e1 = getenv("GP_C1H_SMALL"), *e2 = getenv("GP_C2_SP");  // tuning knobs (results never depend on them)
        a.knobs = ((e1 && atoi(e1) == 1) ? 1 : 0) | ((e2 && atoi(e2) == 0) ? 2 : 0);
        const char *e3 = getenv("GP_WARP_ROW_MAX");  // tuning knob (results never depend on it)
        const int wm = e3 ? atoi(e3) : 2 * kWB;
        a.warp_max = wm < kWarpNet ? kWarpNet : wm > 2 * kWB ? 2 * kWB : wm;
        // Opt-in (GP_GIANT_ROW=<ub>, at most kCtaRow): bit-exact (tests/test_gpu_giant.py, C4
        // identical to the per-CTA path), but measured slower on C4: every row scans the whole
        // presence bitmap (nc / 32 words), so thousands of rows over 4096 entries per level cost
        // more than one CTA per row (contraction 124 -> 435 ms at 4096; the grid-wide variant
        // over 65536 entries: 122 -> 132 ms, the shorter rows left to single CTAs still set
        // the phase).
        const char *e4 = getenv("GP_GIANT_ROW");  // knob (results never depend on it)
        // (<= kCtaRow: the per-CTA rows then never use tout, which holds the groups' accumulators)
        a.giant_ub = prm.dist ? 0 : (e4 ? std::min(std::max(atoi(e4), 0), kCtaRow) : 0);
    }
    if (!prm.dist) {
        const size_t tiles = ((size_t)(prm.n_bound > 0 ? prm.n_bound : 1) + kRT - 1) / kRT + 1;
        gp_status st = ensure_status(ctx, tiles);
        if (st != GP_OK) return st;
        a.status = ctx->status;
        a.epoch = ctx->epoch++ & 0x3FFFFFFFu;  // 30-bit tag (lookback_prefix)
        if (a.epoch == 0) a.epoch = ctx->epoch++ & 0x3FFFFFFFu;
    }
    {
        static int pf = -1;
        if (pf < 0) {
            const char *e = getenv("GP_PROF");
            pf = (e && atoi(e) == 1) ? 1 : 0;
        }
        a.prof = pf;
    }
    void *args[] = {&a};
    LaunchScope ls(ctx, GP_K_CONTRACT);
    const bool big = contract_big(prm.n_bound);
    GP_CUDA(cudaLaunchCooperativeKernel(big ? (const void *)k_contract_level<4> : (const void *)k_contract_level<3>,
                                        dim3(contract_grid(ctx, prm.n_bound)), dim3(kCNT), args,
                                        sizeof(ContractSmem) + 128, ctx->stream));
    ++ctx->launches;
    return GP_OK;
}

}  // namespace gp
