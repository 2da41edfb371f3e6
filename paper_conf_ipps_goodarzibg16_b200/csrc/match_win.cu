// match_win.cu -- matching of a big level (A2-A4) with WINDOWED rounds, for graphs whose
// vertex ids are local (meshes, road networks, geometric graphs: neighbours' ids are close).
//
// The level kernel (match.cu) gathers P_k[x] and P_k[P_k[x]] from L2/HBM with a chain of
// dependent loads per live vertex; each round costs ~10 dependent round trips of the slowest
// warp (C3 level 0: round 1 125 us, round 2 80 us).  Here every CTA (one per SM, 1024
// threads) owns a contiguous vertex range and walks it in sub-chunks of kWinC vertices; for
// each sub-chunk with live vertices it fetches, with one TMA bulk copy, the WINDOW of P_k that
// the sub-chunk's arcs reach two hops out ([c0 - 2D, c1 + 2D], D = the arc-length quantile
// measured in round 1), so every lookup of the round -- the handshake test P_k[P_k[u]], the
// keep test, the rescans' freedom tests -- is a shared-memory load.  Rescanning rows are
// read from global memory, flattened over the lanes of a warp.  Lookups outside the window
// read global memory: results never depend on the window.
//
// Same rule and outputs as k_match_level (R1-R4; PAPER.md P18.s6-13 with the
// handshake): M (partner, FREE for the leftover applied by the contraction), rounds, maximal.
#include <cuda_runtime.h>
#include <stdlib.h>

#include "device_util.cuh"
#include "gp_internal.cuh"

namespace gp {

constexpr int kWT = 1024;                    // threads per CTA (64 registers)
constexpr int kWW = kWT / 32;                // warps per CTA
constexpr int32_t kWinC = 8192;              // vertices per sub-chunk
constexpr int kWinMaxSub = 512;              // sub-chunks per CTA (larger ranges: larger sub-chunks)
constexpr size_t kWinDyn = 196 * 1024;       // dynamic shared memory: the window
constexpr int32_t kWinWords = (int32_t)(kWinDyn / 4);

struct WinArgs {
    const SizeRec *in;
    const int32_t *adjp, *adjncy, *adjwgt;
    int32_t *M;
    int32_t *P0, *P1;  // proposals by round parity
    MatchCtl *ctl;
    int32_t max_rounds;
    uint32_t tie_seed;
};

__device__ __forceinline__ int32_t wld(const int32_t *p) { return __ldcg(p); }
// v, or *gp when useg (a predicated global load instead of a branch)
__device__ __forceinline__ int32_t wld_or(int32_t v, const int32_t *gp, bool useg) {
    asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.global.cg.s32 %0, [%1];\n\t}"
        : "+r"(v)
        : "l"(gp), "r"((unsigned)useg));
    return v;
}

struct Win {
    const int32_t *w;
    int32_t lo, len;
    __device__ __forceinline__ int32_t get(const int32_t *g, int32_t x) const {
        const unsigned d = (unsigned)(x - lo);
        const bool out = d >= (unsigned)len;
        return wld_or(w[out ? 0u : d], g + x, out);
    }
};

__device__ __forceinline__ void win_bulk(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_addr(dst)),
                 "l"(src), "r"(bytes), "r"(smem_addr(bar))
                 : "memory");
}

// max{c in [0, n] : 2*adjp[c] + 5*c <= T} (a kWT-ary search)
__device__ int32_t win_search(const int32_t *adjp, int32_t n, long long T) {
    int32_t lo = 0, hi = n + 1;
    while (hi - lo > 1) {
        const int32_t step = (hi - lo + kWT - 1) / kWT;
        const int32_t c = lo + threadIdx.x * step;
        const bool ok = c < hi && c <= n && 2LL * wld(adjp + c) + 5LL * c <= T;
        const int cnt = __syncthreads_count(ok);
        const int32_t nlo = lo + (cnt - 1) * step, nhi = lo + cnt * step;
        lo = nlo;
        hi = nhi < hi ? nhi : hi;
    }
    return lo;
}

// Heaviest (free after round k, when TEST) neighbour of every lane's vertex u with `need`; the
// rows of the needing lanes are flattened over the warp 32 arcs at a time (coalesced row
// reads; no lane waits for the longest row), per-row maxima by a segmented shuffle max.
// Round 1 (SAMPLE) also feeds the arc-length histogram from the rows of every 64th vertex.
template <bool H, bool TEST, bool SAMPLE>
__device__ __forceinline__ int32_t win_best(const WinArgs &a, const Win &W, const int32_t *Pk, bool need, int32_t u,
                                            unsigned long long *slot, unsigned long long &arcs, int32_t *hist,
                                            int32_t *hmax) {
    const int lane = threadIdx.x & 31;
    const int32_t s = need ? wld(a.adjp + u) : 0;
    const int32_t deg = need ? wld(a.adjp + u + 1) - s : 0;
    const int32_t incl = warp_incl_scan(deg), excl = incl - deg;
    const int32_t T = __shfl_sync(0xffffffffu, incl, 31);
    slot[lane] = 0;
    __syncwarp();
    for (int32_t base = 0; base < T; base += 32) {
        const int32_t e = base + lane;
        const bool valid = e < T;
        int o = 0;
#pragma unroll
        for (int step = 16; step > 0; step >>= 1) {
            const int32_t ex = __shfl_sync(0xffffffffu, excl, o + step);
            if (ex <= e) o += step;
        }
        const int32_t so = __shfl_sync(0xffffffffu, s, o), eo = __shfl_sync(0xffffffffu, excl, o);
        const int32_t uo = __shfl_sync(0xffffffffu, u, o);
        unsigned long long key = 0;
        if (valid) {
            const int32_t j = so + (e - eo);
            const int32_t x = wld(a.adjncy + j), w = wld(a.adjwgt + j);
            bool f = true;
            if (TEST) {
                const int32_t c = W.get(Pk, x);
                f = !(c >= 0 && W.get(Pk, c) == x);
            }
            if (f) key = pack_key<H>(a.tie_seed, w, x);
            if (SAMPLE && (uo & 63) == 0) {
                const uint32_t d = x > uo ? (uint32_t)(x - uo) : (uint32_t)(uo - x);
                const int q = 32 - __clz(d);
                atomicAdd(hist + q, 1);
                atomicMax(hmax + q, (int32_t)d);
            }
        }
        arcs += valid ? 1ull : 0ull;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
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
    return need ? key_vertex<H>(a.tie_seed, bk) : kNone;
}

// the end of a round phase: the CTA's live / pair counts into the round ring (live of the next
// round, matches of this one; slot k + 2 is reset for reuse), then the grid barrier
__device__ __forceinline__ void win_round_bar(MatchCtl *ctl, unsigned &target, int32_t k, int32_t live,
                                              int32_t pairs, int32_t *s) {
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    live = warp_sum(live);
    pairs = warp_sum(pairs);
    if (l == 0) {
        s[w] = live;
        s[kWW + w] = pairs;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        int32_t lt = 0, pt = 0;
        for (int q = 0; q < kWW; ++q) {
            lt += s[q];
            pt += s[kWW + q];
        }
        if (lt) atomicAdd(&ctl->slot[(k + 1) & 3].live, lt);
        if (pt) atomicAdd(&ctl->slot[k & 3].matches, pt);
        if (blockIdx.x == 0) {
            ctl->slot[(k + 2) & 3].live = 0;
            ctl->slot[(k + 2) & 3].matches = 0;
        }
        target += gridDim.x;
        red_release_add_u32(&ctl->bar[0], 1u);
        const long long g0 = spin_start();
        while ((int)(ld_acquire_u32(&ctl->bar[0]) - target) < 0) spin_check(g0);
    }
    __syncthreads();
}

template <bool H>
__global__ void __launch_bounds__(kWT, 1) k_match_win(const __grid_constant__ WinArgs a) {
    extern __shared__ __align__(16) int32_t wsm[];  // the window (kWinWords)
    __shared__ unsigned long long s_slot[kWW * 32];
    __shared__ int32_t s_sub[2][kWinMaxSub];
    __shared__ int32_t s_hist[33], s_hmax[33];
    __shared__ int32_t s_red[2 * kWW];
    __shared__ int32_t s_b[4];
    __shared__ __align__(8) uint64_t s_mbar;
    MatchCtl *ctl = a.ctl;
    const volatile SizeRec *in = a.in;
    if (in->stop) return;  // an earlier level ended the coarsening
    const int32_t n = in->n, nnz = in->nnz;
    if (n <= 0) return;
    const int t = threadIdx.x, b = blockIdx.x, lane = t & 31, wid = t >> 5;
    if (t == 0) {
        mbar_init(&s_mbar, 1);
        fence_mbar_init();
    }
    if (t < 33) {
        s_hist[t] = 0;
        s_hmax[t] = 0;
    }
    __syncthreads();
    unsigned mph = 0, btarget = 0;
    unsigned long long arcs = 0, rows = 0, visits = 0;
    unsigned long long *slot = s_slot + wid * 32;
    trace_mark(ctl->trace, 0);
    // ---- this CTA's vertex range, balanced on 2 * arcs + 5 * vertices, and its sub-chunks ----
    int32_t lo, hi;
    {
        const long long Wt = 2LL * nnz + 5LL * n;
        const int G = gridDim.x;
        lo = b == 0 ? 0 : win_search(a.adjp, n, (long long)b * Wt / G);
        hi = b == G - 1 ? n : win_search(a.adjp, n, (long long)(b + 1) * Wt / G);
    }
    int32_t C = kWinC;
    if ((hi - lo + C - 1) / C > kWinMaxSub) C = (((hi - lo + kWinMaxSub - 1) / kWinMaxSub) + 31) & ~31;
    const int32_t nsub = (hi - lo + C - 1) / C;
    // ---- round 1: proposals of every vertex (no freedom test), M = FREE, arc-length sample ----
    {
        Win W0{wsm, 0, 0};
        int32_t mylive = 0;
        for (int32_t sc = 0; sc < nsub; ++sc) {
            const int32_t c0 = lo + sc * C, c1 = min(hi, c0 + C);
            int32_t sl = 0;
            for (int32_t ib = c0 + wid * 32; ib < c1; ib += kWT) {  // warp-uniform
                const int32_t u = ib + lane;
                const bool inr = u < c1;
                const int32_t p = win_best<H, false, true>(a, W0, a.P1, inr, u, slot, arcs, s_hist, s_hmax);
                if (inr) {
                    a.P1[u] = p;  // round 1 -> parity 1
                    a.M[u] = kFree;
                    if (p < 0) a.P0[u] = kNone;  // no neighbour: dead in both parity buffers
                    sl += p >= 0;
                }
            }
            sl = warp_sum(sl);
            if (lane == 0) s_red[wid] = sl;
            __syncthreads();
            if (t == 0) {
                int32_t x = 0;
                for (int q = 0; q < kWW; ++q) x += s_red[q];
                s_sub[0][sc] = x;
            }
            mylive += sl;
            __syncthreads();
        }
        if (lane != 0) mylive = 0;  // (warp sums above)
        win_round_bar(ctl, btarget, 0, mylive, 0, s_red);
    }
    // window half-width: 2 D, D = the largest sampled arc length once the longest 1/256 of the
    // sampled arcs are set aside
    int32_t D;
    {
        int32_t tot = 0;
        for (int q = 0; q < 33; ++q) tot += s_hist[q];
        const int32_t keep = tot - (tot >> 8);
        int32_t acc = 0, q = 0, mx = 0;
        while (q < 33 && acc < keep) {
            acc += s_hist[q];
            mx = max(mx, s_hmax[q]);
            ++q;
        }
        D = tot > 0 ? mx : 0;
    }
    trace_mark(ctl->trace, 1);
    // ---- rounds: commit of round k + proposals of round k + 1 over windowed sub-chunks ----
    int32_t rounds = 0, maximal = 0, cur = 0;
    for (int k = 1;; ++k) {
        if (t == 0) {
            s_b[0] = *(volatile int32_t *)&ctl->slot[k & 3].live;
            s_b[1] = k > 1 ? *(volatile int32_t *)&ctl->slot[(k - 1) & 3].matches : 0;
        }
        __syncthreads();
        const int32_t live = s_b[0];
        if (s_b[1] > 0) ++rounds;
        __syncthreads();
        if (live == 0) {
            maximal = 1;
            break;
        }
        if (a.max_rounds > 0 && rounds >= a.max_rounds) break;
        if (k > n + 2) __trap();  // each round with proposals matches >= 1 pair
        int32_t *Pk = (k & 1) ? a.P1 : a.P0;
        int32_t *Pn = (k & 1) ? a.P0 : a.P1;
        int32_t mylive = 0, mypairs = 0;
        for (int32_t sc = 0; sc < nsub; ++sc) {
            if (s_sub[cur][sc] == 0) {  // no live vertex left in this sub-chunk
                if (t == 0) s_sub[cur ^ 1][sc] = 0;
                continue;
            }
            const int32_t c0 = lo + sc * C, c1 = min(hi, c0 + C);
            // the window [c0 - 2D, c1 + 2D), 16-byte aligned, at most kWinWords
            long long wl = (long long)c0 - 2LL * D, wh = (long long)c1 + 2LL * D;
            if (wh - wl > kWinWords - 8) {
                const long long h = (kWinWords - 8 - (c1 - c0)) / 2;
                wl = (long long)c0 - (h > 0 ? h : 0);
                wh = wl + kWinWords - 8;
            }
            if (wl < 0) wl = 0;
            if (wh > n) wh = n;
            wl &= ~3LL;
            wh = (wh + 3) & ~3LL;  // (the parity buffers are padded past n)
            Win W{wsm, (int32_t)wl, (int32_t)(wh - wl)};
            __syncthreads();  // the previous window is no longer read
            if (t == 0) {
                asm volatile("fence.proxy.async;" ::: "memory");
                mbar_arrive_expect_tx(&s_mbar, (unsigned)W.len * 4u);
                if (W.len > 0) win_bulk(wsm, Pk + W.lo, (unsigned)W.len * 4u, &s_mbar);
            }
            mbar_wait(&s_mbar, mph);
            mph ^= 1u;
            int32_t sl = 0;
            for (int32_t ib = c0 + wid * 32; ib < c1; ib += kWT) {  // warp-uniform
                const int32_t u = ib + lane;
                int32_t p = -1, q = -1;
                bool lv = false, need = false;
                if (u < c1 && wld(a.M + u) == kFree) {
                    p = W.get(Pk, u);
                    lv = p >= 0;  // else dead: no free neighbour (leftover)
                }
                if (lv) {
                    ++visits;
                    q = W.get(Pk, p);
                    // q == u: handshake (P18.s10-12); else p stays the heaviest free neighbour
                    // while it is free after round k, and u rescans if p matched q
                    need = q != u && q >= 0 && W.get(Pk, q) == p;
                }
                const int32_t b2 = win_best<H, true, false>(a, W, Pk, need, u, slot, arcs, nullptr, nullptr);
                if (!lv) continue;
                if (q == u) {  // matched in round k: both parity buffers hold the partner
                    a.M[u] = p;
                    Pn[u] = p;
                    mypairs += u < p;
                    continue;
                }
                int32_t np = p;
                if (need) {
                    np = b2;
                    ++rows;
                }
                Pn[u] = np;
                // no free neighbour left: dead in both buffers (readers of P_k see p or NONE
                // and decide alike: u is not matched this round)
                if (np < 0) Pk[u] = kNone;
                sl += np >= 0;
            }
            sl = warp_sum(sl);
            if (lane == 0) s_red[wid] = sl;
            __syncthreads();
            if (t == 0) {
                int32_t x = 0;
                for (int q2 = 0; q2 < kWW; ++q2) x += s_red[q2];
                s_sub[cur ^ 1][sc] = x;
            }
            mylive += sl;
        }
        cur ^= 1;
        if (lane != 0) mylive = 0;
        win_round_bar(ctl, btarget, k, mylive, mypairs, s_red);
    }
    trace_mark(ctl->trace, 2);
    // ---- statistics ----
    arcs = warp_sum64(arcs);
    rows = warp_sum64(rows);
    visits = warp_sum64(visits);
    if (lane == 0 && (arcs | rows | visits)) {
        atomicAdd(&ctl->arcs_scanned, arcs);
        atomicAdd(&ctl->rows_scanned, rows);
        atomicAdd(&ctl->live_visits, visits);
    }
    if (b == 0 && t == 0) {
        ctl->rounds = rounds;
        ctl->maximal = maximal;
    }
}

// sampled arcs (rows of every stride-th vertex) longer than n / 64, and all sampled arcs
__global__ void k_locality(const int32_t *adjp, const int32_t *adjncy, int32_t n, int32_t stride,
                           unsigned long long *cnt) {
    unsigned long long lng = 0, all = 0;
    const int32_t lim = n / 64;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i * stride < n;
         i += (long long)gridDim.x * blockDim.x) {
        const int32_t u = (int32_t)(i * stride);
        for (int32_t j = adjp[u]; j < adjp[u + 1]; ++j) {
            const int32_t x = adjncy[j];
            lng += (x > u ? x - u : u - x) > lim;
            ++all;
        }
    }
    lng = warp_sum64(lng);
    all = warp_sum64(all);
    if ((threadIdx.x & 31) == 0 && all) {
        atomicAdd(cnt, lng);
        atomicAdd(cnt + 1, all);
    }
}

// ---------------------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------------------
// Opt-in (GP_WIN=1): bit-exact on every parity case, but measured SLOWER than the level kernel
// on C3 (3.34 vs 2.90 ms; level 0 746 vs 417 us): the flattened round-1 scan costs 3x the level
// kernel's TMA-staged phase 0, and walking every vertex of a live sub-chunk (an M load each,
// 2-3x window amplification) costs more per round than the level kernel's live lists.
bool win_enabled() {
    const char *e = getenv("GP_WIN");  // knob read per call (results never depend on it)
    return e && atoi(e) == 1;
}
int32_t win_min_n() {
    const char *e = getenv("GP_WIN_N");  // tuning knob: smallest level matched with windows
    return e ? atoi(e) : 500000;
}

// local ids: at most 1/256 of the sampled arcs span more than n / 64 ids (one synchronisation,
// once per graph)
gp_status graph_locality(Ctx *ctx, Graph *g, int *out) {
    *out = 0;
    if (g->n <= 0 || g->nnz <= 0) return GP_OK;
    unsigned long long *d = nullptr;
    gp_status st = dev_alloc(ctx, (void **)&d, 16);
    if (st != GP_OK) return st;
    unsigned long long h[2] = {0, 0};
    cudaError_t e = cudaMemsetAsync(d, 0, 16, ctx->stream);
    const int32_t stride = g->n > (1 << 16) ? g->n >> 16 : 1;
    if (e == cudaSuccess) {
        LaunchScope ls(ctx, GP_K_OTHER);
        k_locality<<<148, 256, 0, ctx->stream>>>(g->adjp, g->adjncy, g->n, stride, d);
        e = cudaGetLastError();
        ++ctx->launches;
    }
    if (e == cudaSuccess) e = cudaMemcpyAsync(h, d, 16, cudaMemcpyDeviceToHost, ctx->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
    dev_free(ctx, d);
    if (e != cudaSuccess) return cuda_fail(e, "graph_locality");
    *out = (h[1] > 0 && h[0] * 256 <= h[1]) ? 1 : 0;
    return GP_OK;
}

gp_status enqueue_match_win(Ctx *ctx, const LevelBufs &lb, int32_t *M, MatchCtl *ctl, int32_t max_rounds) {
    WinArgs a;
    a.in = lb.in;
    a.adjp = lb.adjp;
    a.adjncy = lb.adjncy;
    a.adjwgt = lb.adjwgt;
    a.M = M;
    a.P0 = lb.P[0];
    a.P1 = lb.P[1];
    a.ctl = ctl;
    a.max_rounds = max_rounds;
    a.tie_seed = ctx->tie_seed;
    const void *fn = a.tie_seed ? (const void *)k_match_win<true> : (const void *)k_match_win<false>;
    GP_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kWinDyn));
    void *args[] = {&a};
    LaunchScope ls(ctx, GP_K_PROPOSE);
    GP_CUDA(cudaLaunchCooperativeKernel(fn, dim3(ctx->num_sms), dim3(kWT), args, kWinDyn, ctx->stream));
    ++ctx->launches;
    return GP_OK;
}

}  // namespace gp
