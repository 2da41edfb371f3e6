// match.cu -- A1-A4: degree-binned proposals, handshake commit, round loop, leftover.
//
// Rule (PAPER.md P18.s6-13 re-pinned by north_star, R1-R4): in every round each
// free vertex proposes its heaviest free neighbour (ties -> lower id, P12.s23, P18.s7); two
// vertices that propose each other match (handshake; replaces the paper's conflict kernel
// "M[u]=v and M[v]!=u => M[u]=u", P18.s10-12).  Rounds repeat until no free vertex has a
// free neighbour; the leftover pass self-matches the rest (P18.s12-13).
//
// B200 design:
//  * Lazy rescans: after round 1 only vertices whose proposal target was matched rescan
//    their row (their proposal is otherwise still the heaviest free neighbour, because the
//    free set only shrinks).  Result-identical to rescanning everything.
//  * Degree bins (A1, fused into the round-1 kernel): rows with deg <= 2G are scanned by a
//    group of G lanes (G chosen per level from the average degree), deg <= kCtaDeg by a
//    warp, larger rows by a whole CTA (R-MAT hubs).  Warp-shuffle argmax over a packed
//    64-bit key (weight<<32 | ~id).
//  * Owner-writes only: M[u] and P[u] are written by u's own lane; no atomics on M/P, so
//    every schedule gives the same bits.  Worklists are appended with warp-aggregated
//    atomics; their order does not influence any result.
//  * All list-driven kernels use persistent grids (a multiple of the SM count) that read
//    the list length from device memory, so a whole batch of rounds is enqueued without a
//    host round trip; empty speculative rounds cost one near-empty launch each.
#include <cuda_runtime.h>

#include "device_util.cuh"
#include "gp_internal.cuh"

namespace gp {

constexpr int kCtaDeg = 4096;    // rows longer than this are scanned by a whole CTA
constexpr int kUnroll = 4;       // vertices per group per iteration (memory-level parallelism)

struct MatchBufs {
    int32_t *P;
    int32_t *L[2];   // live lists by parity
    int32_t *Rs[2];  // rescan lists: group bin
    int32_t *Rw[2];  // rescan lists: warp bin
    int32_t *Rc[2];  // rescan lists: CTA bin
};

// ---------------------------------------------------------------------------------------
// A1 + A2, round 1: every vertex is free, so no M gathers are needed.  Also initialises
// M[u] = FREE and routes rows longer than 2G to the warp / CTA bins of parity 1.
// ---------------------------------------------------------------------------------------
template <int G>
__global__ void __launch_bounds__(kBlock) k_propose_round1(int32_t n, const int32_t *__restrict__ adjp,
                                                           const int32_t *__restrict__ adjncy,
                                                           const int32_t *__restrict__ adjwgt,
                                                           int32_t *__restrict__ M, int32_t *__restrict__ P,
                                                           MatchBufs b, LevelCtl *ctl) {
    constexpr int GPW = 32 / G;
    const int lane = threadIdx.x & 31, gl = lane % G, grp = lane / G;
    const long long warp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    unsigned long long scanned = 0;
    for (long long base = warp * GPW * kUnroll; base < n; base += nwarps * GPW * kUnroll) {
        int32_t s[kUnroll], e[kUnroll];
#pragma unroll
        for (int i = 0; i < kUnroll; ++i) {
            long long u = base + i * GPW + grp;
            s[i] = 0;
            e[i] = 0;
            if (u < n) {
                s[i] = __ldg(adjp + u);
                e[i] = __ldg(adjp + u + 1);
            }
        }
        int32_t v[kUnroll][2], w[kUnroll][2];
#pragma unroll
        for (int i = 0; i < kUnroll; ++i) {
            const bool small = e[i] - s[i] <= 2 * G;
#pragma unroll
            for (int t = 0; t < 2; ++t) {
                int32_t j = s[i] + t * G + gl;
                v[i][t] = -1;
                w[i][t] = 0;
                if (small && j < e[i]) {
                    v[i][t] = __ldg(adjncy + j);
                    w[i][t] = __ldg(adjwgt + j);
                }
            }
        }
#pragma unroll
        for (int i = 0; i < kUnroll; ++i) {
            unsigned long long key = 0;
#pragma unroll
            for (int t = 0; t < 2; ++t)
                if (v[i][t] >= 0) key = umax64(key, pack_key(w[i][t], v[i][t]));
            key = group_max64<G>(key);
            long long u = base + i * GPW + grp;
            if (gl == 0 && u < n) {
                int32_t deg = e[i] - s[i];
                M[u] = kFree;
                if (deg <= 2 * G) {
                    P[u] = key_vertex(key);
                    scanned += deg;
                } else if (deg <= kCtaDeg) {
                    b.Rw[1][atomicAdd(&ctl->cnt[1].r_warp, 1)] = (int32_t)u;
                } else {
                    b.Rc[1][atomicAdd(&ctl->cnt[1].r_cta, 1)] = (int32_t)u;
                }
            }
        }
    }
    scanned = warp_sum64(scanned);
    if (lane == 0 && scanned) atomicAdd(&ctl->arcs_scanned, scanned);
}

// ---------------------------------------------------------------------------------------
// A2, rounds >= 2: rescan of the group-bin list of parity p (reads M to skip matched).
// ---------------------------------------------------------------------------------------
template <int G>
__global__ void __launch_bounds__(kBlock) k_propose_list(const int32_t *__restrict__ adjp,
                                                         const int32_t *__restrict__ adjncy,
                                                         const int32_t *__restrict__ adjwgt,
                                                         const int32_t *__restrict__ M, int32_t *__restrict__ P,
                                                         const int32_t *__restrict__ list, const int32_t *count) {
    constexpr int GPW = 32 / G;
    const int len = *count;
    const int lane = threadIdx.x & 31, gl = lane % G, grp = lane / G;
    const long long warp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long base = warp * GPW * kUnroll; base < len; base += nwarps * GPW * kUnroll) {
        int32_t s[kUnroll], e[kUnroll], uu[kUnroll];
#pragma unroll
        for (int i = 0; i < kUnroll; ++i) {
            long long k = base + i * GPW + grp;
            uu[i] = -1;
            s[i] = e[i] = 0;
            if (k < len) {
                uu[i] = list[k];
                s[i] = __ldg(adjp + uu[i]);
                e[i] = __ldg(adjp + uu[i] + 1);
            }
        }
        int32_t v[kUnroll][2], w[kUnroll][2];
#pragma unroll
        for (int i = 0; i < kUnroll; ++i)
#pragma unroll
            for (int t = 0; t < 2; ++t) {
                int32_t j = s[i] + t * G + gl;
                v[i][t] = -1;
                w[i][t] = 0;
                if (j < e[i]) {
                    v[i][t] = __ldg(adjncy + j);
                    w[i][t] = __ldg(adjwgt + j);
                }
            }
#pragma unroll
        for (int i = 0; i < kUnroll; ++i)
#pragma unroll
            for (int t = 0; t < 2; ++t)
                if (v[i][t] >= 0 && M[v[i][t]] != kFree) v[i][t] = -1;
#pragma unroll
        for (int i = 0; i < kUnroll; ++i) {
            unsigned long long key = 0;
#pragma unroll
            for (int t = 0; t < 2; ++t)
                if (v[i][t] >= 0) key = umax64(key, pack_key(w[i][t], v[i][t]));
            key = group_max64<G>(key);
            if (gl == 0 && uu[i] >= 0) P[uu[i]] = key_vertex(key);
        }
    }
}

// ---------------------------------------------------------------------------------------
// A2 for long rows: CTA per vertex (CTA bin) then warp per vertex (warp bin).
// ---------------------------------------------------------------------------------------
template <bool kCheckM>
__global__ void __launch_bounds__(kBlock) k_propose_big(const int32_t *__restrict__ adjp,
                                                        const int32_t *__restrict__ adjncy,
                                                        const int32_t *__restrict__ adjwgt,
                                                        const int32_t *__restrict__ M, int32_t *__restrict__ P,
                                                        const int32_t *__restrict__ listC, const int32_t *countC,
                                                        const int32_t *__restrict__ listW, const int32_t *countW,
                                                        LevelCtl *ctl) {
    __shared__ unsigned long long red[kBlock / 32];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int nC = *countC, nW = *countW;
    unsigned long long scanned = 0;
    for (int i = blockIdx.x; i < nC; i += gridDim.x) {
        const int32_t u = listC[i];
        const int32_t s = adjp[u], e = adjp[u + 1];
        unsigned long long key = 0;
        for (int32_t j = s + threadIdx.x; j < e; j += kBlock) {
            int32_t v = __ldg(adjncy + j);
            if (!kCheckM || M[v] == kFree) key = umax64(key, pack_key(__ldg(adjwgt + j), v));
        }
        key = group_max64<32>(key);
        if (lane == 0) red[wib] = key;
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned long long k = 0;
            for (int q = 0; q < kBlock / 32; ++q) k = umax64(k, red[q]);
            P[u] = key_vertex(k);
            scanned += (unsigned long long)(e - s);
        }
        __syncthreads();
    }
    const int gw = blockIdx.x * (kBlock / 32) + wib, nwarps = gridDim.x * (kBlock / 32);
    for (int i = gw; i < nW; i += nwarps) {
        const int32_t u = listW[i];
        const int32_t s = adjp[u], e = adjp[u + 1];
        unsigned long long key = 0;
        for (int32_t j = s + lane; j < e; j += 32) {
            int32_t v = __ldg(adjncy + j);
            if (!kCheckM || M[v] == kFree) key = umax64(key, pack_key(__ldg(adjwgt + j), v));
        }
        key = group_max64<32>(key);
        if (lane == 0) {
            P[u] = key_vertex(key);
            scanned += (unsigned long long)(e - s);
        }
    }
    if (lane == 0 && scanned) atomicAdd(&ctl->arcs_scanned, scanned);
}

// ---------------------------------------------------------------------------------------
// A3: handshake commit over the live list of parity p (round 1: all vertices).
//   P[u] == NONE             -> u is dead for this level (leftover later)
//   P[P[u]] == u             -> M[u] = P[u]             (only u's lane writes M[u])
//   P[u]'s target matched    -> u rescans next round    (lazy rescan)
//   otherwise                -> u stays live with its proposal
// The last CTA to finish closes the round: rounds += (matches > 0), consumed counters = 0.
// ---------------------------------------------------------------------------------------
template <bool kAll, int G>
__global__ void __launch_bounds__(kBlock) k_commit(int32_t n, const int32_t *__restrict__ adjp,
                                                   int32_t *__restrict__ M, const int32_t *__restrict__ P,
                                                   MatchBufs b, LevelCtl *ctl, int p) {
    const int len = kAll ? n : ctl->cnt[p].live;
    const int q = p ^ 1;
    const int32_t *Lp = b.L[p];
    int32_t made = 0, visits = 0;
    const long long stride = (long long)gridDim.x * blockDim.x;
    const long long start = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    // uniform trip count per warp so that warp_append sees all 32 lanes
    for (long long base = start - (threadIdx.x & 31); base < len; base += stride) {
        const long long k = base + (threadIdx.x & 31);
        bool live_next = false, rescan = false;
        int32_t u = -1, deg = 0;
        if (k < len) {
            u = kAll ? (int32_t)k : Lp[k];
            ++visits;
            const int32_t pu = P[u];
            if (pu != kNone) {
                const int32_t qq = P[pu];
                if (qq == u) {
                    M[u] = pu;
                    ++made;
                } else {
                    live_next = true;
                    rescan = (qq != kNone) && (P[qq] == pu);  // pu matched qq this round
                    if (rescan) deg = adjp[u + 1] - adjp[u];
                }
            }
        }
        warp_append(b.L[q], &ctl->cnt[q].live, live_next, u);
        warp_append(b.Rs[q], &ctl->cnt[q].r_small, rescan && deg <= 2 * G, u);
        warp_append(b.Rw[q], &ctl->cnt[q].r_warp, rescan && deg > 2 * G && deg <= kCtaDeg, u);
        warp_append(b.Rc[q], &ctl->cnt[q].r_cta, rescan && deg > kCtaDeg, u);
    }
    made = warp_sum(made);
    visits = warp_sum(visits);
    if ((threadIdx.x & 31) == 0) {
        if (made) atomicAdd(&ctl->matches, made);
        if (visits) atomicAdd(&ctl->live_visits, (unsigned long long)visits);
    }
    // last-block round close
    __shared__ bool last;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) last = atomicAdd(&ctl->blocks_done, 1) == (int)gridDim.x - 1;
    __syncthreads();
    if (last && threadIdx.x == 0) {
        __threadfence();
        volatile LevelCtl *c = ctl;
        if (c->matches > 0) c->rounds = c->rounds + 1;
        c->matches = 0;
        c->cnt[p].live = 0;
        c->cnt[p].r_small = 0;
        c->cnt[p].r_warp = 0;
        c->cnt[p].r_cta = 0;
        c->blocks_done = 0;
        __threadfence();
    }
}

// rows scanned by the group-bin rescans (for the byte model)
__global__ void k_count_rows(const int32_t *count_s, const int32_t *count_w, const int32_t *count_c,
                             LevelCtl *ctl) {
    if (threadIdx.x == 0)
        atomicAdd(&ctl->rows_scanned, (unsigned long long)(*count_s + *count_w + *count_c));
}

// number of live vertices that still have a proposal (exact `maximal` flag under a cap)
__global__ void k_count_proposing(const int32_t *__restrict__ L, const int32_t *count, const int32_t *__restrict__ P,
                                  int32_t *out) {
    const int len = *count;
    int32_t c = 0;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < len; i += (long long)gridDim.x * blockDim.x)
        c += P[L[i]] != kNone;
    c = warp_sum(c);
    if ((threadIdx.x & 31) == 0 && c) atomicAdd(out, c);
}

// A4 leftover: every still-free vertex is matched to itself (P18.s12-13)
__global__ void k_leftover(int32_t n, int32_t *__restrict__ M) {
    for (long long u = (long long)blockIdx.x * blockDim.x + threadIdx.x; u < n;
         u += (long long)gridDim.x * blockDim.x)
        if (M[u] == kFree) M[u] = (int32_t)u;
}

// ---------------------------------------------------------------------------------------
// host driver
// ---------------------------------------------------------------------------------------
static int choose_group(const Graph *g) {
    const double avg = g->n ? (double)g->nnz / g->n : 0.0;
    if (avg <= 3.0) return 4;
    if (avg <= 6.5) return 8;
    return 16;
}

template <int G>
static void launch_round(Ctx *ctx, const Graph *g, int32_t *M, const MatchBufs &b, int round) {
    LevelCtl *ctl = ctx->ctl;
    const int p = round & 1;
    const int grid = persistent_grid(ctx, ctx->max_threads_sm / kBlock);
    {
        LaunchScope ls(ctx, GP_K_PROPOSE);
        if (round == 1) {
            k_propose_round1<G><<<grid, kBlock, 0, ctx->stream>>>(g->n, g->adjp, g->adjncy, g->adjwgt, M, b.P, b,
                                                                  ctl);
        } else {
            k_propose_list<G><<<grid, kBlock, 0, ctx->stream>>>(g->adjp, g->adjncy, g->adjwgt, M, b.P, b.Rs[p],
                                                                &ctl->cnt[p].r_small);
        }
        ++ctx->launches;
    }
    {
        LaunchScope ls(ctx, GP_K_PROPOSE);
        if (round == 1)
            k_propose_big<false><<<grid, kBlock, 0, ctx->stream>>>(g->adjp, g->adjncy, g->adjwgt, M, b.P, b.Rc[p],
                                                                   &ctl->cnt[p].r_cta, b.Rw[p], &ctl->cnt[p].r_warp,
                                                                   ctl);
        else
            k_propose_big<true><<<grid, kBlock, 0, ctx->stream>>>(g->adjp, g->adjncy, g->adjwgt, M, b.P, b.Rc[p],
                                                                  &ctl->cnt[p].r_cta, b.Rw[p], &ctl->cnt[p].r_warp,
                                                                  ctl);
        ++ctx->launches;
    }
    if (round > 1) {
        k_count_rows<<<1, 32, 0, ctx->stream>>>(&ctl->cnt[p].r_small, &ctl->cnt[p].r_warp, &ctl->cnt[p].r_cta, ctl);
        ++ctx->launches;
    }
    {
        LaunchScope ls(ctx, GP_K_COMMIT);
        if (round == 1)
            k_commit<true, G><<<grid, kBlock, 0, ctx->stream>>>(g->n, g->adjp, M, b.P, b, ctl, p);
        else
            k_commit<false, G><<<grid, kBlock, 0, ctx->stream>>>(g->n, g->adjp, M, b.P, b, ctl, p);
        ++ctx->launches;
    }
}

gp_status match_level(Ctx *ctx, const Graph *g, int32_t *M, int32_t max_rounds, bool leftover,
                      MatchResult *res) {
    const int32_t n = g->n;
    *res = MatchResult();
    if (n == 0) return GP_OK;
    // scratch: P, L[2], Rs[2], Rw[2], Rc[2]
    const size_t nn = (size_t)n;
    gp_status st = ensure_scratch(ctx, sizeof(int32_t) * nn * 9);
    if (st != GP_OK) return st;
    int32_t *base = (int32_t *)ctx->scratch;
    MatchBufs b;
    b.P = base;
    for (int q = 0; q < 2; ++q) {
        b.L[q] = base + nn * (1 + q);
        b.Rs[q] = base + nn * (3 + q);
        b.Rw[q] = base + nn * (5 + q);
        b.Rc[q] = base + nn * (7 + q);
    }
    GP_CUDA(cudaMemsetAsync(ctx->ctl, 0, sizeof(LevelCtl), ctx->stream));
    const int G = choose_group(g);
    const int batch = (max_rounds > 0) ? 1 : 4;
    int round = 1;
    bool done = false;
    while (!done) {
        for (int k = 0; k < batch; ++k, ++round) {
            if (max_rounds > 0 && round > max_rounds) break;
            if (G == 4) launch_round<4>(ctx, g, M, b, round);
            else if (G == 8) launch_round<8>(ctx, g, M, b, round);
            else launch_round<16>(ctx, g, M, b, round);
        }
        GP_CUDA(cudaGetLastError());
        GP_CUDA(cudaMemcpyAsync(ctx->ctl_host, ctx->ctl, sizeof(LevelCtl), cudaMemcpyDeviceToHost, ctx->stream));
        GP_CUDA(cudaStreamSynchronize(ctx->stream));
        const int next_parity = round & 1;  // parity the next round would read
        const bool live_left = ctx->ctl_host->cnt[next_parity].live > 0;
        if (!live_left) {
            done = true;
            res->maximal = 1;
        } else if (max_rounds > 0 && round > max_rounds) {
            // capped with live vertices left: maximal iff none of them still has a free
            // neighbour after the rescans the next round would do
            done = true;
            const int p = round & 1;
            const int grid = persistent_grid(ctx, ctx->max_threads_sm / kBlock);
            if (G == 4) k_propose_list<4><<<grid, kBlock, 0, ctx->stream>>>(g->adjp, g->adjncy, g->adjwgt, M, b.P, b.Rs[p], &ctx->ctl->cnt[p].r_small);
            else if (G == 8) k_propose_list<8><<<grid, kBlock, 0, ctx->stream>>>(g->adjp, g->adjncy, g->adjwgt, M, b.P, b.Rs[p], &ctx->ctl->cnt[p].r_small);
            else k_propose_list<16><<<grid, kBlock, 0, ctx->stream>>>(g->adjp, g->adjncy, g->adjwgt, M, b.P, b.Rs[p], &ctx->ctl->cnt[p].r_small);
            k_propose_big<true><<<grid, kBlock, 0, ctx->stream>>>(g->adjp, g->adjncy, g->adjwgt, M, b.P, b.Rc[p], &ctx->ctl->cnt[p].r_cta, b.Rw[p], &ctx->ctl->cnt[p].r_warp, ctx->ctl);
            GP_CUDA(cudaMemsetAsync(&ctx->ctl->matches, 0, sizeof(int32_t), ctx->stream));
            k_count_proposing<<<grid, kBlock, 0, ctx->stream>>>(b.L[p], &ctx->ctl->cnt[p].live, b.P, &ctx->ctl->matches);
            ctx->launches += 3;
            GP_CUDA(cudaMemcpyAsync(ctx->ctl_host, ctx->ctl, sizeof(LevelCtl), cudaMemcpyDeviceToHost, ctx->stream));
            GP_CUDA(cudaStreamSynchronize(ctx->stream));
            res->maximal = ctx->ctl_host->matches == 0;
        }
    }
    res->rounds = ctx->ctl_host->rounds;
    res->arcs_scanned = (int64_t)ctx->ctl_host->arcs_scanned;
    res->rows_scanned = (int64_t)ctx->ctl_host->rows_scanned + n;
    res->live_visits = (int64_t)ctx->ctl_host->live_visits;
    if (leftover) {
        LaunchScope ls(ctx, GP_K_OTHER);
        k_leftover<<<persistent_grid(ctx, 4), kBlock, 0, ctx->stream>>>(n, M);
        ++ctx->launches;
        GP_CUDA(cudaGetLastError());
    }
    return GP_OK;
}

}  // namespace gp
