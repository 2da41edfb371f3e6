// gp_internal.cuh -- internal structures and device helpers of libgpcoarsen (sm_100a).
// Shares nothing with oracle/ (DESIGN.md §1).  Citations: PAPER.md "P<line>.s<k>".
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/gp.h"

namespace gp {

constexpr int32_t kFree = -1;  // M[u] while u is unmatched
constexpr int32_t kNone = -1;  // P[u] when u has no free neighbour

constexpr uint32_t kTagCtx = 0x47504358u;    // "GPCX"
constexpr uint32_t kTagGraph = 0x47504752u;  // "GPGR"
constexpr uint32_t kTagHier = 0x47504849u;   // "GPHI"

constexpr int kBlock = 256;  // threads per CTA of the streaming kernels

// ---------------------------------------------------------------------------------------
// device-side control block of one level (one memset per level)
// ---------------------------------------------------------------------------------------
struct RoundCounters {
    int32_t live;     // entries of the live list of this parity
    int32_t r_small;  // rescan list, group bin
    int32_t r_warp;   // rescan list, warp bin
    int32_t r_cta;    // rescan list, CTA bin
};

struct LevelCtl {
    RoundCounters cnt[2];       // by round parity
    int32_t matches;            // new matches in the current round
    int32_t rounds;             // rounds that created >= 1 match (R4)
    int32_t blocks_done;        // last-block detection of the commit kernel
    int32_t n_coarse;           // written by the cmap scan
    int32_t cnnz;               // written by the count scan
    int32_t n_big_w, n_big_c, n_big_g;  // contraction big-row bins
    uint32_t tile_ctr[8];       // dynamic tile counters of the scans of this level
    unsigned long long arcs_scanned;
    unsigned long long rows_scanned;
    unsigned long long live_visits;
    int32_t pad[4];
};

}  // namespace gp

// ---------------------------------------------------------------------------------------
// host-side handles (the opaque types of include/gp.h)
// ---------------------------------------------------------------------------------------
struct gp_ctx_s;
struct gp_graph_s;
struct gp_hier_s;

namespace gp {
using Ctx = ::gp_ctx_s;
using Graph = ::gp_graph_s;
using Hier = ::gp_hier_s;
struct TimedLaunch {
    int kind;
    cudaEvent_t a, b;
};
struct Level;
}  // namespace gp

struct gp_graph_s {
    uint32_t tag = gp::kTagGraph;
    gp::Ctx *ctx = nullptr;
    int32_t n = 0, nnz = 0;
    int32_t *adjp = nullptr, *adjncy = nullptr, *adjwgt = nullptr, *vwgt = nullptr;
    bool borrowed = false;  // owned by a hierarchy
};

namespace gp {
struct Level {
    int32_t n = 0, nnz = 0, n_coarse = 0, cnnz = 0, rounds = 0, maximal = 0, stop_reason = 0;
    int64_t arcs_scanned = 0, rows_scanned = 0, live_visits = 0;
    int32_t *match = nullptr, *cmap = nullptr;
    Graph *coarse = nullptr;
};
}  // namespace gp

struct gp_hier_s {
    uint32_t tag = gp::kTagHier;
    gp::Ctx *ctx = nullptr;
    std::vector<gp::Level> levels;
};

struct gp_ctx_s {
    uint32_t tag = gp::kTagCtx;
    int device = 0;
    cudaStream_t stream = nullptr;
    int num_sms = 148;
    int max_threads_sm = 2048;
    gp_alloc_fn alloc = nullptr;
    gp_dealloc_fn dealloc = nullptr;
    void *alloc_user = nullptr;

    // grow-only scratch of the level pipeline
    void *scratch = nullptr;
    size_t scratch_bytes = 0;
    gp::LevelCtl *ctl = nullptr;       // device
    gp::LevelCtl *ctl_host = nullptr;  // pinned mirror
    unsigned long long *status = nullptr;  // look-back tile status words
    size_t status_words = 0;
    uint32_t epoch = 1;  // look-back epoch (no memset between scans)

    // instrumentation
    bool timing = false;
    std::vector<gp::TimedLaunch> pending;
    std::vector<cudaEvent_t> event_pool;
    gp_kernel_stats stats[GP_K_COUNT] = {};
    int64_t launches = 0;
};

namespace gp {

// ---------------------------------------------------------------------------------------
// error plumbing (thread-local detail)
// ---------------------------------------------------------------------------------------
void set_error(const std::string &msg);
gp_status cuda_fail(cudaError_t e, const char *what);

#define GP_CUDA(call)                                       \
    do {                                                    \
        cudaError_t e__ = (call);                           \
        if (e__ != cudaSuccess) return ::gp::cuda_fail(e__, #call); \
    } while (0)

// allocation through the context's allocator (stream-ordered)
gp_status dev_alloc(Ctx *ctx, void **p, size_t bytes);
void dev_free(Ctx *ctx, void *p);

// instrumentation brackets
void launch_begin(Ctx *ctx, int kind, cudaEvent_t *a);
void launch_end(Ctx *ctx, int kind, cudaEvent_t a);

struct LaunchScope {
    Ctx *ctx;
    int kind;
    cudaEvent_t a = nullptr;
    LaunchScope(Ctx *c, int k) : ctx(c), kind(k) { launch_begin(ctx, kind, &a); }
    ~LaunchScope() { launch_end(ctx, kind, a); }
};

// grid of a persistent/grid-stride kernel: a multiple of the SM count
inline int persistent_grid(const Ctx *ctx, int blocks_per_sm) { return ctx->num_sms * blocks_per_sm; }

// ---------------------------------------------------------------------------------------
// level pipeline entry points (implemented in match.cu / contract.cu / validate.cu)
// ---------------------------------------------------------------------------------------
struct MatchResult {
    int32_t rounds = 0, maximal = 0;
    int64_t arcs_scanned = 0, rows_scanned = 0, live_visits = 0;
};

// A1-A4 without the leftover pass.  M receives FREE for unmatched vertices unless
// `leftover` is set.  Uses ctx->ctl (memset by the call).
gp_status match_level(Ctx *ctx, const Graph *g, int32_t *M, int32_t max_rounds, bool leftover,
                      MatchResult *res);

// A4 leftover (optional) + A5-A8: cmap and coarse graph.  M may contain FREE entries when
// `apply_leftover` is set (they become self-matches and M is updated in place).
gp_status contract_level(Ctx *ctx, const Graph *g, int32_t *M, int32_t *CM, bool apply_leftover,
                         Graph **coarse_out);

gp_status graph_totals_and_validate(Ctx *ctx, const Graph *g, bool validate);

gp_status ensure_scratch(Ctx *ctx, size_t bytes);
gp_status ensure_status(Ctx *ctx, size_t words);

}  // namespace gp
