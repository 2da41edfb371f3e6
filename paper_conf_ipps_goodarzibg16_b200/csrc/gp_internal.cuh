// gp_internal.cuh -- internal structures and device helpers of libgpcoarsen (sm_100a).
// Shares nothing with oracle/ (DESIGN.md §1).  Citations: PAPER.md "P<line>.s<k>".
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <utility>
#include <vector>

#include "../../include/gp.h"

namespace gp {

constexpr int32_t kFree = -1;  // M[u] while u is unmatched
constexpr int32_t kNone = -1;  // P[u] when u has no free neighbour

constexpr uint32_t kTagCtx = 0x47504358u;    // "GPCX"
constexpr uint32_t kTagGraph = 0x47504752u;  // "GPGR"
constexpr uint32_t kTagHier = 0x47504849u;   // "GPHI"

constexpr int kBlock = 256;  // threads per CTA of the streaming kernels

// gp_graph_create flag used inside the library only (not in gp.h): measure the weight totals
// but do not fail on them (gp_graph_create_dist checks the GLOBAL totals on every rank)
constexpr uint32_t kInternalNoTotalsCheck = 0x80000000u;

// ---------------------------------------------------------------------------------------
// device-side control blocks of one level (zeroed once per gp_coarsen_to call)
// ---------------------------------------------------------------------------------------
struct alignas(16) RoundSlot {  // read as one 16-byte load
    int32_t live;     // live-list length of the round this slot belongs to
    int32_t nhub;     // hub rows waiting for the hub phase
    int32_t matches;  // matches made by the round's commit
    int32_t claim;    // phase-k work claims (groups of 32*kVL live entries) beyond the first
};

constexpr int kTrace = 48;  // phase timestamps per kernel (debug tracing)

struct MatchCtl {
    unsigned long long trace[kTrace];  // %globaltimer at phase boundaries (block 0; debug)
    unsigned bar[2];   // grid barrier
    unsigned chunk_ctr;  // dynamic phase-0 chunk claims
    unsigned pad0;
    RoundSlot slot[4]; // ring by round number
    int32_t rounds, maximal;
    unsigned long long arcs_scanned, rows_scanned, live_visits;
    int32_t pad[2];
    // GP_PROF=1 only: per round k < 16, the slowest warp's phase-k time (ns), the live-list
    // length and the rows rescanned by a thread / by a whole warp
    unsigned long long wmax[16];
    int32_t lens[16], trows[16], wrows[16];
    // GP_PROF=1: round-k grid barrier: ~(first CTA arrival), last arrival, last release (ns)
    unsigned long long barr[16][3];
    // parking: per round (ring k & 3) the wake tasks (matched vertices with parked neighbours)
    // and the woken vertices to resolve within the round
    int32_t nwake[4], nres[4];
    // GP_PROF=1: per round k < 16, how the live vertices ended: kept their target / took the
    // cached second choice / matched (rescans: trows)
    int32_t nkeep[16], nsec[16], nmatch[16];
    // GP_PROF=2: clock64 checkpoints of warp 0 of block 0 through its first phase-k group of
    // round k < 16 (cycles since the phase started)
    long long ck[16][12];
};

constexpr int kMaxContractCtas = 1024;  // grid cap of the contraction kernel
constexpr int kMaxGiant = 4096;         // C1h rows merged by CTA groups per level (contract.cu)

struct ContractCtl {
    unsigned long long trace[kTrace];
    unsigned bar[2];
    int32_t n_coarse, cnnz, n_huge;
    unsigned blocks_done;
    unsigned tile_ctr;  // dynamic C2a warp-tile claims
    unsigned hub_ctr;   // dynamic C1h row claims
    unsigned big_ctr;   // C2b: tiles of > kBigTile merged entries listed for the balanced copy
    int32_t big_flag;   // C2a: some tile has > kBigTile merged entries
    int32_t chunk1[2 * kMaxContractCtas];  // C1 chunk sums {#leaders, sum ub} per owner CTA
    int32_t chunk2[kMaxContractCtas];      // C2 chunk sums of merged entries per owner CTA
    unsigned long long dbg[8];             // debug: slowest C2a warp tile (ns<<32 | tile), paths
    int32_t n_giant;                       // C1h rows merged by CTA groups (ub > giant_ub)
    unsigned gbar[32];                     // their group barriers
    int32_t giant[kMaxGiant];
};

// per-graph device size record: the producer of a coarse graph writes it
struct SizeRec {
    int32_t n, nnz;
    int32_t stop;        // 1: do not coarsen this graph further
    int32_t stop_reason; // GP_STOP_* of the level that produced it
};

struct LevelDev {
    MatchCtl match;
    ContractCtl contract;
    SizeRec out;  // sizes of this level's coarse graph
};

// written by the device into mapped pinned host memory when a level completes
struct LevelReport {
    int32_t n_coarse, cnnz, stop, stop_reason;
    int32_t ready, skipped, pad[2];
};

// device pointers one level's kernels use
struct LevelBufs {
    const SizeRec *in;  // sizes (+ stop flag) of this level's input graph
    const int32_t *adjp, *adjncy, *adjwgt, *vwgt;
    int32_t *P[2], *L[2], *H, *S;                     // matching scratch
    int32_t *off, *cnt, *tile_start, *huge, *lofs;  // contraction scratch
    int32_t *tagg1, *ttot;  // tile aggregates of C1 and tile totals of C2
    int4 *seg;
    unsigned long long *gkeys, *tout;
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
struct DistComm;  // dist.cu: NCCL or loopback collectives of the sharded path
// one rank's piece of a sharded level: M / CM are indexed by GLOBAL fine vertex id (length =
// the level's n_global; only [vbase, vbase + nloc) is this rank's), coarse is the rank's
// shard of the coarse graph
struct DistPiece {
    int rank = 0;
    int32_t vbase = 0, nloc = 0;
    int32_t *M = nullptr, *CM = nullptr;
    ::gp_graph_s *coarse = nullptr;
};
}  // namespace gp

struct gp_graph_s {
    uint32_t tag = gp::kTagGraph;
    gp::Ctx *ctx = nullptr;
    int32_t n = 0, nnz = 0;
    int32_t *adjp = nullptr, *adjncy = nullptr, *adjwgt = nullptr, *vwgt = nullptr;
    gp::SizeRec *sizes = nullptr;  // device copy of {n, nnz, stop}
    bool owns_sizes = true;
    bool borrowed = false;  // owned by a hierarchy
    int locality = -1;      // ids local (1) or not (0), measured on first use (match_win.cu)
    // sharded graphs (NCCL contexts): this rank's rows are the global vertices
    // [vbase, vbase + n); ranges[r] .. ranges[r+1] is rank r's range; adjncy holds global ids
    bool dist = false;
    int rank = 0;
    int32_t vbase = 0, n_global = 0, nnz_global = 0;
    std::vector<int32_t> ranges;
    // weight totals measured at creation (R14; the sharded create checks the global sums)
    unsigned long long sum_adjwgt = 0, sum_vwgt = 0;
    bool counted = false;  // included in ctx->live_objects
    bool arena = false;    // arrays live in a hierarchy arena (small.cu): not freed individually
};

namespace gp {
struct Level {
    int32_t n = 0, nnz = 0, n_coarse = 0, cnnz = 0, rounds = 0, maximal = 0, stop_reason = 0;
    int64_t arcs_scanned = 0, rows_scanned = 0, live_visits = 0;
    int32_t *match = nullptr, *cmap = nullptr;
    Graph *coarse = nullptr;
    std::vector<DistPiece> pieces;  // sharded levels: one piece per local rank
    bool arena = false;             // match / cmap / coarse arrays live in a hierarchy arena
    bool borrowed = false;          // folded sharded level: its arrays belong to a sub-hierarchy
};
}  // namespace gp

struct gp_hier_s {
    uint32_t tag = gp::kTagHier;
    gp::Ctx *ctx = nullptr;
    std::vector<gp::Level> levels;
    gp::LevelDev *levdev = nullptr;  // per-level control blocks (coarse graphs' size records)
    bool counted = false;  // included in ctx->live_objects
    std::vector<void *> arenas;  // device arenas of tail levels (small.cu), freed with the hierarchy
    std::vector<gp_hier_s *> subs;        // folded levels of a sharded hierarchy (dist.cu)
    std::vector<gp_graph_s *> extra;      // empty coarse pieces of folded levels
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
    int32_t *pinned = nullptr;  // small pinned host buffer for read-backs
    gp::LevelReport *reports = nullptr;     // mapped pinned host memory (device-written)
    gp::LevelReport *reports_dev = nullptr; // its device alias
    int32_t max_reports = 0;
    unsigned long long *status = nullptr;  // look-back tile status words
    size_t status_words = 0;
    uint32_t epoch = 1;  // look-back epoch (no memset between scans)
    // tie priority of the matching launches of the current call (R17): set by the ABI entry
    // (gp_match_level_ex / gp_coarsen_to from its opts) before it enqueues any match launch
    uint32_t tie_seed = 0;

    // sharded path: NCCL (one local rank) or loopback (all ranks simulated); null = 1 GPU
    gp::DistComm *comm = nullptr;

    // graphs and hierarchies alive on this context (their buffers came from its allocator:
    // gp_ctx_set_allocator refuses to switch allocators while any exist)
    int64_t live_objects = 0;

    // instrumentation
    bool timing = false;
    std::vector<gp::TimedLaunch> pending;
    std::vector<cudaEvent_t> event_pool;
    gp_kernel_stats stats[GP_K_COUNT] = {};
    std::vector<std::pair<int, float>> launch_log;  // (kind, ms) of every timed launch since the last reset
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

// enqueue the persistent matching kernel of one level (A1-A4; leftover optional).
// mode: kMatchWhole (everything in one launch) or one phase per launch for the sharded
// driver (dist.cu), whose rows are the vertices [vbase, vbase + n) of a larger graph.
constexpr int kMatchWhole = 0;   // phase 0, every round and the leftover pass in one launch
constexpr int kMatchPhase0 = 1;  // phase 0 (+ its hub rows): the round-1 proposals
constexpr int kMatchRound = 2;   // commit of round k + proposals of round k+1 (+ hub rows)
constexpr int kMatchFinish = 3;  // leftover self-matches + statistics
gp_status enqueue_match(Ctx *ctx, const LevelBufs &lb, int32_t *M, MatchCtl *ctl, int32_t max_rounds, bool leftover,
                        double avg_deg_hint, int32_t vbase = 0, int mode = kMatchWhole, int k = 0);
// enqueue the persistent contraction kernel of one level (A4 leftover + A5-A8)
struct ContractParams {
    bool leftover;
    int32_t threshold, stall_pct, level, max_levels;
    int32_t n_bound, nnz_bound;
    // sharded levels only (see ContractArgs in contract.cu)
    int32_t dist = 0, cbase = 0, tb = 0, nnz_ub = 0;
};
constexpr int kContractTileBudget = 256;  // C2 warp-tile budget (upper-bound entries), kWB
int contract_grid(Ctx *ctx, int32_t n_bound);
gp_status enqueue_contract(Ctx *ctx, const LevelBufs &lb, int32_t *M, int32_t *CM, Graph *coarse, ContractCtl *ctl,
                           SizeRec *out_sizes, LevelReport *report, const ContractParams &prm);
size_t contract_tiles(int32_t n, int32_t nnz);

// weight totals (stored in g->sum_*) and, with `validate`, the GP_VALIDATE contract;
// check_totals = false skips the INT32_MAX test (the sharded create checks global sums)
gp_status graph_totals_and_validate(Ctx *ctx, Graph *g, bool validate, bool check_totals = true);

// The calling thread's current device is switched to `dev` for the scope of an ABI call and
// restored afterwards (each entry point runs on its context's device; the caller's current
// device is left as it was).
struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        int cur = -1;
        if (cudaGetDevice(&cur) == cudaSuccess && cur != dev && cudaSetDevice(dev) == cudaSuccess) prev = cur;
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
    DeviceGuard(const DeviceGuard &) = delete;
    DeviceGuard &operator=(const DeviceGuard &) = delete;
};
constexpr int kMaxDevices = 64;  // per-device caches of kernel attributes / occupancy

// coarse-level tail in one CTA (small.cu): every remaining level of a graph that fits one SM's
// shared memory, in one launch
struct SmallLaunch {
    const SizeRec *in;
    const int32_t *adjp, *adjncy, *adjwgt, *vwgt;
    void *slots;  // device array of per-level output descriptors
    int32_t nslots, level0, cap_n, cap_nnz;
    LevelDev *levdev;
    LevelReport *reports;
    int32_t threshold, stall_pct, max_levels, max_rounds;
};
bool small_fits(int32_t n, int32_t nnz);
bool small_use(int32_t n_bound, int32_t nnz_bound);
size_t small_slot_ints(int32_t n, int32_t nnz);
void small_slot_carve(int32_t *base, int32_t n, int32_t nnz, void *out_slot);
size_t small_slot_desc_bytes();
gp_status enqueue_small(Ctx *ctx, const SmallLaunch &L);
// coarse-level tail in one thread-block cluster (medium.cu): the same per-level outputs as the
// single-CTA tail, graph and state in global memory (L2), for levels too big for one SM
struct MediumLaunch : SmallLaunch {
    void *scratch;  // medium_scratch_bytes(cap_n, cap_nnz)
};
bool medium_use(int32_t n_bound, int32_t nnz_bound);
size_t medium_scratch_bytes(int32_t n, int32_t nnz);
gp_status enqueue_medium(Ctx *ctx, const MediumLaunch &L);
// windowed matching rounds for graphs with local ids (match_win.cu)
gp_status enqueue_match_win(Ctx *ctx, const LevelBufs &lb, int32_t *M, MatchCtl *ctl, int32_t max_rounds);
gp_status graph_locality(Ctx *ctx, Graph *g, int *out);
bool win_enabled();
int32_t win_min_n();
// partitioned grid tail (part.cu): every remaining level in one cooperative launch over all SMs,
// each CTA's vertex range and rows in shared memory; same per-level outputs as small.cu
struct PartLaunch : SmallLaunch {
    void *scratch;  // part_scratch_bytes(cap_n, cap_nnz)
};
bool part_fits(Ctx *ctx, int32_t n, int32_t nnz);
bool part_use(Ctx *ctx, int32_t n_bound, int32_t nnz_bound);
size_t part_scratch_bytes(int32_t n, int32_t nnz);
gp_status enqueue_part(Ctx *ctx, const PartLaunch &L);

// refinement of un-coarsening (refine.cu)
gp_status refine_graph(Ctx *ctx, const Graph *g, int32_t *d_part, const gp_refine_opts &o, int32_t *moves_out,
                       int32_t *passes_out);

// projection of un-coarsening (project.cu): cms = CM of levels to..from (fine to coarse)
gp_status enqueue_project(Ctx *ctx, const int32_t *const *cms, int nlev, int32_t n, const int32_t *part_c,
                          int32_t *part_f);

// sharded path (dist.cu)
gp_status dist_coarsen_to(Graph *g, const gp_coarsen_opts *opts, Hier **out);
// the single-GPU level pipeline (gp_abi.cu); ctx->tie_seed must be set
gp_status coarsen_single(Graph *g, const gp_coarsen_opts *opts, Hier **out);
gp_status dist_comm_create_nccl(Ctx *ctx, const void *uid, int rank, int nranks);
gp_status dist_comm_create_loopback(Ctx *ctx, int nranks);
void dist_comm_destroy(Ctx *ctx);
gp_status dist_unique_id(void *out128);
int dist_rank(const Ctx *ctx);    // -1 loopback, else the rank
int dist_nranks(const Ctx *ctx);  // 1 without a communicator
gp_status dist_allgather_i32(Ctx *ctx, const int32_t *h_send, int32_t count, int32_t *h_recv);  // host values
void graph_release(Graph *g);
void hier_release(Hier *h);
gp_status alloc_graph_arrays(Ctx *ctx, Graph *g, int32_t n_bound, int32_t nnz_bound, bool own_sizes);

gp_status ensure_scratch(Ctx *ctx, size_t bytes);
// carve one level's scratch pointers out of ctx->scratch (sized for n, nnz)
gp_status level_scratch(Ctx *ctx, int32_t n, int32_t nnz, LevelBufs *lb);
gp_status ensure_status(Ctx *ctx, size_t words);

}  // namespace gp
