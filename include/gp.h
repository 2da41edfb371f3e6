/*
 * gp.h -- C ABI of the B200-native GP-metis coarsening path.
 *
 * Method: B. Goodarzi, M. Burtscher, D. Goswami, "Parallel Graph Partitioning on a CPU-GPU
 * Architecture", IPDPS-W 2016 (/root/reference/PAPER.md; "P<line>.s<k>" = line, sentence).
 * The library implements the coarsening phase (PAPER §III.A, P16.s21-P20.s33) with the
 * deterministic matching rule pinned by north_star (readings R1-R16):
 * iterated mutual-heaviest-neighbour handshake rounds, ties to the lower vertex id, then a
 * leftover self-match pass.  All results are bit-identical across runs and launch
 * configurations and equal to the oracle (oracle/oracle.c).
 *
 * Conventions shared by every entry point
 *   * Graphs are undirected, weighted CSR (P16.s17-19): adjp[n+1] (adjp[0] = 0,
 *     adjp[n] = nnz = 2|E|), adjncy[nnz] (neighbour ids in [0, n)), adjwgt[nnz] (edge
 *     weights >= 1, equal in both directions), vwgt[n] (vertex weights >= 1).  All ids,
 *     offsets and weights are int32 (R14): n < 2^31, nnz < 2^31, sum(vwgt) and
 *     sum(adjwgt) <= INT32_MAX (checked by gp_graph_create; then no coarse level can
 *     overflow).  No self-loops, no duplicate arcs; neighbour order is arbitrary (R17).
 *   * "d_" pointers are device pointers on the context's device; "h_" pointers are host.
 *   * Everything is enqueued on the context's CUDA stream.  Calls documented as
 *     "synchronous" block the calling thread until the stream has drained their work.
 *   * Errors: every call returns a gp_status; on failure outputs are left untouched (or
 *     set to NULL for handle outputs), nothing is leaked, and gp_last_error() returns a
 *     thread-local human-readable detail.  No C++ exception crosses the ABI.
 *   * Handles (gp_ctx, gp_graph, gp_hier) are library-owned and released with gp_free.
 *     A graph or hierarchy must be freed before its context.  Handles are not
 *     thread-safe; use one context per host thread.
 *   * Devices: every call runs on its handle's device and leaves the calling thread's current
 *     CUDA device as it found it, so contexts on several devices can be mixed in one process.
 */
#ifndef GP_H
#define GP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif
#if defined(__GNUC__)
#pragma GCC visibility push(default) /* the ABI is exported even under -fvisibility=hidden */
#endif

typedef int32_t gp_vid; /* vertex id and CSR offset */
typedef int32_t gp_wgt; /* vertex / edge weight       */

typedef enum {
    GP_OK = 0,
    GP_ERR_INVALID_ARG = 1,   /* NULL handle / pointer, negative size, bad option      */
    GP_ERR_INVALID_GRAPH = 2, /* GP_VALIDATE found a CSR that breaks the input contract */
    GP_ERR_OVERFLOW = 3,      /* sum(vwgt) or sum(adjwgt) exceeds INT32_MAX (R14)       */
    GP_ERR_OUT_OF_MEMORY = 4, /* device or pinned-host allocation failed               */
    GP_ERR_CUDA = 5,          /* a CUDA runtime call failed; see gp_last_error()       */
    GP_ERR_NCCL = 6,          /* an NCCL call of the sharded path failed (or libnccl is missing) */
    GP_ERR_INTERNAL = 7       /* library invariant violated (a bug)                     */
} gp_status;

typedef struct gp_ctx_s *gp_ctx;
typedef struct gp_graph_s *gp_graph;
typedef struct gp_hier_s *gp_hier;

/* Optional device allocator (e.g. the torch caching allocator).  Both must be
 * stream-ordered on `stream`.  With NULL callbacks the library uses cudaMallocAsync on the
 * device's default memory pool (retained between calls). */
typedef void *(*gp_alloc_fn)(size_t bytes, void *stream, void *user);
typedef void (*gp_dealloc_fn)(void *ptr, void *stream, void *user);

/* Context: binds a CUDA device and stream.
 *   device       CUDA device ordinal.
 *   cuda_stream  cudaStream_t to enqueue on (NULL = the legacy default stream).
 * Fails with GP_ERR_CUDA when the device is absent (there is no CPU fallback). */
gp_status gp_ctx_create(int device, void *cuda_stream, gp_ctx *out);
/* Route the context's device allocations through alloc/dealloc (both or neither; NULL, NULL
 * restores cudaMallocAsync).  GP_ERR_INVALID_ARG while graphs or hierarchies created on this
 * context are alive (their buffers would be released through the wrong allocator); the
 * context's internal scratch is released first.  Synchronous. */
gp_status gp_ctx_set_allocator(gp_ctx ctx, gp_alloc_fn alloc, gp_dealloc_fn dealloc, void *user);
/* Number of SMs of the context's device (launch sizing is a multiple of it). */
gp_status gp_ctx_num_sms(gp_ctx ctx, int32_t *out);

/* gp_graph_create flags */
#define GP_INPUT_DEVICE 0x1u /* the four input arrays are device pointers (else host)   */
#define GP_VALIDATE 0x2u     /* check the input contract on the device before use       */

/* Create a library-owned device-resident graph from CSR arrays (P16.s17-19).
 *   n       number of vertices (>= 0)
 *   adjp    n+1 offsets; adjncy/adjwgt adjp[n] entries; vwgt n entries
 *   adjwgt  NULL => every edge weight 1;  vwgt NULL => every vertex weight 1
 *   flags   GP_INPUT_DEVICE: inputs are device pointers (copied device-to-device,
 *           stream-ordered); otherwise host pointers (copied host-to-device; pinned host
 *           memory makes the copy asynchronous).
 *           GP_VALIDATE: GP_ERR_INVALID_GRAPH unless adjp[0]=0, adjp monotone, ids in
 *           range, no self-loops, weights >= 1, no duplicate arcs and symmetric arcs with
 *           equal weights -- all exact for rows in any order (sorted rows: adjacent
 *           duplicates + binary search for the reverse arc; otherwise per-row hash sets in
 *           a temporary 16 B/arc device table); the first offending vertex is named in
 *           gp_last_error().
 * The weight totals are always checked (GP_ERR_OVERFLOW).  Synchronous (reads back the
 * totals).  The inputs may be reused once the call returns. */
gp_status gp_graph_create(gp_ctx ctx, gp_vid n, const gp_vid *adjp, const gp_vid *adjncy,
                          const gp_wgt *adjwgt, const gp_wgt *vwgt, uint32_t flags,
                          gp_graph *out);

/* Borrowed device pointers and sizes of a graph (valid until the graph is freed). */
gp_status gp_graph_view(gp_graph g, gp_vid *n, gp_vid *nnz, const gp_vid **d_adjp,
                        const gp_vid **d_adjncy, const gp_wgt **d_adjwgt, const gp_wgt **d_vwgt);

/* Copy a graph to caller-owned host buffers (sizes from gp_graph_view; any pointer may be
 * NULL to skip that array).  Synchronous. */
gp_status gp_graph_download(gp_graph g, gp_vid *h_adjp, gp_vid *h_adjncy, gp_wgt *h_adjwgt,
                            gp_wgt *h_vwgt);

/* One matching level (P16.s23-25, P18.s6-13; rule R1-R4):
 *   rounds of { every free vertex proposes its heaviest free neighbour (ties -> lower id);
 *               mutual proposals match }
 *   until no free vertex has a free neighbour (maximal) or max_rounds rounds were made,
 *   then every still-free vertex is matched to itself (leftover, P18.s12-13).
 *   d_match     caller-owned device int32[n]; receives M (M[M[u]] = u; M[u] = u for
 *               singletons)
 *   max_rounds  0 = run to the fixpoint; > 0 caps the rounds (result not maximal)
 *   rounds_out  NULL => asynchronous; else synchronous and receives the number of rounds
 *               that created at least one match (R4). */
gp_status gp_match_level(gp_graph g, gp_vid *d_match, int32_t max_rounds, int32_t *rounds_out);

/* gp_match_level with a tie priority (R17 of DESIGN.md §2; P18.s8: "If all the edges have the
 * same weight, a random matching (RM) ... where each vertex chooses one of its unmatched
 * vertices randomly").  Among neighbours of equal edge weight the proposal goes to the lower
 * h_s(v) = lowbias32(v ^ tie_seed) instead of the lower id (lowbias32: x ^= x>>16;
 * x *= 0x7feb352d; x ^= x>>15; x *= 0x846ca68b; x ^= x>>16, all mod 2^32).  tie_seed = 0 is
 * exactly gp_match_level.  The result is deterministic for a given seed; heavier edges still
 * win, so only ties (all of them on unit-weight graphs) are decided "randomly".  The rule is
 * the default rule on the vertices relabeled by h_s, so it is maximal and terminates alike. */
gp_status gp_match_level_ex(gp_graph g, gp_vid *d_match, int32_t max_rounds, uint32_t tie_seed,
                            int32_t *rounds_out);

/* Contraction of one level (P18.s16-27 cmap; P12.s26-28, P20.s0-26 contraction):
 *   d_match     a valid matching of g (output of gp_match_level), device int32[n]
 *   d_cmap      caller-owned device int32[n]; receives CM: leaders (u <= M[u]) get
 *               consecutive coarse ids in id order, partners copy their leader's id (R7)
 *   coarse_out  new graph handle owned by the caller: cvwgt[c] = sum of the pair's
 *               vertex weights; a coarse row is the union of both fine rows mapped by CM,
 *               the collapsed edge dropped (R9), repeated coarse neighbours merged with
 *               weights summed (R8), sorted by ascending coarse id (R10).
 * Synchronous (the coarse sizes are read back to size the outputs). */
gp_status gp_contract_level(gp_graph g, const gp_vid *d_match, gp_vid *d_cmap, gp_graph *coarse_out);

/* Level loop (P10.s16, P20.s27-31, P12.s30; R12, R13). */
typedef struct {
    gp_vid threshold;        /* coarsen while n > threshold                                 */
    int32_t stall_ratio_pct; /* stop after a level with 100*n_c > pct*n; 0 => 95            */
    int32_t max_levels;      /* 0 => 64                                                     */
    int32_t max_rounds;      /* per level; 0 => fixpoint (maximal matchings)               */
    uint32_t tie_seed;       /* 0 => lower id wins ties (north_star); else the RM tie
                                priority of gp_match_level_ex at every level (R17)          */
} gp_coarsen_opts;

#define GP_STOP_NONE 0      /* more levels follow                                          */
#define GP_STOP_THRESHOLD 1 /* the coarse graph has n <= threshold                         */
#define GP_STOP_STALL 2     /* the level shrank by less than (100 - stall_ratio_pct) %     */
#define GP_STOP_MAX_LEVELS 3

/* Coarsen g level by level; the hierarchy keeps every level's M, CM and coarse graph (the
 * paper's pointer arrays, P20.s27).  g itself is not modified or owned.  Synchronous. */
gp_status gp_coarsen_to(gp_graph g, const gp_coarsen_opts *opts, gp_hier *out);

/* One level of a hierarchy; every pointer/handle is borrowed from the hierarchy. */
typedef struct {
    gp_vid n, nnz;           /* the fine graph of this level                               */
    gp_vid n_coarse, cnnz;   /* its coarse graph                                           */
    int32_t rounds;          /* handshake rounds that created >= 1 match (R4)              */
    int32_t maximal;         /* 1 iff the matching reached the fixpoint                    */
    int32_t stop_reason;     /* GP_STOP_* (GP_STOP_NONE except on the last level)          */
    int32_t reserved;
    int64_t arcs_scanned;    /* adjacency entries read by the propose step (all rounds)    */
    int64_t rows_scanned;    /* rows (re)scanned by the propose step                       */
    int64_t live_visits;     /* vertex visits of the commit step (all rounds)              */
    const gp_vid *d_match;   /* device int32[n]                                            */
    const gp_vid *d_cmap;    /* device int32[n]                                            */
    gp_graph coarse;         /* borrowed: do not gp_free                                   */
    /* sharded hierarchies (gp_ctx_create_dist): n, nnz, n_coarse, cnnz, rounds are GLOBAL;
     * d_match / d_cmap / coarse are this rank's piece: the fine vertices
     * [v_begin, v_begin + n_local) and the coarse vertices [cv_begin, cv_begin + n_coarse_local)
     * (coarse ids stay globally contiguous per rank and equal to the 1-GPU numbering).
     * Loopback contexts hold every piece: those three are NULL, use the download calls.
     * Single GPU: v_begin = cv_begin = 0, n_local = n, n_coarse_local = n_coarse.            */
    gp_vid v_begin, n_local, cv_begin, n_coarse_local;
} gp_level;

gp_status gp_hier_num_levels(gp_hier h, int32_t *out);
gp_status gp_hier_level(gp_hier h, int32_t i, gp_level *out);

/* Copy a level's M and CM to caller-owned host buffers (either may be NULL).  Synchronous.
 * Sharded hierarchies: this rank's piece (n_local entries); loopback: all n entries. */
gp_status gp_hier_download_level(gp_hier h, int32_t i, gp_vid *h_match, gp_vid *h_cmap);

/* Copy a level's coarse graph to caller-owned host buffers (any may be NULL): adjp
 * [n_coarse_local + 1], adjncy / adjwgt [its arcs], vwgt [n_coarse_local]; column ids are
 * global coarse ids.  Loopback: the whole coarse graph (pieces concatenated).  Synchronous.
 * *n_out / *nnz_out (nullable) receive the row and arc counts of what is copied. */
gp_status gp_hier_download_coarse(gp_hier h, int32_t i, gp_vid *h_adjp, gp_vid *h_adjncy, gp_wgt *h_adjwgt,
                                  gp_wgt *h_vwgt, gp_vid *n_out, gp_vid *nnz_out);

/* Projection of un-coarsening (P12 "the coarser graph is projected back to the finer graph
 * by transferring the partition assignment of each vertex"; P20-P22 "by considering the CM
 * array and saved pointer arrays"): labels of the coarse graph made by level from_level
 * are carried down to level to_level's fine graph,
 *     part_l[u] = part_{l+1}[CM_l[u]]   for l = from_level, ..., to_level
 * in ONE kernel launch (no intermediate level's labels are written).
 *   d_part_coarse  device int32[n_coarse of from_level] (any label values)
 *   d_part_fine    device int32[n of to_level], caller-owned, written
 * 0 <= to_level <= from_level < levels.  Asynchronous (context stream).  Single-GPU
 * hierarchies only (GP_ERR_INVALID_ARG for sharded ones). */
gp_status gp_project(gp_hier h, int32_t from_level, int32_t to_level, const gp_vid *d_part_coarse,
                     gp_vid *d_part_fine);

/* ---- un-coarsening: refinement (PAPER.md P22.s1-22) -----------------
 * Lock-free refinement of a k-way labelling on one graph (reading R18 of DESIGN.md §2): per
 * pass two iterations, the first moving vertices only to HIGHER partition ids, the second only
 * to LOWER ones (the paper's ordering method, P22.s8-10).  In an iteration every boundary
 * vertex v of partition s requests the neighbouring partition d (in the iteration's direction)
 * with the largest gain w(v,d) - w(v,s) > 0 (ties: lower d) if s keeps >= min_w and d stays
 * <= max_w (P22.s4-7); each destination explores its requests in (gain desc, vertex asc) order
 * and accepts them while its weight stays <= max_w (P22.s16-19); accepted vertices move
 * together.  max_w = ceil(W (100 + imbalance_pct) / (100 k)), min_w = floor(W (100 -
 * imbalance_pct) / (100 k)), W = sum(vwgt).  Stops after a pass without moves or max_passes.
 * Deterministic: equal to the oracle bit for bit. */
typedef struct {
    int32_t nparts;         /* k, 1..1024                                            */
    int32_t imbalance_pct;  /* balance tolerance in percent (the paper uses 3)       */
    int32_t max_passes;     /* passes per level (each = two directed iterations)     */
} gp_refine_opts;

/* Refine d_part (device int32[n], labels in [0, nparts), updated in place) on graph g.
 * moves_out / passes_out (nullable) receive the accepted moves and the passes run.
 * Synchronous (one host read per iteration decides early termination).  Single-GPU graphs. */
gp_status gp_refine(gp_graph g, gp_vid *d_part, const gp_refine_opts *opts, int32_t *moves_out,
                    int32_t *passes_out);

/* Un-coarsening on the GPU (P12.s41-46; P20.s41-P22.s22): starting from d_part_coarse (device
 * int32[n_coarse of the last level]), for every level from the coarsest to level 0: project
 * one level (as gp_project) and refine on that level's fine graph (gp_refine).  g0 is the graph
 * the hierarchy was built from (its level-0 fine graph).  d_part_fine: device int32[n of g0],
 * caller-owned, receives the level-0 labels.  moves_out (nullable): total moves.
 * Synchronous.  Single-GPU hierarchies only. */
gp_status gp_uncoarsen(gp_hier h, gp_graph g0, const gp_vid *d_part_coarse, gp_vid *d_part_fine,
                       const gp_refine_opts *opts, int32_t *moves_out);

/* ---- sharded coarsening over several GPUs -------------------
 * Vertex ranges are sharded over the ranks of one node (one process per GPU).  Each rank
 * owns the contiguous global ids [v_begin, v_end) and holds their CSR rows with GLOBAL
 * column ids.  Every handshake round ends with an all-gather of the boundary proposals
 * (a vertex with a neighbour on another rank publishes (v, P[v], P[P[v]] when P[v] is its
 * own)); per level the leader counts are all-gathered into the rank offsets of the coarse
 * ids (the north_star's "allreduce'd prefix"), the boundary CM values are all-gathered and
 * the rows of non-leader partners are sent to their leader's rank, already mapped to coarse
 * ids.  All results are bit-identical to the 1-GPU path for any number of ranks.
 *
 * gp_nccl_unique_id   rank 0 creates the NCCL id (128 bytes) and broadcasts it (e.g. with
 *                     torch.distributed); GP_ERR_NCCL when libnccl.so.2 cannot be loaded.
 * gp_ctx_create_dist  collective over the nranks processes; `device` is this rank's GPU.
 * gp_ctx_create_loopback  one process, one GPU, `nranks` simulated ranks: every collective
 *                     becomes device-to-device copies between the ranks' private buffers
 *                     (the same kernels and the same exchange layout as NCCL).  For tests and
 *                     for single-GPU runs of the sharded protocol.
 * gp_graph_create_dist  (NCCL contexts) this rank's shard: n_global vertices in total, rows
 *                     v_begin..v_end-1 given by adjp_local[v_end - v_begin + 1] (local offsets,
 *                     adjp_local[0] = 0), adjncy/adjwgt (global ids), vwgt.  Collective: the
 *                     shards must tile [0, n_global) in rank order.  Flags as gp_graph_create.
 *                     On a loopback context, gp_graph_create makes the whole graph and
 *                     gp_coarsen_to splits it into nranks equal vertex ranges.
 * gp_coarsen_to on a sharded graph (or any graph of a loopback context) runs the sharded
 *                     driver; collective. */
gp_status gp_nccl_unique_id(void *out_128_bytes);
gp_status gp_ctx_create_dist(int device, void *cuda_stream, const void *nccl_unique_id, int rank, int nranks,
                             gp_ctx *out);
gp_status gp_ctx_create_loopback(int device, void *cuda_stream, int nranks, gp_ctx *out);
/* rank / nranks of a context: single GPU 0 / 1; NCCL rank / nranks; loopback -1 / nranks. */
gp_status gp_ctx_dist_info(gp_ctx ctx, int32_t *rank, int32_t *nranks);
gp_status gp_graph_create_dist(gp_ctx ctx, gp_vid n_global, gp_vid v_begin, gp_vid v_end, const gp_vid *adjp_local,
                               const gp_vid *adjncy, const gp_wgt *adjwgt, const gp_wgt *vwgt, uint32_t flags,
                               gp_graph *out);

/* Release any gp_ctx / gp_graph / gp_hier (handles are tagged); NULL is a no-op.
 * Levels borrowed from a hierarchy are released with the hierarchy. */
void gp_free(void *handle);

const char *gp_status_string(gp_status s);
/* Detail of the last failure on the calling thread ("" if none). */
const char *gp_last_error(void);

/* ---- instrumentation (used by bench.py; off by default) --------------------------------
 * With timing enabled the library brackets every launch of the listed kernel families
 * with CUDA events on the context stream and accumulates launch counts and device time. */
typedef enum {
    GP_K_PROPOSE = 0,  /* A1+A2: degree-binned heaviest-free-neighbour proposals         */
    GP_K_COMMIT = 1,   /* A3: handshake commit + worklists                               */
    GP_K_CMAP = 2,     /* A4 leftover + A5 cmap scan (+ A6 sizing)                       */
    GP_K_CONTRACT = 3, /* A7: merge by coarse id                                          */
    GP_K_ASSEMBLE = 4, /* A6/A8 scans + compaction                                        */
    GP_K_OTHER = 5,
    GP_K_COUNT = 6
} gp_kernel_kind;

typedef struct {
    int64_t launches;
    double ms; /* summed CUDA-event time of those launches */
} gp_kernel_stats;

gp_status gp_ctx_set_timing(gp_ctx ctx, int32_t enable);
/* Synchronous: drains pending events into the totals, then copies them out. */
gp_status gp_ctx_kernel_stats(gp_ctx ctx, gp_kernel_kind kind, gp_kernel_stats *out);
gp_status gp_ctx_reset_stats(gp_ctx ctx);
/* Synchronous: the timed launches since the last reset, in launch order: kinds[i] (a
 * gp_kernel_kind) and ms[i] (CUDA-event time); up to cap entries are copied, *count receives
 * the total (nullable).  gp_coarsen_to enqueues level l's matching then its contraction, so a
 * call's launches map to its levels in order (speculative levels after the stop come last). */
gp_status gp_ctx_launch_times(gp_ctx ctx, int32_t cap, int32_t *kinds, float *ms, int32_t *count);
/* Kernel launches made through this context since creation (all families). */
gp_status gp_ctx_launch_count(gp_ctx ctx, int64_t *out);

#if defined(__GNUC__)
#pragma GCC visibility pop
#endif
#ifdef __cplusplus
}
#endif
#endif /* GP_H */
