// gp_abi.cu -- the C ABI of include/gp.h: handles, memory, errors, instrumentation and the
// level driver gp_coarsen_to (A9: P10.s16, P20.s27-31, P12.s30; readings R12, R13).
#include <cuda_runtime.h>

#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "gp_internal.cuh"

namespace gp {

gp_status fill_ones(Ctx *ctx, int32_t *p, long long len);

static thread_local std::string g_last_error;

void set_error(const std::string &msg) { g_last_error = msg; }

gp_status cuda_fail(cudaError_t e, const char *what) {
    set_error(std::string(what) + ": " + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ")");
    if (e == cudaErrorMemoryAllocation) return GP_ERR_OUT_OF_MEMORY;
    return GP_ERR_CUDA;
}

gp_status dev_alloc(Ctx *ctx, void **p, size_t bytes) {
    *p = nullptr;
    if (bytes == 0) bytes = 16;
    if (ctx->alloc) {
        *p = ctx->alloc(bytes, (void *)ctx->stream, ctx->alloc_user);
        if (!*p) {
            set_error("user allocator returned NULL for " + std::to_string(bytes) + " bytes");
            return GP_ERR_OUT_OF_MEMORY;
        }
        return GP_OK;
    }
    cudaError_t e = cudaMallocAsync(p, bytes, ctx->stream);
    if (e != cudaSuccess) {
        *p = nullptr;
        return cuda_fail(e, "cudaMallocAsync");
    }
    return GP_OK;
}

void dev_free(Ctx *ctx, void *p) {
    if (!p) return;
    if (ctx->dealloc) ctx->dealloc(p, (void *)ctx->stream, ctx->alloc_user);
    else cudaFreeAsync(p, ctx->stream);
}

gp_status ensure_scratch(Ctx *ctx, size_t bytes) {
    if (bytes <= ctx->scratch_bytes) return GP_OK;
    dev_free(ctx, ctx->scratch);
    ctx->scratch = nullptr;
    ctx->scratch_bytes = 0;
    size_t want = bytes + bytes / 8;
    gp_status st = dev_alloc(ctx, &ctx->scratch, want);
    if (st != GP_OK) return st;
    ctx->scratch_bytes = want;
    return GP_OK;
}

gp_status ensure_status(Ctx *ctx, size_t words) {
    if (words <= ctx->status_words) return GP_OK;
    dev_free(ctx, ctx->status);
    ctx->status = nullptr;
    ctx->status_words = 0;
    size_t want = words + 64;
    gp_status st = dev_alloc(ctx, (void **)&ctx->status, want * sizeof(unsigned long long));
    if (st != GP_OK) return st;
    GP_CUDA(cudaMemsetAsync(ctx->status, 0, want * sizeof(unsigned long long), ctx->stream));
    ctx->status_words = want;
    return GP_OK;
}

// ---- instrumentation -------------------------------------------------------------------
static cudaEvent_t take_event(Ctx *ctx) {
    if (!ctx->event_pool.empty()) {
        cudaEvent_t e = ctx->event_pool.back();
        ctx->event_pool.pop_back();
        return e;
    }
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    return e;
}

void launch_begin(Ctx *ctx, int kind, cudaEvent_t *a) {
    (void)kind;
    *a = nullptr;
    if (!ctx->timing) return;
    *a = take_event(ctx);
    cudaEventRecord(*a, ctx->stream);
}

void launch_end(Ctx *ctx, int kind, cudaEvent_t a) {
    if (!ctx->timing || !a) return;
    cudaEvent_t b = take_event(ctx);
    cudaEventRecord(b, ctx->stream);
    ctx->pending.push_back({kind, a, b});
}

static void drain_events(Ctx *ctx) {
    if (ctx->pending.empty()) return;
    cudaStreamSynchronize(ctx->stream);
    for (auto &t : ctx->pending) {
        float ms = 0.f;
        if (cudaEventElapsedTime(&ms, t.a, t.b) == cudaSuccess) {
            ctx->stats[t.kind].ms += ms;
            ctx->stats[t.kind].launches += 1;
            ctx->launch_log.push_back({t.kind, ms});
        }
        ctx->event_pool.push_back(t.a);
        ctx->event_pool.push_back(t.b);
    }
    ctx->pending.clear();
}

void graph_release(Graph *g) {
    if (!g) return;
    Ctx *ctx = g->ctx;
    if (!g->arena) {
        dev_free(ctx, g->adjp);
        dev_free(ctx, g->adjncy);
        dev_free(ctx, g->adjwgt);
        dev_free(ctx, g->vwgt);
    }
    if (g->owns_sizes) dev_free(ctx, g->sizes);
    if (g->counted) --ctx->live_objects;
    g->tag = 0;
    delete g;
}

void hier_release(Hier *h) {
    if (!h) return;
    for (auto &l : h->levels) {
        if (l.borrowed) continue;  // owned by a sub-hierarchy (folded sharded levels)
        if (!l.arena) {
            dev_free(h->ctx, l.match);
            dev_free(h->ctx, l.cmap);
        }
        graph_release(l.coarse);
        for (auto &p : l.pieces) {
            dev_free(h->ctx, p.M);
            dev_free(h->ctx, p.CM);
            graph_release(p.coarse);
        }
    }
    for (Hier *sub : h->subs) hier_release(sub);
    for (Graph *x : h->extra) graph_release(x);
    dev_free(h->ctx, h->levdev);
    for (void *p : h->arenas) dev_free(h->ctx, p);
    if (h->counted) --h->ctx->live_objects;
    h->tag = 0;
    delete h;
}

// graph arrays with 4 ints of padding (TMA bulk copies round ranges up to 16 bytes)
gp_status alloc_graph_arrays(Ctx *ctx, Graph *g, int32_t n_bound, int32_t nnz_bound, bool own_sizes) {
    if (!g->counted) {
        g->counted = true;
        ++ctx->live_objects;
    }
    gp_status st = dev_alloc(ctx, (void **)&g->adjp, sizeof(int32_t) * ((size_t)n_bound + 4));
    if (st == GP_OK) st = dev_alloc(ctx, (void **)&g->vwgt, sizeof(int32_t) * ((size_t)n_bound + 4));
    if (st == GP_OK) st = dev_alloc(ctx, (void **)&g->adjncy, sizeof(int32_t) * ((size_t)nnz_bound + 4));
    if (st == GP_OK) st = dev_alloc(ctx, (void **)&g->adjwgt, sizeof(int32_t) * ((size_t)nnz_bound + 4));
    g->owns_sizes = own_sizes;
    if (st == GP_OK && own_sizes) st = dev_alloc(ctx, (void **)&g->sizes, sizeof(SizeRec));
    return st;
}

gp_status level_scratch(Ctx *ctx, int32_t n, int32_t nnz, LevelBufs *lb) {
    // per-vertex arrays: a multiple of 4 ints, padded by >= 4 (16-byte aligned TMA windows that
    // may round up past n, match_win.cu)
    const size_t nn = ((size_t)(n > 0 ? n : 1) + 7) & ~(size_t)3;
    const size_t tiles = contract_tiles(n, nnz);
    const size_t ints = 14 * nn + 1 + 3 * tiles + 32;
    const size_t ibytes = ((ints * 4 + 255) / 256) * 256;
    const size_t kbytes = ((8 * ((size_t)nnz + 4) + 255) / 256) * 256;
    gp_status st = ensure_scratch(ctx, ibytes + 2 * kbytes);
    if (st != GP_OK) return st;
    int32_t *p = (int32_t *)ctx->scratch;
    lb->seg = (int4 *)p; p += 4 * nn;  // first: 16-byte aligned
    lb->P[0] = p; p += nn;
    lb->P[1] = p; p += nn;
    lb->L[0] = p; p += nn;
    lb->L[1] = p; p += nn;
    lb->H = p; p += nn;
    lb->S = p; p += nn;
    lb->off = p; p += nn + 1;
    lb->cnt = p; p += nn;
    lb->huge = p; p += nn;
    lb->lofs = p; p += nn;
    lb->tagg1 = p; p += tiles;
    lb->ttot = p; p += tiles;
    lb->tile_start = p; p += tiles + 8;
    lb->gkeys = (unsigned long long *)((char *)ctx->scratch + ibytes);
    lb->tout = (unsigned long long *)((char *)ctx->scratch + ibytes + kbytes);
    return GP_OK;
}

static void set_graph_bufs(LevelBufs *lb, const Graph *g) {
    lb->in = g->sizes;
    lb->adjp = g->adjp;
    lb->adjncy = g->adjncy;
    lb->adjwgt = g->adjwgt;
    lb->vwgt = g->vwgt;
}

template <typename T>
static bool tagged(const void *p, uint32_t tag) {
    return p && static_cast<const T *>(p)->tag == tag;
}

}  // namespace gp

using namespace gp;

#define GP_TRY_BEGIN try {
#define GP_TRY_END                                           \
    }                                                        \
    catch (const std::bad_alloc &) {                         \
        set_error("host allocation failed");                 \
        return GP_ERR_OUT_OF_MEMORY;                         \
    }                                                        \
    catch (...) {                                            \
        set_error("internal exception");                     \
        return GP_ERR_INTERNAL;                              \
    }

extern "C" {

const char *gp_status_string(gp_status s) {
    switch (s) {
        case GP_OK: return "GP_OK";
        case GP_ERR_INVALID_ARG: return "GP_ERR_INVALID_ARG";
        case GP_ERR_INVALID_GRAPH: return "GP_ERR_INVALID_GRAPH";
        case GP_ERR_OVERFLOW: return "GP_ERR_OVERFLOW";
        case GP_ERR_OUT_OF_MEMORY: return "GP_ERR_OUT_OF_MEMORY";
        case GP_ERR_CUDA: return "GP_ERR_CUDA";
        case GP_ERR_NCCL: return "GP_ERR_NCCL";
        case GP_ERR_INTERNAL: return "GP_ERR_INTERNAL";
    }
    return "GP_ERR_UNKNOWN";
}

const char *gp_last_error(void) { return g_last_error.c_str(); }

gp_status gp_ctx_create(int device, void *cuda_stream, gp_ctx *out) {
    if (!out) {
        set_error("gp_ctx_create: out is NULL");
        return GP_ERR_INVALID_ARG;
    }
    *out = nullptr;
    GP_TRY_BEGIN
    int ndev = 0;
    GP_CUDA(cudaGetDeviceCount(&ndev));
    if (device < 0 || device >= ndev) {
        set_error("gp_ctx_create: no CUDA device " + std::to_string(device));
        return GP_ERR_INVALID_ARG;
    }
    DeviceGuard dg(device);  // the caller's current device is restored on return
    cudaDeviceProp prop;
    GP_CUDA(cudaGetDeviceProperties(&prop, device));
    if (prop.major < 10) {
        set_error("gp_ctx_create: device is sm_" + std::to_string(prop.major) + std::to_string(prop.minor) +
                  ", this library is built for sm_100a");
        return GP_ERR_CUDA;
    }
    if (!prop.cooperativeLaunch) {
        set_error("gp_ctx_create: device does not support cooperative launches");
        return GP_ERR_CUDA;
    }
    Ctx *ctx = new Ctx();
    ctx->device = device;
    ctx->stream = (cudaStream_t)cuda_stream;
    ctx->num_sms = prop.multiProcessorCount;
    ctx->max_threads_sm = prop.maxThreadsPerMultiProcessor;
    // retain freed pool memory between calls (stream-ordered allocator)
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess) {
        uint64_t thr = UINT64_MAX;
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    gp_status st = GP_OK;
    cudaError_t e = cudaHostAlloc((void **)&ctx->pinned, 4096, cudaHostAllocDefault);
    if (e != cudaSuccess) st = cuda_fail(e, "cudaHostAlloc(pinned)");
    if (st == GP_OK) {
        ctx->max_reports = 256;
        e = cudaHostAlloc((void **)&ctx->reports, sizeof(LevelReport) * ctx->max_reports, cudaHostAllocMapped);
        if (e != cudaSuccess) st = cuda_fail(e, "cudaHostAlloc(mapped reports)");
    }
    if (st == GP_OK) {
        e = cudaHostGetDevicePointer((void **)&ctx->reports_dev, ctx->reports, 0);
        if (e != cudaSuccess) st = cuda_fail(e, "cudaHostGetDevicePointer");
    }
    if (st != GP_OK) {
        gp_free(ctx);
        return st;
    }
    *out = ctx;
    return GP_OK;
    GP_TRY_END
}

gp_status gp_ctx_set_allocator(gp_ctx ctx, gp_alloc_fn alloc, gp_dealloc_fn dealloc, void *user) {
    if (!tagged<Ctx>(ctx, kTagCtx) || ((alloc == nullptr) != (dealloc == nullptr))) {
        set_error("gp_ctx_set_allocator: bad context or callbacks");
        return GP_ERR_INVALID_ARG;
    }
    if (ctx->live_objects > 0) {
        set_error("gp_ctx_set_allocator: " + std::to_string(ctx->live_objects) +
                  " graph(s) / hierarchy(ies) still hold buffers of the current allocator; free them first");
        return GP_ERR_INVALID_ARG;
    }
    DeviceGuard dg(ctx->device);
    // the context's own scratch was allocated with the previous allocator: release it first
    cudaStreamSynchronize(ctx->stream);
    dev_free(ctx, ctx->scratch);
    dev_free(ctx, ctx->status);
    ctx->scratch = nullptr;
    ctx->scratch_bytes = 0;
    ctx->status = nullptr;
    ctx->status_words = 0;
    ctx->alloc = alloc;
    ctx->dealloc = dealloc;
    ctx->alloc_user = user;
    return GP_OK;
}

gp_status gp_ctx_num_sms(gp_ctx ctx, int32_t *out) {
    if (!tagged<Ctx>(ctx, kTagCtx) || !out) return GP_ERR_INVALID_ARG;
    *out = ctx->num_sms;
    return GP_OK;
}

}  // extern "C"

// gp_graph_create with the totals check optional (check_totals = false: the sharded create,
// which checks the global totals after an all-gather on every rank)
static gp_status graph_create_impl(gp_ctx ctx, gp_vid n, const gp_vid *adjp, const gp_vid *adjncy,
                                   const gp_wgt *adjwgt, const gp_wgt *vwgt, uint32_t flags, bool check_totals,
                                   gp_graph *out) {
    if (out) *out = nullptr;
    if (!tagged<Ctx>(ctx, kTagCtx) || !out || n < 0 || !adjp) {
        set_error("gp_graph_create: bad context, output, n or adjp");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    const bool dev = flags & GP_INPUT_DEVICE;
    const cudaMemcpyKind kind = dev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    DeviceGuard dg(ctx->device);
    int32_t nnz = 0;
    if (dev) {
        GP_CUDA(cudaMemcpyAsync(ctx->pinned, adjp + n, sizeof(int32_t), cudaMemcpyDeviceToHost, ctx->stream));
        GP_CUDA(cudaStreamSynchronize(ctx->stream));
        nnz = ctx->pinned[0];
    } else {
        nnz = adjp[n];
    }
    if (nnz < 0) {
        set_error("gp_graph_create: adjp[n] < 0");
        return GP_ERR_INVALID_GRAPH;
    }
    if (nnz > 0 && !adjncy) {
        set_error("gp_graph_create: adjncy is NULL");
        return GP_ERR_INVALID_ARG;
    }
    Graph *g = new Graph();
    g->ctx = ctx;
    g->n = n;
    g->nnz = nnz;
    gp_status st = alloc_graph_arrays(ctx, g, n, nnz, true);
    cudaError_t e = cudaSuccess;
    if (st == GP_OK) e = cudaMemcpyAsync(g->adjp, adjp, sizeof(int32_t) * ((size_t)n + 1), kind, ctx->stream);
    if (st == GP_OK && e == cudaSuccess && nnz > 0)
        e = cudaMemcpyAsync(g->adjncy, adjncy, sizeof(int32_t) * (size_t)nnz, kind, ctx->stream);
    if (st == GP_OK && e == cudaSuccess && nnz > 0) {
        if (adjwgt) e = cudaMemcpyAsync(g->adjwgt, adjwgt, sizeof(int32_t) * (size_t)nnz, kind, ctx->stream);
        else st = fill_ones(ctx, g->adjwgt, nnz);
    }
    if (st == GP_OK && e == cudaSuccess && n > 0) {
        if (vwgt) e = cudaMemcpyAsync(g->vwgt, vwgt, sizeof(int32_t) * (size_t)n, kind, ctx->stream);
        else st = fill_ones(ctx, g->vwgt, n);
    }
    if (st == GP_OK && e == cudaSuccess) {
        SizeRec r{n, nnz, 0, 0};
        memcpy(ctx->pinned + 16, &r, sizeof(r));
        e = cudaMemcpyAsync(g->sizes, ctx->pinned + 16, sizeof(SizeRec), cudaMemcpyHostToDevice, ctx->stream);
    }
    if (st == GP_OK && e != cudaSuccess) st = cuda_fail(e, "gp_graph_create: copy");
    if (st == GP_OK)  // synchronises
        st = graph_totals_and_validate(ctx, g, flags & GP_VALIDATE, check_totals);
    if (st != GP_OK) {
        std::string keep = g_last_error;
        cudaStreamSynchronize(ctx->stream);
        graph_release(g);
        g_last_error = keep;
        return st;
    }
    *out = g;
    return GP_OK;
    GP_TRY_END
}

extern "C" {

gp_status gp_graph_create(gp_ctx ctx, gp_vid n, const gp_vid *adjp, const gp_vid *adjncy, const gp_wgt *adjwgt,
                          const gp_wgt *vwgt, uint32_t flags, gp_graph *out) {
    return graph_create_impl(ctx, n, adjp, adjncy, adjwgt, vwgt, flags & (GP_INPUT_DEVICE | GP_VALIDATE), true, out);
}

gp_status gp_graph_view(gp_graph g, gp_vid *n, gp_vid *nnz, const gp_vid **d_adjp, const gp_vid **d_adjncy,
                        const gp_wgt **d_adjwgt, const gp_wgt **d_vwgt) {
    if (!tagged<Graph>(g, kTagGraph)) {
        set_error("gp_graph_view: not a graph handle");
        return GP_ERR_INVALID_ARG;
    }
    if (n) *n = g->n;
    if (nnz) *nnz = g->nnz;
    if (d_adjp) *d_adjp = g->adjp;
    if (d_adjncy) *d_adjncy = g->adjncy;
    if (d_adjwgt) *d_adjwgt = g->adjwgt;
    if (d_vwgt) *d_vwgt = g->vwgt;
    return GP_OK;
}

gp_status gp_graph_download(gp_graph g, gp_vid *h_adjp, gp_vid *h_adjncy, gp_wgt *h_adjwgt, gp_wgt *h_vwgt) {
    if (!tagged<Graph>(g, kTagGraph)) {
        set_error("gp_graph_download: not a graph handle");
        return GP_ERR_INVALID_ARG;
    }
    Ctx *ctx = g->ctx;
    DeviceGuard dg(ctx->device);
    cudaStream_t s = ctx->stream;
    if (h_adjp) GP_CUDA(cudaMemcpyAsync(h_adjp, g->adjp, sizeof(int32_t) * ((size_t)g->n + 1), cudaMemcpyDeviceToHost, s));
    if (h_adjncy && g->nnz)
        GP_CUDA(cudaMemcpyAsync(h_adjncy, g->adjncy, sizeof(int32_t) * (size_t)g->nnz, cudaMemcpyDeviceToHost, s));
    if (h_adjwgt && g->nnz)
        GP_CUDA(cudaMemcpyAsync(h_adjwgt, g->adjwgt, sizeof(int32_t) * (size_t)g->nnz, cudaMemcpyDeviceToHost, s));
    if (h_vwgt && g->n) GP_CUDA(cudaMemcpyAsync(h_vwgt, g->vwgt, sizeof(int32_t) * (size_t)g->n, cudaMemcpyDeviceToHost, s));
    GP_CUDA(cudaStreamSynchronize(s));
    return GP_OK;
}

// a SizeRec copy of g with stop = 0 (the first level of a call never inherits a stop flag)
static gp_status fresh_sizes(Ctx *ctx, const Graph *g, SizeRec *dst) {
    SizeRec r{g->n, g->nnz, 0, 0};
    memcpy(ctx->pinned + 32, &r, sizeof(r));
    GP_CUDA(cudaMemcpyAsync(dst, ctx->pinned + 32, sizeof(SizeRec), cudaMemcpyHostToDevice, ctx->stream));
    return GP_OK;
}

static double avg_degree(int32_t n, int32_t nnz) { return n > 0 ? (double)nnz / n : 0.0; }

gp_status gp_match_level(gp_graph g, gp_vid *d_match, int32_t max_rounds, int32_t *rounds_out) {
    return gp_match_level_ex(g, d_match, max_rounds, 0u, rounds_out);
}

gp_status gp_match_level_ex(gp_graph g, gp_vid *d_match, int32_t max_rounds, uint32_t tie_seed,
                            int32_t *rounds_out) {
    if (!tagged<Graph>(g, kTagGraph) || (!d_match && g->n > 0) || max_rounds < 0) {
        set_error("gp_match_level: bad graph, match buffer or max_rounds");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    Ctx *ctx = g->ctx;
    DeviceGuard dg(ctx->device);
    ctx->tie_seed = tie_seed;
    if (ctx->comm) {
        set_error("gp_match_level: per-level calls are single-GPU; sharded graphs use gp_coarsen_to");
        return GP_ERR_INVALID_ARG;
    }
    if (g->n == 0) {
        if (rounds_out) *rounds_out = 0;
        return GP_OK;
    }
    LevelBufs lb;
    gp_status st = level_scratch(ctx, g->n, g->nnz, &lb);
    if (st != GP_OK) return st;
    LevelDev *ld = nullptr;
    st = dev_alloc(ctx, (void **)&ld, sizeof(LevelDev));
    if (st != GP_OK) return st;
    set_graph_bufs(&lb, g);
    lb.in = &ld->out;
    st = fresh_sizes(ctx, g, &ld->out);
    if (st == GP_OK) {
        cudaError_t e = cudaMemsetAsync(&ld->match, 0, sizeof(MatchCtl), ctx->stream);
        if (e != cudaSuccess) st = cuda_fail(e, "memset");
    }
    if (st == GP_OK) st = enqueue_match(ctx, lb, d_match, &ld->match, max_rounds, true, avg_degree(g->n, g->nnz));
    if (st == GP_OK && rounds_out) {
        cudaError_t e = cudaMemcpyAsync(ctx->pinned, &ld->match.rounds, sizeof(int32_t), cudaMemcpyDeviceToHost,
                                        ctx->stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
        if (e != cudaSuccess) st = cuda_fail(e, "gp_match_level");
        else *rounds_out = ctx->pinned[0];
    }
    dev_free(ctx, ld);
    return st;
    GP_TRY_END
}

gp_status gp_contract_level(gp_graph g, const gp_vid *d_match, gp_vid *d_cmap, gp_graph *coarse_out) {
    if (coarse_out) *coarse_out = nullptr;
    if (!tagged<Graph>(g, kTagGraph) || !coarse_out || ((!d_match || !d_cmap) && g->n > 0)) {
        set_error("gp_contract_level: bad graph or buffers");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    Ctx *ctx = g->ctx;
    DeviceGuard dg(ctx->device);
    if (ctx->comm) {
        set_error("gp_contract_level: per-level calls are single-GPU; sharded graphs use gp_coarsen_to");
        return GP_ERR_INVALID_ARG;
    }
    LevelBufs lb;
    gp_status st = level_scratch(ctx, g->n, g->nnz, &lb);
    if (st != GP_OK) return st;
    LevelDev *ld = nullptr;
    st = dev_alloc(ctx, (void **)&ld, sizeof(LevelDev));
    if (st != GP_OK) return st;
    Graph *cg = new Graph();
    cg->ctx = ctx;
    st = alloc_graph_arrays(ctx, cg, g->n, g->nnz, true);
    set_graph_bufs(&lb, g);
    lb.in = &ld->out;
    if (st == GP_OK) st = fresh_sizes(ctx, g, &ld->out);
    if (st == GP_OK) {
        cudaError_t e = cudaMemsetAsync(&ld->contract, 0, sizeof(ContractCtl), ctx->stream);
        if (e != cudaSuccess) st = cuda_fail(e, "memset");
    }
    ContractParams prm{false, -1, 100, 0, INT32_MAX, g->n, g->nnz};
    if (st == GP_OK)
        st = enqueue_contract(ctx, lb, const_cast<int32_t *>(d_match), d_cmap, cg, &ld->contract, cg->sizes, nullptr,
                              prm);
    if (st == GP_OK) {
        cudaError_t e = cudaMemcpyAsync(ctx->pinned, cg->sizes, sizeof(SizeRec), cudaMemcpyDeviceToHost, ctx->stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
        if (e != cudaSuccess) st = cuda_fail(e, "gp_contract_level");
    }
    if (st == GP_OK) {
        cg->n = ctx->pinned[0];
        cg->nnz = ctx->pinned[1];
        // the coarse graph is a regular input graph from now on
        st = fresh_sizes(ctx, cg, cg->sizes);
    }
    dev_free(ctx, ld);
    if (st != GP_OK) {
        std::string keep = g_last_error;
        cudaStreamSynchronize(ctx->stream);
        graph_release(cg);
        g_last_error = keep;
        return st;
    }
    *coarse_out = cg;
    return GP_OK;
    GP_TRY_END
}

// ---------------------------------------------------------------------------------------
// gp_coarsen_to: pipelined level enqueue.  Each level is two persistent cooperative
// kernels (matching, contraction).  All sizes travel through device memory, so the host
// never waits for a level before enqueuing the next one: it keeps kAhead levels in flight,
// sizing level l's outputs by the tightest size it has observed so far (a coarse graph is
// never larger than its fine graph), and learns each level's result from a report the
// contraction kernel writes into mapped host memory.  A level whose predecessor decided to
// stop (threshold / stall / max_levels) exits immediately and is discarded.
// ---------------------------------------------------------------------------------------
constexpr int kAhead = 2;
constexpr int kTailSlots = 12;  // levels per coarse-level tail launch (arena slots)

static bool debug_on() {
    static int on = -1;
    if (on < 0) on = getenv("GP_DEBUG") ? 1 : 0;
    return on == 1;
}
#define GP_DBG(...)                               \
    do {                                          \
        if (debug_on()) {                         \
            fprintf(stderr, "[gp] " __VA_ARGS__); \
            fflush(stderr);                       \
        }                                         \
    } while (0)

}  // extern "C"

namespace gp {
// the single-GPU level pipeline of gp_coarsen_to (also run by the sharded driver once the graph
// is folded onto every rank, dist.cu)
gp_status coarsen_single(Graph *g, const gp_coarsen_opts *opts, Hier **out) {
    Ctx *ctx = g->ctx;
    const int32_t pct = opts->stall_ratio_pct ? opts->stall_ratio_pct : 95;
    int32_t max_levels = opts->max_levels ? opts->max_levels : 64;
    if (max_levels > ctx->max_reports) max_levels = ctx->max_reports;
    Hier *h = new Hier();
    h->ctx = ctx;
    h->counted = true;
    ++ctx->live_objects;
    if (g->n <= opts->threshold) {
        *out = h;
        return GP_OK;
    }
    gp_status st = GP_OK;
    std::vector<Level> lv;  // enqueued levels (L.n / L.nnz hold the size bounds used)
    // tightest known upper bound of the next level's input: the last observed coarse sizes
    int32_t tight_n = g->n, tight_m = g->nnz;
    LevelBufs lb;
    st = level_scratch(ctx, g->n, g->nnz, &lb);  // level 0 is the largest
    if (st == GP_OK) st = dev_alloc(ctx, (void **)&h->levdev, sizeof(LevelDev) * (size_t)(max_levels + 1));
    if (st == GP_OK) {
        cudaError_t e = cudaMemsetAsync(h->levdev, 0, sizeof(LevelDev) * (size_t)(max_levels + 1), ctx->stream);
        if (e != cudaSuccess) st = cuda_fail(e, "memset(levdev)");
    }
    // level 0 reads its sizes from levdev[max_levels].out (a fresh, stop-free copy)
    SizeRec *in0 = (st == GP_OK) ? &h->levdev[max_levels].out : nullptr;
    if (st == GP_OK) st = fresh_sizes(ctx, g, in0);
    for (int i = 0; i < max_levels; ++i) ctx->reports[i].ready = 0;

    // id locality of the input graph (measured once per graph; coarse graphs keep it: coarse ids
    // follow the leaders' id order)
    bool use_win = false;
    if (st == GP_OK && win_enabled() && g->n >= win_min_n()) {  // opt-in (GP_WIN=1)
        if (g->locality < 0) st = graph_locality(ctx, g, &g->locality);
        use_win = g->locality == 1;
    }
    auto enqueue_level = [&](int l) -> gp_status {
        const Graph *in = (l == 0) ? g : lv[l - 1].coarse;
        const int32_t n_b = tight_n, m_b = tight_m;
        Level L;
        L.n = n_b;
        L.nnz = m_b;
        gp_status s2 = dev_alloc(ctx, (void **)&L.match, sizeof(int32_t) * (size_t)(n_b > 0 ? n_b : 1));
        if (s2 == GP_OK) s2 = dev_alloc(ctx, (void **)&L.cmap, sizeof(int32_t) * (size_t)(n_b > 0 ? n_b : 1));
        Graph *cg = nullptr;
        if (s2 == GP_OK) {
            cg = new Graph();
            cg->ctx = ctx;
            cg->borrowed = true;
            s2 = alloc_graph_arrays(ctx, cg, n_b, m_b, false);
            cg->sizes = &h->levdev[l].out;
        }
        L.coarse = cg;
        lv.push_back(L);  // registered before any failure so that it gets released
        if (s2 != GP_OK) return s2;
        LevelBufs b = lb;
        set_graph_bufs(&b, in);
        b.in = (l == 0) ? in0 : in->sizes;
        if (use_win && n_b >= win_min_n())  // windowed rounds for graphs with local ids (match_win.cu)
            s2 = enqueue_match_win(ctx, b, L.match, &h->levdev[l].match, opts->max_rounds);
        else
            s2 = enqueue_match(ctx, b, L.match, &h->levdev[l].match, opts->max_rounds, false, avg_degree(n_b, m_b));
        if (s2 != GP_OK) return s2;
        ContractParams prm{true, opts->threshold, pct, l, max_levels, n_b, m_b};
        return enqueue_contract(ctx, b, L.match, L.cmap, cg, &h->levdev[l].contract, &h->levdev[l].out,
                                &ctx->reports_dev[l], prm);
    };

    // Coarse-level tail (small.cu): once the level bounds fit one SM's
    // shared memory, ONE launch of one CTA runs every remaining level.  The host creates the
    // levels up front (arrays in one arena slot per level) and reads their reports as usual.
    std::vector<std::vector<unsigned char>> keep_host;
    // at most kTailSlots levels per tail launch (each slot is sized by the first level's
    // bounds): a hierarchy that goes deeper continues with another launch from the last tail
    // level's output, so the arena stays small (60 slots of C3's level-5 bounds were 1.6 GB,
    // re-mapped per call when the sharded ranks fold onto this pipeline: loopback 13 -> 25 ms)
    auto tail_slots = [&](int l0) -> int {
        int ns = max_levels - l0;
        const char *e = getenv("GP_TAIL_SLOTS");  // tuning knob (results never depend on it)
        const int cap = e && atoi(e) > 0 ? atoi(e) : kTailSlots;
        return cap < ns ? cap : ns;
    };
    auto enqueue_tail = [&](int l0) -> gp_status {
        const int32_t n_b = tight_n, m_b = tight_m;
        const int ns = tail_slots(l0);
        const size_t slot = small_slot_ints(n_b, m_b);
        void *arena = nullptr, *desc = nullptr;
        gp_status s2 = dev_alloc(ctx, &arena, sizeof(int32_t) * slot * (size_t)ns);
        if (s2 == GP_OK) h->arenas.push_back(arena);
        if (s2 == GP_OK) s2 = dev_alloc(ctx, &desc, small_slot_desc_bytes() * (size_t)ns);
        if (s2 == GP_OK) h->arenas.push_back(desc);
        if (s2 != GP_OK) return s2;
        std::vector<unsigned char> hd((size_t)ns * small_slot_desc_bytes());
        for (int i = 0; i < ns; ++i) {
            int32_t *base = static_cast<int32_t *>(arena) + slot * (size_t)i;
            small_slot_carve(base, n_b, m_b, hd.data() + (size_t)i * small_slot_desc_bytes());
            struct D { int32_t *M, *CM, *cadjp, *cadjncy, *cadjwgt, *cvwgt; };
            const D *d = reinterpret_cast<const D *>(hd.data() + (size_t)i * small_slot_desc_bytes());
            Level L;
            L.n = n_b;
            L.nnz = m_b;
            L.arena = true;
            L.match = d->M;
            L.cmap = d->CM;
            Graph *cg = new Graph();
            cg->ctx = ctx;
            cg->borrowed = true;
            cg->arena = true;
            cg->owns_sizes = false;
            cg->adjp = d->cadjp;
            cg->adjncy = d->cadjncy;
            cg->adjwgt = d->cadjwgt;
            cg->vwgt = d->cvwgt;
            cg->sizes = &h->levdev[l0 + i].out;
            cg->counted = true;
            ++ctx->live_objects;
            L.coarse = cg;
            lv.push_back(L);
        }
        // the descriptors are small: a pinned staging copy is not needed (synchronous copy)
        GP_CUDA(cudaMemcpyAsync(desc, hd.data(), hd.size(), cudaMemcpyHostToDevice, ctx->stream));
        const Graph *in = (l0 == 0) ? g : lv[l0 - 1].coarse;
        SmallLaunch sl;
        sl.in = (l0 == 0) ? in0 : in->sizes;
        sl.adjp = in->adjp;
        sl.adjncy = in->adjncy;
        sl.adjwgt = in->adjwgt;
        sl.vwgt = in->vwgt;
        sl.slots = desc;
        sl.nslots = ns;
        sl.level0 = l0;
        sl.cap_n = n_b;
        sl.cap_nnz = m_b;
        sl.levdev = h->levdev;
        sl.reports = ctx->reports_dev;
        sl.threshold = opts->threshold;
        sl.stall_pct = pct;
        sl.max_levels = max_levels;
        sl.max_rounds = opts->max_rounds;
        if (small_use(n_b, m_b)) {
            s2 = enqueue_small(ctx, sl);
        } else if (part_use(ctx, n_b, m_b) && !medium_use(n_b, m_b)) {  // all SMs, shared-memory partitions
            PartLaunch pl;
            static_cast<SmallLaunch &>(pl) = sl;
            void *scr = nullptr;
            s2 = dev_alloc(ctx, &scr, part_scratch_bytes(n_b, m_b));
            if (s2 == GP_OK) {
                h->arenas.push_back(scr);
                pl.scratch = scr;
                s2 = enqueue_part(ctx, pl);
            }
        } else {  // one thread-block cluster, state in global memory
            MediumLaunch ml;
            static_cast<SmallLaunch &>(ml) = sl;
            void *scr = nullptr;
            s2 = dev_alloc(ctx, &scr, medium_scratch_bytes(n_b, m_b));
            if (s2 == GP_OK) {
                h->arenas.push_back(scr);
                ml.scratch = scr;
                s2 = enqueue_medium(ctx, ml);
            }
        }
        keep_host.push_back(std::move(hd));  // read by the async copy: alive until the final sync
        return s2;
    };

    int enq = 0, obs = 0, last_real = -1;
    bool stop_seen = false;
    while (st == GP_OK) {
        while (st == GP_OK && !stop_seen && enq < max_levels && enq - obs < kAhead) {
            if (small_use(tight_n, tight_m) || medium_use(tight_n, tight_m) || part_use(ctx, tight_n, tight_m)) {
                GP_DBG("enqueue tail levels %d.. in one CTA / cluster (bounds n=%d nnz=%d)\n", enq, tight_n, tight_m);
                const int ns = tail_slots(enq);
                st = enqueue_tail(enq);
                enq += ns;
                break;
            }
            GP_DBG("enqueue level %d (bounds n=%d nnz=%d)\n", enq, tight_n, tight_m);
            st = enqueue_level(enq);
            ++enq;
        }
        if (st != GP_OK || obs == enq) break;
        volatile LevelReport *r = &ctx->reports[obs];
        const auto t_wait = std::chrono::steady_clock::now();
        while (!r->ready) {
            if (std::chrono::steady_clock::now() - t_wait > std::chrono::seconds(120)) {
                set_error("gp_coarsen_to: level " + std::to_string(obs) + " did not report within 120 s");
                st = GP_ERR_INTERNAL;
                break;
            }
            const cudaError_t q = cudaStreamQuery(ctx->stream);
            if (q != cudaSuccess && q != cudaErrorNotReady) {
                st = cuda_fail(q, "gp_coarsen_to: level kernel");
                break;
            }
            if (q == cudaSuccess && !r->ready) {  // stream drained without a report: a bug
                set_error("gp_coarsen_to: level finished without a report");
                st = GP_ERR_INTERNAL;
                break;
            }
        }
        if (st != GP_OK) break;
        GP_DBG("level %d reported: n_c=%d cnnz=%d stop=%d reason=%d skipped=%d\n", obs, r->n_coarse, r->cnnz, r->stop,
               r->stop_reason, r->skipped);
        if (!r->skipped) {
            last_real = obs;
            lv[obs].n_coarse = r->n_coarse;
            lv[obs].cnnz = r->cnnz;
            lv[obs].stop_reason = r->stop_reason;
            tight_n = r->n_coarse;
            tight_m = r->cnnz;
            if (r->stop) stop_seen = true;
        }
        ++obs;
    }
    cudaError_t e = cudaStreamSynchronize(ctx->stream);
    if (st == GP_OK && e != cudaSuccess) st = cuda_fail(e, "gp_coarsen_to");
    if (st == GP_OK && last_real >= 0) {
        // per-level statistics of the matching kernels (one small copy)
        std::vector<LevelDev> hd((size_t)last_real + 1);
        e = cudaMemcpy(hd.data(), h->levdev, sizeof(LevelDev) * hd.size(), cudaMemcpyDeviceToHost);
        if (e != cudaSuccess) st = cuda_fail(e, "gp_coarsen_to: stats");
        for (int l = 0; st == GP_OK && l <= last_real; ++l) {
            Level &L = lv[l];
            L.n = (l == 0) ? g->n : lv[l - 1].n_coarse;
            L.nnz = (l == 0) ? g->nnz : lv[l - 1].cnnz;
            L.rounds = hd[l].match.rounds;
            L.maximal = hd[l].match.maximal;
            L.arcs_scanned = (int64_t)hd[l].match.arcs_scanned;
            L.rows_scanned = (int64_t)hd[l].match.rows_scanned + L.n;
            L.live_visits = (int64_t)hd[l].match.live_visits;
            L.coarse->n = L.n_coarse;
            L.coarse->nnz = L.cnnz;
            if (debug_on()) {
                const unsigned long long *mt = hd[l].match.trace, *ct = hd[l].contract.trace;
                fprintf(stderr, "[gp] level %d n=%d nnz=%d rounds=%d | match us:", l, L.n, L.nnz, L.rounds);
                for (int q = 1; q < kTrace && mt[q]; ++q) fprintf(stderr, " %.1f", (mt[q] - mt[q - 1]) * 1e-3);
                fprintf(stderr, " | contract us (c1a bar c1b bar hub c2a bar c2b):");
                for (int q = 1; q < 9; ++q)
                    fprintf(stderr, " %.1f", ct[q] && ct[q - 1] ? ((long long)ct[q] - (long long)ct[q - 1]) * 1e-3 : 0.0);
                fprintf(stderr, " | gap to contract %.1f us\n", ct[0] && mt[1] ? ((long long)ct[0] - (long long)mt[0]) * 1e-3 : 0.0);
                if (hd[l].contract.dbg[6]) {
                    const unsigned long long *d = hd[l].contract.dbg;
                    fprintf(stderr, "[gp]   c1h rows: sum of upper bounds %llu, slowest row %.1f us (ub %llu)\n", d[6],
                            (d[7] >> 24) * 1e-3, d[7] & 0xFFFFFFull);
                }
                if (hd[l].contract.dbg[4]) {
                    const unsigned long long *d = hd[l].contract.dbg;
                    fprintf(stderr, "[gp]   c2a tiles %llu: slowest %.1f us (tile %llu), mean %.2f us, max warp-merged rows %llu (tile %llu), max rows %llu, warp-merged rows %llu\n",
                            d[4], (d[0] >> 32) * 1e-3, d[0] & 0xffffffffull, d[3] * 1e-3 / d[4], d[1] >> 32,
                            d[1] & 0xffffffffull, d[2] >> 32, d[5]);
                }
                if (hd[l].match.ck[1][8]) {
                    fprintf(stderr, "[gp]   warp-0 checkpoints per round (cycles: claim u p+S qq/rr decide rescan push | loop-exit flush):");
                    for (int k = 1; k < 16 && hd[l].match.ck[k][8]; ++k) {
                        fprintf(stderr, " [");
                        for (int j = 0; j < 9; ++j) fprintf(stderr, "%s%lld", j ? " " : "", hd[l].match.ck[k][j]);
                        fprintf(stderr, "]");
                    }
                    fprintf(stderr, "\n");
                }
                if (hd[l].match.barr[0][0])  // the partitioned grid tail (part.cu, GP_PROF=1)
                    fprintf(stderr, "[gp]   part: slowest CTA round-1 proposals %.1f us, merges %.1f us, copy %.1f us\n",
                            hd[l].match.wmax[0] * 1e-3, hd[l].match.barr[0][0] * 1e-3, hd[l].match.barr[0][1] * 1e-3);
                if (hd[l].match.lens[1]) {
                    fprintf(stderr, "[gp]   per round (live | slowest warp us | rows rescanned thread / warp):");
                    for (int k = 1; k < 16 && hd[l].match.lens[k]; ++k)
                        fprintf(stderr, " [%d %.1f %d/%d]", hd[l].match.lens[k], hd[l].match.wmax[k] * 1e-3,
                                hd[l].match.trows[k], hd[l].match.wrows[k]);
                    fprintf(stderr, "\n");
                    fprintf(stderr, "[gp]   per round (matched / kept target / second choice, impl path):");
                    for (int k = 1; k < 16 && hd[l].match.lens[k]; ++k)
                        fprintf(stderr, " [%d %d %d]", hd[l].match.nmatch[k], hd[l].match.nkeep[k], hd[l].match.nsec[k]);
                    fprintf(stderr, "\n");
                    fprintf(stderr, "[gp]   round barriers (arrival spread | last arrival -> last release, us):");
                    for (int k = 1; k < 16 && hd[l].match.barr[k][1]; ++k)
                        fprintf(stderr, " [%.1f %.1f]", (hd[l].match.barr[k][1] - ~hd[l].match.barr[k][0]) * 1e-3,
                                ((long long)hd[l].match.barr[k][2] - (long long)hd[l].match.barr[k][1]) * 1e-3);
                    fprintf(stderr, "\n");
                }
            }
        }
    }
    // keep levels 0..last_real, release the rest (speculative levels after the stop)
    for (int l = 0; l < (int)lv.size(); ++l) {
        if (st == GP_OK && l <= last_real) {
            h->levels.push_back(lv[l]);
        } else {
            if (!lv[l].arena) {
                dev_free(ctx, lv[l].match);
                dev_free(ctx, lv[l].cmap);
            }
            graph_release(lv[l].coarse);
        }
    }
    if (st != GP_OK) {
        std::string keep = g_last_error;
        cudaStreamSynchronize(ctx->stream);
        hier_release(h);
        g_last_error = keep;
        return st;
    }
    *out = h;
    return GP_OK;
}
}  // namespace gp

extern "C" {

gp_status gp_coarsen_to(gp_graph g, const gp_coarsen_opts *opts, gp_hier *out) {
    if (out) *out = nullptr;
    if (!tagged<Graph>(g, kTagGraph) || !opts || !out || opts->threshold < 0 || opts->stall_ratio_pct < 0 ||
        opts->max_levels < 0 || opts->max_rounds < 0) {
        set_error("gp_coarsen_to: bad graph, options or output");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    Ctx *ctx = g->ctx;
    DeviceGuard dg(ctx->device);
    ctx->tie_seed = opts->tie_seed;
    if (ctx->comm) return dist_coarsen_to(g, opts, out);  // sharded path (dist.cu)
    return coarsen_single(g, opts, out);
    GP_TRY_END
}

gp_status gp_hier_num_levels(gp_hier h, int32_t *out) {
    if (!tagged<Hier>(h, kTagHier) || !out) {
        set_error("gp_hier_num_levels: bad handle");
        return GP_ERR_INVALID_ARG;
    }
    *out = (int32_t)h->levels.size();
    return GP_OK;
}

gp_status gp_hier_level(gp_hier h, int32_t i, gp_level *out) {
    if (!tagged<Hier>(h, kTagHier) || !out || i < 0 || i >= (int32_t)h->levels.size()) {
        set_error("gp_hier_level: bad handle or level index");
        return GP_ERR_INVALID_ARG;
    }
    const Level &l = h->levels[i];
    gp_level o;
    memset(&o, 0, sizeof(o));
    o.n = l.n;
    o.nnz = l.nnz;
    o.n_coarse = l.n_coarse;
    o.cnnz = l.cnnz;
    o.rounds = l.rounds;
    o.maximal = l.maximal;
    o.stop_reason = l.stop_reason;
    o.arcs_scanned = l.arcs_scanned;
    o.rows_scanned = l.rows_scanned;
    o.live_visits = l.live_visits;
    o.d_match = l.match;
    o.d_cmap = l.cmap;
    o.coarse = l.coarse;
    o.v_begin = 0;
    o.n_local = l.n;
    o.cv_begin = 0;
    o.n_coarse_local = l.n_coarse;
    if (!l.pieces.empty()) {  // sharded level
        o.d_match = nullptr;
        o.d_cmap = nullptr;
        o.coarse = nullptr;
        if (l.pieces.size() == 1) {  // NCCL: this rank's piece
            const DistPiece &p = l.pieces[0];
            o.d_match = p.M + p.vbase;
            o.d_cmap = p.CM + p.vbase;
            o.coarse = p.coarse;
            o.v_begin = p.vbase;
            o.n_local = p.nloc;
            o.cv_begin = p.coarse ? p.coarse->vbase : 0;
            o.n_coarse_local = p.coarse ? p.coarse->n : 0;
        }
    }
    *out = o;
    return GP_OK;
}

gp_status gp_hier_download_level(gp_hier h, int32_t i, gp_vid *h_match, gp_vid *h_cmap) {
    if (!tagged<Hier>(h, kTagHier) || i < 0 || i >= (int32_t)h->levels.size()) {
        set_error("gp_hier_download_level: bad handle or level index");
        return GP_ERR_INVALID_ARG;
    }
    const Level &l = h->levels[i];
    DeviceGuard dg(h->ctx->device);
    cudaStream_t s = h->ctx->stream;
    if (!l.pieces.empty()) {  // sharded: the pieces' owned slices, in rank order
        size_t o = 0;
        for (const DistPiece &p : l.pieces) {
            if (h_match && p.nloc)
                GP_CUDA(cudaMemcpyAsync(h_match + o, p.M + p.vbase, sizeof(int32_t) * (size_t)p.nloc,
                                        cudaMemcpyDeviceToHost, s));
            if (h_cmap && p.nloc)
                GP_CUDA(cudaMemcpyAsync(h_cmap + o, p.CM + p.vbase, sizeof(int32_t) * (size_t)p.nloc,
                                        cudaMemcpyDeviceToHost, s));
            o += (size_t)p.nloc;
        }
        GP_CUDA(cudaStreamSynchronize(s));
        return GP_OK;
    }
    if (h_match && l.n) GP_CUDA(cudaMemcpyAsync(h_match, l.match, sizeof(int32_t) * (size_t)l.n, cudaMemcpyDeviceToHost, s));
    if (h_cmap && l.n) GP_CUDA(cudaMemcpyAsync(h_cmap, l.cmap, sizeof(int32_t) * (size_t)l.n, cudaMemcpyDeviceToHost, s));
    GP_CUDA(cudaStreamSynchronize(s));
    return GP_OK;
}

gp_status gp_hier_download_coarse(gp_hier h, int32_t i, gp_vid *h_adjp, gp_vid *h_adjncy, gp_wgt *h_adjwgt,
                                  gp_wgt *h_vwgt, gp_vid *n_out, gp_vid *nnz_out) {
    if (!tagged<Hier>(h, kTagHier) || i < 0 || i >= (int32_t)h->levels.size()) {
        set_error("gp_hier_download_coarse: bad handle or level index");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    const Level &l = h->levels[i];
    std::vector<const Graph *> parts;
    if (l.pieces.empty()) parts.push_back(l.coarse);
    else
        for (const DistPiece &p : l.pieces) parts.push_back(p.coarse);
    DeviceGuard dg(h->ctx->device);
    cudaStream_t s = h->ctx->stream;
    int32_t rows = 0, arcs = 0;
    for (const Graph *c : parts) {
        if (!c) {
            set_error("gp_hier_download_coarse: level has no coarse graph");
            return GP_ERR_INTERNAL;
        }
        if (h_adjp) {
            GP_CUDA(cudaMemcpyAsync(h_adjp + rows, c->adjp, sizeof(int32_t) * ((size_t)c->n + 1), cudaMemcpyDeviceToHost, s));
        }
        if (h_adjncy && c->nnz)
            GP_CUDA(cudaMemcpyAsync(h_adjncy + arcs, c->adjncy, sizeof(int32_t) * (size_t)c->nnz, cudaMemcpyDeviceToHost, s));
        if (h_adjwgt && c->nnz)
            GP_CUDA(cudaMemcpyAsync(h_adjwgt + arcs, c->adjwgt, sizeof(int32_t) * (size_t)c->nnz, cudaMemcpyDeviceToHost, s));
        if (h_vwgt && c->n)
            GP_CUDA(cudaMemcpyAsync(h_vwgt + rows, c->vwgt, sizeof(int32_t) * (size_t)c->n, cudaMemcpyDeviceToHost, s));
        GP_CUDA(cudaStreamSynchronize(s));
        if (h_adjp)  // piece offsets are local: shift them to the concatenation
            for (int32_t r = 0; r <= c->n; ++r) h_adjp[rows + r] += arcs;
        rows += c->n;
        arcs += c->nnz;
    }
    if (n_out) *n_out = rows;
    if (nnz_out) *nnz_out = arcs;
    return GP_OK;
    GP_TRY_END
}

gp_status gp_project(gp_hier h, int32_t from_level, int32_t to_level, const gp_vid *d_part_coarse,
                     gp_vid *d_part_fine) {
    if (!tagged<Hier>(h, kTagHier) || to_level < 0 || from_level < to_level ||
        from_level >= (int32_t)h->levels.size() || !d_part_coarse || !d_part_fine) {
        set_error("gp_project: bad handle, level range or buffers");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    DeviceGuard dg(h->ctx->device);
    std::vector<const int32_t *> cms;
    for (int32_t l = to_level; l <= from_level; ++l) {
        if (!h->levels[l].pieces.empty()) {
            set_error("gp_project: single-GPU hierarchies only");
            return GP_ERR_INVALID_ARG;
        }
        cms.push_back(h->levels[l].cmap);
    }
    return enqueue_project(h->ctx, cms.data(), (int)cms.size(), h->levels[to_level].n, d_part_coarse, d_part_fine);
    GP_TRY_END
}

gp_status gp_refine(gp_graph g, gp_vid *d_part, const gp_refine_opts *opts, int32_t *moves_out, int32_t *passes_out) {
    if (!tagged<Graph>(g, kTagGraph) || !opts || (!d_part && g->n > 0)) {
        set_error("gp_refine: bad graph, labels or options");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    Ctx *ctx = g->ctx;
    DeviceGuard dg(ctx->device);
    if (ctx->comm || g->dist) {
        set_error("gp_refine: single-GPU graphs only");
        return GP_ERR_INVALID_ARG;
    }
    return refine_graph(ctx, g, d_part, *opts, moves_out, passes_out);
    GP_TRY_END
}

gp_status gp_uncoarsen(gp_hier h, gp_graph g0, const gp_vid *d_part_coarse, gp_vid *d_part_fine,
                       const gp_refine_opts *opts, int32_t *moves_out) {
    if (!tagged<Hier>(h, kTagHier) || !tagged<Graph>(g0, kTagGraph) || !opts || !d_part_coarse || !d_part_fine) {
        set_error("gp_uncoarsen: bad hierarchy, graph, labels or options");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    Ctx *ctx = h->ctx;
    DeviceGuard dg(ctx->device);
    const int L = (int)h->levels.size();
    if (L == 0 || g0->n != h->levels[0].n || g0->ctx != ctx) {
        set_error("gp_uncoarsen: g0 is not the fine graph of this hierarchy's level 0");
        return GP_ERR_INVALID_ARG;
    }
    for (const Level &l : h->levels)
        if (!l.pieces.empty()) {
            set_error("gp_uncoarsen: single-GPU hierarchies only");
            return GP_ERR_INVALID_ARG;
        }
    // two label buffers (the coarsest labels are read in place)
    int32_t *buf[2] = {nullptr, nullptr};
    gp_status st = dev_alloc(ctx, (void **)&buf[0], sizeof(int32_t) * (size_t)(g0->n + 1));
    if (st == GP_OK) st = dev_alloc(ctx, (void **)&buf[1], sizeof(int32_t) * (size_t)(g0->n + 1));
    const int32_t *cur = d_part_coarse;
    int32_t total = 0;
    for (int l = L - 1; st == GP_OK && l >= 0; --l) {
        int32_t *dst = (l == 0) ? d_part_fine : buf[l & 1];
        const int32_t *cm = h->levels[l].cmap;
        st = enqueue_project(ctx, &cm, 1, h->levels[l].n, cur, dst);  // P20.s41-P22.s0
        const Graph *fine = (l == 0) ? g0 : h->levels[l - 1].coarse;
        int32_t mv = 0;
        if (st == GP_OK) st = refine_graph(ctx, fine, dst, *opts, &mv, nullptr);  // P22.s1-22
        total += mv;
        cur = dst;
    }
    cudaError_t e = cudaStreamSynchronize(ctx->stream);
    dev_free(ctx, buf[0]);
    dev_free(ctx, buf[1]);
    if (st == GP_OK && e != cudaSuccess) st = cuda_fail(e, "gp_uncoarsen");
    if (st == GP_OK && moves_out) *moves_out = total;
    return st;
    GP_TRY_END
}

gp_status gp_nccl_unique_id(void *out128) {
    if (!out128) return GP_ERR_INVALID_ARG;
    return dist_unique_id(out128);
}

static gp_status attach_comm(gp_ctx ctx, gp_status st) {
    if (st != GP_OK) {
        std::string keep = g_last_error;
        gp_free(ctx);
        g_last_error = keep;
    }
    return st;
}

gp_status gp_ctx_create_dist(int device, void *cuda_stream, const void *nccl_unique_id, int rank, int nranks,
                             gp_ctx *out) {
    if (!out || !nccl_unique_id || nranks < 1 || rank < 0 || rank >= nranks) {
        set_error("gp_ctx_create_dist: bad id, rank or nranks");
        if (out) *out = nullptr;
        return GP_ERR_INVALID_ARG;
    }
    gp_status st = gp_ctx_create(device, cuda_stream, out);
    if (st != GP_OK) return st;
    DeviceGuard dg(device);
    st = attach_comm(*out, dist_comm_create_nccl(*out, nccl_unique_id, rank, nranks));
    if (st != GP_OK) *out = nullptr;
    return st;
}

gp_status gp_ctx_create_loopback(int device, void *cuda_stream, int nranks, gp_ctx *out) {
    if (!out || nranks < 1) {
        set_error("gp_ctx_create_loopback: bad nranks");
        if (out) *out = nullptr;
        return GP_ERR_INVALID_ARG;
    }
    gp_status st = gp_ctx_create(device, cuda_stream, out);
    if (st != GP_OK) return st;
    DeviceGuard dg(device);
    st = attach_comm(*out, dist_comm_create_loopback(*out, nranks));
    if (st != GP_OK) *out = nullptr;
    return st;
}

gp_status gp_ctx_dist_info(gp_ctx ctx, int32_t *rank, int32_t *nranks) {
    if (!tagged<Ctx>(ctx, kTagCtx)) return GP_ERR_INVALID_ARG;
    if (rank) *rank = dist_rank(ctx);
    if (nranks) *nranks = dist_nranks(ctx);
    return GP_OK;
}

gp_status gp_graph_create_dist(gp_ctx ctx, gp_vid n_global, gp_vid v_begin, gp_vid v_end, const gp_vid *adjp_local,
                               const gp_vid *adjncy, const gp_wgt *adjwgt, const gp_wgt *vwgt, uint32_t flags,
                               gp_graph *out) {
    if (out) *out = nullptr;
    if (!tagged<Ctx>(ctx, kTagCtx) || !out || !ctx->comm || dist_rank(ctx) < 0 || n_global < 0 || v_begin < 0 ||
        v_end < v_begin || v_end > n_global) {
        set_error("gp_graph_create_dist: needs an NCCL context and 0 <= v_begin <= v_end <= n_global");
        return GP_ERR_INVALID_ARG;
    }
    if (flags & GP_VALIDATE) {
        set_error("gp_graph_create_dist: GP_VALIDATE checks whole graphs (use a single-GPU context)");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    // Every rank reaches the all-gather even when its local create failed, so that a failure
    // (or an overflow of the GLOBAL weight totals, R14) is reported on all ranks together
    // instead of leaving the others waiting in a collective.
    gp_graph g = nullptr;
    gp_status st = graph_create_impl(ctx, v_end - v_begin, adjp_local, adjncy, adjwgt, vwgt, flags, false, &g);
    const int G = dist_nranks(ctx), me = dist_rank(ctx);
    const unsigned long long sa = g ? g->sum_adjwgt : 0ull, sv = g ? g->sum_vwgt : 0ull;
    int32_t mine[8] = {v_begin, v_end, g ? g->nnz : 0, (int32_t)st, (int32_t)(uint32_t)sa, (int32_t)(uint32_t)(sa >> 32),
                       (int32_t)(uint32_t)sv, (int32_t)(uint32_t)(sv >> 32)};
    std::vector<int32_t> all(8 * (size_t)G);
    const std::string local_err = st != GP_OK ? g_last_error : std::string();
    gp_status gst = dist_allgather_i32(ctx, mine, 8, all.data());
    if (gst != GP_OK) {
        if (g) gp_free(g);
        return gst;
    }
    long long nnz = 0;
    unsigned long long tot_a = 0, tot_v = 0;
    std::vector<int32_t> ranges(G + 1);
    for (int r = 0; r < G; ++r) {
        const int32_t *a = &all[8 * (size_t)r];
        if (st == GP_OK && a[3] != GP_OK) {
            set_error("gp_graph_create_dist: rank " + std::to_string(r) + " failed to create its shard (" +
                      gp_status_string((gp_status)a[3]) + ")");
            st = (gp_status)a[3];
        }
        ranges[r] = a[0];
        nnz += a[2];
        tot_a += (unsigned long long)(uint32_t)a[4] | ((unsigned long long)(uint32_t)a[5] << 32);
        tot_v += (unsigned long long)(uint32_t)a[6] | ((unsigned long long)(uint32_t)a[7] << 32);
        if (st == GP_OK && (a[0] != (r == 0 ? 0 : all[8 * ((size_t)r - 1) + 1]) || (r == G - 1 && a[1] != n_global))) {
            set_error("gp_graph_create_dist: the shards do not tile [0, n_global) in rank order");
            st = GP_ERR_INVALID_ARG;
        }
    }
    if (st == GP_OK && nnz > INT32_MAX) {
        set_error("gp_graph_create_dist: total arcs exceed INT32_MAX");
        st = GP_ERR_OVERFLOW;
    }
    if (st == GP_OK && (tot_a > (unsigned long long)INT32_MAX || tot_v > (unsigned long long)INT32_MAX)) {
        set_error("gp_graph_create_dist: global weight totals exceed INT32_MAX: sum(adjwgt)=" + std::to_string(tot_a) +
                  " sum(vwgt)=" + std::to_string(tot_v));
        st = GP_ERR_OVERFLOW;
    }
    if (st != GP_OK) {
        std::string keep = local_err.empty() ? g_last_error : local_err;
        if (g) gp_free(g);
        g_last_error = keep;
        return st;
    }
    ranges[G] = n_global;
    g->dist = true;
    g->rank = me;
    g->vbase = v_begin;
    g->n_global = n_global;
    g->nnz_global = (int32_t)nnz;
    g->ranges = ranges;
    *out = g;
    return GP_OK;
    GP_TRY_END
}

void gp_free(void *handle) {
    if (!handle) return;
    const uint32_t tag = *static_cast<const uint32_t *>(handle);
    if (tag == kTagGraph) {
        Graph *g = static_cast<Graph *>(handle);
        DeviceGuard dg(g->ctx->device);
        if (!g->borrowed) graph_release(g);
    } else if (tag == kTagHier) {
        Hier *h = static_cast<Hier *>(handle);
        DeviceGuard dg(h->ctx->device);
        hier_release(h);
    } else if (tag == kTagCtx) {
        Ctx *ctx = static_cast<Ctx *>(handle);
        DeviceGuard dg(ctx->device);
        cudaStreamSynchronize(ctx->stream);
        dist_comm_destroy(ctx);
        drain_events(ctx);
        for (auto e : ctx->event_pool) cudaEventDestroy(e);
        dev_free(ctx, ctx->scratch);
        dev_free(ctx, ctx->status);
        cudaStreamSynchronize(ctx->stream);
        if (ctx->pinned) cudaFreeHost(ctx->pinned);
        if (ctx->reports) cudaFreeHost(ctx->reports);
        ctx->tag = 0;
        delete ctx;
    }
}

gp_status gp_ctx_set_timing(gp_ctx ctx, int32_t enable) {
    if (!tagged<Ctx>(ctx, kTagCtx)) return GP_ERR_INVALID_ARG;
    DeviceGuard dg(ctx->device);
    drain_events(ctx);
    ctx->timing = enable != 0;
    return GP_OK;
}

gp_status gp_ctx_kernel_stats(gp_ctx ctx, gp_kernel_kind kind, gp_kernel_stats *out) {
    if (!tagged<Ctx>(ctx, kTagCtx) || !out || kind < 0 || kind >= GP_K_COUNT) return GP_ERR_INVALID_ARG;
    DeviceGuard dg(ctx->device);
    drain_events(ctx);
    *out = ctx->stats[kind];
    return GP_OK;
}

gp_status gp_ctx_reset_stats(gp_ctx ctx) {
    if (!tagged<Ctx>(ctx, kTagCtx)) return GP_ERR_INVALID_ARG;
    DeviceGuard dg(ctx->device);
    drain_events(ctx);
    for (auto &s : ctx->stats) s = gp_kernel_stats{0, 0.0};
    ctx->launch_log.clear();
    return GP_OK;
}

gp_status gp_ctx_launch_times(gp_ctx ctx, int32_t cap, int32_t *kinds, float *ms, int32_t *count) {
    if (!tagged<Ctx>(ctx, kTagCtx) || cap < 0 || (cap > 0 && (!kinds || !ms))) return GP_ERR_INVALID_ARG;
    DeviceGuard dg(ctx->device);
    drain_events(ctx);
    const int32_t n = (int32_t)ctx->launch_log.size();
    for (int32_t i = 0; i < n && i < cap; ++i) {
        kinds[i] = ctx->launch_log[(size_t)i].first;
        ms[i] = ctx->launch_log[(size_t)i].second;
    }
    if (count) *count = n;
    return GP_OK;
}

gp_status gp_ctx_launch_count(gp_ctx ctx, int64_t *out) {
    if (!tagged<Ctx>(ctx, kTagCtx) || !out) return GP_ERR_INVALID_ARG;
    *out = ctx->launches;
    return GP_OK;
}

}  // extern "C"
