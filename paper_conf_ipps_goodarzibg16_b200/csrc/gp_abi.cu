// gp_abi.cu -- the C ABI of include/gp.h: handles, memory, errors, instrumentation and the
// level driver gp_coarsen_to (A9: P10.s16, P20.s27-31, P12.s30; readings R12, R13).
#include <cuda_runtime.h>

#include <cstring>
#include <new>
#include <string>

#include "gp_internal.cuh"

namespace gp {

gp_status contract_set_attributes();
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
        }
        ctx->event_pool.push_back(t.a);
        ctx->event_pool.push_back(t.b);
    }
    ctx->pending.clear();
}

static void graph_release(Graph *g) {
    if (!g) return;
    Ctx *ctx = g->ctx;
    dev_free(ctx, g->adjp);
    dev_free(ctx, g->adjncy);
    dev_free(ctx, g->adjwgt);
    dev_free(ctx, g->vwgt);
    g->tag = 0;
    delete g;
}

static void hier_release(Hier *h) {
    if (!h) return;
    for (auto &l : h->levels) {
        dev_free(h->ctx, l.match);
        dev_free(h->ctx, l.cmap);
        graph_release(l.coarse);
    }
    h->tag = 0;
    delete h;
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
    GP_CUDA(cudaSetDevice(device));
    cudaDeviceProp prop;
    GP_CUDA(cudaGetDeviceProperties(&prop, device));
    if (prop.major < 10) {
        set_error("gp_ctx_create: device is sm_" + std::to_string(prop.major) + std::to_string(prop.minor) +
                  ", this library is built for sm_100a");
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
    gp_status st = contract_set_attributes();
    if (st == GP_OK) st = dev_alloc(ctx, (void **)&ctx->ctl, sizeof(LevelCtl));
    if (st == GP_OK) {
        cudaError_t e = cudaMallocHost((void **)&ctx->ctl_host, sizeof(LevelCtl));
        if (e != cudaSuccess) st = cuda_fail(e, "cudaMallocHost");
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
    // existing buffers were allocated with the previous allocator: release them first
    cudaStreamSynchronize(ctx->stream);
    dev_free(ctx, ctx->scratch);
    dev_free(ctx, ctx->status);
    dev_free(ctx, ctx->ctl);
    ctx->scratch = nullptr;
    ctx->scratch_bytes = 0;
    ctx->status = nullptr;
    ctx->status_words = 0;
    ctx->ctl = nullptr;
    ctx->alloc = alloc;
    ctx->dealloc = dealloc;
    ctx->alloc_user = user;
    return dev_alloc(ctx, (void **)&ctx->ctl, sizeof(LevelCtl));
}

gp_status gp_ctx_num_sms(gp_ctx ctx, int32_t *out) {
    if (!tagged<Ctx>(ctx, kTagCtx) || !out) return GP_ERR_INVALID_ARG;
    *out = ctx->num_sms;
    return GP_OK;
}

gp_status gp_graph_create(gp_ctx ctx, gp_vid n, const gp_vid *adjp, const gp_vid *adjncy, const gp_wgt *adjwgt,
                          const gp_wgt *vwgt, uint32_t flags, gp_graph *out) {
    if (out) *out = nullptr;
    if (!tagged<Ctx>(ctx, kTagCtx) || !out || n < 0 || !adjp) {
        set_error("gp_graph_create: bad context, output or n");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    const bool dev = flags & GP_INPUT_DEVICE;
    const cudaMemcpyKind kind = dev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    GP_CUDA(cudaSetDevice(ctx->device));
    int32_t nnz = 0;
    if (dev) {
        GP_CUDA(cudaMemcpyAsync(&ctx->ctl_host->pad[0], adjp + n, sizeof(int32_t), cudaMemcpyDeviceToHost,
                                ctx->stream));
        GP_CUDA(cudaStreamSynchronize(ctx->stream));
        nnz = ctx->ctl_host->pad[0];
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
    gp_status st = dev_alloc(ctx, (void **)&g->adjp, sizeof(int32_t) * ((size_t)n + 1));
    if (st == GP_OK) st = dev_alloc(ctx, (void **)&g->adjncy, sizeof(int32_t) * (size_t)nnz);
    if (st == GP_OK) st = dev_alloc(ctx, (void **)&g->adjwgt, sizeof(int32_t) * (size_t)nnz);
    if (st == GP_OK) st = dev_alloc(ctx, (void **)&g->vwgt, sizeof(int32_t) * (size_t)n);
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
    if (st == GP_OK && e != cudaSuccess) st = cuda_fail(e, "gp_graph_create: copy");
    if (st == GP_OK) st = graph_totals_and_validate(ctx, g, flags & GP_VALIDATE);
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

gp_status gp_match_level(gp_graph g, gp_vid *d_match, int32_t max_rounds, int32_t *rounds_out) {
    if (!tagged<Graph>(g, kTagGraph) || (!d_match && g->n > 0) || max_rounds < 0) {
        set_error("gp_match_level: bad graph, match buffer or max_rounds");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    Ctx *ctx = g->ctx;
    MatchResult r;
    gp_status st = match_level(ctx, g, d_match, max_rounds, true, &r);
    if (st != GP_OK) return st;
    if (rounds_out) {
        GP_CUDA(cudaStreamSynchronize(ctx->stream));
        *rounds_out = r.rounds;
    }
    return GP_OK;
    GP_TRY_END
}

gp_status gp_contract_level(gp_graph g, const gp_vid *d_match, gp_vid *d_cmap, gp_graph *coarse_out) {
    if (coarse_out) *coarse_out = nullptr;
    if (!tagged<Graph>(g, kTagGraph) || !coarse_out || ((!d_match || !d_cmap) && g->n > 0)) {
        set_error("gp_contract_level: bad graph or buffers");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    Graph *c = nullptr;
    gp_status st = contract_level(g->ctx, g, const_cast<int32_t *>(d_match), d_cmap, false, &c);
    if (st != GP_OK) return st;
    *coarse_out = c;
    return GP_OK;
    GP_TRY_END
}

gp_status gp_coarsen_to(gp_graph g, const gp_coarsen_opts *opts, gp_hier *out) {
    if (out) *out = nullptr;
    if (!tagged<Graph>(g, kTagGraph) || !opts || !out || opts->threshold < 0 || opts->stall_ratio_pct < 0 ||
        opts->max_levels < 0 || opts->max_rounds < 0) {
        set_error("gp_coarsen_to: bad graph, options or output");
        return GP_ERR_INVALID_ARG;
    }
    GP_TRY_BEGIN
    Ctx *ctx = g->ctx;
    const int32_t pct = opts->stall_ratio_pct ? opts->stall_ratio_pct : 95;
    const int32_t max_levels = opts->max_levels ? opts->max_levels : 64;
    Hier *h = new Hier();
    h->ctx = ctx;
    const Graph *cur = g;
    gp_status st = GP_OK;
    while (cur->n > opts->threshold && (int32_t)h->levels.size() < max_levels) {
        Level lv;
        lv.n = cur->n;
        lv.nnz = cur->nnz;
        st = dev_alloc(ctx, (void **)&lv.match, sizeof(int32_t) * (size_t)cur->n);
        if (st == GP_OK) st = dev_alloc(ctx, (void **)&lv.cmap, sizeof(int32_t) * (size_t)cur->n);
        MatchResult mr;
        if (st == GP_OK) st = match_level(ctx, cur, lv.match, opts->max_rounds, false, &mr);
        Graph *cg = nullptr;
        if (st == GP_OK) st = contract_level(ctx, cur, lv.match, lv.cmap, true, &cg);
        if (st != GP_OK) {
            dev_free(ctx, lv.match);
            dev_free(ctx, lv.cmap);
            break;
        }
        cg->borrowed = true;
        lv.coarse = cg;
        lv.rounds = mr.rounds;
        lv.maximal = mr.maximal;
        lv.arcs_scanned = mr.arcs_scanned;
        lv.rows_scanned = mr.rows_scanned;
        lv.live_visits = mr.live_visits;
        lv.n_coarse = cg->n;
        lv.cnnz = cg->nnz;
        h->levels.push_back(lv);
        const bool stall = 100LL * cg->n > (long long)pct * cur->n;
        cur = cg;
        if (stall) {
            h->levels.back().stop_reason = GP_STOP_STALL;
            break;
        }
    }
    if (st != GP_OK) {
        std::string keep = g_last_error;
        cudaStreamSynchronize(ctx->stream);
        hier_release(h);
        g_last_error = keep;
        return st;
    }
    if (!h->levels.empty() && h->levels.back().stop_reason == GP_STOP_NONE)
        h->levels.back().stop_reason = (cur->n <= opts->threshold) ? GP_STOP_THRESHOLD : GP_STOP_MAX_LEVELS;
    *out = h;
    return GP_OK;
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
    *out = o;
    return GP_OK;
}

gp_status gp_hier_download_level(gp_hier h, int32_t i, gp_vid *h_match, gp_vid *h_cmap) {
    if (!tagged<Hier>(h, kTagHier) || i < 0 || i >= (int32_t)h->levels.size()) {
        set_error("gp_hier_download_level: bad handle or level index");
        return GP_ERR_INVALID_ARG;
    }
    const Level &l = h->levels[i];
    cudaStream_t s = h->ctx->stream;
    if (h_match && l.n) GP_CUDA(cudaMemcpyAsync(h_match, l.match, sizeof(int32_t) * (size_t)l.n, cudaMemcpyDeviceToHost, s));
    if (h_cmap && l.n) GP_CUDA(cudaMemcpyAsync(h_cmap, l.cmap, sizeof(int32_t) * (size_t)l.n, cudaMemcpyDeviceToHost, s));
    GP_CUDA(cudaStreamSynchronize(s));
    return GP_OK;
}

void gp_free(void *handle) {
    if (!handle) return;
    const uint32_t tag = *static_cast<const uint32_t *>(handle);
    if (tag == kTagGraph) {
        Graph *g = static_cast<Graph *>(handle);
        if (!g->borrowed) graph_release(g);
    } else if (tag == kTagHier) {
        hier_release(static_cast<Hier *>(handle));
    } else if (tag == kTagCtx) {
        Ctx *ctx = static_cast<Ctx *>(handle);
        cudaStreamSynchronize(ctx->stream);
        drain_events(ctx);
        for (auto e : ctx->event_pool) cudaEventDestroy(e);
        dev_free(ctx, ctx->scratch);
        dev_free(ctx, ctx->status);
        dev_free(ctx, ctx->ctl);
        cudaStreamSynchronize(ctx->stream);
        if (ctx->ctl_host) cudaFreeHost(ctx->ctl_host);
        ctx->tag = 0;
        delete ctx;
    }
}

gp_status gp_ctx_set_timing(gp_ctx ctx, int32_t enable) {
    if (!tagged<Ctx>(ctx, kTagCtx)) return GP_ERR_INVALID_ARG;
    drain_events(ctx);
    ctx->timing = enable != 0;
    return GP_OK;
}

gp_status gp_ctx_kernel_stats(gp_ctx ctx, gp_kernel_kind kind, gp_kernel_stats *out) {
    if (!tagged<Ctx>(ctx, kTagCtx) || !out || kind < 0 || kind >= GP_K_COUNT) return GP_ERR_INVALID_ARG;
    drain_events(ctx);
    *out = ctx->stats[kind];
    return GP_OK;
}

gp_status gp_ctx_reset_stats(gp_ctx ctx) {
    if (!tagged<Ctx>(ctx, kTagCtx)) return GP_ERR_INVALID_ARG;
    drain_events(ctx);
    for (auto &s : ctx->stats) s = gp_kernel_stats{0, 0.0};
    return GP_OK;
}

gp_status gp_ctx_launch_count(gp_ctx ctx, int64_t *out) {
    if (!tagged<Ctx>(ctx, kTagCtx) || !out) return GP_ERR_INVALID_ARG;
    *out = ctx->launches;
    return GP_OK;
}

}  // extern "C"
