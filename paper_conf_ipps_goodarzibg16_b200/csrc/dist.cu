// dist.cu -- the sharded coarsening path: contiguous vertex ranges over the ranks of one node
// (DESIGN.md §7).  Results are bit-identical to the 1-GPU path.
//
// Every rank runs the SAME level kernels as one GPU (match.cu / contract.cu) on its rows;
// only the exchange steps are new:
//   per handshake round   all-gather of boundary records (v, P[v], P[P[v]] if P[v] is the
//                         owner's, else -2) + each rank's live count and match flag.  The
//                         receiver writes P[v] (and P[P[v]]) into its own globally indexed P,
//                         so the unchanged "x free after round k" test P[P[x]] != x sees the
//                         ghost state exactly as the 1-GPU kernel does (the free set only
//                         shrinks and every round reads the previous round's P: the rule's
//                         synchronous rounds, R1-R4, make the sharded run equal the 1-GPU run).
//   per level             all-gather of the leader counts -> rank offsets of the coarse ids
//                         (P18.s16-27's scan, split into per-rank scans + the rank prefix);
//                         all-gather of boundary (v, M[v], CM[v] or -1) records; the rows of
//                         non-leader partners whose leader lives on another rank are sent
//                         to it (grouped send/recv) with CM of every neighbour attached; the
//                         contraction kernel then merges local + shipped rows (P12.s26-28).
// Transport: NCCL over NVLink (one process per GPU; libnccl.so.2 is dlopen'ed) or "loopback"
// (all ranks simulated in one process on one GPU, collectives = device copies between the
// ranks' private buffers): the same kernels, buffers and layouts.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>  // types only: the library is loaded at run time

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "device_util.cuh"
#include "gp_internal.cuh"

namespace gp {

// ---------------------------------------------------------------------------------------
// NCCL, loaded at run time (torch's bundled libnccl.so.2 is picked up when already loaded)
// ---------------------------------------------------------------------------------------
struct NcclApi {
    bool ok = false;
    std::string why;
    ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*AllGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Send)(const void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char *(*GetErrorString)(ncclResult_t) = nullptr;
};

static NcclApi &nccl() {
    static NcclApi api;
    static bool tried = false;
    if (tried) return api;
    tried = true;
    void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
        api.why = std::string("cannot load libnccl.so.2: ") + dlerror();
        return api;
    }
#define GP_SYM(field, name)                                                   \
    api.field = reinterpret_cast<decltype(api.field)>(dlsym(h, name));       \
    if (!api.field) {                                                         \
        api.why = std::string("libnccl.so.2 lacks ") + name;                  \
        return api;                                                           \
    }
    GP_SYM(GetUniqueId, "ncclGetUniqueId");
    GP_SYM(CommInitRank, "ncclCommInitRank");
    GP_SYM(CommDestroy, "ncclCommDestroy");
    GP_SYM(AllGather, "ncclAllGather");
    GP_SYM(Send, "ncclSend");
    GP_SYM(Recv, "ncclRecv");
    GP_SYM(GroupStart, "ncclGroupStart");
    GP_SYM(GroupEnd, "ncclGroupEnd");
    GP_SYM(GetErrorString, "ncclGetErrorString");
#undef GP_SYM
    api.ok = true;
    return api;
}

static gp_status nccl_fail(ncclResult_t r, const char *what) {
    set_error(std::string(what) + ": " + (nccl().GetErrorString ? nccl().GetErrorString(r) : "nccl error"));
    return GP_ERR_NCCL;
}
#define GP_NCCL(call)                                         \
    do {                                                      \
        ncclResult_t r__ = (call);                            \
        if (r__ != ncclSuccess) return nccl_fail(r__, #call); \
    } while (0)

struct DistComm {
    int nranks = 1;
    int rank = 0;  // -1: loopback (every rank lives in this process)
    ncclComm_t comm = nullptr;
    bool loopback() const { return rank < 0; }
    int nlocal() const { return loopback() ? nranks : 1; }
    int grank(int i) const { return loopback() ? i : rank; }
};

gp_status dist_unique_id(void *out128) {
    NcclApi &api = nccl();
    if (!api.ok) {
        set_error(api.why);
        return GP_ERR_NCCL;
    }
    ncclUniqueId id;
    GP_NCCL(api.GetUniqueId(&id));
    memcpy(out128, &id, sizeof(id));
    return GP_OK;
}

int dist_rank(const Ctx *ctx) { return ctx->comm ? ctx->comm->rank : 0; }
int dist_nranks(const Ctx *ctx) { return ctx->comm ? ctx->comm->nranks : 1; }

gp_status dist_comm_create_nccl(Ctx *ctx, const void *uid, int rank, int nranks) {
    NcclApi &api = nccl();
    if (!api.ok) {
        set_error(api.why);
        return GP_ERR_NCCL;
    }
    ncclUniqueId id;
    memcpy(&id, uid, sizeof(id));
    DistComm *c = new DistComm();
    c->nranks = nranks;
    c->rank = rank;
    ncclResult_t r = api.CommInitRank(&c->comm, nranks, id, rank);
    if (r != ncclSuccess) {
        delete c;
        return nccl_fail(r, "ncclCommInitRank");
    }
    ctx->comm = c;
    return GP_OK;
}

gp_status dist_comm_create_loopback(Ctx *ctx, int nranks) {
    DistComm *c = new DistComm();
    c->nranks = nranks;
    c->rank = -1;
    ctx->comm = c;
    return GP_OK;
}

void dist_comm_destroy(Ctx *ctx) {
    if (!ctx->comm) return;
    if (ctx->comm->comm && nccl().ok) nccl().CommDestroy(ctx->comm->comm);
    delete ctx->comm;
    ctx->comm = nullptr;
}

// all-gather of `count` int32 from every local rank's send[i] into every local rank's
// recv[i] (nranks * count ints, rank order)
static gp_status allgather(Ctx *ctx, const std::vector<int32_t *> &send, const std::vector<int32_t *> &recv,
                           size_t count) {
    DistComm *c = ctx->comm;
    if (count == 0) return GP_OK;
    if (!c->loopback()) {
        GP_NCCL(nccl().AllGather(send[0], recv[0], count, ncclInt32, c->comm, ctx->stream));
        return GP_OK;
    }
    for (int r = 0; r < c->nranks; ++r)
        for (int s = 0; s < c->nranks; ++s)
            GP_CUDA(cudaMemcpyAsync(recv[r] + (size_t)s * count, send[s], count * 4, cudaMemcpyDeviceToDevice,
                                    ctx->stream));
    return GP_OK;
}

// point-to-point exchange: local rank i sends scount[i][d] ints at send[i] + soff[i][d] to
// rank d, which receives them at recv[d] + roff[d][i] (offsets/counts in int32 units, global
// rank indices; rank-to-self traffic is never generated by the driver)
using Mat = std::vector<std::vector<long long>>;
static gp_status exchange(Ctx *ctx, const std::vector<int32_t *> &send, const Mat &scount, const Mat &soff,
                          const std::vector<int32_t *> &recv, const Mat &rcount, const Mat &roff) {
    DistComm *c = ctx->comm;
    const int G = c->nranks;
    if (!c->loopback()) {
        const int me = c->rank;
        GP_NCCL(nccl().GroupStart());
        for (int d = 0; d < G; ++d)
            if (d != me && scount[me][d] > 0)
                GP_NCCL(nccl().Send(send[0] + soff[me][d], (size_t)scount[me][d], ncclInt32, d, c->comm, ctx->stream));
        for (int s = 0; s < G; ++s)
            if (s != me && rcount[me][s] > 0)
                GP_NCCL(nccl().Recv(recv[0] + roff[me][s], (size_t)rcount[me][s], ncclInt32, s, c->comm, ctx->stream));
        GP_NCCL(nccl().GroupEnd());
        return GP_OK;
    }
    for (int s = 0; s < G; ++s)
        for (int d = 0; d < G; ++d)
            if (d != s && scount[s][d] > 0)
                GP_CUDA(cudaMemcpyAsync(recv[d] + roff[d][s], send[s] + soff[s][d], (size_t)scount[s][d] * 4,
                                        cudaMemcpyDeviceToDevice, ctx->stream));
    return GP_OK;
}

gp_status dist_allgather_i32(Ctx *ctx, const int32_t *h_send, int32_t count, int32_t *h_recv) {
    DistComm *c = ctx->comm;
    if (c->loopback()) {
        set_error("dist_allgather_i32: host values of a loopback context");
        return GP_ERR_INTERNAL;
    }
    int32_t *d = nullptr;
    gp_status st = dev_alloc(ctx, (void **)&d, sizeof(int32_t) * (size_t)count * (c->nranks + 1));
    if (st != GP_OK) return st;
    cudaError_t e = cudaMemcpyAsync(d, h_send, sizeof(int32_t) * count, cudaMemcpyHostToDevice, ctx->stream);
    if (e != cudaSuccess) st = cuda_fail(e, "allgather h2d");
    if (st == GP_OK) st = allgather(ctx, {d}, {d + count}, (size_t)count);
    if (st == GP_OK) {
        e = cudaMemcpyAsync(h_recv, d + count, sizeof(int32_t) * count * c->nranks, cudaMemcpyDeviceToHost, ctx->stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
        if (e != cudaSuccess) st = cuda_fail(e, "allgather d2h");
    }
    dev_free(ctx, d);
    return st;
}

// ---------------------------------------------------------------------------------------
// kernels of the exchange steps (plain grid-stride kernels; every one is HBM/latency-light)
// ---------------------------------------------------------------------------------------
constexpr int kDT = 256;
constexpr int32_t kNoPP = -2;  // record field "P[P[v]] not known to v's owner"

__device__ __forceinline__ bool in_range(int32_t x, int32_t lo, int32_t hi) { return x >= lo && x < hi; }
__device__ __forceinline__ int owner_of(int32_t x, const int32_t *ranges, int G) {
    int s = 0;
    while (s + 1 < G && x >= ranges[s + 1]) ++s;
    return s;
}

static int grid_for(long long items, int per_block = kDT) {
    long long b = (items + per_block - 1) / per_block;
    if (b < 1) b = 1;
    if (b > 148 * 16) b = 148 * 16;
    return (int)b;
}

// boundary vertices: local rows with a neighbour outside [vbase, vbase + nloc)
__global__ void k_boundary(const int32_t *adjp, const int32_t *adjncy, int32_t nloc, int32_t vbase, int32_t *B,
                           int32_t *count) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long base = (long long)blockIdx.x * blockDim.x; base < nloc; base += stride) {
        const long long r = base + threadIdx.x;
        bool f = false;
        if (r < nloc) {
            const int32_t s = adjp[r], e = adjp[r + 1];
            for (int32_t j = s; j < e && !f; ++j) f = !in_range(adjncy[j], vbase, vbase + nloc);
        }
        warp_append(B, count, f, vbase + (int32_t)r);
    }
}

// round records: header {live, made, count, 0} + count x {v, P[v], P[P[v]] or kNoPP}
__global__ void k_pack_match(const int32_t *B, int32_t nb, const int32_t *P, int32_t vbase, int32_t nloc,
                             const int32_t *live_src, int32_t live_const, const int32_t *made_src, int32_t *buf) {
    const long long t0 = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (t0 == 0) {
        buf[0] = live_src ? *(volatile const int32_t *)live_src : live_const;
        buf[1] = made_src ? *(volatile const int32_t *)made_src : 0;
        buf[2] = nb;
        buf[3] = 0;
    }
    for (long long i = t0; i < nb; i += (long long)gridDim.x * blockDim.x) {
        const int32_t v = B[i];
        const int32_t p = P[v];
        const int32_t pp = (p >= 0 && in_range(p, vbase, vbase + nloc)) ? P[p] : kNoPP;
        buf[4 + 3 * i] = v;
        buf[4 + 3 * i + 1] = p;
        buf[4 + 3 * i + 2] = pp;
    }
}

__global__ void k_unpack_match(const int32_t *recv, long long RS, int G, int me, int32_t maxb, int32_t *P) {
    const long long tot = (long long)G * maxb;
    for (long long idx = (long long)blockIdx.x * blockDim.x + threadIdx.x; idx < tot;
         idx += (long long)gridDim.x * blockDim.x) {
        const int s = (int)(idx / maxb);
        const int32_t i = (int32_t)(idx % maxb);
        if (s == me) continue;
        const int32_t *rb = recv + (size_t)s * RS;
        if (i >= rb[2]) continue;
        const int32_t v = rb[4 + 3 * i], p = rb[4 + 3 * i + 1], pp = rb[4 + 3 * i + 2];
        P[v] = p;
        if (pp != kNoPP) P[p] = pp;  // p is interior to v's owner: its proposal rides along
    }
}

// contraction, step 1: leader flags + per-destination counts of the rows to ship
// cnt layout: [0] leaders (written by the scan), [1 + d] rows to d, [1 + G + d] arcs to d
__global__ void k_dc_flags(const int32_t *M, const int32_t *adjp, int32_t nloc, int32_t vbase, const int32_t *ranges,
                           int G, int32_t *lead, int32_t *cnt) {
    for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < nloc; r += (long long)gridDim.x * blockDim.x) {
        const int32_t u = vbase + (int32_t)r, m = M[u];
        lead[r] = u <= m;  // P18.s18 (R7)
        if (u > m && !in_range(m, vbase, vbase + nloc)) {
            const int d = owner_of(m, ranges, G);
            atomicAdd(&cnt[1 + d], 1);
            atomicAdd(&cnt[1 + G + d], adjp[r + 1] - adjp[r]);
        }
    }
}

// step 2: CM of the local leaders (rank offset + local exclusive scan) and of local partners
__global__ void k_dc_cm(const int32_t *M, const int32_t *lead, const int32_t *pos, int32_t nloc, int32_t vbase,
                        int32_t cbase, int32_t *CM) {
    for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < nloc; r += (long long)gridDim.x * blockDim.x) {
        if (!lead[r]) continue;
        const int32_t u = vbase + (int32_t)r, m = M[u], c = cbase + pos[r];
        CM[u] = c;
        if (m != u && in_range(m, vbase, vbase + nloc)) CM[m] = c;  // P18.s26
    }
}

// CM records: header {0, 0, count, 0} + count x {v, M[v], CM[v] or -1 (leader is remote)}
__global__ void k_pack_cm(const int32_t *B, int32_t nb, const int32_t *M, const int32_t *CM, int32_t vbase,
                          int32_t nloc, int32_t *buf) {
    const long long t0 = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (t0 == 0) {
        buf[0] = buf[1] = buf[3] = 0;
        buf[2] = nb;
    }
    for (long long i = t0; i < nb; i += (long long)gridDim.x * blockDim.x) {
        const int32_t v = B[i], m = M[v];
        const bool known = v <= m || in_range(m, vbase, vbase + nloc);
        buf[4 + 3 * i] = v;
        buf[4 + 3 * i + 1] = m;
        buf[4 + 3 * i + 2] = known ? CM[v] : -1;
    }
}

// pass 1: known CM values; pass 2: CM of a published non-leader = CM of its leader (the
// leader is a boundary vertex of its own rank, so pass 1 delivered it)
__global__ void k_unpack_cm(const int32_t *recv, long long RS, int G, int me, int32_t maxb, int32_t *CM, int pass) {
    const long long tot = (long long)G * maxb;
    for (long long idx = (long long)blockIdx.x * blockDim.x + threadIdx.x; idx < tot;
         idx += (long long)gridDim.x * blockDim.x) {
        const int s = (int)(idx / maxb);
        const int32_t i = (int32_t)(idx % maxb);
        if (s == me) continue;
        const int32_t *rb = recv + (size_t)s * RS;
        if (i >= rb[2]) continue;
        const int32_t v = rb[4 + 3 * i], m = rb[4 + 3 * i + 1], c = rb[4 + 3 * i + 2];
        if (pass == 1 && c >= 0) CM[v] = c;
        if (pass == 2 && c < 0) CM[v] = CM[m];
    }
}

// local non-leaders whose leader is remote copy the leader's CM (delivered by the exchange)
__global__ void k_dc_cm_remote(const int32_t *M, int32_t nloc, int32_t vbase, int32_t *CM) {
    for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < nloc; r += (long long)gridDim.x * blockDim.x) {
        const int32_t u = vbase + (int32_t)r, m = M[u];
        if (u > m && !in_range(m, vbase, vbase + nloc)) CM[u] = CM[m];
    }
}

// ship rows: to destination d go records {leader, deg, vwgt, arc offset} at soff_rec[d] and
// arcs {x, w, CM[x]} at soff_arc[d]; cursors cur[d] (records) and cur[G + d] (arcs)
__global__ void k_ship_pack(const int32_t *M, const int32_t *adjp, const int32_t *adjncy, const int32_t *adjwgt,
                            const int32_t *vwgt, const int32_t *CM, int32_t nloc, int32_t vbase, const int32_t *ranges,
                            int G, const long long *soff_rec, const long long *soff_arc, int32_t *cur, int32_t *buf) {
    for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < nloc; r += (long long)gridDim.x * blockDim.x) {
        const int32_t u = vbase + (int32_t)r, m = M[u];
        if (!(u > m && !in_range(m, vbase, vbase + nloc))) continue;
        const int d = owner_of(m, ranges, G);
        const int32_t s = adjp[r], deg = adjp[r + 1] - s;
        const int32_t slot = atomicAdd(&cur[d], 1);
        const int32_t ao = atomicAdd(&cur[G + d], deg);
        int32_t *rec = buf + soff_rec[d] + 4LL * slot;
        rec[0] = m;
        rec[1] = deg;
        rec[2] = vwgt[r];
        rec[3] = ao;
        int32_t *arc = buf + soff_arc[d] + 3LL * ao;
        for (int32_t j = 0; j < deg; ++j) {
            const int32_t x = adjncy[s + j];
            arc[3 * j] = x;
            arc[3 * j + 1] = adjwgt[s + j];
            arc[3 * j + 2] = CM[x];
        }
    }
}

// received rows of one source: arcs appended to the extended adjacency at abase, CM of
// their endpoints cached, rowinfo[leader row] = {start, deg, vwgt}
__global__ void k_ship_unpack(const int32_t *rbuf, int32_t nrec, int32_t abase, int32_t vbase, int32_t *ext_adjncy,
                              int32_t *ext_adjwgt, int32_t *CM, int4 *rowinfo) {
    const int32_t *arcs = rbuf + 4LL * nrec;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nrec; i += (long long)gridDim.x * blockDim.x) {
        const int32_t l = rbuf[4 * i], deg = rbuf[4 * i + 1], vw = rbuf[4 * i + 2], ao = rbuf[4 * i + 3];
        rowinfo[l - vbase] = make_int4(abase + ao, deg, vw, 1);
        for (int32_t j = 0; j < deg; ++j) {
            const int32_t x = arcs[3LL * (ao + j)];
            ext_adjncy[abase + ao + j] = x;
            ext_adjwgt[abase + ao + j] = arcs[3LL * (ao + j) + 1];
            CM[x] = arcs[3LL * (ao + j) + 2];
        }
    }
}

// per coarse row c (local leader row r): the two fine segments, the merged-row upper bound
// (P20.s5-8) and the coarse vertex weight (P12.s27)
__global__ void k_dc_seg(const int32_t *M, const int32_t *adjp, const int32_t *vwgt, const int32_t *lead,
                         const int32_t *pos, const int4 *rowinfo, int32_t nloc, int32_t vbase, int4 *seg, int32_t *ub,
                         int32_t *cvwgt) {
    for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < nloc; r += (long long)gridDim.x * blockDim.x) {
        if (!lead[r]) continue;
        const int32_t u = vbase + (int32_t)r, m = M[u], c = pos[r];
        const int32_t su = adjp[r], du = adjp[r + 1] - su;
        int4 sg = make_int4(su, du, 0, 0);
        int32_t vw = vwgt[r];
        if (m != u) {
            if (in_range(m, vbase, vbase + nloc)) {
                const int32_t rm = m - vbase;
                sg.z = adjp[rm];
                sg.w = adjp[rm + 1] - sg.z;
                vw += vwgt[rm];
            } else {
                const int4 ri = rowinfo[r];
                sg.z = ri.x;
                sg.w = ri.y;
                vw += ri.z;
            }
        }
        seg[c] = sg;
        ub[c] = sg.y + sg.w;
        cvwgt[c] = vw;
    }
}

// C2 warp-tile starts and the rows with ub > kWB (merged by C1h); publishes n_coarse/n_huge
__global__ void k_dc_tiles(const int32_t *off, int32_t nc, int32_t tb, int32_t ntiles2, int32_t *tile_start,
                           int32_t *huge, ContractCtl *ctl) {
    const long long t0 = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (t0 == 0) {
        tile_start[0] = 0;
        tile_start[ntiles2] = nc;
        ctl->n_coarse = nc;
    }
    for (long long c = t0; c < nc; c += (long long)gridDim.x * blockDim.x) {
        const int32_t o = off[c], d = off[c + 1] - o;
        for (int32_t t2 = o / tb + 1; t2 <= (o + d) / tb && t2 < ntiles2; ++t2) tile_start[t2] = (int32_t)c + 1;
        if (d > kContractTileBudget) huge[atomicAdd(&ctl->n_huge, 1)] = (int32_t)c;
    }
}

// ---- device-wide exclusive scan (out[n] = total; *total_dst = total if non-null) ---------
constexpr int kScanPT = 8;
constexpr int kScanItems = kDT * kScanPT;

__global__ void k_scan_reduce(const int32_t *in, int32_t n, int32_t *partial) {
    const long long b0 = (long long)blockIdx.x * kScanItems;
    int32_t s = 0;
    for (int q = 0; q < kScanPT; ++q) {
        const long long i = b0 + (long long)threadIdx.x * kScanPT + q;
        if (i < n) s += in[i];
    }
    __shared__ int32_t sm[40];
    int32_t tot;
    block_excl_scan<kDT>(s, sm, tot);
    if (threadIdx.x == 0) partial[blockIdx.x] = tot;
}

__global__ void k_scan_top(int32_t *partial, int32_t nb) {
    __shared__ int32_t sm[40];
    int32_t carry = 0;
    for (int32_t b0 = 0; b0 < nb; b0 += kDT) {
        const int32_t i = b0 + threadIdx.x;
        const int32_t v = i < nb ? partial[i] : 0;
        int32_t tot;
        const int32_t ex = block_excl_scan<kDT>(v, sm, tot);
        if (i < nb) partial[i] = carry + ex;
        carry += tot;
    }
    if (threadIdx.x == 0) partial[nb] = carry;
}

__global__ void k_scan_down(const int32_t *in, int32_t n, const int32_t *partial, int32_t nb, int32_t *out,
                            int32_t *total_dst) {
    const long long b0 = (long long)blockIdx.x * kScanItems;
    int32_t v[kScanPT], s = 0;
    for (int q = 0; q < kScanPT; ++q) {
        const long long i = b0 + (long long)threadIdx.x * kScanPT + q;
        v[q] = i < n ? in[i] : 0;
        s += v[q];
    }
    __shared__ int32_t sm[40];
    int32_t tot;
    int32_t run = partial[blockIdx.x] + block_excl_scan<kDT>(s, sm, tot);
    for (int q = 0; q < kScanPT; ++q) {
        const long long i = b0 + (long long)threadIdx.x * kScanPT + q;
        if (i < n) out[i] = run;
        run += v[q];
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        out[n] = partial[nb];
        if (total_dst) *total_dst = partial[nb];
    }
}

// ---------------------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------------------
#define GP_LAUNCH(...)                                        \
    do {                                                      \
        __VA_ARGS__;                                          \
        ++ctx->launches;                                      \
        cudaError_t e__ = cudaGetLastError();                 \
        if (e__ != cudaSuccess) return cuda_fail(e__, "dist kernel launch"); \
    } while (0)

// stream-ordered buffers released together
struct Arena {
    Ctx *ctx;
    std::vector<void *> ptrs;
    explicit Arena(Ctx *c) : ctx(c) {}
    ~Arena() {
        for (void *p : ptrs) dev_free(ctx, p);
    }
    template <typename T>
    gp_status get(T **p, size_t count) {
        gp_status st = dev_alloc(ctx, (void **)p, sizeof(T) * (count > 0 ? count : 1) + 64);
        if (st == GP_OK) ptrs.push_back((void *)*p);
        return st;
    }
};

static gp_status scan_excl(Ctx *ctx, Arena &ar, const int32_t *in, int32_t n, int32_t *out, int32_t *total_dst) {
    const int32_t nb = (n + kScanItems - 1) / kScanItems;
    int32_t *partial = nullptr;
    gp_status st = ar.get(&partial, (size_t)nb + 1);
    if (st != GP_OK) return st;
    if (nb > 0) GP_LAUNCH(k_scan_reduce<<<nb, kDT, 0, ctx->stream>>>(in, n, partial));
    GP_LAUNCH(k_scan_top<<<1, kDT, 0, ctx->stream>>>(partial, nb));
    GP_LAUNCH(k_scan_down<<<nb > 0 ? nb : 1, kDT, 0, ctx->stream>>>(in, n, partial, nb, out, total_dst));
    return GP_OK;
}

// one rank's shard of a level's input graph
struct Shard {
    int rank = 0;                // global rank
    Graph *g = nullptr;          // rows [vbase, vbase + nloc), global column ids
    bool owned = false;          // a temporary slice made by the loopback splitter
};

static gp_status copy_host(Ctx *ctx, void *dst, const void *src, size_t bytes) {
    GP_CUDA(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, ctx->stream));
    GP_CUDA(cudaStreamSynchronize(ctx->stream));
    return GP_OK;
}

// loopback: split a whole graph into G equal vertex ranges
static gp_status split_graph(Ctx *ctx, const Graph *g, int G, std::vector<Shard> &out) {
    std::vector<int32_t> ranges(G + 1), apos(G + 1);
    for (int i = 0; i <= G; ++i) ranges[i] = (int32_t)((long long)g->n * i / G);
    for (int i = 0; i <= G; ++i) {
        gp_status st = copy_host(ctx, &apos[i], g->adjp + ranges[i], sizeof(int32_t));
        if (st != GP_OK) return st;
    }
    for (int i = 0; i < G; ++i) {
        Graph *s = new Graph();
        s->ctx = ctx;
        s->dist = true;
        s->rank = i;
        s->vbase = ranges[i];
        s->n = ranges[i + 1] - ranges[i];
        s->nnz = apos[i + 1] - apos[i];
        s->n_global = g->n;
        s->nnz_global = g->nnz;
        s->ranges = ranges;
        out.push_back({i, s, true});
        gp_status st = alloc_graph_arrays(ctx, s, s->n, s->nnz, true);
        if (st != GP_OK) return st;
        // local offsets = global offsets - adjp[vbase]: copy, then subtract on the device
        std::vector<int32_t> hp((size_t)s->n + 1);
        st = copy_host(ctx, hp.data(), g->adjp + s->vbase, sizeof(int32_t) * hp.size());
        if (st != GP_OK) return st;
        for (auto &x : hp) x -= apos[i];
        GP_CUDA(cudaMemcpyAsync(s->adjp, hp.data(), sizeof(int32_t) * hp.size(), cudaMemcpyHostToDevice, ctx->stream));
        GP_CUDA(cudaStreamSynchronize(ctx->stream));  // hp leaves scope
        if (s->nnz > 0) {
            GP_CUDA(cudaMemcpyAsync(s->adjncy, g->adjncy + apos[i], sizeof(int32_t) * s->nnz, cudaMemcpyDeviceToDevice,
                                    ctx->stream));
            GP_CUDA(cudaMemcpyAsync(s->adjwgt, g->adjwgt + apos[i], sizeof(int32_t) * s->nnz, cudaMemcpyDeviceToDevice,
                                    ctx->stream));
        }
        if (s->n > 0)
            GP_CUDA(cudaMemcpyAsync(s->vwgt, g->vwgt + s->vbase, sizeof(int32_t) * s->n, cudaMemcpyDeviceToDevice,
                                    ctx->stream));
        SizeRec r{s->n, s->nnz, 0, 0};
        GP_CUDA(cudaMemcpyAsync(s->sizes, &r, sizeof(r), cudaMemcpyHostToDevice, ctx->stream));
        GP_CUDA(cudaStreamSynchronize(ctx->stream));
    }
    return GP_OK;
}

// folding: one rank's piece of the gathered coarse graph -> rows of the full CSR
__global__ void k_fold_adjp(const int32_t *piece_adjp, int32_t rows, int32_t arc_base, int32_t *full_adjp) {
    for (int32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < rows; r += gridDim.x * blockDim.x)
        full_adjp[r] = piece_adjp[r] + arc_base;
}

// Folding (PT-Scotch's folding, P14.s21-23): once the coarse graph has at
// most GP_FOLD_N vertices (default 500 000; 0 = never), every rank gathers it whole and finishes
// the hierarchy on the single-GPU pipeline (tail kernels included) -- redundantly on every
// rank, with no per-round collective.  The results are the 1-GPU results by construction.
static int32_t fold_limit() {
    const char *e = getenv("GP_FOLD_N");  // knob read per call (results never depend on it)
    return e ? atoi(e) : 500000;
}

// per-rank working state of one level
struct RankWork {
    Shard sh;
    int32_t vbase = 0, nloc = 0, nnz = 0;
    int32_t *M = nullptr, *CM = nullptr;  // kept by the hierarchy (global-indexed)
    int32_t *P[2] = {nullptr, nullptr}, *S = nullptr, *L[2] = {nullptr, nullptr}, *H = nullptr;
    int32_t *B = nullptr, *nbp = nullptr;
    int32_t *rs = nullptr, *rr = nullptr;  // record send / receive buffers
    int32_t *ranges = nullptr;             // device copy of the level's rank ranges
    LevelDev *ld = nullptr;
    SizeRec *in = nullptr;
    int32_t nb = 0;
    // contraction
    int32_t *lead = nullptr, *pos = nullptr, *cnt = nullptr;
    int32_t nlead = 0, cbase = 0;
    Graph *coarse = nullptr;
};

static double avg_deg(long long n, long long nnz) { return n > 0 ? (double)nnz / (double)n : 0.0; }

gp_status dist_coarsen_to(Graph *g0, const gp_coarsen_opts *opts, Hier **out) {
    Ctx *ctx = g0->ctx;
    DistComm *comm = ctx->comm;
    const int G = comm->nranks;
    const int NL = comm->nlocal();
    const int32_t pct = opts->stall_ratio_pct ? opts->stall_ratio_pct : 95;
    const int32_t max_levels = opts->max_levels ? opts->max_levels : 64;
    Hier *h = new Hier();
    h->ctx = ctx;
    h->counted = true;
    ++ctx->live_objects;
    *out = nullptr;
    std::vector<Shard> shards;
    gp_status st = GP_OK;
    if (comm->loopback()) {
        if (g0->dist) {
            set_error("gp_coarsen_to: a loopback context shards a whole graph itself");
            delete h;
            return GP_ERR_INVALID_ARG;
        }
        st = split_graph(ctx, g0, G, shards);
    } else {
        if (!g0->dist || g0->rank != comm->rank) {
            set_error("gp_coarsen_to: an NCCL context needs this rank's shard (gp_graph_create_dist)");
            delete h;
            return GP_ERR_INVALID_ARG;
        }
        shards.push_back({comm->rank, g0, false});
    }
    auto release_shards = [&]() {
        for (auto &s : shards)
            if (s.owned) graph_release(s.g);
        shards.clear();
    };
    if (st != GP_OK) {
        release_shards();
        delete h;
        return st;
    }
    int32_t N = g0->dist ? g0->n_global : g0->n;
    long long NNZ = g0->dist ? g0->nnz_global : g0->nnz;
    std::vector<int32_t> ranges = shards[0].g->ranges;
    int32_t *pin = ctx->pinned;  // 4096 B: headers / counts (pinned, synchronous use)

    std::vector<RankWork> W;
    // results of one level (set by run_level)
    int32_t rounds = 0, maximal = 0, NC = 0;
    int32_t prev_rounds = 7;  // round count of the previous level (first batch size of the next)
    long long CNNZ = 0;
    int64_t stat_arcs = 0, stat_rows = 0, stat_visits = 0;
    std::vector<int32_t> cranges;
    // one level; GP_CUDA / GP_LAUNCH return from this lambda, the caller releases W on error
    auto run_level = [&](int level, Arena &ar) -> gp_status {
        gp_status st = GP_OK;
        // ---- allocations -------------------------------------------------------------
        for (int i = 0; i < NL && st == GP_OK; ++i) {
            RankWork &w = W[i];
            w.sh = shards[i];
            w.vbase = w.sh.g->vbase;
            w.nloc = w.sh.g->n;
            w.nnz = w.sh.g->nnz;
            st = dev_alloc(ctx, (void **)&w.M, sizeof(int32_t) * ((size_t)N + 1));
            if (st == GP_OK) st = dev_alloc(ctx, (void **)&w.CM, sizeof(int32_t) * ((size_t)N + 1));
            if (st != GP_OK) break;
            st = ar.get(&w.P[0], N);
            if (st == GP_OK) st = ar.get(&w.P[1], N);
            if (st == GP_OK) st = ar.get(&w.S, N);
            if (st == GP_OK) st = ar.get(&w.L[0], w.nloc);
            if (st == GP_OK) st = ar.get(&w.L[1], w.nloc);
            if (st == GP_OK) st = ar.get(&w.H, w.nloc);
            if (st == GP_OK) st = ar.get(&w.B, w.nloc);
            if (st == GP_OK) st = ar.get(&w.nbp, 4);
            if (st == GP_OK) st = ar.get(&w.ranges, G + 1);
            if (st == GP_OK) st = ar.get(&w.ld, 1);
            if (st == GP_OK) st = ar.get(&w.in, 1);
            if (st == GP_OK) st = ar.get(&w.lead, (size_t)w.nloc + 1);
            if (st == GP_OK) st = ar.get(&w.pos, (size_t)w.nloc + 1);
            if (st == GP_OK) st = ar.get(&w.cnt, 1 + 2 * (size_t)G);
            if (st != GP_OK) break;
            GP_CUDA(cudaMemsetAsync(w.ld, 0, sizeof(LevelDev), ctx->stream));
            GP_CUDA(cudaMemsetAsync(w.nbp, 0, 16, ctx->stream));
            GP_CUDA(cudaMemsetAsync(w.cnt, 0, sizeof(int32_t) * (1 + 2 * (size_t)G), ctx->stream));
            GP_CUDA(cudaMemcpyAsync(w.ranges, ranges.data(), sizeof(int32_t) * (G + 1), cudaMemcpyHostToDevice, ctx->stream));
            SizeRec r{w.nloc, w.nnz, 0, 0};
            GP_CUDA(cudaMemcpyAsync(w.in, &r, sizeof(r), cudaMemcpyHostToDevice, ctx->stream));
            GP_CUDA(cudaStreamSynchronize(ctx->stream));  // r leaves scope
            // boundary list of this level
            if (w.nloc > 0)
                GP_LAUNCH(k_boundary<<<grid_for(w.nloc), kDT, 0, ctx->stream>>>(w.sh.g->adjp, w.sh.g->adjncy, w.nloc,
                                                                               w.vbase, w.B, w.nbp));
        }
        if (st != GP_OK) return st;
        // record buffers sized by the largest boundary of any rank
        int32_t maxb = 0;
        {
            std::vector<int32_t> nbs(G, 0);
            for (int i = 0; i < NL; ++i) {
                GP_CUDA(cudaMemcpyAsync(pin + i, W[i].nbp, sizeof(int32_t), cudaMemcpyDeviceToHost, ctx->stream));
            }
            GP_CUDA(cudaStreamSynchronize(ctx->stream));
            if (comm->loopback()) {
                for (int i = 0; i < NL; ++i) nbs[i] = pin[i];
            } else {
                int32_t mine = pin[0];
                st = dist_allgather_i32(ctx, &mine, 1, nbs.data());
                if (st != GP_OK) return st;
            }
            for (int i = 0; i < NL; ++i) W[i].nb = comm->loopback() ? nbs[i] : nbs[comm->rank];
            maxb = *std::max_element(nbs.begin(), nbs.end());
        }
        const long long RS = 4 + 3LL * maxb;  // ints per rank in a record all-gather
        for (int i = 0; i < NL && st == GP_OK; ++i) {
            st = ar.get(&W[i].rs, (size_t)RS);
            if (st == GP_OK) st = ar.get(&W[i].rr, (size_t)RS * G);
        }
        if (st != GP_OK) return st;
        std::vector<int32_t *> vs(NL), vr(NL);
        for (int i = 0; i < NL; ++i) {
            vs[i] = W[i].rs;
            vr[i] = W[i].rr;
        }
        auto bufs_of = [&](RankWork &w) {
            LevelBufs b{};
            b.in = w.in;
            b.adjp = w.sh.g->adjp;
            b.adjncy = w.sh.g->adjncy;
            b.adjwgt = w.sh.g->adjwgt;
            b.vwgt = w.sh.g->vwgt;
            b.P[0] = w.P[0];
            b.P[1] = w.P[1];
            b.L[0] = w.L[0];
            b.L[1] = w.L[1];
            b.H = w.H;
            b.S = w.S;
            return b;
        };
        auto unpack_match = [&](int parity) -> gp_status {
            for (int i = 0; i < NL; ++i)
                GP_LAUNCH(k_unpack_match<<<grid_for((long long)G * maxb), kDT, 0, ctx->stream>>>(
                    W[i].rr, RS, G, comm->grank(i), maxb, W[i].P[parity]));
            return GP_OK;
        };
        const double ad = avg_deg(N, NNZ);
        // ---- matching: phase 0, then one launch + one exchange per round ----------------
        for (int i = 0; i < NL && st == GP_OK; ++i) {
            RankWork &w = W[i];
            st = enqueue_match(ctx, bufs_of(w), w.M, &w.ld->match, opts->max_rounds, true, ad, w.vbase, kMatchPhase0);
            if (st == GP_OK)
                GP_LAUNCH(k_pack_match<<<grid_for(w.nb), kDT, 0, ctx->stream>>>(w.B, w.nb, w.P[1], w.vbase, w.nloc,
                                                                                nullptr, w.nloc, nullptr, w.rs));
        }
        if (st == GP_OK) st = allgather(ctx, vs, vr, (size_t)RS);
        if (st == GP_OK) st = unpack_match(1);
        rounds = 0;
        maximal = 0;
        // Rounds are enqueued in batches with ONE host synchronisation per batch: after the
        // fixpoint a round is a no-op (empty live lists, unchanged boundary records), so the
        // rounds of a batch beyond the last live one change nothing; every round's gathered
        // header {live, made} is copied to its own pinned slot and the batch is evaluated in
        // order (rounds that made a match are counted, R4).  With a max_rounds cap the batch
        // is 1 (a round past the cap would change the result).  The batch grows geometrically
        // from the previous level's round count.
        int batch = opts->max_rounds > 0 ? 1 : std::max(2, std::min(16, prev_rounds + 1));
        bool done = false;
        for (int k = 1; st == GP_OK && !done;) {
            if (k > N + 2) {
                set_error("dist: round loop did not terminate (protocol bug)");
                st = GP_ERR_INTERNAL;
                break;
            }
            const int kb = std::max(1, std::min(batch, 1024 / (2 * G)));  // header slots in the 4 KiB pinned buffer
            for (int b = 0; b < kb && st == GP_OK; ++b) {
                const int kk = k + b;
                for (int i = 0; i < NL && st == GP_OK; ++i) {
                    RankWork &w = W[i];
                    GP_CUDA(cudaMemsetAsync(w.ld->match.bar, 0, sizeof(w.ld->match.bar), ctx->stream));
                    st = enqueue_match(ctx, bufs_of(w), w.M, &w.ld->match, opts->max_rounds, true, ad, w.vbase,
                                       kMatchRound, kk);
                    if (st == GP_OK)
                        GP_LAUNCH(k_pack_match<<<grid_for(w.nb), kDT, 0, ctx->stream>>>(
                            w.B, w.nb, w.P[(kk + 1) & 1], w.vbase, w.nloc, &w.ld->match.slot[(kk + 1) & 3].live, 0,
                            &w.ld->match.slot[kk & 3].matches, w.rs));
                }
                if (st == GP_OK) st = allgather(ctx, vs, vr, (size_t)RS);
                if (st == GP_OK) st = unpack_match((kk + 1) & 1);
                // every rank's header {live, made} of round kk (all in the first local receive buffer)
                if (st == GP_OK)
                    GP_CUDA(cudaMemcpy2DAsync(pin + (size_t)b * 2 * G, 2 * sizeof(int32_t), W[0].rr, RS * sizeof(int32_t),
                                              2 * sizeof(int32_t), G, cudaMemcpyDeviceToHost, ctx->stream));
            }
            if (st != GP_OK) break;
            GP_CUDA(cudaStreamSynchronize(ctx->stream));
            for (int b = 0; b < kb && !done; ++b) {
                long long live = 0;
                bool made = false;
                for (int s = 0; s < G; ++s) {
                    live += pin[(size_t)b * 2 * G + 2 * s];
                    made = made || pin[(size_t)b * 2 * G + 2 * s + 1] != 0;
                }
                if (made) ++rounds;
                if (live == 0) {
                    maximal = 1;
                    done = true;
                } else if (opts->max_rounds > 0 && rounds >= opts->max_rounds) {
                    done = true;
                }
            }
            k += kb;
            if (opts->max_rounds == 0) batch = std::min(2 * batch, 64);
        }
        prev_rounds = rounds;
        for (int i = 0; i < NL && st == GP_OK; ++i)  // leftover pass (P18.s12-13)
            st = enqueue_match(ctx, bufs_of(W[i]), W[i].M, &W[i].ld->match, opts->max_rounds, true, ad, W[i].vbase,
                               kMatchFinish);
        if (st != GP_OK) return st;
        // ---- contraction ---------------------------------------------------------------
        // (1) leader flags, local scan, counts of rows / arcs to ship per destination
        const int CW = 1 + 2 * G;
        std::vector<int32_t *> cs(NL), cr(NL);
        for (int i = 0; i < NL && st == GP_OK; ++i) {
            RankWork &w = W[i];
            if (w.nloc > 0)
                GP_LAUNCH(k_dc_flags<<<grid_for(w.nloc), kDT, 0, ctx->stream>>>(w.M, w.sh.g->adjp, w.nloc, w.vbase,
                                                                               w.ranges, G, w.lead, w.cnt));
            st = scan_excl(ctx, ar, w.lead, w.nloc, w.pos, w.cnt);
            cs[i] = w.cnt;
            if (st == GP_OK) st = ar.get(&cr[i], (size_t)CW * G);
        }
        if (st == GP_OK) st = allgather(ctx, cs, cr, (size_t)CW);
        std::vector<int32_t> counts((size_t)CW * G);
        if (st == GP_OK) {
            cudaError_t e = cudaMemcpyAsync(counts.data(), cr[0], sizeof(int32_t) * counts.size(), cudaMemcpyDeviceToHost,
                                            ctx->stream);
            if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
            if (e != cudaSuccess) st = cuda_fail(e, "dist counts");
        }
        if (st != GP_OK) return st;
        std::vector<int32_t> nlead(G);
        cranges.assign(G + 1, 0);
        Mat shipv(G, std::vector<long long>(G)), shipa(G, std::vector<long long>(G));
        for (int s = 0; s < G; ++s) {
            nlead[s] = counts[(size_t)s * CW];
            for (int d = 0; d < G; ++d) {
                shipv[s][d] = counts[(size_t)s * CW + 1 + d];
                shipa[s][d] = counts[(size_t)s * CW + 1 + G + d];
            }
            cranges[s + 1] = cranges[s] + nlead[s];  // rank offsets of the coarse ids
        }
        NC = cranges[G];
        // (2) CM of local leaders, boundary CM exchange, CM of non-leaders with remote leaders
        for (int i = 0; i < NL && st == GP_OK; ++i) {
            RankWork &w = W[i];
            const int r = comm->grank(i);
            w.nlead = nlead[r];
            w.cbase = cranges[r];
            if (w.nloc > 0)
                GP_LAUNCH(k_dc_cm<<<grid_for(w.nloc), kDT, 0, ctx->stream>>>(w.M, w.lead, w.pos, w.nloc, w.vbase,
                                                                            w.cbase, w.CM));
            GP_LAUNCH(k_pack_cm<<<grid_for(w.nb), kDT, 0, ctx->stream>>>(w.B, w.nb, w.M, w.CM, w.vbase, w.nloc, w.rs));
        }
        if (st == GP_OK) st = allgather(ctx, vs, vr, (size_t)RS);
        for (int pass = 1; pass <= 2 && st == GP_OK; ++pass)
            for (int i = 0; i < NL; ++i)
                GP_LAUNCH(k_unpack_cm<<<grid_for((long long)G * maxb), kDT, 0, ctx->stream>>>(
                    W[i].rr, RS, G, comm->grank(i), maxb, W[i].CM, pass));
        for (int i = 0; i < NL && st == GP_OK; ++i)
            if (W[i].nloc > 0)
                GP_LAUNCH(k_dc_cm_remote<<<grid_for(W[i].nloc), kDT, 0, ctx->stream>>>(W[i].M, W[i].nloc, W[i].vbase,
                                                                                      W[i].CM));
        // (3) ship the rows of non-leaders to their leader's rank
        Mat scount(G, std::vector<long long>(G, 0)), soff = scount, rcount = scount, roff = scount;
        for (int s = 0; s < G; ++s) {
            long long o = 0;
            for (int d = 0; d < G; ++d) {
                scount[s][d] = 4 * shipv[s][d] + 3 * shipa[s][d];
                soff[s][d] = o;
                o += scount[s][d];
            }
        }
        for (int d = 0; d < G; ++d) {
            long long o = 0;
            for (int s = 0; s < G; ++s) {
                rcount[d][s] = scount[s][d];
                roff[d][s] = o;
                o += rcount[d][s];
            }
        }
        std::vector<int32_t *> ss(NL), sr(NL);
        std::vector<int32_t *> ext_adj(NL), ext_wgt(NL);
        std::vector<int4 *> rowinfo(NL);
        std::vector<long long> nnz_ub(NL);
        for (int i = 0; i < NL && st == GP_OK; ++i) {
            RankWork &w = W[i];
            const int r = comm->grank(i);
            long long stot = 0, rtot = 0, rarcs = 0, sarcs = 0;
            for (int d = 0; d < G; ++d) {
                stot += scount[r][d];
                rtot += rcount[r][d];
                rarcs += shipa[d][r];
                sarcs += shipa[r][d];
            }
            nnz_ub[i] = (long long)w.nnz - sarcs + rarcs;
            st = ar.get(&ss[i], (size_t)stot);
            if (st == GP_OK) st = ar.get(&sr[i], (size_t)rtot);
            if (st == GP_OK) st = ar.get(&ext_adj[i], (size_t)(w.nnz + rarcs) + 4);
            if (st == GP_OK) st = ar.get(&ext_wgt[i], (size_t)(w.nnz + rarcs) + 4);
            if (st == GP_OK) st = ar.get(&rowinfo[i], (size_t)w.nloc);
            if (st != GP_OK) break;
            if (stot > 0) {
                std::vector<long long> hrec(G), harc(G);
                for (int d = 0; d < G; ++d) {
                    hrec[d] = soff[r][d];
                    harc[d] = soff[r][d] + 4 * shipv[r][d];
                }
                long long *drec = nullptr;
                int32_t *cur = nullptr;
                st = ar.get(&drec, 2 * (size_t)G);
                if (st == GP_OK) st = ar.get(&cur, 2 * (size_t)G);
                if (st != GP_OK) break;
                memcpy(pin, hrec.data(), sizeof(long long) * G);
                memcpy(pin + 2 * G, harc.data(), sizeof(long long) * G);
                GP_CUDA(cudaMemcpyAsync(drec, pin, sizeof(long long) * 2 * G, cudaMemcpyHostToDevice, ctx->stream));
                GP_CUDA(cudaMemsetAsync(cur, 0, sizeof(int32_t) * 2 * G, ctx->stream));
                GP_LAUNCH(k_ship_pack<<<grid_for(w.nloc), kDT, 0, ctx->stream>>>(
                    w.M, w.sh.g->adjp, w.sh.g->adjncy, w.sh.g->adjwgt, w.sh.g->vwgt, w.CM, w.nloc, w.vbase, w.ranges, G,
                    drec, drec + G, cur, ss[i]));
                GP_CUDA(cudaStreamSynchronize(ctx->stream));  // pin is reused
            }
            if (w.nnz > 0) {
                GP_CUDA(cudaMemcpyAsync(ext_adj[i], w.sh.g->adjncy, sizeof(int32_t) * w.nnz, cudaMemcpyDeviceToDevice,
                                        ctx->stream));
                GP_CUDA(cudaMemcpyAsync(ext_wgt[i], w.sh.g->adjwgt, sizeof(int32_t) * w.nnz, cudaMemcpyDeviceToDevice,
                                        ctx->stream));
            }
        }
        if (st == GP_OK) st = exchange(ctx, ss, scount, soff, sr, rcount, roff);
        for (int i = 0; i < NL && st == GP_OK; ++i) {
            RankWork &w = W[i];
            const int r = comm->grank(i);
            long long abase = w.nnz;
            for (int s = 0; s < G; ++s) {
                if (shipv[s][r] > 0)
                    GP_LAUNCH(k_ship_unpack<<<grid_for(shipv[s][r]), kDT, 0, ctx->stream>>>(
                        sr[i] + roff[r][s], (int32_t)shipv[s][r], (int32_t)abase, w.vbase, ext_adj[i], ext_wgt[i], w.CM,
                        rowinfo[i]));
                abase += shipa[s][r];
            }
        }
        // (4) contraction inputs + the persistent contraction kernel in sharded mode
        std::vector<int32_t> cnnz_loc(NL, 0);
        for (int i = 0; i < NL && st == GP_OK; ++i) {
            RankWork &w = W[i];
            const int32_t nc = w.nlead;
            const int32_t ubn = (int32_t)nnz_ub[i];
            int4 *seg = nullptr;
            int32_t *ub = nullptr, *off = nullptr, *cntv = nullptr, *tstart = nullptr, *huge = nullptr, *lofs = nullptr,
                    *ttot = nullptr;
            unsigned long long *gkeys = nullptr, *tout = nullptr;
            int32_t tb = kContractTileBudget;
            while (tb > 32 && (long long)ubn < 4LL * tb * contract_grid(ctx, w.nloc) * 8) tb >>= 1;
            const int32_t ntiles2 = ubn > 0 ? (ubn + tb - 1) / tb : 0;
            st = ar.get(&seg, nc);
            if (st == GP_OK) st = ar.get(&ub, (size_t)nc + 1);
            if (st == GP_OK) st = ar.get(&off, (size_t)nc + 1);
            if (st == GP_OK) st = ar.get(&cntv, nc);
            if (st == GP_OK) st = ar.get(&tstart, (size_t)ntiles2 + 2);
            if (st == GP_OK) st = ar.get(&huge, nc);
            if (st == GP_OK) st = ar.get(&lofs, nc);
            if (st == GP_OK) st = ar.get(&ttot, (size_t)ntiles2 + 1);
            if (st == GP_OK) st = ar.get(&gkeys, (size_t)ubn + 4);
            if (st == GP_OK) st = ar.get(&tout, (size_t)ubn + 4);
            if (st != GP_OK) break;
            Graph *cg = new Graph();
            cg->ctx = ctx;
            cg->borrowed = true;
            cg->dist = true;
            cg->rank = comm->grank(i);
            cg->vbase = w.cbase;
            cg->n = nc;
            cg->n_global = NC;
            cg->ranges = cranges;
            w.coarse = cg;
            st = alloc_graph_arrays(ctx, cg, nc, ubn, true);
            if (st != GP_OK) break;
            if (w.nloc > 0)
                GP_LAUNCH(k_dc_seg<<<grid_for(w.nloc), kDT, 0, ctx->stream>>>(w.M, w.sh.g->adjp, w.sh.g->vwgt, w.lead,
                                                                             w.pos, rowinfo[i], w.nloc, w.vbase, seg, ub,
                                                                             cg->vwgt));
            st = scan_excl(ctx, ar, ub, nc, off, nullptr);
            if (st != GP_OK) break;
            GP_LAUNCH(k_dc_tiles<<<grid_for(nc), kDT, 0, ctx->stream>>>(off, nc, tb, ntiles2, tstart, huge,
                                                                        &w.ld->contract));
            if (nc > 0) {
                LevelBufs b = bufs_of(w);
                b.adjncy = ext_adj[i];
                b.adjwgt = ext_wgt[i];
                b.off = off;
                b.cnt = cntv;
                b.tile_start = tstart;
                b.huge = huge;
                b.lofs = lofs;
                b.ttot = ttot;
                b.tagg1 = ttot;  // unused in sharded mode
                b.seg = seg;
                b.gkeys = gkeys;
                b.tout = tout;
                ContractParams prm{false, opts->threshold, pct, level, max_levels, w.nloc, ubn};
                prm.dist = 1;
                prm.cbase = w.cbase;
                prm.tb = tb;
                prm.nnz_ub = ubn;
                st = enqueue_contract(ctx, b, w.M, w.CM, cg, &w.ld->contract, &w.ld->out, nullptr, prm);
                if (st != GP_OK) break;
                GP_CUDA(cudaMemcpyAsync(pin, &w.ld->out, sizeof(SizeRec), cudaMemcpyDeviceToHost, ctx->stream));
                GP_CUDA(cudaStreamSynchronize(ctx->stream));
                cnnz_loc[i] = pin[1];
            } else {
                GP_CUDA(cudaMemsetAsync(cg->adjp, 0, sizeof(int32_t), ctx->stream));
            }
            cg->nnz = cnnz_loc[i];
            SizeRec rr{cg->n, cg->nnz, 0, 0};
            GP_CUDA(cudaMemcpyAsync(cg->sizes, &rr, sizeof(rr), cudaMemcpyHostToDevice, ctx->stream));
            GP_CUDA(cudaStreamSynchronize(ctx->stream));
        }
        // global coarse arc count
        CNNZ = 0;
        if (st == GP_OK) {
            if (comm->loopback()) {
                for (int i = 0; i < NL; ++i) CNNZ += cnnz_loc[i];
            } else {
                std::vector<int32_t> all(G);
                st = dist_allgather_i32(ctx, &cnnz_loc[0], 1, all.data());
                for (int s = 0; s < G; ++s) CNNZ += all[s];
            }
        }
        // statistics of the matching (this process's ranks)
        stat_arcs = stat_rows = stat_visits = 0;
        for (int i = 0; i < NL && st == GP_OK; ++i) {
            MatchCtl mc;
            GP_CUDA(cudaMemcpyAsync(&mc, &W[i].ld->match, sizeof(mc), cudaMemcpyDeviceToHost, ctx->stream));
            GP_CUDA(cudaStreamSynchronize(ctx->stream));
            stat_arcs += (int64_t)mc.arcs_scanned;
            stat_rows += (int64_t)mc.rows_scanned + W[i].nloc;
            stat_visits += (int64_t)mc.live_visits;
        }
        return st;
    };

    // gather the (small) coarse graph onto every rank and finish on the single-GPU pipeline
    auto fold = [&](int levels_done) -> gp_status {
        std::vector<long long> rows(G), arcs(G), abase(G + 1, 0);
        for (int r = 0; r < G; ++r) rows[r] = ranges[r + 1] - ranges[r];
        if (comm->loopback()) {
            for (int i = 0; i < NL; ++i) arcs[i] = shards[i].g->nnz;
        } else {
            int32_t mine = shards[0].g->nnz;
            std::vector<int32_t> all(G);
            gp_status s2 = dist_allgather_i32(ctx, &mine, 1, all.data());
            if (s2 != GP_OK) return s2;
            for (int r = 0; r < G; ++r) arcs[r] = all[r];
        }
        long long maxr = 0, maxa = 0;
        for (int r = 0; r < G; ++r) {
            maxr = std::max(maxr, rows[r]);
            maxa = std::max(maxa, arcs[r]);
            abase[r + 1] = abase[r] + arcs[r];
        }
        const long long PS = (maxr + 4) + (maxr + 4) + 2 * (maxa + 4);  // adjp | vwgt | adjncy | adjwgt
        const long long oV = maxr + 4, oA = 2 * (maxr + 4), oW = oA + maxa + 4;
        Arena ar(ctx);
        std::vector<int32_t *> vs(NL), vr(NL);
        for (int i = 0; i < NL; ++i) {
            gp_status s2 = ar.get(&vs[i], (size_t)PS);
            if (s2 == GP_OK) s2 = ar.get(&vr[i], (size_t)PS * G);
            if (s2 != GP_OK) return s2;
            const Graph *sg = shards[i].g;
            GP_CUDA(cudaMemcpyAsync(vs[i], sg->adjp, sizeof(int32_t) * ((size_t)sg->n + 1), cudaMemcpyDeviceToDevice,
                                    ctx->stream));
            if (sg->n > 0)
                GP_CUDA(cudaMemcpyAsync(vs[i] + oV, sg->vwgt, sizeof(int32_t) * (size_t)sg->n, cudaMemcpyDeviceToDevice,
                                        ctx->stream));
            if (sg->nnz > 0) {
                GP_CUDA(cudaMemcpyAsync(vs[i] + oA, sg->adjncy, sizeof(int32_t) * (size_t)sg->nnz,
                                        cudaMemcpyDeviceToDevice, ctx->stream));
                GP_CUDA(cudaMemcpyAsync(vs[i] + oW, sg->adjwgt, sizeof(int32_t) * (size_t)sg->nnz,
                                        cudaMemcpyDeviceToDevice, ctx->stream));
            }
        }
        gp_status s2 = allgather(ctx, vs, vr, (size_t)PS);
        if (s2 != GP_OK) return s2;
        // the whole coarse graph on this process (every local rank would hold the same bytes)
        Graph *fg = new Graph();
        fg->ctx = ctx;
        fg->n = N;
        fg->nnz = (int32_t)NNZ;
        s2 = alloc_graph_arrays(ctx, fg, N, (int32_t)NNZ, true);
        for (int r = 0; s2 == GP_OK && r < G; ++r) {
            const int32_t *pc = vr[0] + (size_t)r * PS;
            if (rows[r] > 0) {
                GP_LAUNCH(k_fold_adjp<<<grid_for(rows[r]), kDT, 0, ctx->stream>>>(pc, (int32_t)rows[r], (int32_t)abase[r],
                                                                                 fg->adjp + ranges[r]));
                GP_CUDA(cudaMemcpyAsync(fg->vwgt + ranges[r], pc + oV, sizeof(int32_t) * (size_t)rows[r],
                                        cudaMemcpyDeviceToDevice, ctx->stream));
            }
            if (arcs[r] > 0) {
                GP_CUDA(cudaMemcpyAsync(fg->adjncy + abase[r], pc + oA, sizeof(int32_t) * (size_t)arcs[r],
                                        cudaMemcpyDeviceToDevice, ctx->stream));
                GP_CUDA(cudaMemcpyAsync(fg->adjwgt + abase[r], pc + oW, sizeof(int32_t) * (size_t)arcs[r],
                                        cudaMemcpyDeviceToDevice, ctx->stream));
            }
        }
        const int32_t tail_words[2] = {(int32_t)NNZ, 0};
        const SizeRec rec{N, (int32_t)NNZ, 0, 0};
        if (s2 == GP_OK) {
            GP_CUDA(cudaMemcpyAsync(fg->adjp + N, tail_words, sizeof(int32_t), cudaMemcpyHostToDevice, ctx->stream));
            GP_CUDA(cudaMemcpyAsync(fg->sizes, &rec, sizeof(rec), cudaMemcpyHostToDevice, ctx->stream));
            GP_CUDA(cudaStreamSynchronize(ctx->stream));  // host words leave scope; the arena is freed
        }
        Hier *sub = nullptr;
        gp_coarsen_opts o2 = *opts;
        o2.max_levels = max_levels - levels_done;
        o2.stall_ratio_pct = pct;
        if (s2 == GP_OK) s2 = coarsen_single(fg, &o2, &sub);
        cudaStreamSynchronize(ctx->stream);
        graph_release(fg);
        if (s2 != GP_OK) return s2;
        h->subs.push_back(sub);
        // the folded levels, as sharded levels whose piece on rank 0 is the whole level
        for (const Level &ls : sub->levels) {
            Level L;
            L.n = ls.n;
            L.nnz = ls.nnz;
            L.n_coarse = ls.n_coarse;
            L.cnnz = ls.cnnz;
            L.rounds = ls.rounds;
            L.maximal = ls.maximal;
            L.stop_reason = ls.stop_reason;
            L.arcs_scanned = ls.arcs_scanned;
            L.rows_scanned = ls.rows_scanned;
            L.live_visits = ls.live_visits;
            L.borrowed = true;
            for (int i = 0; i < NL; ++i) {
                DistPiece p;
                p.rank = comm->grank(i);
                if (p.rank == 0) {
                    p.vbase = 0;
                    p.nloc = ls.n;
                    p.M = ls.match;
                    p.CM = ls.cmap;
                    p.coarse = ls.coarse;
                } else {  // an empty piece (zero rows, adjp = {0})
                    Graph *eg = new Graph();
                    eg->ctx = ctx;
                    h->extra.push_back(eg);
                    gp_status s3 = alloc_graph_arrays(ctx, eg, 0, 0, true);
                    if (s3 != GP_OK) return s3;
                    GP_CUDA(cudaMemsetAsync(eg->adjp, 0, sizeof(int32_t), ctx->stream));
                    eg->vbase = ls.n_coarse;
                    p.vbase = ls.n;  // M + vbase: one past the end of the level's arrays
                    p.nloc = 0;
                    p.M = ls.match;
                    p.CM = ls.cmap;
                    p.coarse = eg;
                }
                L.pieces.push_back(p);
            }
            h->levels.push_back(L);
        }
        return GP_OK;
    };

    for (int level = 0; st == GP_OK && N > opts->threshold && level < max_levels; ++level) {
        W.assign(NL, RankWork());
        {
            Arena ar(ctx);
            st = run_level(level, ar);
        }
        // hierarchy level (pieces own M, CM and the coarse shard; released with h even when
        // the level failed half way)
        Level L;
        L.n = N;
        L.nnz = (int32_t)NNZ;
        L.n_coarse = NC;
        L.cnnz = (int32_t)CNNZ;
        L.rounds = rounds;
        L.maximal = maximal;
        for (int i = 0; i < NL; ++i) {
            DistPiece p;
            p.rank = comm->grank(i);
            p.vbase = W[i].vbase;
            p.nloc = W[i].nloc;
            p.M = W[i].M;
            p.CM = W[i].CM;
            p.coarse = W[i].coarse;
            if (p.coarse) p.coarse->nnz_global = (int32_t)CNNZ;
            L.pieces.push_back(p);
        }
        L.arcs_scanned = stat_arcs;
        L.rows_scanned = stat_rows;
        L.live_visits = stat_visits;
        // stop rule (P12.s30, P20.s30; R12, R13) on the global sizes
        int32_t reason = GP_STOP_NONE;
        if (100LL * NC > (long long)pct * N) reason = GP_STOP_STALL;
        else if (NC <= opts->threshold) reason = GP_STOP_THRESHOLD;
        else if (level + 1 >= max_levels) reason = GP_STOP_MAX_LEVELS;
        L.stop_reason = reason;
        h->levels.push_back(L);
        if (st != GP_OK) break;
        // the coarse shards are the next level's input
        release_shards();
        for (int i = 0; i < NL; ++i) shards.push_back({comm->grank(i), W[i].coarse, false});
        N = NC;
        NNZ = CNNZ;
        ranges = cranges;
        if (reason != GP_STOP_NONE) break;
        if (N <= fold_limit() && level + 1 < max_levels) {
            st = fold(level + 1);
            break;
        }
    }
    release_shards();
    if (st != GP_OK) {
        cudaStreamSynchronize(ctx->stream);
        hier_release(h);
        return st;
    }
    cudaError_t e = cudaStreamSynchronize(ctx->stream);
    if (e != cudaSuccess) {
        hier_release(h);
        return cuda_fail(e, "dist_coarsen_to");
    }
    *out = h;
    return GP_OK;
}

}  // namespace gp
