// validate.cu -- weight totals (R14) and the GP_VALIDATE input contract (R15) on the device.
#include <cuda_runtime.h>

#include <cstring>
#include <string>

#include "device_util.cuh"
#include "gp_internal.cuh"

namespace gp {

struct ValidateOut {
    unsigned long long sum_adjwgt, sum_vwgt;
    unsigned long long fp_fwd, fp_rev;  // arc fingerprints (unused since the exact hash check)
    int32_t first_bad;                  // smallest offending vertex (INT32_MAX = none)
    int32_t bad_mask;                   // which checks failed
    int32_t unsorted;                   // some row is not strictly increasing
    int32_t pad;
};

enum : int32_t {
    kBadOffsets = 1,
    kBadRange = 2,
    kBadSelfLoop = 4,
    kBadWeight = 8,
    kBadVwgt = 16,
    kBadDuplicate = 32,
    kBadAsymmetric = 64,
};

__device__ __forceinline__ unsigned long long mix64(unsigned long long z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
__device__ __forceinline__ unsigned long long arc_fp(int32_t u, int32_t v, int32_t w) {
    return mix64(mix64(((unsigned long long)(uint32_t)u << 32) | (uint32_t)v) ^ (uint32_t)w);
}

__device__ __forceinline__ void flag_bad(ValidateOut *o, int32_t u, int32_t what) {
    atomicMin(&o->first_bad, u);
    atomicOr(&o->bad_mask, what);
}

__global__ void k_totals(int32_t n, int32_t nnz, const int32_t *__restrict__ adjwgt,
                         const int32_t *__restrict__ vwgt, ValidateOut *o) {
    unsigned long long a = 0, v = 0;
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nnz; i += stride)
        a += (unsigned long long)(uint32_t)adjwgt[i];
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride)
        v += (unsigned long long)(uint32_t)vwgt[i];
    a = warp_sum64(a);
    v = warp_sum64(v);
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(&o->sum_adjwgt, a);
        atomicAdd(&o->sum_vwgt, v);
    }
}

__global__ void k_fill(int32_t *p, long long len, int32_t value) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < len; i += (long long)gridDim.x * blockDim.x)
        p[i] = value;
}

__global__ void k_check_offsets(int32_t n, int32_t nnz, const int32_t *__restrict__ adjp, ValidateOut *o) {
    for (long long u = (long long)blockIdx.x * blockDim.x + threadIdx.x; u < n; u += (long long)gridDim.x * blockDim.x) {
        const int32_t a = adjp[u], b = adjp[u + 1];
        if ((u == 0 && a != 0) || b < a || a < 0 || b > nnz || (u == n - 1 && b != nnz)) flag_bad(o, (int32_t)u, kBadOffsets);
    }
}

__global__ void k_check_rows(int32_t n, const int32_t *__restrict__ adjp, const int32_t *__restrict__ adjncy,
                             const int32_t *__restrict__ adjwgt, const int32_t *__restrict__ vwgt, ValidateOut *o) {
    unsigned long long f = 0, r = 0;
    int unsorted = 0;
    for (long long uu = (long long)blockIdx.x * blockDim.x + threadIdx.x; uu < n; uu += (long long)gridDim.x * blockDim.x) {
        const int32_t u = (int32_t)uu;
        if (vwgt[u] < 1) flag_bad(o, u, kBadVwgt);
        int32_t prev = -1;
        for (int32_t j = adjp[u]; j < adjp[u + 1]; ++j) {
            const int32_t v = adjncy[j], w = adjwgt[j];
            if (v < 0 || v >= n) {
                flag_bad(o, u, kBadRange);
                continue;
            }
            if (v == u) flag_bad(o, u, kBadSelfLoop);
            if (w < 1) flag_bad(o, u, kBadWeight);
            if (v == prev) flag_bad(o, u, kBadDuplicate);
            if (v < prev) unsorted = 1;
            prev = v;
            f += arc_fp(u, v, w);
            r += arc_fp(v, u, w);
        }
    }
    f = warp_sum64(f);
    r = warp_sum64(r);
    unsorted = __any_sync(0xffffffffu, unsorted);
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(&o->fp_fwd, f);
        atomicAdd(&o->fp_rev, r);
        if (unsorted) atomicOr(&o->unsorted, 1);
    }
}

// exact symmetry when every row is sorted: (v,u) must exist with the same weight
__global__ void k_check_symmetry_sorted(int32_t n, const int32_t *__restrict__ adjp,
                                        const int32_t *__restrict__ adjncy, const int32_t *__restrict__ adjwgt,
                                        ValidateOut *o) {
    for (long long uu = (long long)blockIdx.x * blockDim.x + threadIdx.x; uu < n; uu += (long long)gridDim.x * blockDim.x) {
        const int32_t u = (int32_t)uu;
        for (int32_t j = adjp[u]; j < adjp[u + 1]; ++j) {
            const int32_t v = adjncy[j], w = adjwgt[j];
            int32_t lo = adjp[v], hi = adjp[v + 1];
            while (lo < hi) {
                int32_t mid = (lo + hi) >> 1;
                if (adjncy[mid] < u) lo = mid + 1;
                else hi = mid;
            }
            if (lo >= adjp[v + 1] || adjncy[lo] != u || adjwgt[lo] != w) flag_bad(o, u, kBadAsymmetric);
        }
    }
}

// Exact check of rows in ANY order (R15): every row gets an open-addressing set of its arc
// positions, p(u) = next_pow2(2 deg u) slots at tbl[4 adjp[u]] (p < 4 deg u, load <= 1/2).
// Insert: a probe that meets an arc with the same neighbour is a duplicate.  Then every arc
// (u, v, w) must find an arc (v, u) with weight w in v's set (no duplicates => symmetric
// multiset, exactly).  A warp per row (hub rows stay balanced inside the warp).
__device__ __forceinline__ uint32_t vslot_hash(uint32_t v) {
    v ^= v >> 16; v *= 0x7feb352du; v ^= v >> 15; v *= 0x846ca68bu; v ^= v >> 16;
    return v;
}
__device__ __forceinline__ uint32_t row_slots(int32_t deg) {
    uint32_t p = 1;
    while (p < 2u * (uint32_t)deg) p <<= 1;
    return p;
}
__global__ void k_hash_insert(int32_t n, const int32_t *__restrict__ adjp, const int32_t *__restrict__ adjncy,
                              int32_t *tbl, ValidateOut *o) {
    const int lane = threadIdx.x & 31;
    const long long w0 = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long uu = w0; uu < n; uu += nw) {
        const int32_t u = (int32_t)uu, s = adjp[u], e = adjp[u + 1];
        if (e - s < 2) continue;  // a single arc cannot be a duplicate
        const uint32_t mask = row_slots(e - s) - 1;
        int32_t *t = tbl + 4LL * s;
        for (int32_t j = s + lane; j < e; j += 32) {
            const int32_t v = adjncy[j];
            uint32_t h = vslot_hash((uint32_t)v) & mask;
            for (;;) {
                const int32_t old = atomicCAS(t + h, 0, j + 1);
                if (old == 0) break;
                if (adjncy[old - 1] == v) {
                    flag_bad(o, u, kBadDuplicate);
                    break;
                }
                h = (h + 1) & mask;
            }
        }
    }
}
__global__ void k_hash_symmetry(int32_t n, const int32_t *__restrict__ adjp, const int32_t *__restrict__ adjncy,
                                const int32_t *__restrict__ adjwgt, const int32_t *__restrict__ tbl, ValidateOut *o) {
    const int lane = threadIdx.x & 31;
    const long long w0 = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long uu = w0; uu < n; uu += nw) {
        const int32_t u = (int32_t)uu, s = adjp[u], e = adjp[u + 1];
        for (int32_t j = s + lane; j < e; j += 32) {
            const int32_t v = adjncy[j], w = adjwgt[j];
            const int32_t vs = adjp[v], ve = adjp[v + 1];
            bool ok = false;
            if (ve - vs == 1) {
                ok = adjncy[vs] == u && adjwgt[vs] == w;
            } else if (ve - vs > 1) {
                const uint32_t mask = row_slots(ve - vs) - 1;
                const int32_t *t = tbl + 4LL * vs;
                uint32_t h = vslot_hash((uint32_t)u) & mask;
                for (;;) {
                    const int32_t k = t[h];
                    if (k == 0) break;  // u is not in v's row
                    if (adjncy[k - 1] == u) {
                        ok = adjwgt[k - 1] == w;
                        break;
                    }
                    h = (h + 1) & mask;
                }
            }
            if (!ok) flag_bad(o, u, kBadAsymmetric);
        }
    }
}

static std::string describe(int32_t mask) {
    std::string s;
    if (mask & kBadOffsets) s += " offsets(adjp[0]=0, monotone, adjp[n]=nnz)";
    if (mask & kBadRange) s += " neighbour-id-out-of-range";
    if (mask & kBadSelfLoop) s += " self-loop";
    if (mask & kBadWeight) s += " edge-weight<1";
    if (mask & kBadVwgt) s += " vertex-weight<1";
    if (mask & kBadDuplicate) s += " duplicate-arc";
    if (mask & kBadAsymmetric) s += " asymmetric-arc";
    return s;
}

gp_status graph_totals_and_validate(Ctx *ctx, Graph *g, bool validate, bool check_totals) {
    ValidateOut *d = nullptr;
    gp_status st = dev_alloc(ctx, (void **)&d, sizeof(ValidateOut));
    if (st != GP_OK) return st;
    ValidateOut h;
    memset(&h, 0, sizeof(h));
    h.first_bad = INT32_MAX;
    cudaStream_t s = ctx->stream;
    const int grid = persistent_grid(ctx, 4);
    int32_t *tbl = nullptr;
    cudaError_t e = cudaMemcpyAsync(d, &h, sizeof(h), cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess && validate && g->n > 0) {
        k_check_offsets<<<grid, kBlock, 0, s>>>(g->n, g->nnz, g->adjp, d);
        e = cudaMemcpyAsync(&h, d, sizeof(h), cudaMemcpyDeviceToHost, s);
        if (e == cudaSuccess) e = cudaStreamSynchronize(s);
        if (e == cudaSuccess && h.bad_mask == 0) {
            k_check_rows<<<grid, kBlock, 0, s>>>(g->n, g->adjp, g->adjncy, g->adjwgt, g->vwgt, d);
            e = cudaMemcpyAsync(&h, d, sizeof(h), cudaMemcpyDeviceToHost, s);
            if (e == cudaSuccess) e = cudaStreamSynchronize(s);
            if (e == cudaSuccess && h.bad_mask == 0 && !h.unsorted) {
                k_check_symmetry_sorted<<<grid, kBlock, 0, s>>>(g->n, g->adjp, g->adjncy, g->adjwgt, d);
                ++ctx->launches;
            } else if (e == cudaSuccess && h.bad_mask == 0 && h.unsorted && g->nnz > 0) {
                // unsorted rows: exact per-row hash sets (duplicates first, then symmetry)
                const size_t tb = sizeof(int32_t) * 4 * (size_t)g->nnz;
                st = dev_alloc(ctx, (void **)&tbl, tb);
                if (st == GP_OK) e = cudaMemsetAsync(tbl, 0, tb, s);
                if (st == GP_OK && e == cudaSuccess) {
                    k_hash_insert<<<grid, kBlock, 0, s>>>(g->n, g->adjp, g->adjncy, tbl, d);
                    e = cudaMemcpyAsync(&h, d, sizeof(h), cudaMemcpyDeviceToHost, s);
                    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
                    if (e == cudaSuccess && h.bad_mask == 0)
                        k_hash_symmetry<<<grid, kBlock, 0, s>>>(g->n, g->adjp, g->adjncy, g->adjwgt, tbl, d);
                    ctx->launches += 2;
                }
            }
        }
        ctx->launches += 2;
    }
    if (st == GP_OK && e == cudaSuccess && (!validate || h.bad_mask == 0)) {
        k_totals<<<grid, kBlock, 0, s>>>(g->n, g->nnz, g->adjwgt, g->vwgt, d);
        ++ctx->launches;
        e = cudaMemcpyAsync(&h, d, sizeof(h), cudaMemcpyDeviceToHost, s);
        if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    }
    dev_free(ctx, tbl);
    dev_free(ctx, d);
    if (st != GP_OK) return st;
    if (e != cudaSuccess) return cuda_fail(e, "graph validation");
    if (validate && h.bad_mask) {
        set_error("GP_VALIDATE: first offending vertex " + std::to_string(h.first_bad) + ":" + describe(h.bad_mask));
        return GP_ERR_INVALID_GRAPH;
    }
    g->sum_adjwgt = h.sum_adjwgt;
    g->sum_vwgt = h.sum_vwgt;
    if (check_totals && (h.sum_adjwgt > (unsigned long long)INT32_MAX || h.sum_vwgt > (unsigned long long)INT32_MAX)) {
        set_error("weight totals exceed INT32_MAX: sum(adjwgt)=" + std::to_string(h.sum_adjwgt) +
                  " sum(vwgt)=" + std::to_string(h.sum_vwgt));
        return GP_ERR_OVERFLOW;
    }
    return GP_OK;
}

gp_status fill_ones(Ctx *ctx, int32_t *p, long long len) {
    if (len <= 0) return GP_OK;
    k_fill<<<persistent_grid(ctx, 4), kBlock, 0, ctx->stream>>>(p, len, 1);
    ++ctx->launches;
    GP_CUDA(cudaGetLastError());
    return GP_OK;
}

}  // namespace gp
