// Microbenchmark of one matching round of the partitioned grid tail (part.cu) in isolation:
// 148 CTAs x 512 threads, each CTA a 530-vertex slice of a 280-wide lattice with its rows and
// a proposal window in shared memory; per-warp cycles of the round loop for code variants.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -o /tmp/pr scripts/micro/part_round.cu
#include "../../paper_conf_ipps_goodarzibg16_b200/csrc/part.cu"

namespace gp {
void set_error(const std::string &) {}
gp_status cuda_fail(cudaError_t, const char *) { return GP_ERR_CUDA; }
void launch_begin(Ctx *, int, cudaEvent_t *) {}
void launch_end(Ctx *, int, cudaEvent_t) {}
gp_status dev_alloc(Ctx *, void **, size_t) { return GP_OK; }
void dev_free(Ctx *, void *) {}
}  // namespace gp

using namespace gp;
constexpr int SIDE = 280, NV = 530;

template <int VAR>
__global__ void __launch_bounds__(512, 1) k_round(const int32_t *Pg, int32_t *Pn, long long *cyc, int32_t n) {
    extern __shared__ __align__(16) int32_t sw[];
    const int t = threadIdx.x, b = blockIdx.x;
    PartView V;
    V.n = n;
    V.lo = b * NV;
    V.hi = V.lo + NV;
    V.nv = NV;
    V.garcs = false;
    V.loff = 0;
    V.aoff = 0;
    V.a0 = 0;
    V.sap = sw;
    V.M = sw + 544;
    V.cnt = V.M + 544;
    V.sadj = V.cnt + 544;
    V.swgt = V.sadj + 4 * 544;
    V.win = V.swgt + 4 * 544;
    V.wlo = max(0, V.lo - 2 * SIDE);
    V.wlen = min(n, V.hi + 2 * SIDE) - V.wlo;
    V.gadjp = nullptr;
    V.gadjncy = nullptr;
    V.gadjwgt = nullptr;
    for (int i = t; i <= NV; i += 512) V.sap[i] = 4 * i;
    for (int i = t; i < NV; i += 512) {
        const int u = V.lo + i;
        const int nb[4] = {u - 1, u + 1, u - SIDE, u + SIDE};
        for (int q = 0; q < 4; ++q) {
            V.sadj[4 * i + q] = min(max(nb[q], 0), n - 1);
            V.swgt[4 * i + q] = 1 + ((u * 7 + q * 13) % 100);
        }
        V.M[i] = kFree;
    }
    for (int i = t; i < V.wlen; i += 512) V.win[i] = Pg[V.wlo + i];
    __syncthreads();
    const int32_t *Pk = Pg;
    int32_t live = 0;
    __syncwarp();
    const long long c0 = clock64();
    for (int32_t i = t; i < V.nv; i += 512) {
        if (V.M[i] != kFree) continue;
        const int32_t u = V.lo + i;
        const int32_t p = V.wget(Pk, u);
        if (p < 0) continue;
        const int32_t q = V.wget(Pk, p);
        if (q == u) {
            V.M[i] = p;
            Pn[u] = p;
            continue;
        }
        int32_t np = p;
        if (VAR == 2) {  // pure shared lookups (no predicated global fallback)
            if (q >= 0 && V.win[q - V.wlo] == p) {
                unsigned long long best = 0;
                for (int32_t j = V.rs(i); j < V.rs(i + 1); ++j) {
                    const int32_t x = V.sadj[j], c = V.win[x - V.wlo];
                    if (!(c >= 0 && V.win[c - V.wlo] == x)) best = umax64(best, pack_key<false>(0u, V.swgt[j], x));
                }
                np = key_vertex<false>(0u, best);
            }
        } else if (VAR == 1 || (q >= 0 && V.wget(Pk, q) == p)) np = part_best<false>(V, Pk, 0u, i, true);
        Pn[u] = np;
        live += np >= 0;
    }
    __syncwarp();
    const long long c1 = clock64();
    if ((t & 31) == 0) cyc[b * 16 + (t >> 5)] = c1 - c0;
    if (live == 12345) Pn[0] = live;
}

int main() {
    const int n = 148 * NV;
    int32_t *P, *Pn;
    long long *cyc;
    cudaMalloc(&P, 4 * (n + 64));
    cudaMalloc(&Pn, 4 * (n + 64));
    cudaMalloc(&cyc, 8 * 148 * 16);
    int32_t *h = new int32_t[n];
    for (int u = 0; u < n; ++u) {  // proposals: right neighbour for even, left for odd (pairs), some chains
        int p = (u % 3 == 0) ? u + 1 : (u % 3 == 1 ? u - 1 : u + SIDE);
        h[u] = (p >= 0 && p < n) ? p : -1;
    }
    cudaMemcpy(P, h, 4 * n, cudaMemcpyHostToDevice);
    const int smem = 200 * 1024;
    long long hc[148 * 16];
    auto run = [&](auto kern, const char *name) {
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        for (int rep = 0; rep < 3; ++rep) kern<<<148, 512, smem>>>(P, Pn, cyc, n);
        cudaDeviceSynchronize();
        cudaMemcpy(hc, cyc, sizeof(hc), cudaMemcpyDeviceToHost);
        long long mx = 0, sum = 0;
        for (int i = 0; i < 148 * 16; ++i) {
            mx = hc[i] > mx ? hc[i] : mx;
            sum += hc[i];
        }
        printf("%-28s mean %.0f max %lld cycles per warp (%s)\n", name, (double)sum / (148 * 16), mx,
               cudaGetErrorString(cudaGetLastError()));
    };
    run(k_round<0>, "keep + rescans");
    run(k_round<1>, "rescan every live vertex");
    run(k_round<2>, "keep + rescans, pure LDS");
    return 0;
}
