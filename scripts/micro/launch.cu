// Launch-overhead microbenchmarks (B200): back-to-back cooperative launches of empty kernels in
// the level kernels' shapes, with and without a __threadfence_system + mapped-host write.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/launch launch.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_empty(int *p) {
    extern __shared__ int s[];
    if (threadIdx.x == 0 && blockIdx.x == 0 && p) s[0] = p[0];
}
__global__ void k_fence_sys(volatile int *host) {
    __syncthreads();
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        __threadfence_system();
        *host = 1;
    }
}
int main() {
    cudaStream_t st;
    cudaStreamCreate(&st);
    int *hm, *dm;
    cudaHostAlloc((void **)&hm, 64, cudaHostAllocMapped);
    cudaHostGetDevicePointer((void **)&dm, hm, 0);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    struct Cfg { int grid, block, smem; bool coop; const char *name; } cfgs[] = {
        {296, 512, 110 * 1024, true, "coop 296x512, 110 KB smem (match shape)"},
        {592, 256, 33 * 1024, true, "coop 592x256, 33 KB smem (contract shape)"},
        {296, 512, 110 * 1024, false, "plain 296x512, 110 KB smem"},
        {1, 1024, 210 * 1024, false, "plain 1x1024, 210 KB smem (tail shape)"},
        {148, 128, 0, false, "plain 148x128"},
    };
    cudaFuncSetAttribute(k_empty, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
    for (auto &c : cfgs) {
        for (int rep = 0; rep < 2; ++rep) {
            const int iters = 200;
            int *nul = nullptr;
            void *args[] = {&nul};
            cudaEventRecord(a, st);
            for (int i = 0; i < iters; ++i) {
                if (c.coop) cudaLaunchCooperativeKernel((void *)k_empty, c.grid, c.block, args, c.smem, st);
                else k_empty<<<c.grid, c.block, c.smem, st>>>(nullptr);
            }
            cudaEventRecord(b, st);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            if (rep) printf("%-48s %.2f us per launch (back to back)\n", c.name, ms * 1e3 / iters);
        }
    }
    for (int rep = 0; rep < 2; ++rep) {
        const int iters = 200;
        cudaEventRecord(a, st);
        for (int i = 0; i < iters; ++i) k_fence_sys<<<592, 256, 0, st>>>(dm);
        cudaEventRecord(b, st);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (rep) printf("%-48s %.2f us per launch\n", "592x256 + threadfence_system + mapped write", ms * 1e3 / iters);
    }
    printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
