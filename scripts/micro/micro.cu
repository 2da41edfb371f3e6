// Microbenchmarks of the latencies the level kernels' rounds are made of (B200):
//   grid barrier (the library's monotone-counter barrier) at 296 CTAs x 512 threads,
//   dependent L2-hit load latency (pointer chase over a 16 MB array, 1 warp and 4736 warps),
//   __syncthreads round of one CTA.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/micro micro.cu
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void red_release(unsigned *p, unsigned v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ void gbar(unsigned *bar, unsigned &epoch, unsigned nb, int sleep) {
    __syncthreads();
    if (threadIdx.x == 0) {
        ++epoch;
        red_release(bar, 1u);
        while ((int)(ld_acquire(bar) - epoch * nb) < 0)
            if (sleep) __nanosleep(sleep);
    }
    __syncthreads();
}
__global__ void k_bar(unsigned *bar, int iters, int sleep, unsigned long long *t) {
    unsigned epoch = 0;
    unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) gbar(bar, epoch, gridDim.x, sleep);
    if (blockIdx.x == 0 && threadIdx.x == 0) *t = clock64() - t0;
}
__global__ void k_chase(const int *next, int steps, int start_stride, unsigned long long *t, int *sink) {
    int x = (blockIdx.x * blockDim.x + threadIdx.x) * start_stride % (1 << 22);
    unsigned long long t0 = clock64();
    for (int i = 0; i < steps; ++i) x = __ldcg(next + x);
    unsigned long long dt = clock64() - t0;
    if (threadIdx.x == 0 && blockIdx.x == 0) *t = dt;
    if (x == -7) *sink = x;
}
__global__ void k_init(int *next, int n) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        next[i] = (int)(((long long)i * 2654435761LL + 12345) % n);
}
int main() {
    unsigned *bar;
    unsigned long long *t, ht;
    int *next, *sink;
    cudaMalloc(&bar, 8);
    cudaMalloc(&t, 8);
    cudaMalloc(&sink, 4);
    const int n = 1 << 22;  // 16 MB: L2-resident
    cudaMalloc(&next, n * 4);
    k_init<<<1024, 256>>>(next, n);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    int configs[][3] = {{296, 512, 20}, {296, 512, 0}, {148, 512, 20}, {148, 1024, 20}, {64, 512, 20}, {16, 512, 20}};
    for (auto &c : configs) {
        for (int rep = 0; rep < 2; ++rep) {
            cudaMemset(bar, 0, 8);
            void *args[] = {&bar, nullptr, nullptr, &t};
            int iters = 1000, sleep = c[2];
            args[1] = &iters;
            args[2] = &sleep;
            cudaEventRecord(a);
            cudaLaunchCooperativeKernel((void *)k_bar, c[0], c[1], args, 0, 0);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            if (rep) printf("grid barrier %4d CTAs x %4d thr, nanosleep %2d: %.2f us per barrier\n", c[0], c[1], c[2], ms * 1e3 / iters);
        }
    }
    int chase_cfg[][2] = {{1, 32}, {148, 32}, {296, 512}, {1184, 128}};
    for (auto &c : chase_cfg) {
        for (int rep = 0; rep < 2; ++rep) {
            int steps = 2000;
            cudaEventRecord(a);
            k_chase<<<c[0], c[1]>>>(next, steps, 7919, t, sink);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            cudaMemcpy(&ht, t, 8, cudaMemcpyDeviceToHost);
            if (rep) printf("L2 pointer chase %4d x %4d threads: %.0f cycles/load (%.3f us/load by events)\n", c[0], c[1], (double)ht / steps, ms * 1e3 / steps);
        }
    }
    return 0;
}
